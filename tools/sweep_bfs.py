#!/usr/bin/env python
"""Direction-optimizing BFS switch point sweep on RMAT-<scale>: hybrid BFS
(top-down while the frontier holds <= V / alpha entries, then bottom-up) for
several alpha, per variant; depths checked equal across points.

    python tools/sweep_bfs.py --alphas 16,32,64,128,256 --variants typeptr,cuda
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))

import numpy as np  # noqa: E402

import synth  # noqa: E402
from apps_bench import Env  # noqa: E402
from paper_conf_asplos_zhangar21_b200 import vf  # noqa: E402
from paper_conf_asplos_zhangar21_b200.graph import Graph  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--scale", type=int, default=24)
    ap.add_argument("--alphas", default="16,32,64,128,256")
    ap.add_argument("--variants", default="typeptr,cuda")
    a = ap.parse_args()
    ctx = vf.Ctx(0, cuda_heap_bytes=8 << 30)
    env = Env(ctx)
    offs, col = synth.rmat_graph(a.scale, seed=1)
    src = int(np.argmax(np.diff(offs.astype(np.int64))))
    ref = None
    for v in a.variants.split(","):
        g = Graph(ctx, offs, col, v)
        for al in [int(x) for x in a.alphas.split(",")]:
            out = {}

            def run():
                out["r"] = g.bfs(src, mode="hybrid", alpha=al)
            ms = env.timed(run, 3, 1)
            d = out["r"][0].cpu().numpy()
            ok = True
            if ref is None:
                ref = d
            else:
                ok = bool(np.array_equal(ref, d))
            print(json.dumps({"variant": v, "alpha": al, "bfs_ms": ms, "calls": out["r"][2], "levels": out["r"][1],
                              "agree": ok}), flush=True)
        del g
        env.free()
    ctx.close()


if __name__ == "__main__":
    main()

#!/usr/bin/env python
"""Config-4 launch-shape sweep: hub chunk size C x grid-level type sort (gsort)
for BFS (hybrid) / CC / one PageRank iteration on RMAT-<scale>, per variant.

    python tools/sweep_graph.py --scale 24 --variants typeptr,cuda --chunks 256,64 --gsort 0,1

One JSON line per (variant, C, gsort) on stdout; CUDA events on the app
stream (apps_bench.Env.timed). Depths and labels are checked against the
first configuration's (exact), PageRank ranks to 1e-5.
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
import torch  # noqa: E402

import synth  # noqa: E402
from apps_bench import Env  # noqa: E402
from paper_conf_asplos_zhangar21_b200 import vf  # noqa: E402
from paper_conf_asplos_zhangar21_b200.graph import Graph  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--scale", type=int, default=24)
    ap.add_argument("--variants", default="typeptr,cuda")
    ap.add_argument("--chunks", default="256,64")
    ap.add_argument("--gsort", default="0,1")
    ap.add_argument("--pr-iters", type=int, default=10)
    ap.add_argument("--hot", default="0", help="hot_degree values (graph.slot_order)")
    a = ap.parse_args()
    ctx = vf.Ctx(0, cuda_heap_bytes=8 << 30)
    env = Env(ctx)
    offs, col = synth.rmat_graph(a.scale, seed=1)
    src = int(np.argmax(np.diff(offs.astype(np.int64))))
    ref = None
    for v in a.variants.split(","):
        for C in [int(x) for x in a.chunks.split(",")]:
            for gs, hd in [(int(x), int(h)) for x in a.gsort.split(",") for h in a.hot.split(",")]:
                vf.set_tuning("gsort", gs)
                g = Graph(ctx, offs, col, v, chunk=C, hot_degree=hd)
                ms_b = env.timed(lambda: g.bfs(src), 2, 1)
                d = g.by_id(g.depth).cpu().numpy()
                ms_c = env.timed(lambda: g.cc(), 1, 1)
                lab = g.by_id(g.lab[0]).cpu().numpy()
                g.pr_init()
                ms_p = env.timed(lambda: g.pr_iteration(), a.pr_iters, 2)
                rk = g.by_id(g.rk[0]).cpu().numpy().astype(np.float64)
                ok = True
                if ref is None:
                    ref = (d, lab, rk)
                else:
                    ok = bool(np.array_equal(ref[0], d) and np.array_equal(ref[1], lab)
                              and np.allclose(rk, ref[2], rtol=1e-5, atol=0))
                print(json.dumps({"variant": v, "C": C, "gsort": gs, "hot_degree": hd, "bfs_ms": ms_b, "cc_ms": ms_c,
                                  "pr_iter_ms": ms_p, "agree": ok}), flush=True)
                del g
                env.free()
    vf.set_tuning("gsort", -1)
    ctx.close()


if __name__ == "__main__":
    main()

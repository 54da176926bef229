#!/usr/bin/env python
"""Run a few steps of one app for ncu captures (no timing is reported here).

  ncu --set full --kernel-name-base demangled -k 'regex:graph::App, 4' -c 1 \
      python tools/prof_app.py graph-pr --variant typeptr
"""
from __future__ import annotations

import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_asplos_zhangar21_b200 import apps, vf  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("app")
    ap.add_argument("--variant", default="typeptr")
    ap.add_argument("--scale", type=int, default=24)
    ap.add_argument("--steps", type=int, default=3)
    a = ap.parse_args()
    ctx = vf.Ctx(0, cuda_heap_bytes=8 << 30)
    if a.app.startswith("graph-en"):
        from paper_conf_asplos_zhangar21_b200.graph_en import GraphEN
        offs, col = synth.rmat_graph(a.scale, seed=1)
        g = GraphEN(ctx, offs, col, a.variant)
        src = int(np.argmax(np.diff(offs.astype(np.int64))))
        if a.app == "graph-en-pr":
            g.pr_init()
            for _ in range(a.steps):
                g.pr_iteration()
        elif a.app == "graph-en-cc":
            g.cc(max_iters=a.steps)
        else:
            g.bfs(src)
    elif a.app.startswith("graph"):
        from paper_conf_asplos_zhangar21_b200.graph import Graph
        offs, col = synth.rmat_graph(a.scale, seed=1)
        g = Graph(ctx, offs, col, a.variant)
        src = int(np.argmax(np.diff(offs.astype(np.int64))))
        if a.app == "graph-pr":
            g.pr_init()
            for _ in range(a.steps):
                g.pr_iteration()
        elif a.app == "graph-cc":
            g.cc(max_iters=a.steps)
        elif a.app == "graph-bfs-hybrid":
            g.bfs(src, mode="hybrid")
        else:
            g.bfs(src)
    elif a.app == "stut":
        from paper_conf_asplos_zhangar21_b200.stut import Stut
        s = Stut(ctx, synth.stut_lattice(2048, 2048, seed=12, v_pull=4.0), a.variant)
        for _ in range(a.steps):
            s.step()
    elif a.app == "nbody":
        from paper_conf_asplos_zhangar21_b200.nbody import Nbody
        nb = Nbody(ctx, synth.nbody_system(65536, seed=10), a.variant)
        for _ in range(a.steps):
            nb.step()
    elif a.app == "collide":
        from paper_conf_asplos_zhangar21_b200.collide import Collide
        c = Collide(ctx, synth.collide_system(1 << 24, seed=13), a.variant)
        for _ in range(a.steps):
            c.step()
    elif a.app == "traf":
        from paper_conf_asplos_zhangar21_b200.traf import Traf
        t = Traf(ctx, synth.traf_world(3277, 4096, seed=11), a.variant)
        for _ in range(a.steps):
            t.step()
    elif a.app == "gen":
        g = apps.Gen(ctx, 4096, 4096, synth.soup(4096, 4096, seed=42), a.variant)
        for _ in range(a.steps):
            g.gen()
    elif a.app == "ray":
        from paper_conf_asplos_zhangar21_b200.ray import Ray
        types, P = synth.ray_scene(10000, seed=7)
        r = Ray(ctx, types, P, a.variant)
        cam = synth.ray_camera(1920, 1080)
        for _ in range(a.steps):
            r.render(1920, 1080, cam)
    elif a.app == "gol":
        g = apps.Gol(ctx, 256, 256, synth.soup(256, 256, seed=42), a.variant)
        for _ in range(a.steps):
            g.gen()
    else:
        raise SystemExit(f"unknown app {a.app}")
    torch.cuda.synchronize()
    ctx.close()


if __name__ == "__main__":
    main()

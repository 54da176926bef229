#!/usr/bin/env python
"""Sweep the grouped-kernel knobs (regroup, unroll, prefetch) per app on one
B200 for COAL / TypePointer: ms per step, CUDA-event timed after warm-up.

  python tools/sweep_apps.py --apps gol,gen,stut,traf --out profiles/sweep_apps_r1
"""
from __future__ import annotations

import argparse
import itertools
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_asplos_zhangar21_b200 import apps, vf  # noqa: E402


def ev_time(fn, steps, warm=3):
    for _ in range(warm):
        fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(steps):
        fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / steps


def graphed(gen_fn, gens):
    """CUDA graph of `gens` generations (launch-bound app): returns replay, per-gen divisor."""
    s = torch.cuda.Stream()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for _ in range(gens):
            gen_fn(stream=s)
    return g.replay, gens


def make(ctx, app, variant):
    if app == "gol":
        return apps.Gol(ctx, 256, 256, synth.soup(256, 256, seed=42), variant).gen, 200
    if app == "golgraph":
        g = apps.Gol(ctx, 256, 256, synth.soup(256, 256, seed=42), variant)
        return g, 5
    if app == "gen":
        return apps.Gen(ctx, 4096, 4096, synth.soup(4096, 4096, seed=42), variant).gen, 20
    if app == "stut":
        from paper_conf_asplos_zhangar21_b200.stut import Stut
        return Stut(ctx, synth.stut_lattice(2048, 2048, seed=12, v_pull=4.0), variant).step, 20
    if app == "traf":
        from paper_conf_asplos_zhangar21_b200.traf import Traf
        return Traf(ctx, synth.traf_world(3277, 4096, seed=11), variant).step, 20
    raise SystemExit(app)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--apps", default="gol,gen,stut,traf")
    ap.add_argument("--out", default="gpurun_out/sweep_apps")
    a = ap.parse_args()
    ctx = vf.Ctx(0, cuda_heap_bytes=1 << 30)
    rows = []
    for app in a.apps.split(","):
        for variant in ("sharedoa", "coal", "typeptr"):
            step, n = make(ctx, app, variant)
            grid = [(-1, -1, -1)] if variant == "sharedoa" else itertools.product((0, 1), (1, 2, 4), (0, 2))
            for rg, u, pf in grid:
                vf.set_tuning("regroup", 1 if rg < 0 else rg)
                vf.set_tuning("unroll", u)
                vf.set_tuning("prefetch", pf)
                if app == "golgraph":  # tuning is read at capture time: one graph per config
                    replay, per = graphed(step.gen, 100)
                    ms = ev_time(replay, n) / per
                else:
                    ms = ev_time(step, n)
                r = dict(app=app, variant=variant, regroup=rg, unroll=u, prefetch=pf, ms=ms)
                rows.append(r)
                print(json.dumps(r), flush=True)
            vf.set_tuning("regroup", 1)
            vf.set_tuning("unroll", -1)
            vf.set_tuning("prefetch", -1)
            del step
            ctx.reset()
    os.makedirs(os.path.dirname(a.out) or ".", exist_ok=True)
    with open(a.out + ".jsonl", "w") as f:
        for r in rows:
            f.write(json.dumps(r) + "\n")
    with open(a.out + ".md", "w") as f:
        f.write("| app | variant | regroup | unroll | prefetch | ms/step |\n|---|---|---|---|---|---|\n")
        for r in rows:
            f.write(f"| {r['app']} | {r['variant']} | {r['regroup']} | {r['unroll']} | {r['prefetch']} | "
                    f"{r['ms']:.4f} |\n")


if __name__ == "__main__":
    main()

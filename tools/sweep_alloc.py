#!/usr/bin/env python
"""Allocator sensitivity (the paper's Fig. 10a / 10b, §8.2
P:2727-2747) re-measured on one B200.

Fig. 10a: COAL (and, for reference, SharedOA / TypePointer) throughput per app
as the number of objects in the FIRST region of each type (before doubling,
P:979-985) sweeps 4K -> 4M (x4 steps as the caption says, plus the 128K / 2M
points the text cites, reading G27). VA reservation is OFF (`reserve_va = 0`):
every region is its own cudaMalloc, so the range table really has
K = sum_t ceil(log2(n_t / init + 1)) rows and COAL's binary search pays
ceil(log2 K) steps (K is recorded).
Fig. 10b: SharedOA external fragmentation = unused slots x object bytes /
allocated region bytes, over the app's regions.

  python tools/sweep_alloc.py --out profiles/alloc_sweep_r1 [--quick]
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_asplos_zhangar21_b200 import apps, vf  # noqa: E402
from paper_conf_asplos_zhangar21_b200.collide import Collide  # noqa: E402
from paper_conf_asplos_zhangar21_b200.stut import Stut  # noqa: E402
from paper_conf_asplos_zhangar21_b200.traf import Traf  # noqa: E402

INITS = [4096, 16384, 65536, 131072, 262144, 1 << 20, 2 << 20, 4 << 20]


def ev_time(fn, steps, warm=2):
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


def frag(ctx, app):
    regs = [r for r in ctx.regions() if r["app"] == app]
    cap = sum(r["cap_objs"] * r["obj_bytes"] for r in regs)
    used = sum(r["used_objs"] * r["obj_bytes"] for r in regs)
    return (cap - used) / cap if cap else 0.0, len(regs)


def make(app, ctx, variant, quick):
    if app == "micro":
        n = (1 << 22) if quick else (1 << 24)
        types = synth.micro_types(n, 4, "random", seed=42)
        m = apps.Micro(ctx, n, 4, variant=variant, types_np=types, init_np=synth.micro_init(n, seed=42))
        return vf.APP_MICRO, m.step, n
    if app == "micro32":
        n = (1 << 22) if quick else (1 << 24)
        types = synth.micro_types(n, 32, "random", seed=42)
        m = apps.Micro(ctx, n, 32, variant=variant, types_np=types, init_np=synth.micro_init(n, seed=42))
        return vf.APP_MICRO, m.step, n
    if app == "gen":
        W = 1024 if quick else 4096
        g = apps.Gen(ctx, W, W, synth.soup(W, W, seed=42), variant)
        return vf.APP_GEN, g.gen, W * W
    if app == "traf":
        R = 400 if quick else 3277
        t = Traf(ctx, synth.traf_world(R, 4096, seed=11), variant)
        return vf.APP_TRAF, t.step, t.calls_per_step
    if app == "stut":
        W = 512 if quick else 2048
        st = Stut(ctx, synth.stut_lattice(W, W, seed=12, v_pull=4.0), variant)
        return vf.APP_STUT, st.step, st.calls_per_step
    if app == "collide":
        N = (1 << 20) if quick else (1 << 22)
        c = Collide(ctx, synth.collide_system(N, seed=13), variant)
        return vf.APP_COLLIDE, c.step, 2 * N
    raise ValueError(app)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--apps", default="micro,micro32,gen,traf,stut,collide")
    ap.add_argument("--variants", default="sharedoa,coal,typeptr")
    ap.add_argument("--out", default="gpurun_out/alloc_sweep")
    ap.add_argument("--quick", action="store_true")
    a = ap.parse_args()
    rows = []
    for init in INITS:
        ctx = vf.Ctx(0, init_chunk_objs=init, reserve_va=False, cuda_heap_bytes=1 << 28)
        for app in a.apps.split(","):
            for v in a.variants.split(","):
                app_id, step, calls = make(app, ctx, v, a.quick)
                ms = ev_time(step, 10)
                fr, nreg = frag(ctx, app_id)
                K = len(ctx.range_table(app_id))
                row = dict(app=app, variant=v, init_objs=init, ms_per_step=ms, calls_per_s=calls / (ms / 1e3),
                           K=K, regions=nreg, ext_frag=fr)
                rows.append(row)
                print(json.dumps(row), flush=True)
                del step
                ctx.reset()
        ctx.close()
    os.makedirs(os.path.dirname(a.out) or ".", exist_ok=True)
    with open(a.out + ".jsonl", "w") as f:
        for r in rows:
            f.write(json.dumps(r) + "\n")
    inits = INITS
    with open(a.out + ".md", "w") as f:
        f.write("Fig. 10a analogue: Gcalls/s per (app, variant) vs objects in the first region "
                "(reserve_va = 0; K = range-table rows)\n\n")
        f.write("| app | variant | " + " | ".join(f"{i // 1024}K" for i in inits) + " |\n")
        f.write("|---|---|" + "---|" * len(inits) + "\n")
        for app in a.apps.split(","):
            for v in a.variants.split(","):
                cells = []
                for i in inits:
                    r = next((x for x in rows if x["app"] == app and x["variant"] == v and x["init_objs"] == i), None)
                    cells.append(f"{r['calls_per_s'] / 1e9:.2f} (K={r['K']})" if r else "-")
                f.write(f"| {app} | {v} | " + " | ".join(cells) + " |\n")
        f.write("\nFig. 10b analogue: SharedOA external fragmentation (unused slot bytes / region bytes)\n\n")
        f.write("| app | " + " | ".join(f"{i // 1024}K" for i in inits) + " |\n")
        f.write("|---|" + "---|" * len(inits) + "\n")
        for app in a.apps.split(","):
            cells = []
            for i in inits:
                r = next((x for x in rows if x["app"] == app and x["variant"] == "sharedoa" and x["init_objs"] == i),
                         None)
                cells.append(f"{100 * r['ext_frag']:.1f}%" if r else "-")
            f.write(f"| {app} | " + " | ".join(cells) + " |\n")
    print("wrote", a.out)


if __name__ == "__main__":
    main()

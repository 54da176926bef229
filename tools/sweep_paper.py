#!/usr/bin/env python
"""The paper's microbenchmark studies re-measured on one B200 (config 2):

  fig12a  calls/s vs number of objects (T = 4, random order)
  fig12b  calls/s vs types per warp k (n fixed, order k-per-warp)
  fig11   TypePointer on device-heap objects vs on typed arenas
  tab1c   COAL / TypePointer with the paper's indirect CALL vs our grouped direct call
          (Table 1 row C, Fig. 5b line 4)

Variants: cuda (device-heap new + virtual call), sharedoa, concord (embedded tag +
switch), coal, typeptr, coal_ind / typeptr_ind (indirect CALL), typeptr_heap, and
the BRANCH ceiling. Every step is CUDA-event timed with the L2 flushed before it.

  python tools/sweep_paper.py --out profiles/paper_sweep_r1
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_asplos_zhangar21_b200 import apps, vf  # noqa: E402

_FLUSH = None


def timeit(m, reps=10, warm=3):
    global _FLUSH
    if _FLUSH is None:
        _FLUSH = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    for _ in range(warm):
        m.step()
    torch.cuda.synchronize()
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(reps)]
    for a, b in evs:
        _FLUSH.zero_()
        a.record()
        m.step()
        b.record()
    torch.cuda.synchronize()
    return sum(a.elapsed_time(b) for a, b in evs) / reps


def measure(ctx, variant, n, T, order, k=None):
    types = synth.micro_types(n, T, order, seed=42, k=k)
    init = synth.micro_init(n, seed=42)
    if variant == "branch":
        m = apps.MicroBranch(ctx, n, T, order, seed=42, k=k, init_np=init)
        ms = timeit(m)
    else:
        base = variant[:-4] if variant.endswith("_ind") else variant
        m = apps.Micro(ctx, n, T, variant=base, types_np=types, init_np=init)
        vf.set_tuning("call", 1 if variant.endswith("_ind") else 0)
        try:
            ms = timeit(m)
        finally:
            vf.set_tuning("call", 0)
    del m
    ctx.reset()
    return ms


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default="gpurun_out/paper_sweep")
    ap.add_argument("--studies", default="fig12a,fig12b,fig11,tab1c")
    ap.add_argument("--cuda-max", type=int, default=1 << 23, help="largest n for device-heap allocation")
    a = ap.parse_args()
    ctx = vf.Ctx(0, cuda_heap_bytes=8 << 30)
    rows = []

    def rec(study, variant, n, T, order, k, ms):
        r = dict(study=study, variant=variant, n=n, T=T, order=order, k=k, ms=ms, gcalls_per_s=n / ms / 1e6)
        rows.append(r)
        print(json.dumps(r), flush=True)

    allv = ["branch", "concord", "sharedoa", "coal", "typeptr", "cuda"]
    studies = a.studies.split(",")
    if "fig12a" in studies:
        for lg in (20, 21, 22, 23, 24, 25):
            n = 1 << lg
            for v in allv:
                if v == "cuda" and n > a.cuda_max:
                    continue
                rec("fig12a", v, n, 4, "random", None, measure(ctx, v, n, 4, "random"))
    if "fig12b" in studies:
        n = 1 << 22
        for k in (1, 2, 4, 8, 16, 32):
            for v in allv:
                rec("fig12b", v, n, 32, "kperwarp", k, measure(ctx, v, n, 32, "kperwarp", k))
    if "fig11" in studies:
        n = 1 << 22
        for T in (4, 32):
            for v in ("cuda", "typeptr_heap", "sharedoa", "typeptr"):
                rec("fig11", v, n, T, "random", None, measure(ctx, v, n, T, "random"))
    if "tab1c" in studies:
        n = 1 << 24
        for T in (1, 4, 16, 32):
            for v in ("sharedoa", "coal_ind", "coal", "typeptr_ind", "typeptr"):
                rec("tab1c", v, n, T, "random", None, measure(ctx, v, n, T, "random"))

    os.makedirs(os.path.dirname(a.out) or ".", exist_ok=True)
    with open(a.out + ".jsonl", "w") as f:
        for r in rows:
            f.write(json.dumps(r) + "\n")
    with open(a.out + ".md", "w") as f:
        for study in studies:
            sub = [r for r in rows if r["study"] == study]
            if not sub:
                continue
            vs = list(dict.fromkeys(r["variant"] for r in sub))
            keyf = (lambda r: (r["n"], r["T"], r["k"]))
            keys = list(dict.fromkeys(keyf(r) for r in sub))
            f.write(f"\n### {study} (Gcalls/s; L2 flushed before every step)\n\n| n | T | k | " + " | ".join(vs) +
                    " |\n|" + "---|" * (3 + len(vs)) + "\n")
            for key in keys:
                d = {r["variant"]: r["gcalls_per_s"] for r in sub if keyf(r) == key}
                f.write(f"| 2^{key[0].bit_length() - 1} | {key[1]} | {key[2] if key[2] else '-'} | " +
                        " | ".join(f"{d[v]:.1f}" if v in d else "—" for v in vs) + " |\n")
    print("wrote", a.out)


if __name__ == "__main__":
    main()

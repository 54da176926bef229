#!/usr/bin/env python
"""Config-2 launch-knob sweep for the COAL / TypePointer grouped kernels
(vf_set_tuning: unroll x prefetch x regroup) at n = 2^26, random order,
T in {4, 32}. Each object set is allocated once and re-dispatched under every
knob setting (CUDA events, inputs >> L2). Run on a B200:

  python tools/sweep_knobs.py --out profiles/sweep_knobs_r1
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_asplos_zhangar21_b200 import apps, vf  # noqa: E402


def timeit(m, reps=30, warm=3):
    for _ in range(warm):
        m.step()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(reps):
        m.step()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / reps


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=1 << 26)
    ap.add_argument("--Ts", default="4,32")
    ap.add_argument("--out", default="gpurun_out/sweep_knobs")
    ap.add_argument("--regroups", default="1,0")
    ap.add_argument("--unrolls", default="1,2,4")
    ap.add_argument("--pfs", default="0,1,2", help="prefetch values (3 = deep pipeline, sorted kernel)")
    a = ap.parse_args()
    ctx = vf.Ctx(0, cuda_heap_bytes=1 << 30)
    rows = []
    for T in [int(x) for x in a.Ts.split(",")]:
        types = synth.micro_types(a.n, T, "random", seed=42)
        init = synth.micro_init(a.n, seed=42)
        for v in ("coal", "typeptr"):
            m = apps.Micro(ctx, a.n, T, variant=v, types_np=types, init_np=init)
            for rg in [int(x) for x in a.regroups.split(",")]:
                for u in [int(x) for x in a.unrolls.split(",")]:
                    for pf in [int(x) for x in a.pfs.split(",")]:
                        vf.set_tuning("regroup", rg)
                        vf.set_tuning("unroll", u)
                        vf.set_tuning("prefetch", pf)
                        ms = timeit(m)
                        rows.append(dict(T=T, variant=v, regroup=rg, unroll=u, prefetch=pf, ms=ms,
                                         gcalls=a.n / ms / 1e6))
                        print(json.dumps(rows[-1]), flush=True)
            for k, val in (("regroup", 1), ("unroll", -1), ("prefetch", -1)):
                vf.set_tuning(k, val)
            rows.append(dict(T=T, variant=v, regroup="default", unroll="default", prefetch="default",
                             ms=timeit(m), gcalls=None))
            rows[-1]["gcalls"] = a.n / rows[-1]["ms"] / 1e6
            print(json.dumps(rows[-1]), flush=True)
            del m
            ctx.reset()
    os.makedirs(os.path.dirname(a.out) or ".", exist_ok=True)
    with open(a.out + ".jsonl", "w") as f:
        for r in rows:
            f.write(json.dumps(r) + "\n")
    with open(a.out + ".md", "w") as f:
        f.write(f"Config 2 knob sweep, n = {a.n}, random order (Gcalls/s)\n\n"
                "| T | variant | regroup | unroll | prefetch | Gcalls/s |\n|---|---|---|---|---|---|\n")
        for r in rows:
            f.write(f"| {r['T']} | {r['variant']} | {r['regroup']} | {r['unroll']} | {r['prefetch']} | "
                    f"{r['gcalls']:.1f} |\n")
    print("wrote", a.out)


if __name__ == "__main__":
    main()

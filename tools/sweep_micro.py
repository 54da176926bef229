#!/usr/bin/env python
"""Config-2 sweep (paper Fig. 12b analogue): calls/s of every dispatch variant over
T in {1,2,4,8,16,32} x {random, sorted} at n = 2^26 per GPU (device-heap CUDA
baseline at n = 2^22, where device `new` finishes in seconds). Writes JSON + a
markdown table. Run on a B200: python tools/sweep_micro.py --out profiles/sweep_micro_r1
"""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_asplos_zhangar21_b200 import apps, vf  # noqa: E402


_FLUSH = None


def timeit(m, reps, warm=3):
    """Per-step CUDA events; the L2 is flushed (512 MiB memset) before every step
    so 2^22-object working sets (< 126 MB L2) are measured from HBM too."""
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


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=1 << 26)
    ap.add_argument("--cuda-n", type=int, default=1 << 22)
    ap.add_argument("--reps", type=int, default=20)
    ap.add_argument("--Ts", default="1,2,4,8,16,32")
    ap.add_argument("--orders", default="random,sorted")
    ap.add_argument("--out", default="gpurun_out/sweep_micro")
    a = ap.parse_args()
    ctx = vf.Ctx(0, cuda_heap_bytes=8 << 30)
    rows = []
    for order in a.orders.split(","):
        for T in [int(x) for x in a.Ts.split(",")]:
            for n, variants in ((a.n, ("sharedoa", "coal", "typeptr")), (a.cuda_n, ("cuda", "sharedoa", "coal", "typeptr"))):
                types = synth.micro_types(n, T, order, seed=42)
                init = synth.micro_init(n, seed=42)
                for v in variants:
                    t0 = time.time()
                    m = apps.Micro(ctx, n, T, variant=v, types_np=types, init_np=init)
                    ta = time.time() - t0
                    ms = timeit(m, a.reps)
                    rows.append(dict(order=order, T=T, n=n, variant=v, ms=ms, calls_per_s=n / ms * 1e3,
                                     alloc_s=ta))
                    print(json.dumps(rows[-1]), flush=True)
                    del m
                ctx.reset()
    os.makedirs(os.path.dirname(a.out) or ".", exist_ok=True)
    json.dump(rows, open(a.out + ".json", "w"), indent=1)
    with open(a.out + ".md", "w") as f:
        f.write("| order | T | n | " + " | ".join(["cuda", "sharedoa", "coal", "typeptr"]) +
                " | coal/sharedoa | typeptr/sharedoa | typeptr/cuda |\n|---|---|---|---|---|---|---|---|---|---|\n")
        for order in a.orders.split(","):
            for T in [int(x) for x in a.Ts.split(",")]:
                for n in (a.n, a.cuda_n):
                    d = {r["variant"]: r["calls_per_s"] / 1e9 for r in rows
                         if r["order"] == order and r["T"] == T and r["n"] == n}
                    fmt = lambda k: f"{d[k]:.1f}" if k in d else "—"
                    rel = lambda x, y: f"{d[x] / d[y]:.2f}" if x in d and y in d else "—"
                    f.write(f"| {order} | {T} | 2^{n.bit_length() - 1} | {fmt('cuda')} | {fmt('sharedoa')} | "
                            f"{fmt('coal')} | {fmt('typeptr')} | {rel('coal', 'sharedoa')} | "
                            f"{rel('typeptr', 'sharedoa')} | {rel('typeptr', 'cuda')} |\n")
    print("wrote", a.out)


if __name__ == "__main__":
    main()

#!/usr/bin/env python
"""Benchmark: virtual calls/s of the config-2 dispatch microbenchmark (BASELINE.json configs[1]).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                    [--variant typeptr] [--T 4] [--order random] [--n 67108864]

One step = one dispatch pass: one virtual `apply()` call on each of the n
polymorphic objects (paper §8.3), through libvf's kernel for the
chosen variant, with the object pointers and objects resident in HBM. With
torchrun (N > 1) every rank runs its own n objects (weak scaling, no
data-path collective: the dispatch is per-object independent); time is the max
over ranks of the CUDA-event time between barriers.

Rank 0 prints ONE JSON line. Besides the contract keys it carries
  variants      calls/s of cuda(device-heap new), sharedoa, coal, typeptr, measured in this run
  roofline      achieved algorithmic GB/s of the dispatch kernel vs MEASURED_PEAKS hbm_gbs
  cpu_baseline  the CPU oracle (tests-only code) timed on a bounded sample on this host
  e2e           the same metric through the C ABI from pinned host buffers
`--impl reference` times the CPU oracle itself (the only reference this paper has).
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

ALG_BYTES_PER_CALL = 16  # 8 B pointer + 4 B field read + 4 B field write
LAYOUT_BYTES_PER_CALL = 40  # 8 B pointer + the 16 B object's sector share read + written


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=500)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--variant", default="typeptr", choices=["cuda", "sharedoa", "coal", "typeptr"])
    ap.add_argument("--T", type=int, default=4)
    ap.add_argument("--order", default="random", choices=["random", "sorted", "kperwarp"])
    ap.add_argument("--n", "--objects", dest="n", type=int, default=1 << 26)
    ap.add_argument("--seed", type=int, default=42)
    ap.add_argument("--cuda-n", type=int, default=1 << 24,
                    help="objects for the same-config comparison with the device-heap CUDA baseline (device "
                         "`new` of 2^24 objects takes ~36 s on B200, of 2^26 ~10 min)")
    ap.add_argument("--apps", default=",".join(("gol", "ray", "nbody", "gen", "traf", "stut", "collide", "graph")),
                    help="per-app block (BASELINE configs 1, 3, 4, 5); '' to skip")
    ap.add_argument("--app-variants", default="cuda,cuda_packed,sharedoa,coal,typeptr")
    ap.add_argument("--app-small", action="store_true",
                    help="per-app block at code-path test sizes (tests only; not a BASELINE config)")
    ap.add_argument("--strong", action="store_true",
                    help="N > 1: split ONE array of --n objects into contiguous blocks (default: weak, --n per GPU)")
    ap.add_argument("--no-variants", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--cpu-sample", type=int, default=1 << 24)
    return ap.parse_args()


# --------------------------------------------------------------------------- clocks
class Clocks:
    REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap",
               0x8: "hw_slowdown", 0x20: "sync_boost", 0x40: "sw_thermal_slowdown",
               0x80: "hw_thermal_slowdown", 0x100: "hw_power_brake_slowdown"}

    def __init__(self, dev):
        self.dev, self.proc, self.lines = dev, None, []

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.dev), "--query-gpu=clocks.sm,clocks.max.sm,clocks_event_reasons.active",
                 "--format=csv,noheader,nounits", "-lms", "50"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if not self.proc:
            return None
        time.sleep(0.06)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=2)
        except Exception:
            self.proc.kill()
        sm, mx, reasons = [], 0.0, set()
        for l in self.lines:
            try:
                a, b, c = [x.strip() for x in l.split(",")]
                sm.append(float(a))
                mx = max(mx, float(b))
                r = int(c, 16)
                for bit, name in self.REASONS.items():
                    if r & bit:
                        reasons.add(name)
            except Exception:
                pass
        if not sm:
            return None
        sm.sort()
        return {"sm_mhz": sm[len(sm) // 2], "sm_max_mhz": mx, "reasons": sorted(reasons), "samples": len(sm)}


# --------------------------------------------------------------------------- helpers
def max_over_ranks(ms, dev):
    import torch
    import torch.distributed as dist
    t = torch.tensor([ms], dtype=torch.float64, device="cpu" if dist.get_backend() == "gloo" else dev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return {}


def ncu_traffic(kernel_key):
    """dram bytes per launch from the committed ncu --set full summary, if present."""
    try:
        d = json.load(open(os.path.join(ROOT, "profiles", "ncu_summary.json")))
        e = d["kernels"].get(kernel_key)
        return None if e is None else e.get("dram_bytes_per_launch")
    except Exception:
        return None


def cpu_model():
    try:
        for l in open("/proc/cpuinfo"):
            if l.startswith("model name"):
                return l.split(":", 1)[1].strip()
    except Exception:
        pass
    return "?"


_SAMPLE = {}


def oracle_micro_sample(args, n_s, reps, threads):
    """Times `reps` oracle passes over an n_s-object sample (inputs generated once)."""
    import numpy as np

    import oracle
    import synth
    if n_s not in _SAMPLE:
        _SAMPLE[n_s] = (synth.micro_types(n_s, args.T, args.order, seed=args.seed),
                        synth.micro_init(n_s, seed=args.seed))
    t, init = _SAMPLE[n_s]
    vals, sec = oracle.micro_run(t, init, args.T, reps, threads=threads)
    assert np.array_equal(vals, init + reps * (t.astype(np.int32) + 1))  # closed form
    return sec


# --------------------------------------------------------------------------- reference arm
def workload_config(args, world):
    """The workload both arms measure (the reference arm times a bounded sample
    of it on the host; its cpu_baseline.sample says which)."""
    strong = getattr(args, "strong", False) and world > 1
    per = f"{args.n} objects in total, contiguous blocks of n/{world} per GPU" if strong else f"{args.n} objects/GPU"
    return {"workload": f"micro: n={per} x T={args.T} types, {args.order} order, "
                        f"1 virtual apply() per object per step",
            "variant": args.variant, "n": args.n, "T": args.T, "order": args.order,
            "seed": args.seed, "object_bytes": 16,
            "l2": "inputs larger than L2 (1.5 GiB objects+pointers per GPU >> 126 MB)",
            "parallelism": f"dp{world} ({'strong: one array split into index blocks' if strong else 'weak: independent object shards'})"}


def run_reference(args, rank, world):
    if rank != 0:
        return
    import oracle
    threads = oracle.max_threads()
    n_s = min(args.n, args.cpu_sample)
    # one step = one pass over a bounded sample of the workload on all host cores;
    # the oracle times its pass loop itself (object allocation is outside, as on the GPU)
    oracle_micro_sample(args, n_s, max(1, args.warmup), threads)
    per = oracle_micro_sample(args, n_s, 1, threads)
    k = max(1, min(args.steps, int(60.0 / max(per, 1e-6))))  # keep the arm to about a minute
    tot = oracle_micro_sample(args, n_s, k, threads)
    v = n_s * k / tot
    out = {"impl": "reference", "metric": "virtual calls/s (config 2 dispatch microbenchmark)",
           "value": v, "unit": "calls/s", "n_gpus": args.gpus, "steps": k, "warmup": args.warmup,
           "ms_per_step": 1e3 * tot / k, "higher_is_better": True, "scaling": "weak",
           "vs_baseline": None, "dtype": "int32", "data": "synthetic",
           "config": workload_config(args, world),
           "cpu_baseline": {"value": v, "unit": "calls/s", "cores": threads, "kind": "oracle",
                            "sample": f"{n_s} objects per step ({args.order}, T={args.T}), one pass, "
                                      f"OpenMP {threads} threads, {cpu_model()}"},
           "e2e": {"value": v, "unit": "calls/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)


# --------------------------------------------------------------------------- our arm
def run_ours(args, rank, world, local):
    import numpy as np
    import torch
    import torch.distributed as dist

    import synth
    from paper_conf_asplos_zhangar21_b200 import apps, vf

    torch.cuda.set_device(local)
    dev = torch.device(f"cuda:{local}")
    ctx = vf.Ctx(local, cuda_heap_bytes=16 << 30)
    s = torch.cuda.Stream(device=dev)
    if args.strong and world > 1:
        # strong scaling: ONE array of args.n objects, contiguous
        # index blocks of n / world per rank (same global draws as N = 1)
        per = -(-args.n // world)
        lo, hi = min(args.n, rank * per), min(args.n, (rank + 1) * per)
        types = synth.micro_types(args.n, args.T, args.order, seed=args.seed)[lo:hi].copy()
        init = synth.micro_init(args.n, seed=args.seed)[lo:hi].copy()
        n = hi - lo
    else:
        n = args.n
        types = synth.micro_types(n, args.T, args.order, seed=args.seed + rank)
        init = synth.micro_init(n, seed=args.seed + rank)
    n_total = args.n if (args.strong and world > 1) else world * n

    def barrier():
        if world > 1:
            dist.barrier()

    def timed(m, steps, warmup):
        with torch.cuda.stream(s):
            for _ in range(warmup):
                m.step(s)
        torch.cuda.synchronize(dev)
        barrier()
        torch.cuda.synchronize(dev)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        l0 = vf.launch_count()
        e0.record(s)
        for _ in range(steps):
            m.step(s)
        e1.record(s)
        torch.cuda.synchronize(dev)
        barrier()
        launches = vf.launch_count() - l0
        ms = e0.elapsed_time(e1)
        if world > 1:
            ms = max_over_ranks(ms, dev)
        return ms, launches

    flush_buf = None

    def timed_flush(m, steps, warmup):
        """Per-step CUDA events with a 512 MiB L2 flush (memset) before each step:
        for working sets that would otherwise stay resident in the 126 MB L2."""
        nonlocal flush_buf
        if flush_buf is None:
            flush_buf = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
        with torch.cuda.stream(s):
            for _ in range(warmup):
                m.step(s)
        torch.cuda.synchronize(dev)
        evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(steps)]
        with torch.cuda.stream(s):
            for a, b in evs:
                flush_buf.zero_()
                a.record(s)
                m.step(s)
                b.record(s)
        torch.cuda.synchronize(dev)
        return sum(a.elapsed_time(b) for a, b in evs)

    results = {}
    # ---- headline variant at the BASELINE size ----
    m = apps.Micro(ctx, n, args.T, variant=args.variant, types_np=types, init_np=init)
    clocks = Clocks(local)
    clocks.start()
    time.sleep(0.5)  # let the sampler come up so it covers the timed region
    ms, launches = timed(m, args.steps, args.warmup)
    clk = clocks.stop()
    step_ms = ms / args.steps
    value = n_total * args.steps / (ms / 1e3)
    # parity spot-check of the timed objects (closed form on a sample; oracle parity lives in tests/)
    reps = args.warmup + args.steps
    vals = m.values().cpu().numpy()
    idx = np.random.default_rng(rank).integers(0, n, 4096)
    ok = bool(np.array_equal(vals[idx], init[idx] + reps * (types[idx].astype(np.int32) + 1)))

    # ---- e2e: pointer array H2D from pinned host memory + dispatch + result checksum D2H ----
    e2e = None
    if not args.no_e2e:
        host_ptrs = m.objs.cpu().pin_memory()
        dev_ptrs = torch.empty_like(m.objs)
        vals_dev = torch.empty(n, dtype=torch.int32, device=dev)
        csum = torch.zeros(1, dtype=torch.int64, device=dev)
        csum_host = torch.zeros(1, dtype=torch.int64).pin_memory()
        get = vf.micro_get_args(vals_dev.data_ptr())
        e2e_steps = max(3, min(20, args.steps))

        def e2e_step():
            # vf_dispatch_host: chunked H2D of the host pointer array on a copy
            # stream, each chunk dispatched as soon as it lands (overlap)
            ctx.dispatch_host(m.v, vf.APP_MICRO, vf.MICRO_APPLY, host_ptrs, dev_ptrs, stream=s)
            ctx.dispatch(m.v, vf.APP_MICRO, vf.MICRO_GET, dev_ptrs, get, stream=s)
            csum.zero_()
            vf.checksum_i32(vals_dev, csum, stream=s)
            csum_host.copy_(csum, non_blocking=True)

        with torch.cuda.stream(s):
            for _ in range(2):
                e2e_step()
            torch.cuda.synchronize(dev)
            barrier()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            for _ in range(e2e_steps):
                e2e_step()
            e1.record(s)
        torch.cuda.synchronize(dev)
        e_ms = e0.elapsed_time(e1)
        if world > 1:
            e_ms = max_over_ranks(e_ms, dev)
        e2e = {"value": n_total * e2e_steps / (e_ms / 1e3), "unit": "calls/s",
               "h2d_bytes_per_step": 8 * n, "d2h_bytes_per_step": 8,
               "path": "pinned host pointer array -> vf_dispatch_host(apply; chunked H2D overlapped with the "
                       "calls) -> vf_dispatch(get) -> vf_checksum_i32 -> 8 B D2H"}
        del host_ptrs, dev_ptrs, vals_dev
    del m
    ctx.reset()

    # ---- the other variants (same config; device-heap CUDA baseline at cuda_n) ----
    if not args.no_variants:
        for variant in ("cuda_packed", "sharedoa", "coal", "typeptr"):
            if variant == args.variant:
                results[variant] = {"calls_per_s": value, "n": n}
                continue
            mv = apps.Micro(ctx, n, args.T, variant=variant, types_np=types, init_np=init)
            vms, _ = timed(mv, max(20, args.steps // 4), args.warmup)
            results[variant] = {"calls_per_s": n_total * max(20, args.steps // 4) / (vms / 1e3), "n": n}
            del mv
            ctx.reset()
        # device-heap `new` baseline (paper's CUDA) at a size it allocates in seconds
        cn = min(args.cuda_n, n)
        small = {}
        for variant in ("cuda", "cuda_packed", "sharedoa", "coal", "typeptr"):
            mv = apps.Micro(ctx, cn, args.T, variant=variant, types_np=types[:cn], init_np=init[:cn])
            vms = timed_flush(mv, 30, args.warmup)
            small[variant] = world * cn * 30 / (vms / 1e3)
            del mv
        ctx.reset()
        results["at_cuda_n"] = {"n": cn, "l2": "flushed (512 MiB memset) before every timed step",
                                **{k: v for k, v in small.items()},
                                "speedup_vs_cuda": {k: v / small["cuda"] for k, v in small.items()}}
        base = results.get("sharedoa", {}).get("calls_per_s")
        if base:
            results["speedup_vs_sharedoa_at_n"] = {k: results[k]["calls_per_s"] / base
                                                   for k in ("cuda_packed", "sharedoa", "coal", "typeptr")}
        if results.get("cuda_packed"):
            results["speedup_vs_cuda_packed_at_n"] = {k: results[k]["calls_per_s"] / results["cuda_packed"]["calls_per_s"]
                                                      for k in ("cuda_packed", "sharedoa", "coal", "typeptr")}

    # ---- CPU baseline: the oracle on this host, bounded sample (rank 0, N=1 only) ----
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu:
        import oracle
        threads = oracle.max_threads()
        n_s = min(n, args.cpu_sample)
        reps_c = 10
        sec = oracle_micro_sample(args, n_s, reps_c, threads)
        cpu = {"value": n_s * reps_c / sec, "unit": "calls/s", "cores": threads, "kind": "oracle",
               "sample": f"{n_s} objects x {reps_c} passes ({args.order}, T={args.T}), OpenMP {threads} "
                         f"threads, {cpu_model()}"}

    # ---- per-app block: BASELINE configs 1, 3, 4, 5 (tools/apps_bench.py) ----
    apps_block = None
    names = [a for a in args.apps.split(",") if a]
    if names:
        sys.path.insert(0, os.path.join(ROOT, "tools"))
        import apps_bench
        env = apps_bench.Env(ctx, rank, world, None, local)

        def log(name, row):
            if rank == 0:
                print(f"# app {name}: {row.get('wall_s', 0):.1f} s", file=sys.stderr, flush=True)

        apps_block = apps_bench.run_apps(env, names, tuple(args.app_variants.split(",")),
                                         cpu=(rank == 0 and world == 1 and not args.no_cpu), clocks_cls=Clocks,
                                         log=log, small=args.app_small)

    pk = peaks()
    hbm = pk.get("hbm_gbs")
    peak_src = "MEASURED_PEAKS.json hbm_gbs (copy, burst), of measured"
    if not hbm:  # file absent on this box: the profiling guide's stated fallback
        hbm, peak_src = 6650.0, "B200_PROFILING.md fallback 6.65 TB/s (MEASURED_PEAKS.json absent), of fallback"
    # the library's default for these variants: the type-sorted tile kernel
    # (vf_set_tuning "regroup" = 1), as in the ncu launch list (profiles/)
    kern = f"k_dispatch_sorted<micro,apply,{'ResolveTP' if args.variant == 'typeptr' else 'ResolveCOAL'}>" \
        if args.variant in ("coal", "typeptr") else "k_dispatch_virtual<micro,apply>"
    achieved = ALG_BYTES_PER_CALL * n / (step_ms / 1e3) / 1e9
    tr = ncu_traffic(f"micro_{args.variant}_T{args.T}_{args.order}")
    roof = {"bound": "hbm", "kernel": kern, "achieved": achieved, "peak": hbm, "unit": "GB/s",
            "frac": (achieved / hbm) if hbm else None,
            "peak_source": peak_src,
            "traffic": tr,
            "alg_bytes_per_call": ALG_BYTES_PER_CALL,
            "layout_floor_bytes_per_call": LAYOUT_BYTES_PER_CALL,
            "layout_floor_frac": (LAYOUT_BYTES_PER_CALL * n / (step_ms / 1e3) / 1e9 / hbm) if hbm else None}
    if rank == 0:
        out = {"metric": "virtual calls/s (config 2 dispatch microbenchmark)", "value": value,
               "unit": "calls/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
               "ms_per_step": step_ms, "higher_is_better": True,
               "scaling": "strong" if (args.strong and world > 1) else "weak",
               "vs_baseline": None, "dtype": "int32", "data": "synthetic",
               "config": workload_config(args, world),
               "gpu_launches": launches, "parity_sample_ok": ok, "roofline": roof, "clocks": clk,
               "e2e": e2e, "cpu_baseline": cpu, "variants": results, "apps": apps_block}
        print(json.dumps(out), flush=True)
    ctx.close()


def main():
    args = parse()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    # test hooks (tests/test_gpu_bench_multirank.py): run N ranks on ONE GPU over
    # gloo (NCCL refuses two ranks on one device); never set by the driver
    if os.environ.get("VF_BENCH_DEVICE") is not None:
        local = int(os.environ["VF_BENCH_DEVICE"])
    if world > 1:
        import torch.distributed as dist
        backend = "gloo" if args.impl == "reference" else os.environ.get("VF_BENCH_BACKEND", "nccl")
        if args.impl != "reference":
            import torch
            torch.cuda.set_device(local)
        dist.init_process_group(backend)
    if args.impl == "reference":
        run_reference(args, rank, world)
    else:
        run_ours(args, rank, world, local)
    if world > 1:
        import torch.distributed as dist
        dist.destroy_process_group()


if __name__ == "__main__":
    main()

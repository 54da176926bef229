"""Per-app measurement of BASELINE.json configs 1, 3, 4 and 5 (the `apps` block of
bench.py's JSON line; also runnable alone: `python tools/apps_bench.py`).

BASELINE metric: "virtual calls/sec per app at 1/2/4/8 B200; speedup vs CUDA
vTable dispatch" (paper methodology: kernel time of the step loop, P:1433-1449;
per-app comparison, Fig. 6).

For every app, at its BASELINE size, every variant runs the SAME step loop:
  cuda         device-heap `new` per object + the compiler's virtual call
  cuda_packed  the same virtual call over objects placement-new'd into one
               index-ordered slab (SURVEY §7 "a fair CUDA baseline" sensitivity point)
  sharedoa     typed arenas + the compiler's virtual call (§4)
  coal         typed arenas + range-table type resolution + grouped direct call (§5)
  typeptr      typed arenas + tagged pointers + grouped direct call (§6)
Time = CUDA events on the launching stream around K steps after W warm-up
steps, barrier + synchronize on both sides, max over ranks. calls/s = virtual
calls issued by all ranks / that time. speedup_vs_cuda = t_cuda / t_variant on
the same config. Device-heap `new` costs ~2.4 s per 4M objects and slows as
the heap fills (measured on B200: 16.8M objects 36 s, 50M ~6 min): the heap
arm runs at the BASELINE size for every app except GEN (3 x 16.8M objects),
which adds a same-config comparison at 2048^2 where all five variants run.
Multi-GPU (world > 1): strong scaling of the same total problem (graph vertex
blocks, GEN row slabs, N-body / collision id blocks, STUT node row slabs, TRAF
ring blocks, ray strips); the heap arm is skipped there (allocation time).
"""
from __future__ import annotations

import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402

ALL_VARIANTS = ("cuda", "cuda_packed", "sharedoa", "coal", "typeptr")
ORDER = ("gol", "ray", "nbody", "gen", "traf", "stut", "collide", "graph")
SMS = 148


def peaks(root=ROOT):
    """MEASURED_PEAKS.json (driver-written), else the profiling guide's fallbacks."""
    try:
        pk = json.load(open(os.path.join(root, "MEASURED_PEAKS.json")))
        hbm, src = float(pk["hbm_gbs"]), "MEASURED_PEAKS.json hbm_gbs (copy)"
        mhz = float(pk.get("sm_max_mhz", 1965.0))
    except Exception:
        hbm, src, mhz = 6650.0, "B200_PROFILING.md fallback 6.65 TB/s (MEASURED_PEAKS.json absent)", 1965.0
    fp32 = SMS * 128 * 2 * mhz * 1e6 / 1e12  # TFLOP/s: 148 SMs x 128 FP32 lanes x FMA x max SM clock
    return {"hbm_gbs": hbm, "hbm_src": src, "fp32_tflops": fp32,
            "fp32_src": f"derived: {SMS} SM x 128 FP32 lanes x 2 FLOP x {mhz:.0f} MHz"}


class Env:
    """Rank / device / stream plumbing shared by the app runs."""

    def __init__(self, ctx, rank=0, world=1, group=None, device=0):
        self.ctx, self.rank, self.world, self.group = ctx, rank, world, group
        self.dev = torch.device(f"cuda:{device}")
        self.s = torch.cuda.Stream(device=self.dev)

    def barrier(self):
        if self.world > 1:
            import torch.distributed as dist
            dist.barrier(group=self.group)

    def _reduce(self, x, dtype, op):
        import torch.distributed as dist
        dev = "cpu" if dist.get_backend(self.group) == "gloo" else self.dev
        t = torch.tensor([x], dtype=dtype, device=dev)
        dist.all_reduce(t, op=op, group=self.group)
        return t.item()

    def max_ms(self, ms: float) -> float:
        if self.world == 1:
            return ms
        import torch.distributed as dist
        return float(self._reduce(ms, torch.float64, dist.ReduceOp.MAX))

    def sum_i(self, x: int) -> int:
        if self.world == 1:
            return int(x)
        import torch.distributed as dist
        return int(self._reduce(int(x), torch.int64, dist.ReduceOp.SUM))

    def timed(self, step, steps: int, warmup: int):
        """ms per step: CUDA events on the app stream around `steps` calls of
        step() after `warmup` calls; barrier + sync on both sides; max over ranks."""
        with torch.cuda.stream(self.s):
            for _ in range(warmup):
                step()
        torch.cuda.synchronize(self.dev)
        self.barrier()
        torch.cuda.synchronize(self.dev)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(self.s):
            e0.record(self.s)
            for _ in range(steps):
                step()
            e1.record(self.s)
        torch.cuda.synchronize(self.dev)
        self.barrier()
        return self.max_ms(e0.elapsed_time(e1)) / steps

    def free(self):
        torch.cuda.synchronize(self.dev)
        self.ctx.reset()
        torch.cuda.empty_cache()


def _roof(bound, per_call, calls_per_s, pk):
    if bound == "alu":
        ach = per_call * calls_per_s / 1e12
        return {"bound": "alu", "achieved": ach, "peak": pk["fp32_tflops"], "unit": "TFLOP/s",
                "frac": ach / pk["fp32_tflops"], "per_call": per_call, "peak_source": pk["fp32_src"]}
    ach = per_call * calls_per_s / 1e9
    return {"bound": bound, "achieved": ach, "peak": pk["hbm_gbs"], "unit": "GB/s", "frac": ach / pk["hbm_gbs"],
            "per_call": per_call, "peak_source": pk["hbm_src"]}


def _ncu(app_variant):
    """ncu DRAM bytes of the app's dominant kernel (profiles/ncu_apps_summary.json, committed)."""
    try:
        return json.load(open(os.path.join(ROOT, "profiles", "ncu_apps_summary.json")))["captures"].get(app_variant)
    except Exception:
        return None


def _traffic(row, key, variant, pk, launches_per_step=1):
    """Real-DRAM roofline of a one-kernel step: the captured launch's DRAM bytes
    (ncu, cold cache) x launches per step / the measured step time."""
    cap = _ncu(f"{key}_{variant}")
    ms = row["variants"].get(variant, {}).get("ms_per_step")
    if not cap or not ms:
        return
    b = cap["dram_bytes"] * launches_per_step
    row["roofline"]["traffic"] = b
    row["roofline"]["real_dram_gbs"] = b / (ms / 1e3) / 1e9
    row["roofline"]["real_frac"] = b / (ms / 1e3) / 1e9 / pk["hbm_gbs"]
    row["roofline"]["traffic_source"] = f"{cap['source']} ({cap['kernel'][:60]}), {variant}"


def _cpu(calls, sec, sample):
    import oracle  # bench.py's cpu_baseline leg (tests-only code, timed, never on the product path)
    return {"value": calls / sec, "unit": "calls/s", "cores": oracle.max_threads(), "kind": "oracle",
            "sample": sample}


def _finish(row, base_key="cuda"):
    v = row["variants"]
    b = v.get(base_key, {}).get("ms_per_step")
    if b:
        row["speedup_vs_cuda"] = {k: b / x["ms_per_step"] for k, x in v.items() if x.get("ms_per_step")}
    return row


def _variants(env, variants, heap_ok=True):
    return [v for v in variants if v != "cuda" or (heap_ok and env.world == 1)]


# ------------------------------------------------------------------ config 1: GOL
def app_gol(env, variants, pk, cpu=True, steps=5, warmup=2, small=False):
    from paper_conf_asplos_zhangar21_b200 import apps
    W = H = 64 if small else 256
    gens = 10 if small else 100
    g0 = synth.soup(W, H, seed=42)
    row = {"config": f"{W}x{H}, {gens} generations per step (one CUDA graph of {gens} fused generations), "
                     "dead border; 2.6 MB working set: L2-resident by construction (replicas only at N > 1)",
           "calls_per_step": W * H * gens * env.world, "variants": {}}
    states = {}
    for v in _variants(env, variants):
        g = apps.Gol(env.ctx, W, H, g0, v)
        torch.cuda.synchronize(env.dev)
        graph = torch.cuda.CUDAGraph()
        with torch.cuda.graph(graph, stream=env.s):
            for _ in range(gens):
                g.gen(stream=env.s)
        ms = env.timed(graph.replay, steps, warmup)
        states[v] = g.current.cpu().numpy()
        row["variants"][v] = {"ms_per_step": ms, "calls_per_s": row["calls_per_step"] / (ms / 1e3)}
        del graph, g
        env.free()
    ref = next(iter(states.values()))
    row["variants_agree"] = all(np.array_equal(ref, s) for s in states.values())
    best = max(row["variants"].values(), key=lambda x: x["calls_per_s"])["calls_per_s"]
    row["roofline"] = _roof("l2", 14, best, pk)
    row["roofline"]["note"] = "14 B/call algorithmic; the 2.6 MB state stays in L2, so HBM is not the bound"
    if cpu and env.rank == 0:
        import oracle
        _, _, _, sec = oracle.gol_run(W, H, g0, gens, threads=oracle.max_threads())
        row["cpu_baseline"] = _cpu(W * H * gens, sec, f"full config ({W}x{H}, {gens} generations)")
    return _finish(row)


# ------------------------------------------------------------------ config 3: ray tracer
def app_ray(env, variants, pk, cpu=True, steps=3, warmup=1, small=False):
    from paper_conf_asplos_zhangar21_b200.ray import Ray
    W, H, S = (192, 108, 500) if small else (1920, 1080, 10000)
    types, P = synth.ray_scene(S, seed=7)
    cam = synth.ray_camera(W, H)
    tcounts = np.bincount(types, minlength=4)
    flops = float((tcounts * np.array([2, 19, 12, 51])).sum() / S)  # formula FLOPs per hit()
    row = {"config": f"{W}x{H}, {S} shapes, 1 primary ray/pixel, 1 frame per step; 8-row strips round-robin "
                     f"over {env.world} GPU(s); scene L1/L2-resident (FP32-bound)",
           "calls_per_step": W * H * S, "variants": {}}
    frames = {}
    for v in _variants(env, variants):
        r = Ray(env.ctx, types, P, v)
        rgb = torch.zeros((H, W, 3), dtype=torch.float32, device=env.dev)
        hid = torch.full((H, W), -1, dtype=torch.int32, device=env.dev)
        ms = env.timed(lambda: r.render_frame(W, H, cam, env.rank, env.world, rgb, hid, env.s), steps, warmup)
        Ray.gather_image(rgb, hid, env.world, env.group)
        frames[v] = hid.cpu().numpy()
        row["variants"][v] = {"ms_per_step": ms, "calls_per_s": W * H * S / (ms / 1e3)}
        del r, rgb, hid
        env.free()
    ref = next(iter(frames.values()))
    row["variants_agree"] = all(np.array_equal(ref, f) for f in frames.values())
    best = max(row["variants"].values(), key=lambda x: x["calls_per_s"])["calls_per_s"]
    row["roofline"] = _roof("alu", flops, best, pk)
    if cpu and env.rank == 0:
        import oracle
        rows = 16
        _, _, calls, sec = oracle.ray_render(W, H, types, P, cam, synth.RAY_ALBEDO, row0=H // 2 - rows // 2,
                                             nrows=rows, threads=oracle.max_threads())
        row["cpu_baseline"] = _cpu(calls, sec, f"{rows} of {H} rows (centre band), full scene")
    return _finish(row)


# ------------------------------------------------------------------ config 5: N-body (all pairs)
def app_nbody(env, variants, pk, cpu=True, steps=10, warmup=3, small=False):
    from paper_conf_asplos_zhangar21_b200.nbody import Nbody
    N = 2048 if small else 65536
    s = synth.nbody_system(N, seed=10)
    row = {"config": f"all-pairs N-body, N={N} bodies, 1 step (one virtual update() per body); id blocks "
                     f"over {env.world} GPU(s) + all-gather of positions; 1 MB positions L2-resident (FP32-bound)",
           "calls_per_step": N, "variants": {}}
    pos = {}
    for v in _variants(env, variants):
        nb = Nbody(env.ctx, s, v, env.rank, env.world, env.group)
        ms = env.timed(lambda: nb.step(env.s), steps, warmup)
        pos[v] = nb.positions()
        row["variants"][v] = {"ms_per_step": ms, "calls_per_s": N / (ms / 1e3)}
        del nb
        env.free()
    ref = next(iter(pos.values()))
    row["variants_agree"] = all(np.array_equal(ref, p) for p in pos.values())
    best = max(row["variants"].values(), key=lambda x: x["calls_per_s"])["calls_per_s"]
    row["roofline"] = _roof("alu", 20.0 * (N - 1), best, pk)
    if cpu and env.rank == 0:
        import oracle
        Ns = 8192
        _, _, sec = oracle.nbody_run(synth.nbody_system(Ns, seed=10), 2, threads=oracle.max_threads())
        row["cpu_baseline"] = _cpu(Ns * 2 * (Ns / N), sec,
                                   f"N={Ns}, 2 steps, rate scaled by {Ns}/{N} (work per call ~ N)")
    return _finish(row)


# ------------------------------------------------------------------ config 5: GEN
def _gen_once(env, v, W, s0, steps, warmup):
    from paper_conf_asplos_zhangar21_b200 import apps
    g = apps.Gen(env.ctx, W, W, s0, v, rank=env.rank, world=env.world, group=env.group)
    ms = env.timed(lambda: g.gen(env.s), steps, warmup)
    st = g.current.cpu().numpy()[g.lo:g.hi].copy()
    del g
    env.free()
    return ms, st


GEN_HEAP_FULL = False  # --gen-heap-full: the device-heap arm also at 4096^2 (~6 min of device `new`)


def app_gen(env, variants, pk, cpu=True, steps=20, warmup=3, small=False):
    W = 256 if small else 4096
    s0 = synth.soup(W, W, seed=42)
    row = {"config": f"{W}x{W} Generations B2/S345/C4, 1 fused generation per step; row slabs over "
                     f"{env.world} GPU(s) + halo rows; 3 x 16.8M objects (> L2)",
           "calls_per_step": W * W, "variants": {}}
    states = {}
    for v in _variants(env, variants, heap_ok=GEN_HEAP_FULL or small):
        ms, states[v] = _gen_once(env, v, W, s0, steps, warmup)
        row["variants"][v] = {"ms_per_step": ms, "calls_per_s": W * W / (ms / 1e3)}
    ref = next(iter(states.values()))
    row["variants_agree"] = all(np.array_equal(ref, s) for s in states.values())
    base = row["variants"].get("cuda_packed", {}).get("ms_per_step")
    if base:
        row["speedup_vs_cuda_packed"] = {k: base / x["ms_per_step"] for k, x in row["variants"].items()}
    # same-config comparison with the device-heap arm (3 x 4.2M `new`s fit the bench budget)
    if "cuda" in variants and env.world == 1 and not GEN_HEAP_FULL:
        W2 = 128 if small else 2048
        s2 = synth.soup(W2, W2, seed=42)
        sub = {"config": f"{W2}x{W2} (all five variants incl. the device-heap CUDA arm; the heap arm at "
                         f"{W}x{W} needs ~6 min of device `new`)", "calls_per_step": W2 * W2, "variants": {}}
        for v in variants:
            ms, _ = _gen_once(env, v, W2, s2, steps, warmup)
            sub["variants"][v] = {"ms_per_step": ms, "calls_per_s": W2 * W2 / (ms / 1e3)}
        row["same_config_with_heap_cuda"] = _finish(sub)
    best = max(row["variants"].values(), key=lambda x: x["calls_per_s"])["calls_per_s"]
    row["roofline"] = _roof("hbm", 14, best, pk)
    if not small and env.world == 1:
        _traffic(row, "gen", "typeptr", pk)  # the fused step is ONE launch per generation
    if cpu and env.rank == 0:
        import oracle
        _, _, _, sec = oracle.gen_run(W, W, s0, 2, threads=oracle.max_threads())
        row["cpu_baseline"] = _cpu(W * W * 2, sec, f"full grid, 2 generations")
    return _finish(row)


# ------------------------------------------------------------------ config 5: TRAF
def app_traf(env, variants, pk, cpu=True, steps=20, warmup=3, small=False):
    from paper_conf_asplos_zhangar21_b200.traf import Traf
    R, L = (37, 512) if small else (3277, 4096)
    w = synth.traf_world(R, L, seed=11)
    nveh = len(w["veh_ring"])
    row = {"config": f"{R} rings x {L} cells, {nveh} vehicles ({R * L + nveh} objects), 1 step = update() per "
                     f"cell + step() per vehicle; ring blocks over {env.world} GPU(s), no exchange",
           "calls_per_step": R * L + nveh, "variants": {}}
    res = {}
    for v in _variants(env, variants):
        t = Traf(env.ctx, w, v, env.rank, env.world)
        ms = env.timed(lambda: t.step(env.s), steps, warmup)
        res[v] = t.state()[0].copy()
        row["variants"][v] = {"ms_per_step": ms, "calls_per_s": row["calls_per_step"] / (ms / 1e3)}
        del t
        env.free()
    ref = next(iter(res.values()))
    row["variants_agree"] = all(np.array_equal(ref, r) for r in res.values())
    best = max(row["variants"].values(), key=lambda x: x["calls_per_s"])["calls_per_s"]
    row["roofline"] = _roof("hbm", (26 * R * L + 38 * nveh) / (R * L + nveh), best, pk)
    if cpu and env.rank == 0:
        import oracle
        _, _, sec = oracle.traf_run(w, 5, threads=oracle.max_threads())
        row["cpu_baseline"] = _cpu((R * L + nveh) * 5, sec, "full world, 5 steps")
    return _finish(row)


# ------------------------------------------------------------------ config 5: STUT
def app_stut(env, variants, pk, cpu=True, steps=20, warmup=3, small=False):
    from paper_conf_asplos_zhangar21_b200.stut import Stut
    W = H = 128 if small else 2048
    w = synth.stut_lattice(W, H, seed=12, v_pull=4.0)
    n, S = W * H, len(w["a"])
    row = {"config": f"{W}x{H} nodes + {S} springs ({n + S} objects), 1 step = force() per spring + move() per "
                     f"node; node row slabs over {env.world} GPU(s) + all-gather of positions",
           "calls_per_step": n + S, "variants": {}}
    res = {}
    for v in _variants(env, variants):
        st = Stut(env.ctx, w, v, env.rank, env.world, env.group)
        ms = env.timed(lambda: st.step(env.s), steps, warmup)
        res[v] = st.positions()
        row["variants"][v] = {"ms_per_step": ms, "calls_per_s": (n + S) / (ms / 1e3)}
        del st
        env.free()
    ref = next(iter(res.values()))
    row["variants_agree"] = all(np.array_equal(ref, r) for r in res.values())
    best = max(row["variants"].values(), key=lambda x: x["calls_per_s"])["calls_per_s"]
    row["roofline"] = _roof("hbm", (64 * S + 140 * n) / (S + n), best, pk)
    if cpu and env.rank == 0:
        import oracle
        _, _, _, sec = oracle.stut_run(w, 2, threads=oracle.max_threads())
        row["cpu_baseline"] = _cpu((n + S) * 2, sec, "full structure, 2 steps")
    return _finish(row)


# ------------------------------------------------------------------ config 5: collision
def app_collide(env, variants, pk, cpu=True, steps=5, warmup=2, small=False):
    from paper_conf_asplos_zhangar21_b200.collide import Collide
    N = (1 << 16) if small else (1 << 24)
    s = synth.collide_system(N, seed=13)
    row = {"config": f"N={N} bodies, cutoff grid G={s['G']}, merging; 1 step = grid + update() + merge() per "
                     f"active body; id blocks over {env.world} GPU(s) + all-gathers", "variants": {}}
    res = {}
    for v in _variants(env, variants):
        c = Collide(env.ctx, s, v, env.rank, env.world, env.group)
        for _ in range(warmup):
            c.step(env.s)
        torch.cuda.synchronize(env.dev)
        a0 = c.calls()
        ms = env.timed(lambda: c.step(env.s), steps, 0)
        calls = env.sum_i(c.calls() - a0) / steps
        res[v] = c.positions()
        row["variants"][v] = {"ms_per_step": ms, "calls_per_s": calls / (ms / 1e3), "calls_per_step": calls}
        del c
        env.free()
    ref = next(iter(res.values()))
    row["variants_agree"] = all(np.array_equal(ref, r) for r in res.values())
    row["calls_per_step"] = next(iter(row["variants"].values()))["calls_per_step"]
    best = max(row["variants"].values(), key=lambda x: x["calls_per_s"])["calls_per_s"]
    row["roofline"] = _roof("hbm", (80 + 68) / 2, best, pk)
    if cpu and env.rank == 0:
        import oracle
        _, _, ocalls, sec = oracle.collide_run(s, 1, threads=oracle.max_threads())
        row["cpu_baseline"] = _cpu(ocalls, sec, f"full system (N={N}), 1 step")
    return _finish(row)


# ------------------------------------------------------------------ config 4: graph
def app_graph(env, variants, pk, cpu=True, scale=24, small=False):
    from paper_conf_asplos_zhangar21_b200.graph import Graph
    scale = 14 if small else scale
    t0 = time.time()
    offs, col = synth.rmat_graph(scale, seed=1)
    gen_s = time.time() - t0
    V, A = len(offs) - 1, len(col)
    src = int(np.argmax(np.diff(offs.astype(np.int64))))
    avg = A / V
    bfs_mode = "hybrid" if env.world == 1 else "bits"
    row = {"config": f"RMAT-{scale} (V={V}, {A} arcs, 4 degree-bucket vertex types), vertex blocks over "
                     f"{env.world} GPU(s); BFS ({bfs_mode}) from the max-degree vertex, CC to convergence, "
                     f"PageRank iteration; input generation {gen_s:.1f} s (host, untimed)",
           "variants": {}}
    sub = {"bfs": {}, "cc": {}, "pr": {}}
    outs = {}
    for v in _variants(env, variants):
        g = Graph(env.ctx, offs, col, v, env.rank, env.world, env.group)
        ms_b = env.timed(lambda: g.bfs(src, mode=bfs_mode), 2, 1)
        calls_b = env.sum_i(g.calls)
        d = g.by_id(g.depth).cpu().numpy()
        ms_c = env.timed(lambda: g.cc(), 1, 1)
        calls_c = env.sum_i(g.calls)
        lab = g.by_id(g.lab[0]).cpu().numpy()
        g.pr_init()
        ms_p = env.timed(lambda: g.pr_iteration(), 10, 2)
        calls_p = env.sum_i(2 * g.E)
        outs[v] = (d, lab)
        sub["bfs"][v] = {"ms_per_step": ms_b, "calls_per_s": calls_b / (ms_b / 1e3), "calls_per_step": calls_b}
        sub["cc"][v] = {"ms_per_step": ms_c, "calls_per_s": calls_c / (ms_c / 1e3), "calls_per_step": calls_c}
        sub["pr"][v] = {"ms_per_step": ms_p, "calls_per_s": calls_p / (ms_p / 1e3), "calls_per_step": calls_p}
        # whole step = one BFS + one CC + one PageRank iteration
        ms = ms_b + ms_c + ms_p
        row["variants"][v] = {"ms_per_step": ms, "calls_per_s": (calls_b + calls_c + calls_p) / (ms / 1e3)}
        del g
        env.free()
    ref = next(iter(outs.values()))
    row["variants_agree"] = all(np.array_equal(ref[0], o[0]) and np.array_equal(ref[1], o[1]) for o in outs.values())
    for k in sub:
        row[k] = _finish({"variants": sub[k]})
    # PageRank per iteration: per vertex 20 B (+20 B for its contribution), per arc 8 B
    best_pr = max(sub["pr"].values(), key=lambda x: x["calls_per_s"])
    row["roofline"] = _roof("hbm", (40 + 8 * avg) / 2, best_pr["calls_per_s"], pk)
    row["roofline"]["kernel"] = "PageRank iteration (pr_contrib + pr_update)"
    if cpu and env.rank == 0:
        import oracle
        types = synth.vertex_types(offs)
        _, psec = oracle.graph_pr(offs, col, types, iters=2, threads=oracle.max_threads())
        row["cpu_baseline"] = _cpu(2 * V * 2, psec, f"full graph, PageRank 2 iterations (2 calls/vertex/iteration)")
    return _finish(row)


def run_apps(env, names=ORDER, variants=ALL_VARIANTS, cpu=True, clocks_cls=None, log=None, small=False):
    pk = peaks()
    out = {}
    for name in names:
        t0 = time.time()
        clk = clocks_cls(env.dev.index) if clocks_cls else None
        if clk:
            clk.start()
            time.sleep(0.3)
        row = globals()[f"app_{name}"](env, variants, pk, cpu=cpu, small=small)
        if small:
            row["scale"] = "small (code-path test sizes, not a BASELINE config)"
        if clk:
            row["clocks"] = clk.stop()
        row["wall_s"] = time.time() - t0
        out[name] = row
        if log:
            log(name, row)
    return out


if __name__ == "__main__":
    import argparse
    ap = argparse.ArgumentParser()
    ap.add_argument("--apps", default=",".join(ORDER))
    ap.add_argument("--variants", default=",".join(ALL_VARIANTS))
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--out", default=None)
    ap.add_argument("--small", action="store_true", help="code-path test sizes")
    ap.add_argument("--gen-heap-full", action="store_true",
                    help="GEN: the device-heap CUDA arm at 4096^2 too (3 x 16.8M device `new`s, ~6 min)")
    a = ap.parse_args()
    globals()["GEN_HEAP_FULL"] = a.gen_heap_full
    from paper_conf_asplos_zhangar21_b200 import vf
    ctx = vf.Ctx(0, cuda_heap_bytes=16 << 30)
    env = Env(ctx)
    from bench import Clocks  # the same nvidia-smi sampler as the contract line
    res = run_apps(env, a.apps.split(","), tuple(a.variants.split(",")), cpu=not a.no_cpu, clocks_cls=Clocks,
                   log=lambda n, r: print(json.dumps({n: r}), flush=True), small=a.small)
    if a.out:
        json.dump(res, open(a.out, "w"), indent=1)
    ctx.close()

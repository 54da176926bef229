#!/usr/bin/env python
"""Round-1 per-app table (kept for GraphChi-vEN, §8f f4, and the GOL persistent forms);
the BASELINE configs' per-app numbers now come from tools/apps_bench.py (bench.py's
`apps` block).

For each app, each dispatch variant: virtual calls/s over the timed steps
(CUDA events on the launching stream, after warm-up), plus the algorithmic
bytes (or FLOPs) per call and the fraction of the measured roof, and the CPU
oracle timed on this host's cores on the same (or a stated sampled) input.
Writes one JSON line per (app, variant) to <out>.jsonl and a table to <out>.md.

  python tools/bench_apps.py --out profiles/apps_r1 [--apps gol,gen,graph,ray,traf] [--quick]
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402  (cpu_baseline leg only)
import synth  # noqa: E402
from paper_conf_asplos_zhangar21_b200 import apps, vf  # noqa: E402
from paper_conf_asplos_zhangar21_b200.graph import Graph  # noqa: E402
from paper_conf_asplos_zhangar21_b200.graph_en import GraphEN  # noqa: E402
from paper_conf_asplos_zhangar21_b200.ray import Ray  # noqa: E402
from paper_conf_asplos_zhangar21_b200.traf import Traf  # noqa: E402
from paper_conf_asplos_zhangar21_b200.nbody import Nbody  # noqa: E402
from paper_conf_asplos_zhangar21_b200.stut import Stut  # noqa: E402
from paper_conf_asplos_zhangar21_b200.collide import Collide  # noqa: E402

VARIANTS = ("cuda", "sharedoa", "coal", "typeptr")
PEAKS = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))) if os.path.exists(
    os.path.join(ROOT, "MEASURED_PEAKS.json")) else {}
HBM = PEAKS.get("hbm_gbs", 6650.0)  # else the B200_PROFILING.md fallback (6.65 TB/s)
SMS = 148
FP32_PEAK = SMS * 128 * 2 * PEAKS.get("sm_max_mhz", 1965.0) * 1e6 / 1e12  # TFLOP/s, derived
ROWS = []


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


def record(app, config, variant, calls_per_step, ms, unit_per_call, unit, bound, extra=None, cpu=None):
    achieved = unit_per_call * calls_per_step / (ms / 1e3) / (1e9 if unit == "GB/s" else 1e12)
    peak = HBM if unit == "GB/s" else FP32_PEAK
    row = dict(app=app, config=config, variant=variant, calls_per_step=calls_per_step, ms_per_step=ms,
               calls_per_s=calls_per_step / (ms / 1e3), roofline=dict(bound=bound, achieved=achieved, peak=peak,
                                                                       unit=unit, frac=achieved / peak,
                                                                       per_call=unit_per_call),
               **(extra or {}))
    if cpu:
        row["cpu_baseline"] = cpu
    ROWS.append(row)
    print(json.dumps(row), flush=True)
    return row


def cpu_info(calls, sec, sample):
    return dict(value=calls / sec, unit="calls/s", cores=oracle.max_threads(), kind="oracle", sample=sample)


# ---------------------------------------------------------------- config 1: GOL
def bench_gol(ctx, quick):
    W = H = 256
    gens = 100
    g0 = synth.soup(W, H, seed=42)
    _, _, _, sec = oracle.gol_run(W, H, g0, gens, threads=oracle.max_threads())
    cpu = cpu_info(W * H * gens, sec, "full config (256x256, 100 generations)")
    for v in VARIANTS:
        g = apps.Gol(ctx, W, H, g0, v)
        s = torch.cuda.Stream()
        torch.cuda.synchronize()
        graph = torch.cuda.CUDAGraph()
        with torch.cuda.graph(graph, stream=s):
            for _ in range(gens):
                g.gen(stream=s)
        ms = ev_time(graph.replay, 5) / gens
        ms_eager = ev_time(g.gen, 50)
        ms_unfused = ev_time(lambda: g.gen(fused=False), 50)
        # 8 B ptr + 1 B nbr + 1 B state out + 4 B counter r/w per next() call
        record("gol", "256x256, 100 gens (CUDA graph of 100 generations)", v, W * H, ms, 14, "GB/s", "l2/latency",
               dict(ms_per_gen_eager=ms_eager, ms_per_gen_eager_unfused=ms_unfused), cpu)
        del graph
        vf.set_tuning("cluster", 1)
        ms_run = ev_time(lambda: g.run(gens), 5) / gens
        vf.set_tuning("cluster", 0)
        record("gol-cluster", "256x256, 100 gens in ONE thread-block cluster launch (vf_gol_run, DSMEM state)", v,
               W * H, ms_run, 14, "GB/s", "l2/latency", None, cpu)
        ms_run = ev_time(lambda: g.run(gens), 5) / gens
        record("gol-coop", "256x256, 100 gens in one cooperative grid-barrier launch (vf_gol_run, cluster=0)", v,
               W * H, ms_run, 14, "GB/s", "l2/latency", None, cpu)
        del g
    ctx.reset()


# ---------------------------------------------------------------- config 5: GEN
def bench_gen(ctx, quick):
    # every variant at the same size (the device-heap arm's 3 x 16.8M `new`s at
    # 4096^2 take ~6 min): the per-app speedups compare one config
    W = H = 1024 if quick else 2048
    gens = 20
    s0 = synth.soup(W, H, seed=42)
    _, _, _, sec = oracle.gen_run(W, H, s0, gens, threads=oracle.max_threads())
    cpu = cpu_info(W * H * gens, sec, f"{W}x{H}, {gens} generations (same input)")
    for v in VARIANTS:
        Wv, sv = W, s0
        g = apps.Gen(ctx, Wv, Wv, sv, v)
        ms = ev_time(g.gen, gens)
        g2 = apps.Gen(ctx, Wv, Wv, sv, v)
        ms_unfused = ev_time(lambda: g2.gen(fused=False), gens)
        # fused step per cell: 8 B ptr + 16 B object r/w + ~1 B state read (9 neighbours from L1/L2) + 1 B write
        record("gen", f"{Wv}x{Wv} B2/S345/C4 (fused step)", v, Wv * Wv, ms, 14, "GB/s", "hbm",
               dict(ms_unfused=ms_unfused), cpu)
        del g2
        del g
        ctx.reset()


# ---------------------------------------------------------------- config 4: graph
def bench_graph(ctx, quick):
    scale = 20 if quick else 24
    t0 = time.time()
    offs, col = synth.rmat_graph(scale, seed=1)
    print(f"# rmat-{scale}: V={len(offs) - 1} arcs={len(col)} gen {time.time() - t0:.1f}s", flush=True)
    types = synth.vertex_types(offs)
    src = int(np.argmax(np.diff(offs.astype(np.int64))))
    V, arcs = len(offs) - 1, len(col)
    thr = oracle.max_threads()
    _, _, bcalls, bsec = oracle.graph_bfs(offs, col, types, src)
    _, _, ccalls, csec = oracle.graph_cc(offs, col, types, threads=thr)
    _, psec = oracle.graph_pr(offs, col, types, iters=5, threads=thr)
    cpu = dict(bfs=cpu_info(bcalls, bsec, "full graph, 1 thread (sequential BFS)"),
               cc=cpu_info(ccalls, csec, "full graph"),
               pr=cpu_info(2 * V * 5, psec, "full graph, 5 iterations (2 virtual calls/vertex/iteration)"))
    avg_deg = arcs / V
    for v in VARIANTS:
        g = Graph(ctx, offs, col, v)
        ms = ev_time(lambda: g.bfs(src), 3, warm=1)
        calls = g.calls
        # per reached vertex: 8 B ptr + 8 B offs + per arc 4 B col + 4 B depth
        record("graph-bfs", f"rmat-{scale} top-down BFS from max-degree vertex", v, calls, ms,
               16 + 8 * avg_deg, "GB/s", "hbm", dict(V=V, arcs=arcs), cpu["bfs"])
        ms = ev_time(lambda: g.bfs(src, mode="hybrid"), 3, warm=1)
        # bottom-up levels dispatch every entry (visited ones return after the 8 B ptr + 16 B object read)
        record("graph-bfs-hybrid", f"rmat-{scale} direction-optimizing BFS (top-down, then bottom-up probes)", v,
               g.calls, ms, 16 + 8 * avg_deg * bcalls / max(g.calls, 1), "GB/s", "hbm", dict(V=V, arcs=arcs),
               cpu["bfs"])
        ms = ev_time(lambda: g.cc(), 2, warm=1)
        record("graph-cc", f"rmat-{scale} Jacobi CC to convergence", v, g.calls, ms, 20 + 8 * avg_deg, "GB/s",
               "hbm", dict(iters=g.calls // V), cpu["cc"])
        g.pr_init()
        ms = ev_time(lambda: g.pr_iteration(), 10, warm=2)
        # per vertex per iteration: contrib (8 ptr + 4 r + 8 c) and update (8 ptr + 8 offs + 4 out) + 8 B/arc
        record("graph-pr", f"rmat-{scale} PageRank iteration", v, 2 * V, ms, (40 + 8 * avg_deg) / 2, "GB/s",
               "hbm", None, cpu["pr"])
        del g
        ctx.reset()


# ---------------------------------------------------------------- §8f f4: GraphChi-vEN
def _graph_en_scale(ctx, scale, variants, tag):
    t0 = time.time()
    offs, col = synth.rmat_graph(scale, seed=1)
    V, A = len(offs) - 1, len(col)
    print(f"# vEN rmat-{scale}: V={V} arcs={A} gen {time.time() - t0:.1f}s", flush=True)
    types = synth.vertex_types(offs)
    src = int(np.argmax(np.diff(offs.astype(np.int64))))
    deg = np.diff(offs.astype(np.int64))
    cpu = None
    if scale <= 20:
        _, _, bvc, bec, bsec = oracle.graph_en_bfs(offs, col, types, src)
        _, it, cvc, cec, csec = oracle.graph_en_cc(offs, col, types)
        _, psec = oracle.graph_en_pr(offs, col, types, iters=5)
        cpu = dict(bfs=cpu_info(bvc + bec, bsec, f"rmat-{scale}, 1 thread"),
                   cc=cpu_info(cvc + cec, csec, f"rmat-{scale}, 1 thread"),
                   pr=cpu_info(5 * (V + 2 * A), psec, f"rmat-{scale}, 5 iterations, 1 thread"))
    for v in variants:
        g = GraphEN(ctx, offs, col, v)
        ms = ev_time(lambda: g.bfs(src), 3, warm=1)
        ec = g.edge_calls_bfs()
        calls = g.vcalls + ec
        # frontier entry: 8 ptr + 16 vertex + 8 offs; out-edge: 8 ptr + 4 dst + 4 depth
        byts = 32 * g.vcalls + 16 * ec
        record("graph-en-bfs", f"{tag} rmat-{scale} vEN top-down BFS", v, calls, ms, byts / calls, "GB/s", "hbm",
               dict(V=V, arcs=A, vertex_calls=g.vcalls, edge_calls=ec), cpu and cpu["bfs"])
        g.cc_init()
        ms = ev_time(lambda: (g.changed.zero_(), g.cc_iteration()), 5, warm=2)
        # vertex 8 ptr + 16 obj + 8 offs + 4 in + 4 out; in-edge get 8 ptr + 4; pull 8 ptr + 4 src + 4 lab + 4
        calls = g.E + 2 * A
        byts = 40 * g.E + 12 * A + 20 * A
        record("graph-en-cc", f"{tag} rmat-{scale} vEN CC iteration", v, calls, ms, byts / calls, "GB/s", "hbm",
               dict(vertex_calls=g.E, edge_calls=2 * A), cpu and cpu["cc"])
        g.pr_init()
        ms = ev_time(lambda: g.pr_iteration(), 5, warm=2)
        # vertex 8 ptr + 16 obj + 8 offs + 4 rank + 8 contrib; in-edge get 8 ptr + 8; pull 8 ptr + 4 src + 8 + 8
        byts = 44 * g.E + 16 * A + 28 * A
        record("graph-en-pr", f"{tag} rmat-{scale} vEN PageRank iteration", v, calls, ms, byts / calls, "GB/s",
               "hbm", dict(vertex_calls=g.E, edge_calls=2 * A), cpu and cpu["pr"])
        del g
        ctx.reset()
        torch.cuda.empty_cache()


EN_FULL = True


def bench_graph_en(ctx, quick):
    # the device-heap CUDA baseline allocates one `new` per edge (~3 us each): all
    # four variants at rmat-18; the typed variants also at the config-4 scale
    _graph_en_scale(ctx, 16 if quick else 18, VARIANTS, "all-variants")
    if EN_FULL:
        _graph_en_scale(ctx, 20 if quick else 24, ("sharedoa", "coal", "typeptr"), "full")


# ---------------------------------------------------------------- config 3: ray
def bench_ray(ctx, quick):
    W, H, S = (480, 270, 10000) if quick else (1920, 1080, 10000)
    types, P = synth.ray_scene(S, seed=7)
    cam = synth.ray_camera(W, H)
    rows = 16 if not quick else 8
    _, _, calls, sec = oracle.ray_render(W, H, types, P, cam, synth.RAY_ALBEDO, row0=H // 2 - rows // 2,
                                         nrows=rows, threads=oracle.max_threads())
    cpu = cpu_info(calls, sec, f"{rows} of {H} rows (centre band), full scene")
    tcounts = np.bincount(types, minlength=4)
    # formula FLOPs per hit() (fma = 2): plane 2, sphere 19, rect 12, triangle 51
    flops = float((tcounts * np.array([2, 19, 12, 51])).sum() / S)
    for v in VARIANTS:
        r = Ray(ctx, types, P, v)
        rgb = torch.empty((H, W, 3), dtype=torch.float32, device="cuda")
        hid = torch.empty((H, W), dtype=torch.int32, device="cuda")
        ms = ev_time(lambda: r.render(W, H, cam, rgb=rgb, hid=hid), 3, warm=1)
        record("ray", f"{W}x{H}, {S} shapes, 1 primary ray/pixel", v, W * H * S, ms, flops, "TFLOP/s", "alu",
               None, cpu)
        del r
        ctx.reset()


# ---------------------------------------------------------------- config 5: TRAF
def bench_traf(ctx, quick):
    R, L = (400, 4096) if quick else (3277, 4096)
    w = synth.traf_world(R, L, seed=11)
    steps = 20
    _, _, sec = oracle.traf_run(w, steps, threads=oracle.max_threads())
    nveh = len(w["veh_ring"])
    cpu = cpu_info((R * L + nveh) * steps, sec, f"full world, {steps} steps")
    for v in VARIANTS:
        t = Traf(ctx, w, v)
        ms = ev_time(t.step, steps)
        # cells: 8 ptr + 16 obj + 2 B writes; vehicles: 8 ptr + 24 obj r/w + ~6 B occupancy
        per_call = (26 * R * L + 38 * nveh) / (R * L + nveh)
        record("traf", f"{R} rings x {L} cells, {nveh} vehicles", v, t.calls_per_step, ms, per_call, "GB/s", "hbm",
               dict(objects=R * L + nveh), cpu)
        del t
        ctx.reset()


# ---------------------------------------------------------------- config 5: N-body (all pairs)
def bench_nbody(ctx, quick):
    N = 16384 if quick else 65536
    steps = 10
    s = synth.nbody_system(N, seed=10)
    Ns = 8192
    _, _, sec = oracle.nbody_run(synth.nbody_system(Ns, seed=10), 2, threads=oracle.max_threads())
    # work per update() call grows with N: scale the sampled rate by Ns/N
    cpu = cpu_info(Ns * 2 * (Ns / N), sec, f"N={Ns}, 2 steps, rate scaled by {Ns}/{N} (work per call ~ N)")
    flops = 20.0 * (N - 1)  # per update(): N-1 pair interactions x 20 formula FLOPs
    for v in VARIANTS:
        nb = Nbody(ctx, s, v)
        ms = ev_time(nb.step, steps)
        record("nbody", f"all-pairs N={N}", v, N, ms, flops, "TFLOP/s", "alu", None, cpu)
        del nb
        ctx.reset()


# ---------------------------------------------------------------- config 5: STUT
def bench_stut(ctx, quick):
    W = H = 512 if quick else 2048
    steps = 20
    w = synth.stut_lattice(W, H, seed=12, v_pull=4.0)
    _, _, _, sec = oracle.stut_run(w, 5, threads=oracle.max_threads())
    n, S = W * H, len(w["a"])
    cpu = cpu_info((n + S) * 5, sec, f"full structure, 5 steps")
    # spring: 8 ptr + 32 obj + 16 pos + 8 F; node: 8 ptr + 24 obj r + 12 w + 8 offs + 24 inc + 48 F + 16 pos
    per_call = (64 * S + 140 * n) / (S + n)
    for v in VARIANTS:
        st = Stut(ctx, w, v)
        ms = ev_time(st.step, steps)
        record("stut", f"{W}x{H} nodes, {S} springs", v, st.calls_per_step, ms, per_call, "GB/s", "hbm",
               dict(objects=n + S), cpu)
        del st
        ctx.reset()


# ---------------------------------------------------------------- config 5: collision (cutoff grid + merging)
def bench_collide(ctx, quick):
    N = (1 << 20) if quick else (1 << 24)
    steps = 10
    s = synth.collide_system(N, seed=13)
    _, _, ocalls, sec = oracle.collide_run(s, 1, threads=oracle.max_threads())
    cpu = cpu_info(ocalls, sec, f"full system (N={N}), 1 step")
    # update: 8 ptr + 24 obj r + 12 obj w + 16 own P + 16 Pm w + 4 near w = 80 B; merge: 8 ptr + 24 obj r
    # + 4 near + 16 Pm + 16 P w = 68 B; neighbour positions are L1/L2-resident
    per_call = (80 + 68) / 2
    for v in VARIANTS:
        c = Collide(ctx, s, v)
        for _ in range(2):
            c.step()
        torch.cuda.synchronize()
        a0 = c.calls()
        ms = ev_time(c.step, steps, warm=0)
        calls = (c.calls() - a0) / steps
        record("collide", f"N={N} bodies, cutoff grid G={s['G']}, merging", v, int(calls), ms, per_call, "GB/s",
               "hbm", dict(objects=N), cpu)
        del c
        ctx.reset()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--apps", default="gol,ray,traf,gen,stut,nbody,collide,graph")
    ap.add_argument("--out", default="gpurun_out/apps")
    ap.add_argument("--quick", action="store_true")
    ap.add_argument("--tune", action="append", default=[], help="libvf tuning knob key=value (vf_set_tuning)")
    ap.add_argument("--en-small-only", action="store_true", help="graph_en: rmat-18 (all variants) only")
    a = ap.parse_args()
    global EN_FULL
    EN_FULL = not a.en_small_only
    for kv in a.tune:
        k, v = kv.split("=")
        vf.set_tuning(k, int(v))
    ctx = vf.Ctx(0, cuda_heap_bytes=16 << 30)
    for name in a.apps.split(","):
        globals()[f"bench_{name}"](ctx, a.quick)
    os.makedirs(os.path.dirname(a.out) or ".", exist_ok=True)
    with open(a.out + ".jsonl", "w") as f:
        for r in ROWS:
            f.write(json.dumps(r) + "\n")
    with open(a.out + ".md", "w") as f:
        f.write("| app | config | variant | calls/step | ms/step | Gcalls/s | vs cuda | achieved | frac | "
                "oracle Gcalls/s (cores) |\n|---|---|---|---|---|---|---|---|---|---|\n")
        for r in ROWS:
            base = next((x for x in ROWS if x["app"] == r["app"] and x["config"] == r["config"]
                         and x["variant"] == "cuda"), None)
            rel = r["calls_per_s"] / base["calls_per_s"] if base else float("nan")
            rf = r["roofline"]
            cpu = r.get("cpu_baseline")
            f.write(f"| {r['app']} | {r['config']} | {r['variant']} | {r['calls_per_step']} | {r['ms_per_step']:.3f} | "
                    f"{r['calls_per_s'] / 1e9:.4g} | {rel:.2f} | {rf['achieved']:.1f} {rf['unit']} | {rf['frac']:.3f} | "
                    f"{(cpu['value'] / 1e9) if cpu else float('nan'):.3f} ({cpu['cores'] if cpu else '-'}) |\n")
    print("wrote", a.out)


if __name__ == "__main__":
    main()

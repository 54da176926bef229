"""CPU ORACLE for "Judging a Type by Its Pointer" (ASPLOS'21) — TEST INFRASTRUCTURE.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` leg may import this package. The product path
(``paper_conf_asplos_zhangar21_b200``) never imports it, and it imports
nothing from the product path: the two share only the seeded input generators
in ``synth/``.

The arithmetic lives in plain C++ (``oracle/*.cpp``, ordinary ``virtual``
methods, objects from plain ``new`` in index order), compiled to
``liboracle.so`` with ``g++ -O2 -ffp-contract=off -fopenmp``. This module is
argument marshalling only. Every function cites its passage in ``oracle.h``.

Pinned (tests/test_oracle_*.py, ``-m "not gpu"``) by: closed forms (micro
val_i = init_i + R(t_i+1), region count ceil(log2(n/4096+1))), brute force
(linear scan vs. Algorithm-1 tree on every edge address), round-trip
invariants (TypePointer), Fig. 3's structural example, and an independent
textbook Game-of-Life plus still-life/oscillator/glider invariants.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
SO = os.path.join(HERE, "liboracle.so")
SOURCES = ["alloc.cpp", "micro.cpp", "gol.cpp", "gen.cpp", "graph.cpp", "graph_en.cpp", "ray.cpp", "traf.cpp", "nbody.cpp", "stut.cpp", "collide.cpp"]
NOT_FOUND = 0xFFFFFFFF


def build(force: bool = False) -> str:
    srcs = [os.path.join(HERE, s) for s in SOURCES]
    hdr = os.path.join(HERE, "oracle.h")
    if not force and os.path.exists(SO):
        newest = max(os.path.getmtime(p) for p in srcs + [hdr, __file__])
        if os.path.getmtime(SO) >= newest:
            return SO
    cmd = ["g++", "-O2", "-std=c++17", "-ffp-contract=off", "-fopenmp", "-fPIC", "-shared",
           "-o", SO] + srcs
    subprocess.run(cmd, check=True)
    return SO


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(SO)
        u64p = ctypes.POINTER(ctypes.c_uint64)
        u32p = ctypes.POINTER(ctypes.c_uint32)
        L.oracle_region_plan.restype = ctypes.c_uint32
        L.oracle_region_plan.argtypes = [ctypes.c_uint64, ctypes.c_uint64, u64p, ctypes.c_uint32]
        L.oracle_build_table.restype = ctypes.c_uint32
        L.oracle_build_table.argtypes = [u64p, u64p, u32p, ctypes.c_uint32, u64p, u64p, u32p]
        L.oracle_coal_lookup.restype = None
        L.oracle_coal_lookup.argtypes = [u64p, u64p, u32p, ctypes.c_uint32, u64p, ctypes.c_uint64, u32p]
        L.oracle_tp_tag.restype = ctypes.c_uint64
        L.oracle_tp_tag.argtypes = [ctypes.c_uint64, ctypes.c_uint32]
        L.oracle_tp_type.restype = ctypes.c_uint32
        L.oracle_tp_type.argtypes = [ctypes.c_uint64]
        L.oracle_tp_strip.restype = ctypes.c_uint64
        L.oracle_tp_strip.argtypes = [ctypes.c_uint64]
        L.oracle_tp_vfunc.restype = ctypes.c_uint64
        L.oracle_tp_vfunc.argtypes = [ctypes.c_uint64, u64p, ctypes.c_uint32, ctypes.c_uint32]
        L.oracle_micro_run.restype = ctypes.c_int
        L.oracle_micro_run.argtypes = [ctypes.c_uint64, ctypes.c_uint32, ctypes.c_void_p, ctypes.c_void_p,
                                       ctypes.c_uint32, ctypes.c_int, ctypes.c_void_p,
                                       ctypes.POINTER(ctypes.c_double)]
        L.oracle_gol_run.restype = ctypes.c_int
        L.oracle_gol_run.argtypes = [ctypes.c_uint32, ctypes.c_uint32, ctypes.c_void_p, ctypes.c_uint32,
                                     ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p,
                                     ctypes.c_void_p, ctypes.POINTER(ctypes.c_double)]
        L.oracle_gen_run.restype = ctypes.c_int
        L.oracle_gen_run.argtypes = [ctypes.c_uint32, ctypes.c_uint32, ctypes.c_void_p, ctypes.c_uint32,
                                     ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint32, ctypes.c_int,
                                     ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
                                     ctypes.POINTER(ctypes.c_double)]
        P, U32, U64 = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64
        L.oracle_graph_bfs.restype = ctypes.c_int
        L.oracle_graph_bfs.argtypes = [U64, P, P, P, U32, P, P, P, ctypes.POINTER(ctypes.c_double)]
        L.oracle_graph_cc.restype = ctypes.c_int
        L.oracle_graph_cc.argtypes = [U64, P, P, P, ctypes.c_int, P, P, P, ctypes.POINTER(ctypes.c_double)]
        L.oracle_graph_en_edge_types.restype = ctypes.c_int
        L.oracle_graph_en_edge_types.argtypes = [U64, P, P, P]
        L.oracle_graph_en_bfs.restype = ctypes.c_int
        L.oracle_graph_en_bfs.argtypes = [U64, P, P, P, U32, P, P, P, P, ctypes.POINTER(ctypes.c_double)]
        L.oracle_graph_en_cc.restype = ctypes.c_int
        L.oracle_graph_en_cc.argtypes = [U64, P, P, P, P, P, P, P, ctypes.POINTER(ctypes.c_double)]
        L.oracle_graph_en_pr.restype = ctypes.c_int
        L.oracle_graph_en_pr.argtypes = [U64, P, P, P, ctypes.c_double, U32, P, ctypes.POINTER(ctypes.c_double)]
        L.oracle_graph_pr.restype = ctypes.c_int
        L.oracle_graph_pr.argtypes = [U64, P, P, P, ctypes.c_double, U32, ctypes.c_int, P,
                                      ctypes.POINTER(ctypes.c_double)]
        L.oracle_ray_render.restype = ctypes.c_int
        L.oracle_ray_render.argtypes = [U32, U32, U32, U32, U32, P, P, P, P, ctypes.c_int, P, P, P,
                                        ctypes.POINTER(ctypes.c_double)]
        L.oracle_traf_run.restype = ctypes.c_int
        L.oracle_traf_run.argtypes = [U32, U32, U32, P, P, P, P, P, U32, U64, P, P, ctypes.c_int, P, P,
                                      ctypes.POINTER(ctypes.c_double)]
        L.oracle_nbody_run.restype = ctypes.c_int
        L.oracle_nbody_run.argtypes = [U32, P, P, P, U32, ctypes.c_float, P, ctypes.c_float, ctypes.c_int, P, P,
                                       ctypes.POINTER(ctypes.c_double)]
        L.oracle_stut_run.restype = ctypes.c_int
        F = ctypes.c_float
        L.oracle_stut_run.argtypes = [U32, P, P, P, P, U32, P, P, P, P, P, P, U32, F, F, F, F, ctypes.c_int, P, P, P,
                                      ctypes.POINTER(ctypes.c_double)]
        L.oracle_collide_run.restype = ctypes.c_int
        L.oracle_collide_run.argtypes = [U32, P, P, P, U32, U32, F, F, F, P, F, ctypes.c_int, P, P, P,
                                         ctypes.POINTER(ctypes.c_double)]
        L.oracle_max_threads.restype = ctypes.c_int
        _lib = L
    return _lib


def _p(a: np.ndarray, ct):
    return a.ctypes.data_as(ctypes.POINTER(ct))


def max_threads() -> int:
    return int(lib().oracle_max_threads())


# ---- allocator / range table / COAL / TypePointer --------------------------
def region_plan(count: int, init_chunk: int = 4096) -> list[int]:
    L = lib()
    k = L.oracle_region_plan(count, init_chunk, None, 0)
    out = np.zeros(max(k, 1), dtype=np.uint64)
    L.oracle_region_plan(count, init_chunk, _p(out, ctypes.c_uint64), k)
    return [int(x) for x in out[:k]]


def build_table(start, nbytes, types):
    start = np.ascontiguousarray(start, dtype=np.uint64)
    nbytes = np.ascontiguousarray(nbytes, dtype=np.uint64)
    types = np.ascontiguousarray(types, dtype=np.uint32)
    n = len(start)
    ts = np.zeros(max(n, 1), np.uint64)
    te = np.zeros(max(n, 1), np.uint64)
    tt = np.zeros(max(n, 1), np.uint32)
    K = lib().oracle_build_table(_p(start, ctypes.c_uint64), _p(nbytes, ctypes.c_uint64),
                                 _p(types, ctypes.c_uint32), n, _p(ts, ctypes.c_uint64),
                                 _p(te, ctypes.c_uint64), _p(tt, ctypes.c_uint32))
    return ts[:K].copy(), te[:K].copy(), tt[:K].copy()


def coal_lookup(t_start, t_end, t_type, addrs) -> np.ndarray:
    t_start = np.ascontiguousarray(t_start, dtype=np.uint64)
    t_end = np.ascontiguousarray(t_end, dtype=np.uint64)
    t_type = np.ascontiguousarray(t_type, dtype=np.uint32)
    addrs = np.ascontiguousarray(addrs, dtype=np.uint64)
    out = np.zeros(len(addrs), dtype=np.uint32)
    lib().oracle_coal_lookup(_p(t_start, ctypes.c_uint64), _p(t_end, ctypes.c_uint64),
                             _p(t_type, ctypes.c_uint32), len(t_start), _p(addrs, ctypes.c_uint64),
                             len(addrs), _p(out, ctypes.c_uint32))
    return out


def tp_tag(addr: int, t: int) -> int:
    return int(lib().oracle_tp_tag(addr, t))


def tp_type(q: int) -> int:
    return int(lib().oracle_tp_type(q))


def tp_strip(q: int) -> int:
    return int(lib().oracle_tp_strip(q))


def tp_vfunc(q: int, vtables, slots: int, func: int) -> int:
    vt = np.ascontiguousarray(vtables, dtype=np.uint64)
    return int(lib().oracle_tp_vfunc(q, _p(vt, ctypes.c_uint64), slots, func))


# ---- apps -----------------------------------------------------------------
def micro_run(types, init, T: int, reps: int, threads: int = 1):
    """Returns (vals int32[n], seconds of the dispatch passes)."""
    types = np.ascontiguousarray(types, dtype=np.uint32)
    init = np.ascontiguousarray(init, dtype=np.int32)
    n = len(types)
    out = np.zeros(n, dtype=np.int32)
    sec = ctypes.c_double(0.0)
    rc = lib().oracle_micro_run(n, T, types.ctypes.data, init.ctypes.data, reps, threads,
                                out.ctypes.data, ctypes.byref(sec))
    if rc != 0:
        raise ValueError(f"oracle_micro_run rc={rc}")
    return out, sec.value


def gol_run(W: int, H: int, alive0, gens: int, torus: bool = False, threads: int = 1):
    """Returns (state uint8[H*W], counter uint16[H*W], pop uint32[gens], seconds)."""
    a = np.ascontiguousarray(alive0, dtype=np.uint8)
    st = np.zeros(W * H, np.uint8)
    ctr = np.zeros(W * H, np.uint16)
    pop = np.zeros(max(gens, 1), np.uint32)
    sec = ctypes.c_double(0.0)
    rc = lib().oracle_gol_run(W, H, a.ctypes.data, gens, int(torus), threads, st.ctypes.data,
                              ctr.ctypes.data, pop.ctypes.data, ctypes.byref(sec))
    if rc != 0:
        raise ValueError(f"oracle_gol_run rc={rc}")
    return st, ctr, pop[:gens].copy(), sec.value


def rule_masks(born, survive):
    """'B2/S345' style digit strings -> bit masks."""
    return sum(1 << int(d) for d in str(born)), sum(1 << int(d) for d in str(survive))


def gen_run(W: int, H: int, state0, gens: int, born="2", survive="345", C: int = 4,
            torus: bool = False, threads: int = 1):
    """Returns (state uint8[H*W], counter uint16[H*W], hist uint32[C], seconds)."""
    bm, sm = rule_masks(born, survive)
    a = np.ascontiguousarray(state0, dtype=np.uint8)
    st = np.zeros(W * H, np.uint8)
    ctr = np.zeros(W * H, np.uint16)
    hist = np.zeros(C, np.uint32)
    sec = ctypes.c_double(0.0)
    rc = lib().oracle_gen_run(W, H, a.ctypes.data, gens, bm, sm, C, int(torus), threads, st.ctypes.data,
                              ctr.ctypes.data, hist.ctypes.data, ctypes.byref(sec))
    if rc != 0:
        raise ValueError(f"oracle_gen_run rc={rc}")
    return st, ctr, hist, sec.value


def _csr(offs, col, types):
    return (np.ascontiguousarray(offs, dtype=np.uint64), np.ascontiguousarray(col, dtype=np.uint32),
            np.ascontiguousarray(types, dtype=np.uint32))


def graph_bfs(offs, col, types, src: int):
    """Returns (depth int32[V], levels, calls, seconds)."""
    offs, col, types = _csr(offs, col, types)
    V = len(offs) - 1
    depth = np.empty(V, np.int32)
    lv, calls, sec = ctypes.c_uint32(), ctypes.c_uint64(), ctypes.c_double()
    rc = lib().oracle_graph_bfs(V, offs.ctypes.data, col.ctypes.data, types.ctypes.data, src,
                                depth.ctypes.data, ctypes.byref(lv), ctypes.byref(calls), ctypes.byref(sec))
    if rc:
        raise ValueError(f"oracle_graph_bfs rc={rc}")
    return depth, lv.value, calls.value, sec.value


def graph_cc(offs, col, types, threads: int = 1):
    """Returns (label uint32[V], iters, calls, seconds)."""
    offs, col, types = _csr(offs, col, types)
    V = len(offs) - 1
    label = np.empty(V, np.uint32)
    it, calls, sec = ctypes.c_uint32(), ctypes.c_uint64(), ctypes.c_double()
    rc = lib().oracle_graph_cc(V, offs.ctypes.data, col.ctypes.data, types.ctypes.data, threads,
                               label.ctypes.data, ctypes.byref(it), ctypes.byref(calls), ctypes.byref(sec))
    if rc:
        raise ValueError(f"oracle_graph_cc rc={rc}")
    return label, it.value, calls.value, sec.value


def graph_pr(offs, col, types, iters: int = 20, d: float = 0.85, threads: int = 1):
    """Returns (rank float32[V], seconds)."""
    offs, col, types = _csr(offs, col, types)
    V = len(offs) - 1
    rank = np.empty(V, np.float32)
    sec = ctypes.c_double()
    rc = lib().oracle_graph_pr(V, offs.ctypes.data, col.ctypes.data, types.ctypes.data, d, iters, threads,
                               rank.ctypes.data, ctypes.byref(sec))
    if rc:
        raise ValueError(f"oracle_graph_pr rc={rc}")
    return rank, sec.value


def graph_en_edge_types(offs, vtypes):
    """GraphChi-vEN edge class of every arc (0 Edge, 1 HubEdge: source is a Hub)."""
    offs = np.ascontiguousarray(offs, dtype=np.uint64)
    vtypes = np.ascontiguousarray(vtypes, dtype=np.uint32)
    V = len(offs) - 1
    et = np.empty(int(offs[-1]), np.uint32)
    lib().oracle_graph_en_edge_types(V, offs.ctypes.data, vtypes.ctypes.data, et.ctypes.data)
    return et


def graph_en_bfs(offs, col, types, src: int):
    """Virtual edges + vertices. Returns (depth int32[V], levels, vertex calls, edge calls, seconds)."""
    offs, col, types = _csr(offs, col, types)
    V = len(offs) - 1
    depth = np.empty(V, np.int32)
    lv, vc, ec, sec = ctypes.c_uint32(), ctypes.c_uint64(), ctypes.c_uint64(), ctypes.c_double()
    rc = lib().oracle_graph_en_bfs(V, offs.ctypes.data, col.ctypes.data, types.ctypes.data, src, depth.ctypes.data,
                                   ctypes.byref(lv), ctypes.byref(vc), ctypes.byref(ec), ctypes.byref(sec))
    if rc:
        raise ValueError(f"oracle_graph_en_bfs rc={rc}")
    return depth, lv.value, vc.value, ec.value, sec.value


def graph_en_cc(offs, col, types):
    """Virtual edges + vertices. Returns (label uint32[V], iters, vertex calls, edge calls, seconds)."""
    offs, col, types = _csr(offs, col, types)
    V = len(offs) - 1
    label = np.empty(V, np.uint32)
    it, vc, ec, sec = ctypes.c_uint32(), ctypes.c_uint64(), ctypes.c_uint64(), ctypes.c_double()
    rc = lib().oracle_graph_en_cc(V, offs.ctypes.data, col.ctypes.data, types.ctypes.data, label.ctypes.data,
                                  ctypes.byref(it), ctypes.byref(vc), ctypes.byref(ec), ctypes.byref(sec))
    if rc:
        raise ValueError(f"oracle_graph_en_cc rc={rc}")
    return label, it.value, vc.value, ec.value, sec.value


def graph_en_pr(offs, col, types, iters: int = 20, d: float = 0.85):
    """Virtual edges + vertices. Returns (rank float32[V], seconds)."""
    offs, col, types = _csr(offs, col, types)
    V = len(offs) - 1
    rank = np.empty(V, np.float32)
    sec = ctypes.c_double()
    rc = lib().oracle_graph_en_pr(V, offs.ctypes.data, col.ctypes.data, types.ctypes.data, d, iters,
                                  rank.ctypes.data, ctypes.byref(sec))
    if rc:
        raise ValueError(f"oracle_graph_en_pr rc={rc}")
    return rank, sec.value


def ray_render(W: int, H: int, types, params, cam, albedo, row0: int = 0, nrows: int | None = None,
               threads: int = 1):
    """Returns (rgb float32[nrows, W, 3], hit_id int32[nrows, W], calls, seconds)."""
    nrows = H - row0 if nrows is None else nrows
    types = np.ascontiguousarray(types, dtype=np.uint32)
    params = np.ascontiguousarray(params, dtype=np.float32)
    cam = np.ascontiguousarray(cam, dtype=np.float32)
    albedo = np.ascontiguousarray(albedo, dtype=np.float32)
    rgb = np.zeros((nrows, W, 3), np.float32)
    hid = np.zeros((nrows, W), np.int32)
    calls, sec = ctypes.c_uint64(), ctypes.c_double()
    rc = lib().oracle_ray_render(W, H, row0, nrows, len(types), types.ctypes.data, params.ctypes.data,
                                 cam.ctypes.data, albedo.ctypes.data, threads, rgb.ctypes.data, hid.ctypes.data,
                                 ctypes.byref(calls), ctypes.byref(sec))
    if rc:
        raise ValueError(f"oracle_ray_render rc={rc}")
    return rgb, hid, calls.value, sec.value


def traf_run(world: dict, steps: int, threads: int = 1):
    """world = synth.traf_world(...); returns (pos uint32[nveh], v uint32[nveh], seconds)."""
    w = {k: (np.ascontiguousarray(v) if isinstance(v, np.ndarray) else v) for k, v in world.items()}
    n = len(w["veh_ring"])
    pos = np.zeros(n, np.uint32)
    vel = np.zeros(n, np.uint32)
    sec = ctypes.c_double()
    rc = lib().oracle_traf_run(w["R"], w["L"], n, w["veh_ring"].ctypes.data, w["veh_pos"].ctypes.data,
                               w["veh_type"].ctypes.data, w["light"].ctypes.data, w["phase"].ctypes.data, steps,
                               w["seed"], w["vmax"].ctypes.data, w["slow_thr"].ctypes.data, threads,
                               pos.ctypes.data, vel.ctypes.data, ctypes.byref(sec))
    if rc:
        raise ValueError(f"oracle_traf_run rc={rc}")
    return pos, vel, sec.value


def nbody_run(sys_: dict, steps: int, threads: int = 1):
    """sys_ = synth.nbody_system(...); returns (pos float32[N,4], vel float32[N,3], seconds)."""
    types = np.ascontiguousarray(sys_["types"], np.uint32)
    pos = np.ascontiguousarray(sys_["pos"], np.float32)
    vel = np.ascontiguousarray(sys_["vel"], np.float32)
    eps2 = np.ascontiguousarray(sys_["eps2"], np.float32)
    N = len(types)
    po = np.zeros((N, 4), np.float32)
    vo = np.zeros((N, 3), np.float32)
    sec = ctypes.c_double()
    rc = lib().oracle_nbody_run(N, types.ctypes.data, pos.ctypes.data, vel.ctypes.data, steps,
                                ctypes.c_float(sys_["dt"]), eps2.ctypes.data, ctypes.c_float(sys_["damp"]), threads,
                                po.ctypes.data, vo.ctypes.data, ctypes.byref(sec))
    if rc:
        raise ValueError(f"oracle_nbody_run rc={rc}")
    return po, vo, sec.value


def stut_run(w: dict, steps: int, threads: int = 1):
    """w = synth.stut_lattice(...) / synth.stut_custom(...); returns
    (pos float32[n,2], vel float32[n,2], broken uint8[S], seconds). See oracle.h."""
    n, S = len(w["types"]), len(w["a"])
    c = lambda a, dt: np.ascontiguousarray(a, dtype=dt)
    types, pos, vel, mass = c(w["types"], np.uint32), c(w["pos"], np.float32), c(w["vel"], np.float32), \
        c(w["mass"], np.float32)
    a, b, L0, k = c(w["a"], np.uint32), c(w["b"], np.uint32), c(w["L0"], np.float32), c(w["k"], np.float32)
    io, inc = c(w["inc_offs"], np.uint32), c(w["inc"], np.uint32)
    po = np.zeros((n, 2), np.float32)
    vo = np.zeros((n, 2), np.float32)
    bo = np.zeros(max(S, 1), np.uint8)
    secs = ctypes.c_double(0)
    rc = lib().oracle_stut_run(n, types.ctypes.data, pos.ctypes.data, vel.ctypes.data, mass.ctypes.data, S,
                               a.ctypes.data, b.ctypes.data, L0.ctypes.data, k.ctypes.data, io.ctypes.data,
                               inc.ctypes.data, steps, float(w["dt"]), float(w["damping"]), float(w["v_pull"]),
                               float(w["break_ratio"]), threads, po.ctypes.data, vo.ctypes.data, bo.ctypes.data,
                               ctypes.byref(secs))
    if rc:
        raise ValueError(f"oracle_stut_run rc={rc}")
    return po, vo, bo[:S], secs.value


def collide_run(sys_: dict, steps: int, threads: int = 1):
    """sys_ = synth.collide_system(...); returns (pos float32[N,4], vel float32[N,4], calls, seconds)."""
    types = np.ascontiguousarray(sys_["types"], np.uint32)
    pos = np.ascontiguousarray(sys_["pos"], np.float32)
    vel = np.ascontiguousarray(sys_["vel"], np.float32)
    eps2 = np.ascontiguousarray(sys_["eps2"], np.float32)
    N = len(types)
    po = np.zeros((N, 4), np.float32)
    vo = np.zeros((N, 4), np.float32)
    calls = ctypes.c_uint64()
    sec = ctypes.c_double()
    rc = lib().oracle_collide_run(N, types.ctypes.data, pos.ctypes.data, vel.ctypes.data, steps, int(sys_["G"]),
                                  float(sys_["rc"]), float(sys_["rm"]), float(sys_["dt"]), eps2.ctypes.data,
                                  float(sys_["damp"]), threads, po.ctypes.data, vo.ctypes.data, ctypes.byref(calls),
                                  ctypes.byref(sec))
    if rc:
        raise ValueError(f"oracle_collide_run rc={rc}")
    return po, vo, calls.value, sec.value

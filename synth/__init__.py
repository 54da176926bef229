"""Seeded synthetic input generators shared by the oracle tests and the CUDA path.

This module holds NONE of the method's arithmetic (no dispatch, no range
lookup, no tagging, no app update rule). It only draws the random numbers the
workloads need, with a counter-based generator, so that both sides receive
byte-identical inputs:

    splitmix64(x): z = x + 0x9E3779B97F4A7C15
                   z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9
                   z = (z ^ (z >> 27)) * 0x94D049BB133111EB
                   return z ^ (z >> 31)              (all mod 2^64)

    draw(seed, stream, i)  = splitmix64(seed ^ (stream << 56) ^ i)
    uniform(u, n)          = floor(u * n / 2^64)     (exact, n < 2^32)
    bernoulli(u, p)        = (u >> 32) < floor(p * 2^32)

Stream ids are fixed per use (constants below). The workload recipes follow
SURVEY.md §8(c)/(d) and are restated in DESIGN.md §"Input recipe".
"""
from __future__ import annotations

import numpy as np

M64 = (1 << 64) - 1

# stream ids (fixed per use)
S_TYPE = 1      # micro: object type draw
S_INIT = 2      # micro: initial val
S_GOL = 3       # GOL / GEN initial soup
S_ADDR = 4      # random probe addresses (tests)
S_GRAPH = 5     # RMAT edges
S_PERM = 6      # vertex permutation
S_SCENE = 7     # ray-tracer scene
S_TRAF = 8      # traffic: vehicle placement / types
S_TRAF_RNG = 9  # traffic: per-step slowdown draws (counter index = id<<24 ^ t)
S_BODY = 10     # n-body initial conditions
S_STUT = 11     # structure perturbation
S_COLL = 12     # collision bodies


def splitmix64(x: np.ndarray | int) -> np.ndarray:
    """Vectorised splitmix64 over uint64 (wrap-around arithmetic)."""
    z = np.asarray(x, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = z + np.uint64(0x9E3779B97F4A7C15)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        z = z ^ (z >> np.uint64(31))
    return z


def splitmix64_int(x: int) -> int:
    """Scalar reference form (pure Python ints) used to pin the vectorised one."""
    z = (x + 0x9E3779B97F4A7C15) & M64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & M64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & M64
    return z ^ (z >> 31)


def draw(seed: int, stream: int, idx: np.ndarray) -> np.ndarray:
    """draw(seed, stream, i) = splitmix64(seed ^ (stream << 56) ^ i)."""
    key = np.uint64(((seed & M64) ^ ((stream & 0xFF) << 56)) & M64)
    return splitmix64(np.asarray(idx, dtype=np.uint64) ^ key)


def uniform(u: np.ndarray, n: int) -> np.ndarray:
    """floor(u * n / 2^64) computed exactly in uint64 for 0 < n < 2^32."""
    assert 0 < n < (1 << 32)
    u = np.asarray(u, dtype=np.uint64)
    n64 = np.uint64(n)
    hi = u >> np.uint64(32)
    lo = u & np.uint64(0xFFFFFFFF)
    with np.errstate(over="ignore"):
        t = hi * n64 + ((lo * n64) >> np.uint64(32))
    return (t >> np.uint64(32)).astype(np.uint32)


def bernoulli(u: np.ndarray, p: float) -> np.ndarray:
    thr = np.uint64(int(p * (1 << 32)))
    return (np.asarray(u, dtype=np.uint64) >> np.uint64(32)) < thr


# --------------------------------------------------------------------------
# Config 2: dispatch microbenchmark (paper §8.3)
# --------------------------------------------------------------------------
ORDERS = ("random", "sorted", "kperwarp")


def micro_types(n: int, T: int, order: str = "random", seed: int = 42, k: int | None = None) -> np.ndarray:
    """Type id per object index, uint32[n].

    random  : t(i) = uniform(draw(seed, S_TYPE, i), T)
    sorted  : t(i) = floor(i*T/n)
    kperwarp: t(i) = (i mod 32) mod k     (Fig. 12b "types per warp", k<=T)
    """
    i = np.arange(n, dtype=np.uint64)
    if order == "random":
        return uniform(draw(seed, S_TYPE, i), T)
    if order == "sorted":
        return ((i * np.uint64(T)) // np.uint64(max(n, 1))).astype(np.uint32)
    if order == "kperwarp":
        k = T if k is None else k
        return ((i % np.uint64(32)) % np.uint64(k)).astype(np.uint32)
    raise ValueError(order)


def micro_init(n: int, seed: int = 42) -> np.ndarray:
    """init_i = draw(seed, S_INIT, i) & 0xFFFF  (int32[n])."""
    return (draw(seed, S_INIT, np.arange(n, dtype=np.uint64)) & np.uint64(0xFFFF)).astype(np.int32)


def random_addresses(n: int, seed: int = 7) -> np.ndarray:
    """Arbitrary u64 probe addresses for lookup tests."""
    return draw(seed, S_ADDR, np.arange(n, dtype=np.uint64))


# --------------------------------------------------------------------------
# Config 1 (GOL) and GEN: initial soup
# --------------------------------------------------------------------------
def soup(W: int, H: int, seed: int = 42, p: float = 0.5) -> np.ndarray:
    """alive[c] for c = y*W + x, uint8[H*W]; p = 0.5 -> lowest bit of the draw."""
    c = np.arange(W * H, dtype=np.uint64)
    u = draw(seed, S_GOL, c)
    if p == 0.5:
        return (u & np.uint64(1)).astype(np.uint8)
    return bernoulli(u, p).astype(np.uint8)


def place(W: int, H: int, cells) -> np.ndarray:
    """Grid with the given (x, y) cells alive (fixture helper)."""
    g = np.zeros(W * H, dtype=np.uint8)
    for x, y in cells:
        g[y * W + x] = 1
    return g


# --------------------------------------------------------------------------
# Config 4: RMAT graph. Native helper synth/rmat.cpp.
# --------------------------------------------------------------------------
_rmat_lib = None


def _rmat():
    global _rmat_lib
    if _rmat_lib is None:
        import ctypes
        import os
        import subprocess
        here = os.path.dirname(os.path.abspath(__file__))
        so, src = os.path.join(here, "libsynth.so"), os.path.join(here, "rmat.cpp")
        if not os.path.exists(so) or os.path.getmtime(so) < os.path.getmtime(src):
            subprocess.run(["g++", "-O2", "-std=c++17", "-fopenmp", "-fPIC", "-shared", "-o", so, src], check=True)
        L = ctypes.CDLL(so)
        P, U32, U64, D = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_double
        L.synth_rmat_edges.argtypes = [U32, U64, D, D, D, U64, U64, P, P]
        L.synth_rmat_edges.restype = None
        L.synth_permutation.argtypes = [U64, U64, U64, P]
        L.synth_permutation.restype = None
        L.synth_csr.argtypes = [U64, U64, P, P, P, P, P]
        L.synth_csr.restype = U64
        _rmat_lib = L
    return _rmat_lib


def build_native() -> None:
    _rmat()


def rmat_graph(scale: int, edge_factor: int = 16, seed: int = 1, A: float = 0.57, B: float = 0.19,
               C: float = 0.19, permute: bool = True):
    """Symmetric, de-duplicated, self-loop-free RMAT CSR: (offs uint64[V+1], col uint32[arcs])."""
    L = _rmat()
    V = 1 << scale
    E = edge_factor * V
    src = np.empty(E, np.uint32)
    dst = np.empty(E, np.uint32)
    L.synth_rmat_edges(scale, E, A, B, C, seed, S_GRAPH, src.ctypes.data, dst.ctypes.data)
    perm = None
    if permute:
        perm = np.empty(V, np.uint32)
        L.synth_permutation(V, seed, S_PERM, perm.ctypes.data)
    offs = np.empty(V + 1, np.uint64)
    col = np.empty(2 * E, np.uint32)
    arcs = L.synth_csr(V, E, src.ctypes.data, dst.ctypes.data, None if perm is None else perm.ctypes.data,
                       offs.ctypes.data, col.ctypes.data)
    return offs, col[:arcs].copy()


def csr_from_edges(V: int, edges):
    """Symmetric CSR of a small explicit undirected edge list (fixtures)."""
    L = _rmat()
    e = np.asarray(edges, dtype=np.uint32).reshape(-1, 2)
    src = np.ascontiguousarray(e[:, 0])
    dst = np.ascontiguousarray(e[:, 1])
    offs = np.empty(V + 1, np.uint64)
    col = np.empty(max(2 * len(e), 1), np.uint32)
    arcs = L.synth_csr(V, len(e), src.ctypes.data, dst.ctypes.data, None, offs.ctypes.data, col.ctypes.data)
    return offs, col[:arcs].copy()


# --------------------------------------------------------------------------
# Config 3: ray-tracer scene (reading G24)
# --------------------------------------------------------------------------
RAY_ALBEDO = np.array([[0.8, 0.8, 0.8], [0.9, 0.2, 0.2], [0.2, 0.9, 0.2], [0.2, 0.3, 0.9]], np.float32)


def _unit(seed, stream, idx):
    """uniform float32 in [0, 1) with 24 random bits (exact)."""
    return ((draw(seed, stream, idx) >> np.uint64(40)).astype(np.float32) * np.float32(2.0 ** -24))


def ray_scene(S: int, seed: int = 7, ground: bool = True):
    """Shapes j = 0..S-1: j = 0 is the ground plane y = -2 (if ground), else type
    1 + (j mod 3) (Sphere, Rect, Triangle); centres uniform in
    [-50,50]x[-30,30]x[-150,-50], sizes uniform in [0.5, 2). Returns
    (types uint32[S], params float32[S, 12])."""
    j = np.arange(S, dtype=np.uint64)
    r = [_unit(seed, S_SCENE, j * np.uint64(16) + np.uint64(k)) for k in range(16)]
    lo = np.array([-50, -30, -150], np.float32)
    hi = np.array([50, 30, -50], np.float32)
    c = np.stack([lo[k] + r[k] * (hi[k] - lo[k]) for k in range(3)], axis=1).astype(np.float32)
    s = (np.float32(0.5) + r[3] * np.float32(1.5)).astype(np.float32)
    types = (1 + (j % np.uint64(3))).astype(np.uint32)
    P = np.zeros((S, 12), np.float32)
    sph = types == 1
    P[sph, 0:3] = c[sph]
    P[sph, 3] = s[sph]
    rect = types == 2
    axis = np.minimum((r[4] * 3).astype(np.int64), 2)
    for a in range(3):
        m = rect & (axis == a)
        oth = [k for k in range(3) if k != a]
        P[m, 0] = a
        P[m, 1] = c[m, a]
        P[m, 2] = c[m, oth[0]] - s[m]
        P[m, 3] = c[m, oth[0]] + s[m]
        P[m, 4] = c[m, oth[1]] - s[m]
        P[m, 5] = c[m, oth[1]] + s[m]
    tri = types == 3
    for v in range(3):
        for k in range(3):
            P[tri, 3 * v + k] = c[tri, k] + s[tri] * (np.float32(2.0) * r[5 + 3 * v + k][tri] - np.float32(1.0))
    if ground and S > 0:
        types[0] = 0
        P[0, :] = 0
        P[0, 0] = -2.0
    return types, P


def ray_camera(W: int, H: int, fov_deg: float = 60.0, light=(0.4, 1.0, 0.6)):
    """fp32 camera constants computed once on the host: [tan(fov/2)*W/H, tan(fov/2), unit light]."""
    th = np.tan(np.deg2rad(fov_deg) / 2.0)
    l = np.asarray(light, np.float64)
    l = l / np.linalg.norm(l)
    return np.array([th * W / H, th, l[0], l[1], l[2]], np.float32)


# --------------------------------------------------------------------------
# Config 5 TRAF: Nagel-Schreckenberg rings (reading G16)
# --------------------------------------------------------------------------
TRAF_VMAX = np.array([5, 3, 4], np.uint32)          # Car, Truck, Bus
TRAF_PSLOW = (0.2, 0.1, 0.3)


def traf_world(R: int, L: int, density: float = 0.25, light_p: float = 1.0 / 32, seed: int = 11,
               p_slow=TRAF_PSLOW):
    """Rings x cells world: vehicles on cells with Bernoulli(density) draws (ring-major
    id order), type uniform in {Car, Truck, Bus}; LightCells with Bernoulli(light_p),
    phase uniform in [0, 20)."""
    N = R * L
    c = np.arange(N, dtype=np.uint64)
    occ = bernoulli(draw(seed, S_TRAF, c), density)
    cells = np.nonzero(occ)[0]
    veh_ring = (cells // L).astype(np.uint32)
    veh_pos = (cells % L).astype(np.uint32)
    vid = np.arange(len(cells), dtype=np.uint64)
    veh_type = uniform(draw(seed, S_TRAF, vid + np.uint64(1 << 40)), 3)
    light = bernoulli(draw(seed, S_TRAF, c + np.uint64(1 << 41)), light_p).astype(np.uint8)
    phase = uniform(draw(seed, S_TRAF, c + np.uint64(1 << 42)), 20)
    slow_thr = np.array([int(p * (1 << 32)) for p in p_slow], np.uint32)
    return dict(R=R, L=L, veh_ring=veh_ring, veh_pos=veh_pos, veh_type=veh_type, light=light, phase=phase,
                seed=seed, vmax=TRAF_VMAX.copy(), slow_thr=slow_thr)


# --------------------------------------------------------------------------
# Config 5 N-body (reading G18)
# --------------------------------------------------------------------------
NBODY_EPS2 = np.array([0.05, 0.01, 0.002], np.float32)  # Star, Planet, Dust softening^2
NBODY_MASS = ((5.0, 10.0), (0.5, 1.0), (0.01, 0.05))     # per-type mass ranges


def nbody_system(N: int, seed: int = 10, dt: float = 1e-3, damp: float = 0.999):
    """Bodies uniform in the unit-ish cube [-1,1]^3, velocities in [-0.1,0.1]^3,
    type = uniform(3) (0 Star, 1 Planet, 2 Dust), mass uniform in the type's range."""
    i = np.arange(N, dtype=np.uint64)
    r = [_unit(seed, S_BODY, i * np.uint64(8) + np.uint64(k)) for k in range(8)]
    types = uniform(draw(seed, S_BODY, i + np.uint64(1 << 40)), 3)
    pos = np.zeros((N, 4), np.float32)
    for k in range(3):
        pos[:, k] = np.float32(2.0) * r[k] - np.float32(1.0)
    lo = np.array([m[0] for m in NBODY_MASS], np.float32)[types]
    hi = np.array([m[1] for m in NBODY_MASS], np.float32)[types]
    pos[:, 3] = lo + r[3] * (hi - lo)
    vel = np.stack([(np.float32(0.2) * r[4 + k] - np.float32(0.1)) for k in range(3)], 1).astype(np.float32)
    return dict(types=types, pos=pos, vel=vel, eps2=NBODY_EPS2.copy(), dt=np.float32(dt), damp=np.float32(damp))


# degree-bucket vertex types (reading G22): Leaf <=1, Low 2-15, Mid 16-255, Hub >=256
DEG_BOUNDS = (1, 15, 255)


def vertex_types(offs) -> np.ndarray:
    deg = np.diff(np.asarray(offs, dtype=np.int64))
    return np.digitize(deg, [DEG_BOUNDS[0] + 1, DEG_BOUNDS[1] + 1, DEG_BOUNDS[2] + 1]).astype(np.uint32)


# --------------------------------------------------------------------------
# Config 5 STUT spring-node structure (reading G17)
# --------------------------------------------------------------------------
STUT_NODE, STUT_ANCHOR, STUT_PULL, STUT_SPRING = 0, 1, 2, 3  # type ids


def stut_lattice(W: int, H: int, seed: int = 12, jitter: float = 0.1, k0: float = 20.0, dt: float = 0.01,
                 damping: float = 0.05, v_pull: float = 1.0, break_ratio: float = 1.5):
    """W x H node lattice, node n = y*W + x at (x, y) (+ seeded jitter for free
    nodes); column 0 = AnchorNode, column W-1 = AnchorPullNode, else Node;
    mass 1 + 0.5u. Springs in the order (y, x, {right, down, diagonal}) with
    rest length 1 (axis) or float32(sqrt 2) (diagonal), stiffness k0(0.5+u).
    Incidence (structure only): for every node the springs touching it in
    ascending spring id, code = (spring << 1) | (node is the spring's b end)."""
    n = W * H
    i = np.arange(n, dtype=np.uint64)
    x = (np.arange(n) % W).astype(np.float32)
    y = (np.arange(n) // W).astype(np.float32)
    types = np.full(n, STUT_NODE, np.uint32)
    types[np.arange(n) % W == 0] = STUT_ANCHOR
    types[np.arange(n) % W == W - 1] = STUT_PULL
    free = types == STUT_NODE
    jx = np.float32(jitter) * (np.float32(2.0) * _unit(seed, S_STUT, 4 * i) - np.float32(1.0))
    jy = np.float32(jitter) * (np.float32(2.0) * _unit(seed, S_STUT, 4 * i + np.uint64(1)) - np.float32(1.0))
    pos = np.stack([np.where(free, x + jx, x), np.where(free, y + jy, y)], 1).astype(np.float32)
    mass = (np.float32(1.0) + np.float32(0.5) * _unit(seed, S_STUT, 4 * i + np.uint64(2))).astype(np.float32)
    a, b, L0 = [], [], []
    nodes = np.arange(n, dtype=np.int64).reshape(H, W)
    diag = np.float32(np.sqrt(2.0))
    # enumerate (y, x, kind) in order via a [H, W, 3] table, -1 = absent
    tab_b = np.full((H, W, 3), -1, np.int64)
    tab_b[:, :-1, 0] = nodes[:, 1:]
    tab_b[:-1, :, 1] = nodes[1:, :]
    tab_b[:-1, :-1, 2] = nodes[1:, 1:]
    tab_a = np.broadcast_to(nodes[:, :, None], (H, W, 3))
    kind = np.broadcast_to(np.arange(3)[None, None, :], (H, W, 3))
    sel = tab_b.reshape(-1) >= 0
    a = tab_a.reshape(-1)[sel].astype(np.uint32)
    b = tab_b.reshape(-1)[sel].astype(np.uint32)
    L0 = np.where(kind.reshape(-1)[sel] == 2, diag, np.float32(1.0)).astype(np.float32)
    S = len(a)
    si = np.arange(S, dtype=np.uint64)
    k = (np.float32(k0) * (np.float32(0.5) + _unit(seed, S_STUT, (si << np.uint64(2)) + np.uint64(3)
                                                   + np.uint64(1 << 40)))).astype(np.float32)
    inc_offs, inc = stut_incidence(n, a, b)
    return dict(W=W, H=H, types=types, pos=pos, vel=np.zeros((n, 2), np.float32), mass=mass, a=a, b=b, L0=L0,
                k=k, inc_offs=inc_offs, inc=inc, dt=np.float32(dt), damping=np.float32(damping),
                v_pull=np.float32(v_pull), break_ratio=np.float32(break_ratio))


def stut_incidence(n: int, a: np.ndarray, b: np.ndarray):
    """CSR of the springs touching each node, ascending spring id; code =
    (s << 1) | is_b. Pure structure (no method arithmetic)."""
    S = len(a)
    s = np.arange(S, dtype=np.uint64)
    node = np.concatenate([np.asarray(a, np.int64), np.asarray(b, np.int64)])
    code = np.concatenate([s << np.uint64(1), (s << np.uint64(1)) | np.uint64(1)]).astype(np.uint32)
    order = np.lexsort((code, node))
    offs = np.zeros(n + 1, np.uint32)
    np.add.at(offs, node + 1, 1)
    return np.cumsum(offs).astype(np.uint32), code[order]


def stut_custom(types, pos, mass, a, b, L0, k, vel=None, dt=0.01, damping=0.0, v_pull=1.0, break_ratio=1.5):
    """A hand-built structure (tests): same dict as stut_lattice."""
    n = len(types)
    a = np.asarray(a, np.uint32)
    b = np.asarray(b, np.uint32)
    inc_offs, inc = stut_incidence(n, a, b)
    return dict(W=n, H=1, types=np.asarray(types, np.uint32), pos=np.asarray(pos, np.float32).reshape(n, 2),
                vel=(np.zeros((n, 2), np.float32) if vel is None else np.asarray(vel, np.float32).reshape(n, 2)),
                mass=np.asarray(mass, np.float32), a=a, b=b, L0=np.asarray(L0, np.float32),
                k=np.asarray(k, np.float32), inc_offs=inc_offs, inc=inc, dt=np.float32(dt),
                damping=np.float32(damping), v_pull=np.float32(v_pull), break_ratio=np.float32(break_ratio))



# --------------------------------------------------------------------------
# Config 5 collision (readings G18 / G19)
# --------------------------------------------------------------------------
COLL_EPS2 = np.array([0.02, 0.01, 0.005], np.float32)  # per type, in units of rc^2 = 1


def collide_system(N: int, seed: int = 13, per_cell: float = 4.0, rm: float = 0.05, dt: float = 0.01,
                   damp: float = 0.999, vmax: float = 0.5):
    """N bodies uniform in [0, G)^3 with cells of side rc = 1 (G = ceil((N/per_cell)^(1/3))),
    velocities uniform in [-vmax, vmax]^3, type uniform(3) (Star / Planet / Dust), masses as
    the N-body system's; merge radius rm. vel is N x 4 (w unused)."""
    G = max(1, int(np.ceil((N / per_cell) ** (1.0 / 3.0))))
    i = np.arange(N, dtype=np.uint64)
    r = [_unit(seed, S_COLL, i * np.uint64(8) + np.uint64(k)) for k in range(7)]
    types = uniform(draw(seed, S_COLL, i + np.uint64(1 << 40)), 3)
    pos = np.zeros((N, 4), np.float32)
    for k in range(3):
        pos[:, k] = np.float32(G) * r[k]
    lo = np.array([m[0] for m in NBODY_MASS], np.float32)[types]
    hi = np.array([m[1] for m in NBODY_MASS], np.float32)[types]
    pos[:, 3] = lo + r[3] * (hi - lo)
    vel = np.zeros((N, 4), np.float32)
    for k in range(3):
        vel[:, k] = np.float32(vmax) * (np.float32(2.0) * r[4 + k] - np.float32(1.0))
    return dict(types=types, pos=pos, vel=vel, eps2=COLL_EPS2.copy(), dt=np.float32(dt), damp=np.float32(damp),
                G=G, rc=np.float32(1.0), rm=np.float32(rm))

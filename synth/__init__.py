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

"""Pins for the oracle's Game of Life (config 1; Table 2).

Pinned against an independent textbook array implementation of Conway's rule
(B3/S23) written here with numpy shifts, against the F3 fixture (glider /
block / blinker invariants, tests/golden/gol_f3.txt), and against counter
invariants of the polymorphic cells (age of a still life = generations).
"""
import os

import numpy as np
import pytest

import oracle
import synth


def textbook_gol(grid2d, gens, torus=False):
    """Conway's rule on a 2-D 0/1 array; returns list of states after each gen."""
    g = grid2d.astype(np.int32)
    out = []
    H, W = g.shape
    for _ in range(gens):
        if torus:
            n = sum(np.roll(np.roll(g, dy, 0), dx, 1)
                    for dy in (-1, 0, 1) for dx in (-1, 0, 1) if (dx, dy) != (0, 0))
        else:
            p = np.pad(g, 1)
            n = sum(p[1 + dy:1 + dy + H, 1 + dx:1 + dx + W]
                    for dy in (-1, 0, 1) for dx in (-1, 0, 1) if (dx, dy) != (0, 0))
        g = ((n == 3) | ((g == 1) & (n == 2))).astype(np.int32)
        out.append(g.copy())
    return out


def load_f3():
    p = os.path.join(os.path.dirname(__file__), "golden", "gol_f3.txt")
    d = {}
    for line in open(p):
        if not line.strip() or line.startswith("#"):
            continue
        k, *rest = line.split()
        d[k] = rest
    cells = lambda k: [tuple(int(v) for v in c.split(",")) for c in d[k]]
    return cells("glider"), cells("block"), cells("blinker"), int(d["population"][0]), int(d["generations"][0])


def test_f3_fixture_invariants():
    glider, block, blinker, pop, gens = load_f3()
    W = H = 16
    g0 = synth.place(W, H, glider + block + blinker)
    for g in range(1, gens + 1):
        st, ctr, pops, _ = oracle.gol_run(W, H, g0, g)
        assert np.all(pops == pop)
        s2 = st.reshape(H, W)
        for (x, y) in block:
            assert s2[y, x] == 1
            assert ctr[y * W + x] == g  # a still-life cell ages once per generation
        if g % 4 == 0:
            k = g // 4
            for (x, y) in glider:
                assert s2[y + k, x + k] == 1
        horiz = g % 2 == 0
        bl = [(2, 12), (3, 12), (4, 12)] if horiz else [(3, 11), (3, 12), (3, 13)]
        for (x, y) in bl:
            assert s2[y, x] == 1
        assert s2.sum() == pop


@pytest.mark.parametrize("torus", [False, True])
@pytest.mark.parametrize("W,H", [(16, 16), (37, 23), (64, 64)])
def test_gol_vs_textbook(W, H, torus):
    g0 = synth.soup(W, H, seed=42)
    ref = textbook_gol(g0.reshape(H, W), 40, torus)
    for gens in (1, 2, 7, 40):
        st, ctr, pops, _ = oracle.gol_run(W, H, g0, gens, torus)
        assert np.array_equal(st.reshape(H, W), ref[gens - 1])
        assert list(pops) == [int(r.sum()) for r in ref[:gens]]


def test_gol_counters_definition():
    # counter = generations since the cell last changed state (age / dead_for),
    # derived from the textbook state sequence
    W, H, G = 24, 24, 30
    g0 = synth.soup(W, H, seed=9)
    seq = [g0.reshape(H, W)] + textbook_gol(g0.reshape(H, W), G)
    st, ctr, _, _ = oracle.gol_run(W, H, g0, G)
    c2 = ctr.reshape(H, W)
    for y in range(H):
        for x in range(W):
            k = 0
            while k < G and seq[G - k][y, x] == seq[G - k - 1][y, x]:
                k += 1
            assert c2[y, x] == k


def test_gol_threads_identical():
    W = H = 256
    g0 = synth.soup(W, H, seed=42)
    a = oracle.gol_run(W, H, g0, 100, False, threads=1)
    b = oracle.gol_run(W, H, g0, 100, False, threads=oracle.max_threads())
    for x, y in zip(a[:3], b[:3]):
        assert np.array_equal(x, y)

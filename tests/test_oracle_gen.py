"""Pins for the oracle's Generations CA (config 5 GEN; Table 2, reading G15).

Pinned against an independent textbook array implementation of the B/S/C rule,
the special case B3/S23/C2 = Conway's Life (textbook GOL), a hand-derived
single-cell decay sequence, and the histogram invariant.
"""
import numpy as np
import pytest

import oracle
import synth
from tests.test_oracle_gol import textbook_gol


def textbook_generations(s2d, gens, born, survive, C, torus=False):
    B = {int(d) for d in str(born)}
    S = {int(d) for d in str(survive)}
    s = s2d.astype(np.int32)
    H, W = s.shape
    out = []
    for _ in range(gens):
        live = (s == 1).astype(np.int32)
        if torus:
            n = sum(np.roll(np.roll(live, dy, 0), dx, 1) for dy in (-1, 0, 1) for dx in (-1, 0, 1)
                    if (dx, dy) != (0, 0))
        else:
            p = np.pad(live, 1)
            n = sum(p[1 + dy:1 + dy + H, 1 + dx:1 + dx + W] for dy in (-1, 0, 1) for dx in (-1, 0, 1)
                    if (dx, dy) != (0, 0))
        born_m = np.isin(n, list(B))
        surv_m = np.isin(n, list(S))
        new = np.zeros_like(s)
        new[(s == 0) & born_m] = 1
        new[(s == 1) & surv_m] = 1
        if C > 2:
            new[(s == 1) & ~surv_m] = 2
        dying = s >= 2
        nxt = s + 1
        new[dying] = np.where(nxt[dying] >= C, 0, nxt[dying])
        s = new
        out.append(s.copy())
    return out


@pytest.mark.parametrize("rule", [("2", "345", 4), ("3", "23", 3), ("34", "34", 5), ("1", "", 2)])
@pytest.mark.parametrize("torus", [False, True])
def test_gen_vs_textbook(rule, torus):
    born, surv, C = rule
    W, H = 41, 29
    s0 = synth.soup(W, H, seed=3)
    ref = textbook_generations(s0.reshape(H, W), 25, born, surv, C, torus)
    for g in (1, 5, 25):
        st, _, hist, _ = oracle.gen_run(W, H, s0, g, born, surv, C, torus)
        assert np.array_equal(st.reshape(H, W), ref[g - 1])
        assert hist.sum() == W * H
        assert list(hist) == [int((ref[g - 1] == k).sum()) for k in range(C)]


def test_gen_b3s23c2_is_life():
    W = H = 48
    s0 = synth.soup(W, H, seed=8)
    ref = textbook_gol(s0.reshape(H, W), 30)
    st, _, _, _ = oracle.gen_run(W, H, s0, 30, "3", "23", 2)
    assert np.array_equal(st.reshape(H, W), ref[-1])


def test_gen_single_cell_decay():
    # a lone alive cell has 0 neighbours: S345 fails -> dying 2 -> 3 -> dead (C = 4)
    W = H = 5
    s0 = synth.place(W, H, [(2, 2)])
    seq = [int(oracle.gen_run(W, H, s0, g, "2", "345", 4)[0][12]) for g in range(1, 5)]
    assert seq == [2, 3, 0, 0]


def test_gen_threads_identical():
    W = H = 128
    s0 = synth.soup(W, H, seed=4)
    a = oracle.gen_run(W, H, s0, 20, threads=1)
    b = oracle.gen_run(W, H, s0, 20, threads=oracle.max_threads())
    for x, y in zip(a[:3], b[:3]):
        assert np.array_equal(x, y)


@pytest.mark.parametrize("rule", [("2", "345", 4), ("34", "34", 6), ("3", "23", 2)])
def test_gen_counters_definition(rule):
    """The counter of a cell's current object (Dead / Alive / Dying; each next()
    call increments it, a type change swaps in the other object with counter 0,
    P:1530-1534 reading G15) = generations since the cell's KIND last changed,
    derived here from the textbook state sequence (all dying states 2..C-1 are
    one kind: the Dying object just advances its stage)."""
    born, surv, C = rule
    W, H, G = 27, 19, 30
    s0 = synth.soup(W, H, seed=12)
    seq = [s0.reshape(H, W).astype(np.int32)] + textbook_generations(s0.reshape(H, W), G, born, surv, C)
    kind = [np.minimum(s, 2) for s in seq]
    _, ctr, _, _ = oracle.gen_run(W, H, s0, G, born, surv, C)
    c2 = ctr.reshape(H, W)
    changed = 0
    for y in range(H):
        for x in range(W):
            k = 0
            while k < G and kind[G - k][y, x] == kind[G - k - 1][y, x]:
                k += 1
            assert c2[y, x] == k
            changed += k < G
    assert 0 < changed < W * H  # both branches of the derivation are exercised

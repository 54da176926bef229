"""Pins for the oracle's TRAF (config 5; Table 2, reading G16).

Pinned against: fixture F5 (free-flow closed form pos_t = sum_{k<=t} min(k, vmax)),
a red light that never turns green (the car stops in front of it forever),
vehicle conservation / one vehicle per cell, and an independent vectorised
numpy textbook Nagel-Schreckenberg implementation of the same rule.
"""
import numpy as np
import pytest

import oracle
import synth


def world(R, L, rings, poss, types, light_cells=(), phases=None, p_slow=(0.0, 0.0, 0.0), seed=1):
    light = np.zeros(R * L, np.uint8)
    phase = np.zeros(R * L, np.uint32)
    for k, c in enumerate(light_cells):
        light[c] = 1
        phase[c] = 0 if phases is None else phases[k]
    return dict(R=R, L=L, veh_ring=np.array(rings, np.uint32), veh_pos=np.array(poss, np.uint32),
                veh_type=np.array(types, np.uint32), light=light, phase=phase, seed=seed,
                vmax=synth.TRAF_VMAX.copy(), slow_thr=np.array([int(p * (1 << 32)) for p in p_slow], np.uint32))


def test_f5_free_flow_closed_form():
    w = world(1, 100, [0], [0], [0])  # one Car (vmax 5), no lights, p_slow = 0
    got = [int(oracle.traf_run(w, t)[0][0]) for t in range(1, 9)]
    assert got == [1, 3, 6, 10, 15, 20, 25, 30]  # increments min(k, 5)
    for t in (1, 4, 17, 40):
        assert int(oracle.traf_run(w, t)[0][0]) == sum(min(k, 5) for k in range(1, t + 1)) % 100


def test_red_light_blocks():
    # light at cell 10, phase 0: red for steps t = 0..7, green for t = 8..19.
    # A Bus (vmax 4) from cell 0: t0 -> 1, t1 -> 3, t2 -> 6, t3 stops in front of
    # the red light at 9 (gap 3), waits through t7, moves on at t8.
    w = world(1, 50, [0], [0], [2], light_cells=[10], phases=[0])
    pos = [int(oracle.traf_run(w, t)[0][0]) for t in range(1, 11)]
    assert pos == [1, 3, 6, 9, 9, 9, 9, 9, 10, 12]


def textbook_nasch(w, steps):
    R, L = w["R"], w["L"]
    ring = w["veh_ring"].astype(np.int64)
    pos = w["veh_pos"].astype(np.int64)
    typ = w["veh_type"].astype(np.int64)
    v = np.zeros_like(pos)
    vmax = w["vmax"].astype(np.int64)[typ]
    thr = w["slow_thr"].astype(np.uint64)[typ]
    ids = np.arange(len(pos), dtype=np.uint64)
    light = w["light"].reshape(R, L).astype(bool)
    phase = w["phase"].reshape(R, L).astype(np.int64)
    for t in range(steps):
        occ = np.zeros((R, L), bool)
        occ[ring, pos] = True
        blocked = light & (((t + phase) % 20) < 8)
        nv = np.minimum(v + 1, vmax)
        gap = np.full_like(pos, 0)
        stop = np.zeros(len(pos), bool)
        for k in range(1, 6):
            c = (pos + k) % L
            hit = occ[ring, c] | blocked[ring, c]
            stop |= hit
            gap += (~stop) & (k <= nv)
        nv = np.minimum(nv, gap)
        u = synth.draw(w["seed"], synth.S_TRAF_RNG, (ids << np.uint64(24)) ^ np.uint64(t))
        slow = (u >> np.uint64(32)) < thr
        nv = np.where(slow & (nv > 0), nv - 1, nv)
        v = nv
        pos = (pos + nv) % L
    return pos.astype(np.uint32), v.astype(np.uint32)


@pytest.mark.parametrize("R,L,steps", [(7, 64, 30), (32, 256, 50)])
def test_traf_vs_textbook_and_invariants(R, L, steps):
    w = synth.traf_world(R, L, seed=R)
    pos, vel, _ = oracle.traf_run(w, steps)
    ref_pos, ref_v = textbook_nasch(w, steps)
    assert np.array_equal(pos, ref_pos) and np.array_equal(vel, ref_v)
    cells = w["veh_ring"].astype(np.int64) * L + pos
    assert len(np.unique(cells)) == len(cells)  # <= 1 vehicle per cell
    assert np.array_equal(np.bincount(w["veh_ring"], minlength=R), np.bincount(cells // L, minlength=R))
    assert np.all(vel <= w["vmax"][w["veh_type"]])


def test_traf_threads_identical():
    w = synth.traf_world(64, 512, seed=3)
    a = oracle.traf_run(w, 40, threads=1)
    b = oracle.traf_run(w, 40, threads=oracle.max_threads())
    assert np.array_equal(a[0], b[0]) and np.array_equal(a[1], b[1])

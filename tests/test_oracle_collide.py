"""Pins for the collision oracle (config 5 at 16M bodies, readings G18 / G19):

* one cell covering everything, no merging -> the all-pairs N-body oracle, bit
  for bit (same formula, same ascending-j order);
* an independent brute-force float64 numpy step (all pairs, cutoff mask,
  nearest-within-rm, mutual merge) agrees, including bodies outside the grid
  (clamped to edge cells) and which bodies get absorbed;
* a head-on pair merges into its mass-weighted centre / momentum;
* total mass is conserved through merges; 1 thread == all threads.
"""
import numpy as np
import pytest

import oracle
import synth


def numpy_step(s, P, V):
    """One collision step in float64 over ALL pairs (no grid)."""
    N = len(P)
    x, m = P[:, :3].astype(np.float64), P[:, 3].astype(np.float64)
    act = m > 0
    eps2 = s["eps2"].astype(np.float64)[s["types"]]
    rc2, rm2 = float(s["rc"]) ** 2, float(s["rm"]) ** 2
    d = x[None, :, :] - x[:, None, :]
    d2 = (d ** 2).sum(-1)
    pair = act[:, None] & act[None, :] & ~np.eye(N, dtype=bool)
    r2 = d2 + eps2[:, None]
    w = np.where(pair & (d2 < rc2), m[None, :] / (r2 * np.sqrt(r2)), 0.0)
    a = (d * w[..., None]).sum(1)
    v = V[:, :3].astype(np.float64) * np.where(s["types"] == 2, float(s["damp"]), 1.0)[:, None]
    v = np.where(act[:, None], v + float(s["dt"]) * a, V[:, :3])
    xn = np.where(act[:, None], x + float(s["dt"]) * v, x)
    cand = np.where(pair & (d2 < rm2), d2, np.inf)
    near = np.where(np.isfinite(cand.min(1)), cand.argmin(1), -1)  # argmin -> smallest id on ties
    Po = np.concatenate([xn, m[:, None]], 1)
    Vo = np.concatenate([v, np.zeros((N, 1))], 1)
    absorbed = np.zeros(N, bool)
    for i in range(N):
        j = near[i]
        if act[i] and j >= 0 and near[j] == i:
            if j > i:
                M = m[i] + m[j]
                Po[i, :3] = (m[i] * xn[i] + m[j] * xn[j]) / M
                Vo[i, :3] = (m[i] * v[i] + m[j] * v[j]) / M
                Po[i, 3] = M
            else:
                Po[i, 3] = 0.0
                Vo[i, :3] = 0.0
                absorbed[i] = True
    return Po, Vo, absorbed


def test_single_cell_no_merge_equals_nbody_oracle():
    nb = synth.nbody_system(300, seed=21)
    s = dict(types=nb["types"], pos=nb["pos"], vel=np.concatenate([nb["vel"], np.zeros((300, 1), np.float32)], 1),
             eps2=nb["eps2"], dt=nb["dt"], damp=nb["damp"], G=1, rc=np.float32(1e18), rm=np.float32(0.0))
    for steps in (1, 4):
        p, v, calls, _ = oracle.collide_run(s, steps)
        p_ref, v_ref, _ = oracle.nbody_run(nb, steps)
        assert np.array_equal(p.view(np.uint32), p_ref.view(np.uint32))
        assert np.array_equal(v[:, :3].view(np.uint32), v_ref.view(np.uint32))
        assert calls == 2 * 300 * steps


@pytest.mark.parametrize("N,outside", [(400, False), (700, True)])
def test_one_step_matches_bruteforce_float64(N, outside):
    s = synth.collide_system(N, seed=N, per_cell=3.0, rm=0.15)
    if outside:  # some bodies beyond the grid: clamped into the edge cells
        s["pos"][:20, 0] = -0.7
        s["pos"][20:40, 2] = np.float32(s["G"]) + 0.4
    p, v, _, _ = oracle.collide_run(s, 1)
    rp, rv, absorbed = numpy_step(s, s["pos"], s["vel"])
    assert absorbed.any()  # the merge path is exercised
    assert np.array_equal(p[:, 3] == 0, rp[:, 3] == 0)
    assert np.allclose(p, rp, rtol=1e-5, atol=1e-5)
    assert np.allclose(v[:, :3], rv[:, :3], rtol=1e-4, atol=1e-4)


def test_head_on_pair_merges_to_centre_of_mass():
    s = synth.collide_system(2, seed=1, rm=0.05)
    s["G"] = 2
    s["types"][:] = 1
    s["pos"][:] = [[0.5, 0.5, 0.5, 2.0], [0.53, 0.5, 0.5, 1.0]]
    s["vel"][:] = [[0.1, 0, 0, 0], [-0.2, 0, 0, 0]]
    p, v, _, _ = oracle.collide_run(s, 1)
    assert p[1, 3] == 0 and np.all(v[1, :3] == 0)  # absorbed by body 0
    assert p[0, 3] == 3.0
    # post-update states from the brute-force step, then the mass-weighted mean
    rp, rv, _ = numpy_step(s, s["pos"], s["vel"])
    assert np.allclose(p[0], rp[0], rtol=1e-6) and np.allclose(v[0, :3], rv[0, :3], rtol=1e-5)
    mom = 2.0 * 0.1 + 1.0 * (-0.2)
    assert abs(3.0 * v[0, 0] - mom) < 1e-3  # momentum of the pair (plus the tiny mutual pull)


def test_mass_conserved_and_bodies_disappear():
    s = synth.collide_system(3000, seed=5, per_cell=4.0, rm=0.12)
    m0 = s["pos"][:, 3].astype(np.float64).sum()
    p, _, calls, _ = oracle.collide_run(s, 6, threads=oracle.max_threads())
    assert (p[:, 3] == 0).sum() > 0
    assert abs(p[:, 3].astype(np.float64).sum() - m0) <= 1e-5 * m0
    assert calls < 2 * 3000 * 6  # absorbed bodies stop being called


def test_threads_identical():
    s = synth.collide_system(5000, seed=8, rm=0.1)
    a = oracle.collide_run(s, 3, threads=1)
    b = oracle.collide_run(s, 3, threads=oracle.max_threads())
    assert np.array_equal(a[0], b[0]) and np.array_equal(a[1], b[1]) and a[2] == b[2]

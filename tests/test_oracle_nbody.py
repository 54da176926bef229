"""Pins for the oracle's all-pairs N-body (config 5, reading G18).

Pinned against: fixture F10 (two equal bodies stay exactly mirror-symmetric,
centre of mass exactly 0), a float64 closed-form single step for N = 2, an
independent float64 numpy integrator of the same equations, and momentum
conservation when softening is type-independent and damping is off.
"""
import numpy as np
import pytest

import oracle
import synth


def system(pos, vel, types, eps2=(0.01, 0.01, 0.01), dt=1e-2, damp=1.0):
    return dict(types=np.array(types, np.uint32), pos=np.array(pos, np.float32), vel=np.array(vel, np.float32),
                eps2=np.array(eps2, np.float32), dt=np.float32(dt), damp=np.float32(damp))


def np_step(pos, vel, types, eps2, dt, damp):
    x, m = pos[:, :3].astype(np.float64), pos[:, 3].astype(np.float64)
    d = x[None, :, :] - x[:, None, :]
    r2 = (d ** 2).sum(-1) + eps2[types][:, None]
    w = m[None, :] / (r2 * np.sqrt(r2))
    np.fill_diagonal(w, 0.0)
    a = (d * w[..., None]).sum(1)
    v = vel.astype(np.float64) * np.where(types == 2, damp, 1.0)[:, None] + dt * a
    out = pos.astype(np.float64).copy()
    out[:, :3] = x + dt * v
    return out, v


def test_f10_two_bodies_symmetric_exact():
    s = system([[0.5, 0, 0, 1.0], [-0.5, 0, 0, 1.0]], [[0, 0, 0], [0, 0, 0]], [1, 1])
    for steps in (1, 2, 5, 20):
        p, v, _ = oracle.nbody_run(s, steps)
        assert p[0, 0] == -p[1, 0] and p[0, 1] == p[1, 1] == 0 and p[0, 2] == p[1, 2] == 0
        assert p[0, 0] + p[1, 0] == 0.0 and v[0, 0] == -v[1, 0]
        assert p[0, 0] < 0.5  # they attract


def test_two_body_single_step_closed_form():
    a = 0.5
    eps2 = 0.01
    dt = 1e-2
    s = system([[a, 0, 0, 2.0], [-a, 0, 0, 1.0]], [[0, 0.1, 0], [0, 0, 0]], [1, 1], eps2=(eps2,) * 3, dt=dt)
    p, v, _ = oracle.nbody_run(s, 1)
    r2 = (2 * a) ** 2 + eps2
    a0 = -1.0 * 2 * a / r2 ** 1.5  # body 0 pulled toward -x by m1 = 1
    a1 = 2.0 * 2 * a / r2 ** 1.5
    assert np.isclose(v[0, 0], dt * a0, rtol=1e-6) and np.isclose(v[1, 0], dt * a1, rtol=1e-6)
    assert np.isclose(p[0, 0], a + dt * dt * a0, rtol=1e-6)
    assert np.isclose(p[0, 1], dt * 0.1, rtol=1e-6)


def test_vs_float64_integrator():
    s = synth.nbody_system(64, seed=3, dt=1e-3)
    pos, vel = s["pos"].astype(np.float64), s["vel"].astype(np.float64)
    for _ in range(3):
        pos, vel = np_step(pos, vel, s["types"], s["eps2"].astype(np.float64), float(s["dt"]), float(s["damp"]))
    p, v, _ = oracle.nbody_run(s, 3)
    np.testing.assert_allclose(p, pos, rtol=1e-5, atol=1e-6)
    np.testing.assert_allclose(v, vel, rtol=1e-4, atol=1e-6)


def test_momentum_conserved_without_damping_and_equal_softening():
    s = synth.nbody_system(256, seed=4)
    s["eps2"] = np.full(3, 0.01, np.float32)
    s["damp"] = np.float32(1.0)
    m = s["pos"][:, 3].astype(np.float64)
    p0 = (m[:, None] * s["vel"]).sum(0)
    _, v, _ = oracle.nbody_run(s, 10)
    p1 = (m[:, None] * v.astype(np.float64)).sum(0)
    scale = (m[:, None] * np.abs(v)).sum()
    assert np.all(np.abs(p1 - p0) <= 1e-5 * scale)


def test_nbody_threads_identical():
    s = synth.nbody_system(512, seed=5)
    a = oracle.nbody_run(s, 4, threads=1)
    b = oracle.nbody_run(s, 4, threads=oracle.max_threads())
    assert np.array_equal(a[0], b[0]) and np.array_equal(a[1], b[1])

"""Pins for the STUT oracle (config 5 structure, reading G17) against closed
forms and invariants that do not come from the oracle itself:

* one spring + one free node = a harmonic oscillator; semi-implicit Euler is
  then a linear map M = [[1-h^2 w^2, h], [-h w^2, 1]] on (u, v) whose n-th
  power (float64 matrix power) gives the trajectory, and which conserves
  v^2 + w^2 u^2 - h w^2 u v exactly (checked in float64 here first);
* damping on a force-free node: v_t = v_0 (1 - h c / m)^t;
* a relaxed lattice translating at v = 1 with h = 2^-7 moves exactly
  (every position and difference is representable: forces are exactly 0);
* linear momentum of a free lattice (no anchors, no damping) is conserved;
* a spring pulled at constant speed breaks at the first step whose start
  length exceeds 1.5 L0 (closed-form step index, far from any rounding tie);
* an independent vectorised float64 numpy integrator of the same equations
  agrees on a jittered anchored/pulled lattice;
* 1 thread == all threads, bit for bit.
"""
import numpy as np
import pytest

import oracle
import synth


def _one_spring(u0=0.1, k=20.0, m=1.0, h=0.01, c=0.0):
    return synth.stut_custom(types=[synth.STUT_ANCHOR, synth.STUT_NODE], pos=[[0, 0], [1.0 + u0, 0]],
                             mass=[1.0, m], a=[0], b=[1], L0=[1.0], k=[k], dt=h, damping=c)


@pytest.mark.parametrize("steps", [1, 7, 100, 400])
def test_single_spring_matches_symplectic_euler_matrix_power(steps):
    u0, k, m, h = 0.1, 20.0, 1.0, 0.01
    w = _one_spring(u0, k, m, h)
    pos, vel, broken, _ = oracle.stut_run(w, steps)
    w2 = k / m
    M = np.array([[1 - h * h * w2, h], [-h * w2, 1.0]])
    u, v = np.linalg.matrix_power(M, steps) @ np.array([u0, 0.0])
    assert abs((pos[1, 0] - 1.0) - u) <= 2e-5 * (1 + steps / 100)
    assert abs(vel[1, 0] - v) <= 2e-4 * (1 + steps / 100)
    assert pos[1, 1] == 0 and vel[1, 1] == 0 and not broken.any()
    assert pos[0, 0] == 0 and pos[0, 1] == 0  # the anchor never moves


def test_single_spring_modified_energy_bounded():
    u0, k, m, h = 0.1, 20.0, 1.0, 0.01
    w2 = k / m
    H = lambda u, v: v * v + w2 * u * u - h * w2 * u * v  # noqa: E731
    H0 = H(u0, 0.0)
    for steps in (50, 333, 1000):
        pos, vel, _, _ = oracle.stut_run(_one_spring(u0, k, m, h), steps)
        assert abs(H(pos[1, 0] - 1.0, vel[1, 0]) - H0) <= 1e-4 * H0


def test_damping_geometric_decay():
    """A node with no springs: F = -c v, so v_t = v_0 (1 - h c/m)^t."""
    h, c, m = 0.01, 0.5, 2.0
    w = synth.stut_custom(types=[synth.STUT_NODE], pos=[[0, 0]], mass=[m], a=[], b=[], L0=[], k=[],
                          vel=[[1.0, -2.0]], dt=h, damping=c)
    for t in (1, 10, 200):
        _, vel, _, _ = oracle.stut_run(w, t)
        r = (1 - h * c / m) ** t
        assert np.allclose(vel[0], [r, -2 * r], rtol=1e-5, atol=0)


def test_relaxed_lattice_translates_exactly():
    W, H = 6, 5
    w = synth.stut_lattice(W, H, seed=1, jitter=0.0, dt=2.0 ** -7, damping=0.0)
    w["types"][:] = synth.STUT_NODE
    w["vel"][:, 0] = 1.0
    for t in (1, 3, 64):
        pos, vel, broken, _ = oracle.stut_run(w, t)
        exp = w["pos"].copy()
        exp[:, 0] += np.float32(t * 2.0 ** -7)
        assert np.array_equal(pos, exp) and np.array_equal(vel, w["vel"]) and not broken.any()


def test_free_lattice_conserves_momentum():
    w = synth.stut_lattice(12, 9, seed=3, jitter=0.15, damping=0.0)
    w["types"][:] = synth.STUT_NODE
    pos, vel, broken, _ = oracle.stut_run(w, 150)
    p = (w["mass"][:, None].astype(np.float64) * vel).sum(0)
    scale = (w["mass"][:, None] * np.abs(vel)).sum()
    assert scale > 1e-2  # it does move
    assert np.all(np.abs(p) <= 1e-5 * scale)
    cm0 = (w["mass"][:, None] * w["pos"]).sum(0) / w["mass"].sum()
    cm = (w["mass"][:, None].astype(np.float64) * pos).sum(0) / w["mass"].sum()
    assert np.allclose(cm, cm0, atol=1e-4)


def test_pulled_spring_breaks_at_closed_form_step():
    """Anchor (0,0) -- spring L0=1 -- pull node starting at (1,0) moving +0.7/s,
    h = 0.01: the start-of-step length is 1 + 0.007 t, > 1.5 first at t = 72
    (1.497 at t = 71), so it is intact after 72 steps and broken after 73."""
    w = synth.stut_custom(types=[synth.STUT_ANCHOR, synth.STUT_PULL], pos=[[0, 0], [1, 0]], mass=[1, 1],
                          a=[0], b=[1], L0=[1.0], k=[5.0], dt=0.01, v_pull=0.7)
    _, _, broken, _ = oracle.stut_run(w, 72)
    assert broken[0] == 0
    pos, _, broken, _ = oracle.stut_run(w, 73)
    assert broken[0] == 1
    assert abs(pos[1, 0] - (1 + 0.007 * 73)) < 1e-5


def _numpy_reference(w, steps):
    """Independent vectorised float64 integrator of the same equations."""
    px = w["pos"][:, 0].astype(np.float64)
    py = w["pos"][:, 1].astype(np.float64)
    vx = w["vel"][:, 0].astype(np.float64)
    vy = w["vel"][:, 1].astype(np.float64)
    m = w["mass"].astype(np.float64)
    a, b = w["a"].astype(np.int64), w["b"].astype(np.int64)
    L0, k = w["L0"].astype(np.float64), w["k"].astype(np.float64)
    free = w["types"] == synth.STUT_NODE
    pull = w["types"] == synth.STUT_PULL
    dt, c = float(w["dt"]), float(w["damping"])
    broken = np.zeros(len(a), bool)
    for _ in range(steps):
        dx, dy = px[b] - px[a], py[b] - py[a]
        ln = np.hypot(dx, dy)
        broken |= ln > float(w["break_ratio"]) * L0
        fs = np.where(broken, 0.0, k * (ln - L0) / ln)
        Fx = np.zeros_like(px)
        Fy = np.zeros_like(py)
        np.add.at(Fx, a, fs * dx)
        np.add.at(Fy, a, fs * dy)
        np.add.at(Fx, b, -fs * dx)
        np.add.at(Fy, b, -fs * dy)
        Fx -= c * vx
        Fy -= c * vy
        vx = np.where(free, vx + dt * Fx / m, vx)
        vy = np.where(free, vy + dt * Fy / m, vy)
        px = np.where(free, px + dt * vx, np.where(pull, px + dt * float(w["v_pull"]), px))
        py = np.where(free, py + dt * vy, py)
    return np.stack([px, py], 1), np.stack([vx, vy], 1), broken


def test_lattice_matches_independent_float64_integrator():
    w = synth.stut_lattice(16, 11, seed=5, jitter=0.1, v_pull=1.0)
    pos, vel, broken, _ = oracle.stut_run(w, 40)
    rp, rv, rb = _numpy_reference(w, 40)
    assert np.allclose(pos, rp, atol=2e-5, rtol=0)
    assert np.allclose(vel, rv, atol=2e-4, rtol=0)
    assert np.array_equal(broken.astype(bool), rb)


def test_lattice_breaks_near_the_pulled_edge():
    w = synth.stut_lattice(24, 8, seed=6, v_pull=4.0)
    _, _, broken, _ = oracle.stut_run(w, 60)
    assert broken.any()
    rp, rv, rb = _numpy_reference(w, 60)
    assert np.array_equal(broken.astype(bool), rb)


def test_threads_identical():
    w = synth.stut_lattice(64, 40, seed=7, v_pull=3.0)
    a = oracle.stut_run(w, 30, threads=1)
    b = oracle.stut_run(w, 30, threads=oracle.max_threads())
    for x, y in zip(a[:3], b[:3]):
        assert np.array_equal(x, y)


def test_lattice_structure():
    W, H = 5, 4
    w = synth.stut_lattice(W, H)
    S = (W - 1) * H + W * (H - 1) + (W - 1) * (H - 1)
    assert len(w["a"]) == S
    deg = np.diff(w["inc_offs"].astype(np.int64))
    assert deg.sum() == 2 * S and deg.max() <= 6
    # every incidence entry names a spring that touches that node at the coded end
    for n in range(W * H):
        for e in w["inc"][w["inc_offs"][n]:w["inc_offs"][n + 1]]:
            s, isb = e >> 1, e & 1
            assert (w["b"][s] if isb else w["a"][s]) == n

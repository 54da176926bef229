"""Pins for the oracle's ray tracer (config 3; Table 2 RAY P:1592-1600, readings G24/G25).

Pinned against closed forms (fixture F8: sphere hit t = 8 on the centre ray, a
rectangle in front wins with t = 5, equal-t duplicates -> lower id; ground
plane t = -2/d_y; a triangle hit at known barycentrics) and against an
independent float64 numpy implementation of the four intersection formulas
(hit ids agree wherever the float64 winner is not a near-tie).
"""
import numpy as np
import pytest

import oracle
import synth

ALB = synth.RAY_ALBEDO


def cam(W, H, fov):
    return synth.ray_camera(W, H, fov)


def shapes(*rows):
    types = np.array([r[0] for r in rows], np.uint32)
    P = np.zeros((len(rows), 12), np.float32)
    for i, r in enumerate(rows):
        P[i, :len(r[1])] = r[1]
    return types, P


def test_f8_sphere_rect_ties():
    W = H = 3
    c = cam(W, H, 90.0)
    t, P = shapes((1, [0, 0, -10, 2]))
    rgb, hid, calls, _ = oracle.ray_render(W, H, t, P, c, ALB)
    assert hid[1, 1] == 0 and calls == 9
    # centre ray d = (0,0,-1): t = 8, normal (0,0,1) -> lambert = l_z
    assert np.allclose(rgb[1, 1], ALB[1] * c[4] + 0.1, rtol=0, atol=1e-7)
    # an axis-aligned square at z = -5 in front of the sphere wins (t = 5)
    t2, P2 = shapes((1, [0, 0, -10, 2]), (2, [2, -5, -1, 1, -1, 1]))
    _, hid2, _, _ = oracle.ray_render(W, H, t2, P2, c, ALB)
    assert hid2[1, 1] == 1
    # equal t duplicates -> lower id wins
    t3, P3 = shapes((1, [0, 0, -10, 2]), (1, [0, 0, -10, 2]))
    _, hid3, _, _ = oracle.ray_render(W, H, t3, P3, c, ALB)
    assert hid3[1, 1] == 0


def test_ground_plane_and_triangle_closed_form():
    W, H = 8, 8
    c = cam(W, H, 60.0)
    # ground plane only: rows below the horizon hit, the rest miss
    t, P = shapes((0, [-2.0]))
    rgb, hid, _, _ = oracle.ray_render(W, H, t, P, c, ALB)
    assert np.all(hid[H // 2:] == 0) and np.all(hid[:H // 2] == -1)
    assert np.all(rgb[:H // 2] == 0)
    # lambert on the plane = l_y for every hit pixel (normal +y)
    assert np.allclose(rgb[H // 2:].reshape(-1, 3), ALB[0] * c[3] + 0.1, atol=1e-6)
    # triangle in z = -3 around the optical axis: centre pixels hit at t = 3 / |d_z|
    t2, P2 = shapes((3, [-1, -1, -3, 1, -1, -3, 0, 1, -3]))
    _, hid2, _, _ = oracle.ray_render(2, 2, t2, P2, cam(2, 2, 10.0), ALB)
    assert np.all(hid2 == 0)


def np_hits(types, P, W, H, c):
    """float64 reference: (t_best, id, second best t) per pixel, plain formulas."""
    ys, xs = np.mgrid[0:H, 0:W]
    u = (xs + 0.5) / W
    v = (ys + 0.5) / H
    d = np.stack([(2 * u - 1) * c[0], (1 - 2 * v) * c[1], -np.ones_like(u, dtype=float)], -1).astype(np.float64)
    d /= np.linalg.norm(d, axis=-1, keepdims=True)
    T = np.full((len(types), H, W), np.inf)
    for j, (ty, p) in enumerate(zip(types, P.astype(np.float64))):
        if ty == 0:
            with np.errstate(divide="ignore", invalid="ignore"):
                t = p[0] / d[..., 1]
        elif ty == 1:
            cc = p[:3]
            b = -(d @ cc)
            disc = b * b - (cc @ cc - p[3] ** 2)
            sq = np.sqrt(np.maximum(disc, 0))
            t = np.where(disc < 0, np.inf, np.where(-b - sq > 1e-4, -b - sq, -b + sq))
        elif ty == 2:
            a = int(p[0])
            oth = [k for k in range(3) if k != a]
            with np.errstate(divide="ignore", invalid="ignore"):
                t = p[1] / d[..., a]
            h = d * t[..., None]
            ok = (h[..., oth[0]] >= p[2]) & (h[..., oth[0]] <= p[3]) & (h[..., oth[1]] >= p[4]) & (h[..., oth[1]] <= p[5])
            t = np.where(ok, t, np.inf)
        else:
            v0, v1, v2 = p[0:3], p[3:6], p[6:9]
            e1, e2 = v1 - v0, v2 - v0
            pv = np.cross(d, e2)
            det = pv @ e1
            with np.errstate(divide="ignore", invalid="ignore"):
                inv = 1 / det
                tv = -v0
                uu = (pv @ tv) * inv
                qv = np.cross(tv, e1)
                vv = (d @ qv) * inv
                t = (qv @ e2) * inv
            ok = (uu >= 0) & (uu <= 1) & (vv >= 0) & (uu + vv <= 1)
            t = np.where(ok, t, np.inf)
        t = np.where(np.isfinite(t) & (t > 1e-4), t, np.inf)
        T[j] = t
    order = np.sort(T, axis=0)
    best = np.argmin(T, axis=0)
    return order[0], np.where(np.isfinite(order[0]), best, -1), order[1] if len(types) > 1 else np.full((H, W), np.inf)


@pytest.mark.parametrize("S,seed", [(40, 1), (200, 2)])
def test_random_scene_vs_float64_reference(S, seed):
    W, H = 96, 54
    types, P = synth.ray_scene(S, seed=seed)
    c = cam(W, H, 60.0)
    rgb, hid, calls, _ = oracle.ray_render(W, H, types, P, c, ALB)
    assert calls == W * H * S
    tb, ref_id, t2 = np_hits(types, P, W, H, c)
    clear = np.isinf(tb) | (t2 - tb > 1e-3 * tb)  # not a near tie
    assert clear.mean() > 0.95
    assert np.array_equal(hid[clear], ref_id[clear])
    assert np.all(rgb[hid < 0] == 0)
    assert np.all(rgb[hid >= 0] >= 0.1 - 1e-7)


def test_ray_rows_and_threads_consistent():
    W, H, S = 64, 36, 150
    types, P = synth.ray_scene(S, seed=5)
    c = cam(W, H, 60.0)
    a = oracle.ray_render(W, H, types, P, c, ALB, threads=1)
    b = oracle.ray_render(W, H, types, P, c, ALB, threads=oracle.max_threads())
    assert np.array_equal(a[0], b[0]) and np.array_equal(a[1], b[1])
    part = oracle.ray_render(W, H, types, P, c, ALB, row0=10, nrows=7)
    assert np.array_equal(part[1], a[1][10:17]) and np.array_equal(part[0], a[0][10:17])

"""GPU parity for config 3 (ray tracer over polymorphic shapes) vs the CPU oracle.

Both sides evaluate the same fp32 operation sequence (explicit fmaf, no
contraction, IEEE sqrt/div), so the hit-id image and the RGB image are
bit-identical; the full 1920x1080 x 10k-shape frame is checked on sampled rows.
"""
import numpy as np
import pytest
import torch

import oracle
import synth
from paper_conf_asplos_zhangar21_b200 import vf
from paper_conf_asplos_zhangar21_b200.ray import Ray

pytestmark = pytest.mark.gpu
VARIANTS = ["cuda", "sharedoa", "coal", "typeptr"]


@pytest.fixture(scope="module")
def ctx():
    c = vf.Ctx(0, cuda_heap_bytes=2 << 30)
    yield c
    c.close()


@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("W,H,S", [(96, 54, 300), (160, 90, 1000), (33, 17, 257)])
def test_ray_parity(ctx, variant, W, H, S):
    types, P = synth.ray_scene(S, seed=7)
    cam = synth.ray_camera(W, H)
    rgb_ref, hid_ref, _, _ = oracle.ray_render(W, H, types, P, cam, synth.RAY_ALBEDO, threads=oracle.max_threads())
    r = Ray(ctx, types, P, variant)
    rgb, hid = r.render(W, H, cam)
    assert np.array_equal(hid.cpu().numpy(), hid_ref)
    assert np.array_equal(rgb.cpu().numpy(), rgb_ref)
    assert ctx.verify(vf.APP_RAY, r.v, r.objs) == 0


def test_ray_strips_multi_rank_layout(ctx):
    """Round-robin 8-row strips over 3 emulated ranks reassemble the frame exactly."""
    W, H, S = 64, 45, 200
    types, P = synth.ray_scene(S, seed=3)
    cam = synth.ray_camera(W, H)
    r = Ray(ctx, types, P, "typeptr")
    full_rgb, full_hid = r.render(W, H, cam)
    acc_hid = torch.full((H, W), -7, dtype=torch.int32, device="cuda")
    for rank in range(3):
        _, hid = r.render_frame(W, H, cam, rank, 3)
        mask = torch.zeros(H, dtype=torch.bool, device="cuda")
        for r0, n in r.strips(H, rank, 3):
            mask[r0:r0 + n] = True
        acc_hid[mask] = hid[mask]
    assert torch.equal(acc_hid, full_hid)


@pytest.mark.slow
def test_ray_full_frame_sampled_rows(ctx):
    """BASELINE config 3 (1920x1080, 10k shapes), bench launch configuration; oracle on 24 sampled rows."""
    W, H, S = 1920, 1080, 10000
    types, P = synth.ray_scene(S, seed=7)
    cam = synth.ray_camera(W, H)
    r = Ray(ctx, types, P, "typeptr")
    rgb, hid = r.render(W, H, cam)
    rgb, hid = rgb.cpu().numpy(), hid.cpu().numpy()
    for row in np.linspace(0, H - 1, 24).astype(int):
        rr, hh, _, _ = oracle.ray_render(W, H, types, P, cam, synth.RAY_ALBEDO, row0=int(row), nrows=1,
                                         threads=oracle.max_threads())
        assert np.array_equal(hh[0], hid[row]) and np.array_equal(rr[0], rgb[row])


def _edge_scene():
    """Shapes that sit on the edges of the hoisted fast path's operand ranges
    (app_ray.cu hit_rays / fast_domain), mixed into a random scene so tiles
    hold both: the fast path must give hit_t's results, or flag the tile for
    the per-operation IEEE re-run."""
    types, P = synth.ray_scene(700, seed=11)
    extra = []
    # tangent sphere: the centre ray (odd W, H: d = (0, 0, -1)) has disc == 0 exactly
    extra.append((1, [1.0, 0.0, -10.0, 1.0]))
    # grazing spheres: disc tiny positive / tiny negative for the centre ray
    extra.append((1, [2.0, 0.0, -20.0, 2.0 * (1 + 2 ** -23)]))
    extra.append((1, [3.0, 0.0, -30.0, 3.0 * (1 - 2 ** -23)]))
    # spheres outside the fast domain (|centre| > 2^40): tile re-run
    extra.append((1, [0.0, 0.0, -3.0e12, 1.0e12]))
    # triangle in the plane y = 0 (contains the origin): det == 0 for the d.y == 0 row
    extra.append((3, [-1.0, 0.0, -5.0, 1.0, 0.0, -5.0, 0.0, 0.0, -8.0]))
    # triangle with huge vertices (outside the fast domain)
    extra.append((3, [-1e10, -1e10, -1e11, 1e10, -1e10, -1e11, 0.0, 1e10, -1e11]))
    # rects: p == 0 (t == 0 -> miss), tiny |p| (outside [2^-60, 2^60]), one per axis
    extra.append((2, [0, 0.0, -1.0, 1.0, -9.0, -1.0]))
    extra.append((2, [1, 1e-30, -1.0, 1.0, -9.0, -1.0]))
    extra.append((2, [2, -4.0, -0.5, 0.5, -0.5, 0.5]))
    extra.append((2, [0, 1e25, -1.0, 1.0, -9.0, -1.0]))
    # planes: the ground (shape 0) plus h == 0 and a tiny h
    extra.append((0, [0.0]))
    extra.append((0, [1e-30]))
    t2 = np.array([t for t, _ in extra], np.uint32)
    P2 = np.zeros((len(extra), 12), np.float32)
    for i, (_, q) in enumerate(extra):
        P2[i, :len(q)] = q
    # interleave: the special shapes land in several tiles and runs
    types = np.concatenate([types[:300], t2[:6], types[300:], t2[6:]])
    P = np.concatenate([P[:300], P2[:6], P[300:], P2[6:]])
    return types, P


@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("W,H", [(65, 37), (33, 17)])
def test_ray_fast_path_edges(ctx, variant, W, H):
    types, P = _edge_scene()
    cam = synth.ray_camera(W, H)
    rgb_ref, hid_ref, _, _ = oracle.ray_render(W, H, types, P, cam, synth.RAY_ALBEDO, threads=oracle.max_threads())
    r = Ray(ctx, types, P, variant)
    rgb, hid = r.render(W, H, cam)
    assert np.array_equal(hid.cpu().numpy(), hid_ref)
    assert np.array_equal(rgb.cpu().numpy(), rgb_ref)


@pytest.mark.parametrize("variant", ["coal", "typeptr"])
@pytest.mark.parametrize("parts", [1, 3, 16])
def test_ray_shape_parts(ctx, variant, parts):
    """The direct kernel over 1 / 3 / 16 shape parts (in-kernel shading vs
    atomicMin of the keys + k_ray_shade) gives the oracle's frame."""
    W, H, S = 200, 120, 2600
    types, P = synth.ray_scene(S, seed=5)
    cam = synth.ray_camera(W, H)
    rgb_ref, hid_ref, _, _ = oracle.ray_render(W, H, types, P, cam, synth.RAY_ALBEDO, threads=oracle.max_threads())
    r = Ray(ctx, types, P, variant)
    vf.set_tuning("ray_parts", parts)
    try:
        rgb, hid = r.render(W, H, cam)
    finally:
        vf.set_tuning("ray_parts", -1)
    assert np.array_equal(hid.cpu().numpy(), hid_ref)
    assert np.array_equal(rgb.cpu().numpy(), rgb_ref)


@pytest.mark.parametrize("variant", VARIANTS)
def test_ray_empty_and_single_shape_scenes(ctx, variant):
    """No shapes at all (every pixel a miss) and a one-shape scene: the oracle's frame."""
    W, H = 17, 9
    cam = synth.ray_camera(W, H)
    for S in (0, 1):
        types, P = synth.ray_scene(S, seed=2)
        rgb_ref, hid_ref, _, _ = oracle.ray_render(W, H, types, P, cam, synth.RAY_ALBEDO)
        r = Ray(ctx, types, P, variant)
        rgb, hid = r.render(W, H, cam)
        assert np.array_equal(hid.cpu().numpy(), hid_ref)
        assert np.array_equal(rgb.cpu().numpy(), rgb_ref)

"""GPU parity for config 5 collision (cutoff-grid softened gravity + mutual-nearest
merging over polymorphic Star / Planet / Dust bodies; readings G18 / G19) vs
the CPU oracle: fp32 with explicit fmaf on both sides, expected bit-exact and
asserted bit-exact (a merge decision is a threshold, so any drift would show
as a different absorbed set); every variant; emulated id-block ranks; the
full 16M-body configuration the bench times."""
import numpy as np
import pytest

import oracle
import synth
from paper_conf_asplos_zhangar21_b200 import vf
from paper_conf_asplos_zhangar21_b200.collide import Collide

pytestmark = pytest.mark.gpu
VARIANTS = ["cuda", "sharedoa", "coal", "typeptr"]


@pytest.fixture(scope="module")
def ctx():
    c = vf.Ctx(0, cuda_heap_bytes=4 << 30)
    yield c
    c.close()


def _run(ctx, s, steps, variant):
    c = Collide(ctx, s, variant)
    for _ in range(steps):
        c.step()
    return c


def _same(c, p_ref, v_ref):
    p, v = c.positions(), c.velocities()
    assert np.array_equal(p.view(np.uint32), p_ref.view(np.uint32))
    assert np.array_equal(v.view(np.uint32), v_ref[:, :3].view(np.uint32))


@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("N,steps,rm", [(1, 2, 0.05), (2, 3, 0.05), (1000, 4, 0.1), (3 * 4096 + 77, 3, 0.12)])
def test_collide_parity(ctx, variant, N, steps, rm):
    s = synth.collide_system(N, seed=N, rm=rm)
    p_ref, v_ref, calls, _ = oracle.collide_run(s, steps, threads=oracle.max_threads())
    c = _run(ctx, s, steps, variant)
    _same(c, p_ref, v_ref)
    assert c.calls() == calls
    assert ctx.verify(vf.APP_COLLIDE, c.v, c.objs) == 0


@pytest.mark.parametrize("variant", ["cuda", "typeptr"])
def test_collide_many_merges_and_outside_grid(ctx, variant):
    """Dense soup with a large merge radius (a sizeable fraction merges every
    step, chains of nearest neighbours), bodies beyond the grid clamped into
    the edge cells; mass is conserved."""
    s = synth.collide_system(20000, seed=3, per_cell=6.0, rm=0.3)
    s["pos"][:300, 0] = -0.7
    s["pos"][300:600, 2] = np.float32(s["G"]) + 0.4
    p_ref, v_ref, calls, _ = oracle.collide_run(s, 5, threads=oracle.max_threads())
    assert (p_ref[:, 3] == 0).sum() > 1000
    c = _run(ctx, s, 5, variant)
    _same(c, p_ref, v_ref)
    assert c.calls() == calls
    p = c.positions()
    m0 = s["pos"][:, 3].astype(np.float64).sum()
    assert abs(p[:, 3].astype(np.float64).sum() - m0) <= 1e-5 * m0


def test_collide_single_cell_is_all_pairs(ctx):
    """G = 1 with rc covering the box and rm = 0: every body sees every other,
    i.e. the all-pairs N-body step; equals the oracle bit for bit."""
    s = synth.collide_system(700, seed=4, rm=0.0)
    s["G"] = 1
    s["rc"] = np.float32(1e6)
    p_ref, v_ref, _, _ = oracle.collide_run(s, 3)
    c = _run(ctx, s, 3, "coal")
    _same(c, p_ref, v_ref)


def test_collide_head_on_pair(ctx):
    s = synth.collide_system(2, seed=1, rm=0.05)
    s["G"] = 2
    s["types"][:] = 1
    s["pos"][:] = [[0.5, 0.5, 0.5, 2.0], [0.53, 0.5, 0.5, 1.0]]
    s["vel"][:] = [[0.1, 0, 0, 0], [-0.2, 0, 0, 0]]
    p_ref, v_ref, _, _ = oracle.collide_run(s, 2)
    c = _run(ctx, s, 2, "typeptr")
    _same(c, p_ref, v_ref)
    assert c.positions()[1, 3] == 0 and c.positions()[0, 3] == 3.0


@pytest.mark.parametrize("world", [2, 3])
def test_collide_block_shards_reassemble(ctx, world):
    """Emulated ranks: each owns an id block and dispatches its bodies over the
    replicated grid; after update the owned slices of Pm / Vm / near are
    stitched, after merge those of P (what the all-gathers do) -> the oracle."""
    N, steps = 5000, 4
    s = synth.collide_system(N, seed=11, rm=0.2)
    p_ref, v_ref, calls, _ = oracle.collide_run(s, steps)
    ranks = [Collide(ctx, s, "typeptr", r, world, exchange=False) for r in range(world)]

    def stitch(name):
        full = getattr(ranks[0], name).clone()
        for c in ranks:
            full[c.lo:c.hi] = getattr(c, name)[c.lo:c.hi]
        for c in ranks:
            getattr(c, name).copy_(full)

    for _ in range(steps):
        for c in ranks:
            c.update()
        for name in ("Pm", "Vm", "near"):
            stitch(name)
        for c in ranks:
            c.merge()
        stitch("P")
    p = ranks[0].positions()
    assert np.array_equal(p.view(np.uint32), p_ref.view(np.uint32))
    v = np.concatenate([c.velocities() for c in ranks])
    assert np.array_equal(v.view(np.uint32), v_ref[:, :3].view(np.uint32))
    assert sum(c.calls() for c in ranks) == calls


def test_collide_full_size_16M(ctx):
    """BASELINE config 5 at its full size (16,777,216 bodies, the bench's
    launch configuration): 2 steps bit-exact vs the oracle on every body."""
    N = 1 << 24
    s = synth.collide_system(N, seed=13)
    p_ref, v_ref, calls, _ = oracle.collide_run(s, 2, threads=oracle.max_threads())
    c = _run(ctx, s, 2, "typeptr")
    _same(c, p_ref, v_ref)
    assert c.calls() == calls
    assert ctx.verify(vf.APP_COLLIDE, c.v, c.objs) == 0

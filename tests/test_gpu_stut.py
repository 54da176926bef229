"""GPU parity for config 5 STUT (spring-node structure, reading G17) vs the CPU
oracle: fp32 with the same explicit-fmaf formula on both sides -> bit-exact
positions, velocities and the identical set of broken springs; every variant;
row-slab sharding with ghost springs."""
import numpy as np
import pytest

import oracle
import synth
from paper_conf_asplos_zhangar21_b200 import vf
from paper_conf_asplos_zhangar21_b200.stut import Stut

pytestmark = pytest.mark.gpu
VARIANTS = ["cuda", "sharedoa", "coal", "typeptr"]


@pytest.fixture(scope="module")
def ctx():
    c = vf.Ctx(0, cuda_heap_bytes=2 << 30)
    yield c
    c.close()


@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("W,H,steps,vp", [(2, 1, 5, 1.0), (17, 9, 60, 4.0), (130, 67, 40, 6.0)])
def test_stut_parity(ctx, variant, W, H, steps, vp):
    w = synth.stut_lattice(W, H, seed=W + H, v_pull=vp)
    pos_ref, vel_ref, br_ref, _ = oracle.stut_run(w, steps, threads=oracle.max_threads())
    s = Stut(ctx, w, variant)
    for _ in range(steps):
        s.step()
    assert np.array_equal(s.positions().view(np.uint32), pos_ref.view(np.uint32))
    assert np.array_equal(s.velocities().view(np.uint32), vel_ref.view(np.uint32))
    assert np.array_equal(s.broken(), br_ref)
    if W > 100:
        assert br_ref.any()  # the fracture path is exercised
    assert ctx.verify(vf.APP_STUT, s.v, s.nodes) == 0
    assert ctx.verify(vf.APP_STUT, s.v, s.springs) == 0


def test_stut_row_slabs_reassemble(ctx):
    """3 emulated ranks (row slabs + ghost springs); positions stitched after
    every step as the all-gather does -> the oracle's state."""
    w = synth.stut_lattice(40, 23, seed=3, v_pull=5.0)
    steps, world = 50, 3
    pos_ref, vel_ref, br_ref, _ = oracle.stut_run(w, steps)
    ranks = [Stut(ctx, w, "typeptr", r, world, exchange=False) for r in range(world)]
    for _ in range(steps):
        for s in ranks:
            s.step()
        full = ranks[0].pos.clone()
        for s in ranks:
            full[s.lo:s.hi] = s.pos[s.lo:s.hi]
        for s in ranks:
            s.pos.copy_(full)
    assert np.array_equal(ranks[0].positions(), pos_ref)
    assert np.array_equal(np.concatenate([s.velocities() for s in ranks]), vel_ref)
    br = np.zeros_like(br_ref)
    for s in ranks:
        own = s.spring_ids[(w["a"][s.spring_ids] >= s.lo) & (w["a"][s.spring_ids] < s.hi)]
        br[own] = s.broken()[own]
    assert np.array_equal(br, br_ref)
    assert sum(s.n_own_springs for s in ranks) == len(w["a"])

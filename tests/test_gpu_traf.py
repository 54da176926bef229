"""GPU parity for config 5 TRAF (Nagel-Schreckenberg over polymorphic cells / vehicles)
vs the CPU oracle: integer state, bit-exact, every variant; plus ring sharding."""
import numpy as np
import pytest

import oracle
import synth
from paper_conf_asplos_zhangar21_b200 import vf
from paper_conf_asplos_zhangar21_b200.traf import Traf

pytestmark = pytest.mark.gpu
VARIANTS = ["cuda", "sharedoa", "coal", "typeptr"]


@pytest.fixture(scope="module")
def ctx():
    c = vf.Ctx(0, cuda_heap_bytes=4 << 30)
    yield c
    c.close()


@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("R,L,steps", [(13, 256, 40), (64, 1024, 60)])
def test_traf_parity(ctx, variant, R, L, steps):
    w = synth.traf_world(R, L, seed=R + L)
    pos_ref, v_ref, _ = oracle.traf_run(w, steps, threads=oracle.max_threads())
    t = Traf(ctx, w, variant)
    for _ in range(steps):
        t.step()
    pos, vel = t.state()
    assert np.array_equal(pos, pos_ref) and np.array_equal(vel, v_ref)
    assert ctx.verify(vf.APP_TRAF, t.v, t.vehs) == 0
    assert ctx.verify(vf.APP_TRAF, t.v, t.cells) == 0


def test_traf_ring_shards_reassemble(ctx):
    """3 emulated ranks, each owning a block of whole rings, give the oracle's state."""
    w = synth.traf_world(10, 512, seed=5)
    pos_ref, v_ref, _ = oracle.traf_run(w, 30)
    pos = np.zeros_like(pos_ref)
    vel = np.zeros_like(v_ref)
    for rank in range(3):
        t = Traf(ctx, w, "typeptr", rank, 3)
        for _ in range(30):
            t.step()
        p, v = t.state()
        pos[t.vid_global] = p
        vel[t.vid_global] = v
    assert np.array_equal(pos, pos_ref) and np.array_equal(vel, v_ref)

"""GPU parity for config 5 GEN (Generations CA over polymorphic Dead/Alive/Dying cells)
vs the CPU oracle: bit-exact state, counters and per-cell type, every variant."""
import numpy as np
import pytest

import oracle
import synth
from paper_conf_asplos_zhangar21_b200 import apps, vf

pytestmark = pytest.mark.gpu
VARIANTS = ["cuda", "sharedoa", "coal", "typeptr"]


@pytest.fixture(scope="module")
def ctx():
    c = vf.Ctx(0, cuda_heap_bytes=4 << 30)
    yield c
    c.close()


@pytest.mark.parametrize("fused", [True, False])
@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("W,H,gens,rule,torus", [(256, 256, 60, ("2", "345", 4), False),
                                                 (77, 45, 40, ("3", "23", 2), False),
                                                 (64, 64, 33, ("34", "34", 6), True)])
def test_gen_parity(ctx, variant, W, H, gens, rule, torus, fused):
    born, surv, C = rule
    s0 = synth.soup(W, H, seed=42)
    st_ref, ctr_ref, hist_ref, _ = oracle.gen_run(W, H, s0, gens, born, surv, C, torus)
    g = apps.Gen(ctx, W, H, s0, variant, born, surv, C, torus)
    for _ in range(gens):
        g.gen(fused=fused)
    st = g.current.cpu().numpy()
    assert np.array_equal(st, st_ref)
    ctr, typ = g.counters()
    assert np.array_equal(ctr.cpu().numpy().view(np.uint16), ctr_ref)
    assert np.array_equal(typ.cpu().numpy(), np.minimum(st_ref, 2))
    assert list(np.bincount(st, minlength=C)) == list(hist_ref)
    assert ctx.verify(vf.APP_GEN, g.v, g.grid) == 0

"""GPU parity for config 1 (Game of Life over polymorphic cells) vs the CPU oracle: bit-exact
state, per-cell counters and population per generation, every variant."""
import numpy as np
import pytest
import torch

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
@pytest.mark.parametrize("W,H,gens,torus", [(256, 256, 100, False), (37, 23, 30, False), (64, 48, 25, True)])
def test_gol_parity(ctx, variant, W, H, gens, torus, fused):
    g0 = synth.soup(W, H, seed=42)
    st_ref, ctr_ref, pop_ref, _ = oracle.gol_run(W, H, g0, gens, torus)
    g = apps.Gol(ctx, W, H, g0, variant, torus)
    pops = []
    for _ in range(gens):
        g.gen(fused=fused)
        pops.append(int(g.current.sum().item()))
    assert np.array_equal(g.current.cpu().numpy(), st_ref)
    ctr, typ = g.counters()
    assert np.array_equal(ctr.cpu().numpy().view(np.uint16), ctr_ref)
    assert np.array_equal(typ.cpu().numpy(), st_ref)
    assert pops == list(pop_ref)
    assert ctx.verify(vf.APP_GOL, g.v, g.grid) == 0


def test_gol_f3_fixture(ctx):
    W = H = 16
    g0 = synth.place(W, H, [(2, 1), (3, 2), (1, 3), (2, 3), (3, 3), (12, 1), (13, 1), (12, 2), (13, 2),
                            (2, 12), (3, 12), (4, 12)])
    for variant in VARIANTS:
        g = apps.Gol(ctx, W, H, g0, variant)
        for gen in range(1, 33):
            g.gen()
            assert int(g.current.sum().item()) == 12
        s = g.current.cpu().numpy().reshape(H, W)
        for (x, y) in [(2, 1), (3, 2), (1, 3), (2, 3), (3, 3)]:
            assert s[y + 8, x + 8] == 1  # 32 gens = 8 glider periods


def test_gol_cuda_graph_capture(ctx):
    """The 100-generation loop captured once as a CUDA graph gives the same result."""
    W = H = 256
    g0 = synth.soup(W, H, seed=42)
    st_ref, ctr_ref, _, _ = oracle.gol_run(W, H, g0, 100)
    g = apps.Gol(ctx, W, H, g0, "typeptr")
    s = torch.cuda.Stream()
    torch.cuda.synchronize()
    graph = torch.cuda.CUDAGraph()
    with torch.cuda.graph(graph, stream=s):
        for _ in range(100):
            g.gen(stream=s)
    graph.replay()
    torch.cuda.synchronize()
    assert np.array_equal(g.current.cpu().numpy(), st_ref)


@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("W,H,gens,torus", [(256, 256, 100, False), (37, 23, 31, False), (64, 48, 25, True),
                                            (1024, 1024, 7, False)])
@pytest.mark.parametrize("cluster", [1, 0])
def test_gol_persistent_run(ctx, variant, W, H, gens, torus, cluster):
    """vf_gol_run: all generations in one launch == the oracle. cluster = 1: grids
    of <= 2^17 cells run in one thread-block cluster (DSMEM state rows); larger
    grids and cluster = 0 use the cooperative grid-barrier kernel (at 1024^2 each
    thread owns several cells)."""
    vf.set_tuning("cluster", cluster)
    g0 = synth.soup(W, H, seed=43)
    st_ref, ctr_ref, _, _ = oracle.gol_run(W, H, g0, gens, torus)
    g = apps.Gol(ctx, W, H, g0, variant, torus)
    g.run(gens)
    assert np.array_equal(g.current.cpu().numpy(), st_ref)
    ctr, typ = g.counters()
    assert np.array_equal(ctr.cpu().numpy().view(np.uint16), ctr_ref)
    assert np.array_equal(typ.cpu().numpy(), st_ref)
    # split runs continue where the last one stopped
    g2 = apps.Gol(ctx, W, H, g0, variant, torus)
    g2.run(gens // 2)
    g2.run(gens - gens // 2)
    assert np.array_equal(g2.current.cpu().numpy(), st_ref)
    vf.set_tuning("cluster", 0)

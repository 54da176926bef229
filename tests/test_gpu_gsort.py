"""Grid-level type sort of the dispatch list for heavy methods (vf_set_tuning
"gsort" = 1): same results as the oracle for every app with
heavy methods (N-body update, graph BFS / CC / PageRank incl. multi-chunk work
entries whose bodies read their ORIGINAL index, collision update), including
null / untypable entries dropped from the sorted list."""
import numpy as np
import pytest

import oracle
import synth
from paper_conf_asplos_zhangar21_b200 import vf

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def ctx():
    c = vf.Ctx(0, cuda_heap_bytes=1 << 30)
    vf.set_tuning("gsort", 1)
    yield c
    vf.set_tuning("gsort", -1)
    c.close()


@pytest.mark.parametrize("variant", ["coal", "typeptr"])
def test_gsort_nbody(ctx, variant):
    from paper_conf_asplos_zhangar21_b200.nbody import Nbody
    s = synth.nbody_system(20000, seed=9)
    p_ref, v_ref, _ = oracle.nbody_run(s, 2)
    nb = Nbody(ctx, s, variant)
    for _ in range(2):
        nb.step()
    assert np.array_equal(nb.positions().view(np.uint32), p_ref.view(np.uint32))
    assert np.array_equal(nb.velocities().view(np.uint32), v_ref.view(np.uint32))


@pytest.mark.parametrize("chunk", [256, 7])
@pytest.mark.parametrize("variant", ["coal", "typeptr"])
def test_gsort_graph(ctx, variant, chunk):
    from paper_conf_asplos_zhangar21_b200.graph import Graph
    offs, col = synth.rmat_graph(15, seed=15)
    t = synth.vertex_types(offs)
    src = int(np.argmax(np.diff(offs.astype(np.int64))))
    depth, levels, _, _ = oracle.graph_bfs(offs, col, t, src)
    label, iters, _, _ = oracle.graph_cc(offs, col, t)
    rank, _ = oracle.graph_pr(offs, col, t, iters=20)
    g = Graph(ctx, offs, col, variant, chunk=chunk)
    for mode in ("topdown", "hybrid", "bits"):
        d, lv, _ = g.bfs(src, mode=mode)
        assert np.array_equal(d.cpu().numpy(), depth) and lv == levels
    lab, it, _ = g.cc()
    assert np.array_equal(lab.cpu().numpy().view(np.uint32), label) and it == iters
    r, _ = g.pagerank(20)
    np.testing.assert_allclose(r.cpu().numpy(), rank, rtol=1e-5, atol=0)


@pytest.mark.parametrize("variant", ["coal", "typeptr"])
def test_gsort_collide(ctx, variant):
    from paper_conf_asplos_zhangar21_b200.collide import Collide
    s = synth.collide_system(20000, seed=11, rm=0.2)
    p_ref, v_ref, calls, _ = oracle.collide_run(s, 3)
    c = Collide(ctx, s, variant)
    for _ in range(3):
        c.step()
    assert np.array_equal(c.positions().view(np.uint32), p_ref.view(np.uint32))
    assert np.array_equal(c.velocities().view(np.uint32), v_ref[:, :3].view(np.uint32))
    assert c.calls() == calls


def test_gsort_nulls_and_untypable(ctx):
    """nulls are skipped and a pointer neither rule types is dropped, as in the
    unsorted dispatch (N-body bodies with a few entries nulled out)."""
    import torch
    from paper_conf_asplos_zhangar21_b200.nbody import Nbody
    s = synth.nbody_system(10000, seed=3)
    nb = Nbody(ctx, s, "typeptr")
    objs = nb.objs.clone()
    objs[::97] = 0
    st = ctx.dispatch_raw(nb.v, vf.APP_NBODY, vf.NBODY_UPDATE, objs.data_ptr(), objs.numel(), nb._args(),
                          vf._stream(None))
    assert st == 0
    vf.set_tuning("gsort", 0)  # per-CTA-tile sort only
    nb2 = Nbody(ctx, s, "typeptr")
    objs2 = nb2.objs.clone()
    objs2[::97] = 0
    ctx.dispatch_raw(nb2.v, vf.APP_NBODY, vf.NBODY_UPDATE, objs2.data_ptr(), objs2.numel(), nb2._args(),
                     vf._stream(None))
    vf.set_tuning("gsort", 1)
    torch.cuda.synchronize()
    assert torch.equal(nb.p[1], nb2.p[1])

"""GPU parity for the GraphChi-vEN apps (virtual edges + vertices; Table 2
P:1566-1588) vs the CPU oracle (oracle/graph_en.cpp).

BFS depths and CC labels (and the CC iteration count) are unique -> bit-exact.
PageRank: Leaf / Low vertices sum their in-edges in oracle order, Mid / Hub
with unrolled accumulators and multi-chunk partials -> 1e-5 relative
(BASELINE north_star). Every variant; RMAT graphs spanning all four vertex
types and both edge types; C = 7 makes most vertices multi-chunk. Edge objects
are checked by brute-force type identity and by reading every arc's (src, dst)
back through its virtual get().
"""
import numpy as np
import pytest
import torch

import oracle
import synth
from paper_conf_asplos_zhangar21_b200 import vf
from paper_conf_asplos_zhangar21_b200.graph_en import GraphEN

pytestmark = pytest.mark.gpu
VARIANTS = ["cuda", "sharedoa", "coal", "typeptr"]


@pytest.fixture(scope="module")
def ctx():
    c = vf.Ctx(0, cuda_heap_bytes=4 << 30)
    yield c
    c.close()


@pytest.fixture(scope="module", params=[12, 16])
def rmat(request):
    offs, col = synth.rmat_graph(request.param, seed=request.param + 100)
    types = synth.vertex_types(offs)
    assert len(np.unique(types)) == 4
    src = int(np.argmax(np.diff(offs.astype(np.int64))))
    depth, levels, vc, ec, _ = oracle.graph_en_bfs(offs, col, types, src)
    label, iters, _, _, _ = oracle.graph_en_cc(offs, col, types)
    rank, _ = oracle.graph_en_pr(offs, col, types, iters=20)
    et = oracle.graph_en_edge_types(offs, types)
    assert set(np.unique(et)) == {0, 1}
    return dict(offs=offs, col=col, src=src, depth=depth, levels=levels, vc=vc, ec=ec, label=label, iters=iters,
                rank=rank, etypes=et)


@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("chunk", [256, 7])
def test_graph_en_parity(ctx, rmat, variant, chunk):
    g = GraphEN(ctx, rmat["offs"], rmat["col"], variant, chunk=chunk)
    offs, col = rmat["offs"], rmat["col"]
    # edge objects: the oracle's edge classes, brute-force type identity, endpoints via virtual get()
    assert np.array_equal(g.etypes.cpu().numpy().astype(np.uint32), rmat["etypes"])
    assert ctx.verify(vf.APP_EDGE, g.v, g.out_edges) == 0
    assert ctx.verify(vf.APP_EDGE, g.v, g.in_edges) == 0
    assert ctx.verify(vf.APP_GRAPH_EN, g.v, g.vobj) == 0
    ep = g.edge_endpoints().cpu().numpy().view(np.uint64)
    deg = np.diff(offs.astype(np.int64))
    srcs = np.repeat(np.arange(len(offs) - 1, dtype=np.uint64), deg)
    assert np.array_equal(ep >> np.uint64(32), srcs)
    assert np.array_equal(ep & np.uint64(0xFFFFFFFF), col.astype(np.uint64))
    # BFS
    depth, levels, vc = g.bfs(rmat["src"])
    assert np.array_equal(depth.cpu().numpy(), rmat["depth"])
    assert levels == rmat["levels"] and vc >= rmat["vc"] and g.edge_calls_bfs() == rmat["ec"]
    # CC (twice: re-initialised)
    for _ in range(2):
        label, iters, _, ec = g.cc()
        assert np.array_equal(label.cpu().numpy().view(np.uint32), rmat["label"])
        assert iters == rmat["iters"] and ec == iters * 2 * len(col)
    # PageRank
    rank, _, _ = g.pagerank(20)
    r = rank.cpu().numpy()
    np.testing.assert_allclose(r, rmat["rank"], rtol=1e-5, atol=0)
    assert int(g.counter.abs().sum()) == 0
    assert abs(float(r.astype(np.float64).sum()) - 1.0) < 1e-4


@pytest.mark.parametrize("variant", ["coal", "typeptr"])
def test_graph_en_fallback_untagged_and_foreign(ctx, variant):
    """Edge pointers the rule cannot type (TP: tag stripped; COAL: the range
    table withheld) fall back to the embedded vTable* and give the same result."""
    offs, col = synth.rmat_graph(11, seed=5)
    types = synth.vertex_types(offs)
    label_ref, iters_ref, _, _, _ = oracle.graph_en_cc(offs, col, types)
    rank_ref, _ = oracle.graph_en_pr(offs, col, types, iters=20)
    g = GraphEN(ctx, offs, col, variant, chunk=16)
    if variant == "typeptr":
        mask = (1 << vf.VA_BITS) - 1
        g.in_edges = g.in_edges & mask  # untagged -> tag 0 -> fallback
    else:
        g.er.K, g.er.P = 1, 1  # only the first range is known -> the rest miss
    label, iters, _, _ = g.cc()
    assert np.array_equal(label.cpu().numpy().view(np.uint32), label_ref) and iters == iters_ref
    rank, _, _ = g.pagerank(20)
    np.testing.assert_allclose(rank.cpu().numpy(), rank_ref, rtol=1e-5, atol=0)


def test_graph_en_f6_fixture(ctx):
    offs, col = synth.csr_from_edges(6, [(0, 1), (1, 2), (2, 3), (4, 5)])
    for variant in VARIANTS:
        g = GraphEN(ctx, offs, col, variant)
        depth, _, _ = g.bfs(0)
        assert list(depth.cpu().numpy()) == [0, 1, 2, 3, -1, -1]
        label, _, _, _ = g.cc()
        assert list(label.cpu().numpy()) == [0, 0, 0, 0, 4, 4]
        torch.cuda.synchronize()


@pytest.mark.parametrize("variant", VARIANTS)
def test_graph_en_degenerate_graphs(ctx, variant):
    """No edges at all (every vertex dangling: PageRank stays uniform), and a
    single edge plus isolated vertices: same results as the oracle."""
    for V, edges in ((5, []), (6, [(2, 4)])):
        offs, col = synth.csr_from_edges(V, edges)
        types = synth.vertex_types(offs)
        g = GraphEN(ctx, offs, col, variant)
        assert g.A == 2 * len(edges)
        d_ref, lv_ref, _, _, _ = oracle.graph_en_bfs(offs, col, types, 2)
        depth, levels, _ = g.bfs(2)
        assert np.array_equal(depth.cpu().numpy(), d_ref) and levels == lv_ref
        l_ref, it_ref, _, _, _ = oracle.graph_en_cc(offs, col, types)
        label, iters, _, _ = g.cc()
        assert np.array_equal(label.cpu().numpy().view(np.uint32), l_ref) and iters == it_ref
        r_ref, _ = oracle.graph_en_pr(offs, col, types, iters=7)
        rank, _, _ = g.pagerank(7)
        np.testing.assert_allclose(rank.cpu().numpy(), r_ref, rtol=1e-6, atol=0)
        if not edges:
            np.testing.assert_allclose(r_ref, 1.0 / V, rtol=1e-6)

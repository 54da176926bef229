"""Pins for the oracle's GraphChi-vEN apps (virtual edges + vertices; Table 2
P:1566-1588, readings G32/G33).

The vEN apps compute the same function as the vE apps through a different
object structure (edge objects carrying the data, in-edge lists built by the
oracle itself), so they are pinned by: fixture F6 (hand-derived depths /
labels), the textbook queue BFS and union-find CC of test_oracle_graph.py,
scipy's connected components, the PageRank closed forms (star, cycle) and the
dense fixed-point solve, bit-equality with the (separately pinned) vE oracle,
and the exact per-app edge-call counts (BFS: sum of reached degrees; CC:
2 * arcs per iteration).
"""
import numpy as np
import pytest
from scipy.sparse import csr_matrix
from scipy.sparse.csgraph import connected_components

import oracle
import synth
from tests.test_oracle_graph import pr_dense, textbook_bfs, union_find_cc


def types_of(offs):
    return synth.vertex_types(offs)


def test_f6_fixture():
    offs, col = synth.csr_from_edges(6, [(0, 1), (1, 2), (2, 3), (4, 5)])
    depth, levels, vc, ec, _ = oracle.graph_en_bfs(offs, col, types_of(offs), 0)
    assert list(depth) == [0, 1, 2, 3, -1, -1]
    assert levels == 4 and vc == 4
    assert ec == 1 + 2 + 2 + 1  # out-degrees of 0, 1, 2, 3
    label, iters, vc, ec, _ = oracle.graph_en_cc(offs, col, types_of(offs))
    assert list(label) == [0, 0, 0, 0, 4, 4]
    assert ec == iters * 2 * len(col) and vc == iters * 6


def test_edge_types_follow_source_bucket():
    # a 300-leaf star: centre is a Hub (deg 300 >= 256), its 300 out-arcs are HubEdges
    offs, col = synth.csr_from_edges(301, [(0, i) for i in range(1, 301)])
    vt = types_of(offs)
    assert vt[0] == 3 and np.all(vt[1:] == 0)
    et = oracle.graph_en_edge_types(offs, vt)
    assert np.all(et[:300] == 1) and np.all(et[300:] == 0) and len(et) == 600


@pytest.mark.parametrize("scale", [8, 11])
def test_bfs_cc_vs_textbook(scale):
    offs, col = synth.rmat_graph(scale, seed=scale)
    t = types_of(offs)
    src = int(np.argmax(np.diff(offs.astype(np.int64))))
    depth, _, vc, ec, _ = oracle.graph_en_bfs(offs, col, t, src)
    ref = textbook_bfs(offs, col, src)
    assert np.array_equal(depth, ref)
    deg = np.diff(offs.astype(np.int64))
    assert vc == int((ref >= 0).sum()) and ec == int(deg[ref >= 0].sum())
    label, _, _, _, _ = oracle.graph_en_cc(offs, col, t)
    assert np.array_equal(label, union_find_cc(offs, col))


def test_cc_vs_scipy_scale14():
    offs, col = synth.rmat_graph(14, seed=4)
    V = len(offs) - 1
    A = csr_matrix((np.ones(len(col)), col.astype(np.int64), offs.astype(np.int64)), shape=(V, V))
    n, comp = connected_components(A, directed=False)
    label, iters, _, _, _ = oracle.graph_en_cc(offs, col, types_of(offs))
    # scipy numbers components arbitrarily: the label must be the min vertex id of the component
    mins = np.full(n, V, np.int64)
    np.minimum.at(mins, comp, np.arange(V))
    assert np.array_equal(label, mins[comp].astype(np.uint32))
    # same labels AND the same iteration count as the vE Jacobi oracle
    l2, it2, _, _ = oracle.graph_cc(offs, col, types_of(offs))
    assert np.array_equal(label, l2) and iters == it2


def test_pr_star_closed_form():
    offs, col = synth.csr_from_edges(4, [(0, 1), (0, 2), (0, 3)])
    r, _ = oracle.graph_en_pr(offs, col, types_of(offs), iters=200)
    d = 0.85
    assert abs(r[0] - (1 + d * 3) / (4 * (1 + d))) < 1e-6
    assert np.allclose(r[1:], (1 - r[0]) / 3, atol=1e-6)


def test_pr_cycle_uniform_every_iteration():
    k = 7
    offs, col = synth.csr_from_edges(k, [(i, (i + 1) % k) for i in range(k)])
    for it in (1, 5, 20):
        r, _ = oracle.graph_en_pr(offs, col, types_of(offs), iters=it)
        assert np.allclose(r, 1.0 / k, rtol=1e-6)


def test_pr_dense_solve_with_dangling():
    V = 9
    offs, col = synth.csr_from_edges(V, [(0, 1), (1, 2), (2, 0), (2, 3), (3, 4), (4, 5), (5, 3), (6, 7)])
    ref = pr_dense(offs, col, 0.85, V)
    r, _ = oracle.graph_en_pr(offs, col, types_of(offs), iters=300)
    assert np.allclose(r, ref, rtol=1e-5, atol=1e-7)


@pytest.mark.parametrize("iters", [1, 20])
def test_pr_bit_equal_to_vertex_only_oracle(iters):
    # in-edges visited in ascending source = CSR row order, same fp64 values and
    # dangling order -> bit-identical to oracle_graph_pr (pinned separately)
    offs, col = synth.rmat_graph(13, seed=6)
    t = types_of(offs)
    a, _ = oracle.graph_en_pr(offs, col, t, iters=iters)
    b, _ = oracle.graph_pr(offs, col, t, iters=iters)
    assert np.array_equal(a, b)
    assert abs(float(a.astype(np.float64).sum()) - 1.0) < 1e-5

"""Pins for the oracle's graph apps (config 4; Table 2, readings G20-G23).

Pinned against: fixture F6 (hand-derived depths / labels), a textbook queue BFS
and union-find CC written here, the Graph500 BFS validation rules, PageRank
closed forms (star, cycle), a dense linear solve of the PageRank fixed point
with dangling redistribution, and mass conservation.
"""
from collections import deque

import numpy as np
import pytest

import oracle
import synth


def types_of(offs):
    return synth.vertex_types(offs)


def textbook_bfs(offs, col, src):
    V = len(offs) - 1
    d = [-1] * V
    d[src] = 0
    q = deque([src])
    while q:
        v = q.popleft()
        for e in range(int(offs[v]), int(offs[v + 1])):
            u = int(col[e])
            if d[u] == -1:
                d[u] = d[v] + 1
                q.append(u)
    return np.array(d, np.int32)


def union_find_cc(offs, col):
    V = len(offs) - 1
    parent = list(range(V))

    def find(x):
        while parent[x] != x:
            parent[x] = parent[parent[x]]
            x = parent[x]
        return x
    for v in range(V):
        for e in range(int(offs[v]), int(offs[v + 1])):
            a, b = find(v), find(int(col[e]))
            if a != b:
                parent[max(a, b)] = min(a, b)
    roots = [find(v) for v in range(V)]
    # label = min vertex id in the component
    mins = {}
    for v, r in enumerate(roots):
        mins[r] = min(mins.get(r, v), v)
    return np.array([mins[r] for r in roots], np.uint32)


def test_f6_fixture():
    offs, col = synth.csr_from_edges(6, [(0, 1), (1, 2), (2, 3), (4, 5)])
    depth, levels, calls, _ = oracle.graph_bfs(offs, col, types_of(offs), 0)
    assert list(depth) == [0, 1, 2, 3, -1, -1]
    assert levels == 4 and calls == 4
    label, _, _, _ = oracle.graph_cc(offs, col, types_of(offs))
    assert list(label) == [0, 0, 0, 0, 4, 4]


@pytest.mark.parametrize("scale", [8, 11])
def test_bfs_cc_vs_textbook(scale):
    offs, col = synth.rmat_graph(scale, seed=scale)
    t = types_of(offs)
    src = int(np.argmax(np.diff(offs.astype(np.int64))))
    depth, _, calls, _ = oracle.graph_bfs(offs, col, t, src)
    ref = textbook_bfs(offs, col, src)
    assert np.array_equal(depth, ref)
    assert calls == int((ref >= 0).sum())
    label, _, _, _ = oracle.graph_cc(offs, col, t)
    assert np.array_equal(label, union_find_cc(offs, col))


def test_bfs_graph500_validation_scale14():
    offs, col = synth.rmat_graph(14, seed=3)
    t = types_of(offs)
    deg = np.diff(offs.astype(np.int64))
    src = int(np.argmax(deg))
    depth, _, _, _ = oracle.graph_bfs(offs, col, t, src)
    V = len(offs) - 1
    rows = np.repeat(np.arange(V), deg)
    du, dv = depth[rows], depth[col]
    assert depth[src] == 0
    both = (du >= 0) & (dv >= 0)
    assert np.all(np.abs(du[both] - dv[both]) <= 1)
    assert not np.any((du >= 0) ^ (dv >= 0))  # an arc never leaves the reached set
    # every reached vertex but src has a parent one level up
    has_parent = np.zeros(V, bool)
    np.logical_or.at(has_parent, rows[(du >= 0) & (dv == du - 1)], True)
    reached = depth >= 0
    assert np.all(has_parent[reached & (np.arange(V) != src)])
    label, _, _, _ = oracle.graph_cc(offs, col, t, threads=oracle.max_threads())
    assert np.array_equal(reached, label == label[src])


def pr_dense(offs, col, d, V):
    deg = np.diff(offs.astype(np.int64))
    W = np.zeros((V, V))
    for u in range(V):
        for e in range(int(offs[u]), int(offs[u + 1])):
            W[int(col[e]), u] = 1.0 / deg[u]
    dang = (deg == 0).astype(float)
    M = np.eye(V) - d * (W + np.outer(np.ones(V), dang) / V)
    return np.linalg.solve(M, np.full(V, (1 - d) / V))


def test_pr_star_closed_form():
    # undirected star: centre 0 + 3 leaves; r_centre = (1 + d m) / (V (1 + d))
    offs, col = synth.csr_from_edges(4, [(0, 1), (0, 2), (0, 3)])
    r, _ = oracle.graph_pr(offs, col, types_of(offs), iters=200)
    d = 0.85
    assert abs(r[0] - (1 + d * 3) / (4 * (1 + d))) < 1e-6
    assert np.allclose(r[1:], (1 - r[0]) / 3, atol=1e-6)


def test_pr_cycle_uniform_every_iteration():
    k = 7
    offs, col = synth.csr_from_edges(k, [(i, (i + 1) % k) for i in range(k)])
    for it in (1, 5, 20):
        r, _ = oracle.graph_pr(offs, col, types_of(offs), iters=it)
        assert np.allclose(r, 1.0 / k, rtol=1e-6)


def test_pr_dense_solve_with_dangling():
    # small graph with a triangle (non-bipartite), a tail, and isolated vertices
    V = 9
    offs, col = synth.csr_from_edges(V, [(0, 1), (1, 2), (2, 0), (2, 3), (3, 4), (4, 5), (5, 3), (6, 7)])
    ref = pr_dense(offs, col, 0.85, V)
    r, _ = oracle.graph_pr(offs, col, types_of(offs), iters=300)
    assert np.allclose(r, ref, rtol=1e-5, atol=1e-7)
    assert abs(ref.sum() - 1) < 1e-12


def test_pr_mass_and_threads_rmat():
    offs, col = synth.rmat_graph(13, seed=5)
    t = types_of(offs)
    a, _ = oracle.graph_pr(offs, col, t, iters=20, threads=1)
    b, _ = oracle.graph_pr(offs, col, t, iters=20, threads=oracle.max_threads())
    assert np.array_equal(a, b)
    assert abs(float(a.astype(np.float64).sum()) - 1.0) < 1e-5

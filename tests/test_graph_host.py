"""Host logic of config 4 (CPU): the hot-first storage slots of graph.py and
the CSR rebuilt in slot space, checked against their definition on small
seeded graphs (no GPU: the rebuild runs on torch's CPU device here).

Definition (graph.py docstring): within each rank's vertex block, slots are
assigned by descending degree, ties by vertex id; slot row s is vertex
inv[s]'s row in the same order with every neighbour replaced by its slot.
"""
import numpy as np
import pytest
import torch

import synth
from paper_conf_asplos_zhangar21_b200 import graph as G


def _perm(deg, V, world, hot=0):
    """Brute force of the slot definition: per block, vertices of degree >=
    hot by descending degree (ties by id), then the rest by id."""
    perm = np.empty(V, np.int64)
    for r in range(world):
        lo, hi, _ = G.block_range(V, r, world)
        key = sorted(range(lo, hi), key=lambda v: (0, -deg[v], v) if deg[v] >= hot else (1, 0, v))
        perm[np.array(key, dtype=np.int64)] = np.arange(lo, hi)
    return perm


@pytest.mark.parametrize("hot", [0, 4, 16, 1 << 30])
@pytest.mark.parametrize("world", [1, 3])
def test_slot_order_matches_definition(hot, world):
    offs, col = synth.rmat_graph(10, seed=7)
    V = len(offs) - 1
    deg = np.diff(offs.astype(np.int64))
    assert np.array_equal(G.slot_order(deg, V, world, hot), _perm(deg, V, world, hot))


@pytest.mark.parametrize("scale,world", [(8, 1), (10, 1), (10, 3)])
def test_csr_by_slot_matches_definition(scale, world):
    offs, col = synth.rmat_graph(scale, seed=3)
    V = len(offs) - 1
    deg = np.diff(offs.astype(np.int64))
    perm = _perm(deg, V, world)
    inv = np.empty_like(perm)
    inv[perm] = np.arange(V)
    offs_s, col_s = G._csr_by_slot(offs, col, torch.from_numpy(perm), torch.from_numpy(inv), "cpu")
    offs_s, col_s = offs_s.numpy(), col_s.numpy().astype(np.int64)
    assert offs_s[0] == 0 and offs_s[-1] == len(col)
    for s in range(V):  # brute force, row by row
        v = inv[s]
        want = perm[col[offs[v]:offs[v + 1]].astype(np.int64)]
        assert np.array_equal(col_s[offs_s[s]:offs_s[s + 1]], want)
    # hot-first inside every block, ownership unchanged
    for r in range(world):
        lo, hi, _ = G.block_range(V, r, world)
        assert set(perm[lo:hi]) == set(range(lo, hi))
        d_slot = deg[inv[lo:hi]]
        assert np.all(d_slot[:-1] >= d_slot[1:])
        ties = d_slot[:-1] == d_slot[1:]
        assert np.all(inv[lo:hi][:-1][ties] < inv[lo:hi][1:][ties])


def test_slot_relabel_preserves_bfs_depths():
    """BFS over the slot CSR, read back by vertex id, equals BFS over the original CSR."""
    offs, col = synth.rmat_graph(9, seed=5)
    V = len(offs) - 1
    deg = np.diff(offs.astype(np.int64))
    perm = _perm(deg, V, 1)
    inv = np.empty_like(perm)
    inv[perm] = np.arange(V)
    offs_s, col_s = G._csr_by_slot(offs, col, torch.from_numpy(perm), torch.from_numpy(inv), "cpu")
    offs_s, col_s = offs_s.numpy(), col_s.numpy()

    def bfs(o, c, src):
        d = np.full(V, -1, np.int64)
        d[src] = 0
        fr = [src]
        while fr:
            nx = []
            for u in fr:
                for w in c[o[u]:o[u + 1]]:
                    if d[w] < 0:
                        d[w] = d[u] + 1
                        nx.append(int(w))
            fr = nx
        return d

    src = int(np.argmax(deg))
    d0 = bfs(offs, col, src)
    d1 = bfs(offs_s, col_s, int(perm[src]))
    assert np.array_equal(d1[perm], d0)

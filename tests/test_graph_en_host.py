"""Host-side logic of the GraphChi-vEN driver (CPU): the in-edge pointer
array is the out-edge array permuted by reverse_arcs, so in_edges[k] for k in
row(v) must be the arc (col[k] -> v)."""
import numpy as np
import torch

import synth
from paper_conf_asplos_zhangar21_b200.graph_en import reverse_arcs


def test_reverse_arcs_pairs_every_arc_with_its_reverse():
    for scale, seed in ((8, 1), (11, 2)):
        offs, col = synth.rmat_graph(scale, seed=seed)
        deg = np.diff(offs.astype(np.int64))
        src = np.repeat(np.arange(len(offs) - 1), deg)
        rev = reverse_arcs(torch.from_numpy(col.astype(np.int64))).numpy()
        # arc rev[k] goes col[k] -> src[k]
        assert np.array_equal(src[rev], col.astype(np.int64))
        assert np.array_equal(col[rev].astype(np.int64), src)
        # a permutation
        assert np.array_equal(np.sort(rev), np.arange(len(col)))


def test_reverse_arcs_fixture():
    offs, col = synth.csr_from_edges(4, [(0, 1), (0, 2), (1, 2), (2, 3)])
    # arcs: 0->1 0->2 | 1->0 1->2 | 2->0 2->1 2->3 | 3->2
    rev = reverse_arcs(torch.from_numpy(col.astype(np.int64))).tolist()
    assert rev == [2, 4, 0, 5, 1, 3, 7, 6]

"""GraphChi-vEN driver: BFS / CC / PageRank with virtual edges AND virtual vertices
(Table 2; readings G32/G33 in DESIGN.md).

Argument marshalling and step sequencing over the C ABI only. Vertices are
VF_APP_GRAPH_EN objects (degree-bucket types, as config 4), edges are
VF_APP_EDGE objects, one per arc of the symmetric CSR (Edge, or HubEdge when
the source is a Hub). Inside every vertex method each edge access is a
virtual call on an edge object; the edge data (labels, PageRank shares) lives
in the edge objects, double-buffered, as in GraphChi. Per iteration:

  CC:  vertex cc_update()  (reads in-edges' get_label(b))      -> label_out
       edge   pull_label() (every arc stores its source's label in buffer 1-b)
  PR:  vertex pr_gather()  (sums in-edges' get_pr(b))          -> rank, contrib
       edge   pull_pr()    (every arc stores contrib[src] in buffer 1-b)
  BFS: vertex bfs_expand() per frontier entry (out-edges' target())

Single GPU (the multi-GPU graph path is config 4's vertex-only app, graph.py).
"""
from __future__ import annotations

import ctypes

import numpy as np
import torch

import synth

from . import vf
from .graph import work_entries

HUB = 3  # vertex type id of Hub (deg >= 256)


def reverse_arcs(col: torch.Tensor) -> torch.Tensor:
    """rev[k] = index of the reverse arc (col[k] -> v) of arc k = (v -> col[k]) in
    a symmetric CSR with sorted rows: a stable sort of the arcs by target lists,
    for each v, the arcs (u -> v) in ascending u, i.e. in the order of v's row."""
    return torch.argsort(col, stable=True)


class GraphEN:
    def __init__(self, ctx: vf.Ctx, offs: np.ndarray, col: np.ndarray, variant: str = "typeptr", chunk: int = 256):
        self.ctx, self.variant = ctx, variant
        self.v = vf.VARIANTS[variant]
        dev = torch.device(f"cuda:{ctx.device}")
        self.dev = dev
        V = len(offs) - 1
        self.V, self.C = V, int(chunk)
        self.A = int(offs[-1])
        deg = np.diff(np.asarray(offs, dtype=np.int64))
        self.deg_np = deg
        vtypes = synth.vertex_types(offs)
        tag = variant == "typeptr"
        self.offs = torch.from_numpy(np.ascontiguousarray(offs, dtype=np.uint64).view(np.int64)).to(dev)
        col_t = torch.from_numpy(np.ascontiguousarray(col, dtype=np.uint32).view(np.int32)).to(dev)
        # ---- vertices
        ctor = np.stack([np.arange(V, dtype=np.uint32), deg.astype(np.uint32)], axis=1).copy()
        ctor_t = torch.from_numpy(ctor.view(np.int32)).to(dev)
        vt = torch.from_numpy(vtypes.astype(np.int32)).to(dev)
        if variant == "cuda":
            self.vobj = ctx.alloc_cuda(vf.APP_GRAPH_EN, vt, ctor_t)
        else:
            self.vobj = ctx.alloc_typed_batch(vf.APP_GRAPH_EN, vt, ctor_t, tag=tag)
        del ctor_t
        # ---- edges: arc k = (src(k) -> col[k]), type HubEdge iff src is a Hub
        deg_t = torch.from_numpy(deg).to(dev)
        src = torch.repeat_interleave(torch.arange(V, dtype=torch.int32, device=dev), deg_t)
        etypes = (vt == HUB).to(torch.int32)[src.long()]
        ector = torch.stack([src, col_t], dim=1).contiguous()
        del src
        if variant == "cuda":
            self.out_edges = ctx.alloc_cuda(vf.APP_EDGE, etypes, ector)
        else:
            self.out_edges = ctx.alloc_typed_batch(vf.APP_EDGE, etypes, ector, tag=tag)
        self.etypes = etypes
        del ector
        # in-edges of v in ascending source order: the arcs (u -> v) sorted stably by v
        rev = reverse_arcs(col_t)
        self.in_edges = self.out_edges[rev].contiguous()
        del rev, col_t
        # ---- nested edge-call resolver (COAL table / TypePointer tag / vTable* fallback)
        self.er = self._resolver()
        # ---- work entries
        evid, ech = work_entries(deg, 0, V, self.C)
        self.E = len(evid)
        self.entries = self.vobj[torch.from_numpy(evid).to(dev)].contiguous()
        self.entry_chunk = torch.from_numpy(ech.view(np.int32)).to(dev)
        self.depth = torch.empty(V, dtype=torch.int32, device=dev)
        self.q = [torch.empty(max(self.E, 1), dtype=torch.int64, device=dev) for _ in range(2)]
        self.qc = [torch.empty(max(self.E, 1), dtype=torch.int32, device=dev) for _ in range(2)]
        self.count = torch.zeros(1, dtype=torch.int32, device=dev)
        self.lab = [torch.empty(V, dtype=torch.int32, device=dev) for _ in range(2)]
        self.changed = torch.zeros(1, dtype=torch.int32, device=dev)
        self.rk = [torch.empty(V, dtype=torch.float32, device=dev) for _ in range(2)]
        self.contrib = torch.empty(V, dtype=torch.float64, device=dev)
        self.dangling = torch.zeros(2, dtype=torch.float64, device=dev)
        self.partial = torch.zeros(max(self.E, 1), dtype=torch.float64, device=dev)
        self.counter = torch.zeros(V, dtype=torch.int32, device=dev)
        self.b = 0
        self.vcalls = self.ecalls = 0
        torch.cuda.synchronize(dev)

    def _resolver(self):
        rt = self.ctx.range_table(vf.APP_EDGE)
        K = len(rt)
        dev = self.dev
        u64 = lambda xs: torch.from_numpy(np.array(xs or [0], dtype=np.uint64).view(np.int64)).to(dev)  # noqa: E731
        self._rt_start = u64([r.start for r in rt])
        self._rt_end = u64([r.end for r in rt])
        self._rt_type = torch.tensor([r.type_id for r in rt] or [0], dtype=torch.int32, device=dev)
        self._vptrs = u64(self.ctx.type_vptrs(vf.APP_EDGE))
        P = 1
        while P < K:
            P *= 2
        rule = vf.TYPEPTR if self.variant == "typeptr" else vf.COAL
        return vf.edge_resolver(self._rt_start.data_ptr(), self._rt_end.data_ptr(), self._rt_type.data_ptr(),
                                self._vptrs.data_ptr(), K, P, rule)

    def _dispatch(self, app, method, objs_ptr, n, args, stream=None):
        st = self.ctx.dispatch_raw(self.v, app, method, objs_ptr, n, args, vf._stream(stream))
        if st:
            self.ctx._check(st, f"graph_en app {app} method {method}")

    def _pull(self, method, slot, contrib=None, label=None, stream=None):
        a = vf.edge_args(0 if contrib is None else contrib.data_ptr(), 0 if label is None else label.data_ptr(), 0,
                         slot)
        self._dispatch(vf.APP_EDGE, method, self.out_edges.data_ptr(), self.A, a, stream)

    def edge_endpoints(self):
        """(src, dst) of every arc read back through the edge objects' virtual get()."""
        out = torch.empty(self.A, dtype=torch.int64, device=self.dev)
        a = vf.edge_args(0, 0, out.data_ptr(), 0)
        self._dispatch(vf.APP_EDGE, vf.EDGE_GET, self.out_edges.data_ptr(), self.A, a)
        return out

    # ---------------------------------------------------------------- BFS
    def bfs(self, src: int):
        """Top-down level-synchronous BFS; returns (depth, levels, vertex calls, edge calls)."""
        L = vf.lib()
        st = L.vf_graph_bfs_init(self.V, self.depth.data_ptr(), src, self.vobj.data_ptr(), self.offs.data_ptr(),
                                 self.C, self.q[0].data_ptr(), self.qc[0].data_ptr(), self.count.data_ptr(),
                                 vf._stream(None))
        if st:
            raise vf.VFError(st, "bfs_init")
        vcalls, level = 0, 0
        n = int(self.count.item())
        while n > 0:
            self.count.zero_()
            a = vf.graph_en_bfs_args(self.offs.data_ptr(), self.out_edges.data_ptr(), self.depth.data_ptr(),
                                     self.vobj.data_ptr(), self.qc[0].data_ptr(), self.q[1].data_ptr(),
                                     self.qc[1].data_ptr(), self.count.data_ptr(), level, self.C, self.er)
            self._dispatch(vf.APP_GRAPH_EN, vf.GRAPH_EN_BFS_EXPAND, self.q[0].data_ptr(), n, a)
            vcalls += n
            n = int(self.count.item())
            self.q[0], self.q[1] = self.q[1], self.q[0]
            self.qc[0], self.qc[1] = self.qc[1], self.qc[0]
            level += 1
        self.vcalls = vcalls
        self.ecalls = None  # sum of reached degrees: edge_calls_bfs()
        return self.depth, level, vcalls

    def edge_calls_bfs(self):
        reached = (self.depth >= 0).cpu().numpy()
        return int(self.deg_np[reached].sum())

    # ---------------------------------------------------------------- CC
    def cc_init(self):
        L = vf.lib()
        L.vf_iota_u32(self.V, self.lab[0].data_ptr(), vf._stream(None))
        L.vf_iota_u32(self.V, self.lab[1].data_ptr(), vf._stream(None))
        self.b = 0
        self._pull(vf.EDGE_PULL_LABEL, 0, label=self.lab[0])

    def cc_iteration(self, stream=None):
        a = vf.graph_en_cc_args(self.offs.data_ptr(), self.in_edges.data_ptr(), self.lab[0].data_ptr(),
                                self.lab[1].data_ptr(), self.changed.data_ptr(), self.entry_chunk.data_ptr(), self.C,
                                self.b, self.er)
        self._dispatch(vf.APP_GRAPH_EN, vf.GRAPH_EN_CC_UPDATE, self.entries.data_ptr(), self.E, a, stream)
        self._pull(vf.EDGE_PULL_LABEL, 1 - self.b, label=self.lab[1], stream=stream)
        self.b = 1 - self.b
        self.lab[0], self.lab[1] = self.lab[1], self.lab[0]
        return self.E, 2 * self.A  # vertex calls, edge calls (nested get_label + pull_label)

    def cc(self, max_iters: int = 10 ** 6):
        """Jacobi min-label propagation until no change; returns (labels, iters, vertex calls, edge calls)."""
        self.cc_init()
        it = vc = ec = 0
        while it < max_iters:
            self.changed.zero_()
            v, e = self.cc_iteration()
            vc, ec, it = vc + v, ec + e, it + 1
            if int(self.changed.item()) == 0:
                break
        self.vcalls, self.ecalls = vc, ec
        return self.lab[0], it, vc, ec

    # ---------------------------------------------------------------- PageRank
    def pr_init(self, d: float = 0.85):
        vf.lib().vf_fill_f32(self.V, self.rk[0].data_ptr(), ctypes.c_float(1.0 / self.V).value, vf._stream(None))
        self.b = 0
        self.dangling.zero_()
        a = self._pr_args(d)
        a.dangling_out_dev = self.dangling.data_ptr()  # D_0 -> dangling[0]
        self._dispatch(vf.APP_GRAPH_EN, vf.GRAPH_EN_PR_INIT, self.entries.data_ptr(), self.E, a)
        self._pull(vf.EDGE_PULL_PR, 0, contrib=self.contrib)

    def _pr_args(self, d):
        D_in = self.dangling.data_ptr() + 8 * self.b
        D_out = self.dangling.data_ptr() + 8 * (1 - self.b)
        return vf.graph_en_pr_args(self.offs.data_ptr(), self.in_edges.data_ptr(), self.rk[0].data_ptr(),
                                   self.rk[1].data_ptr(), self.contrib.data_ptr(), D_in, D_out, (1.0 - d) / self.V, d,
                                   float(self.V), self.entry_chunk.data_ptr(), self.partial.data_ptr(),
                                   self.counter.data_ptr(), self.C, self.b, self.er)

    def pr_iteration(self, d: float = 0.85, stream=None):
        """One iteration: virtual pr_gather() per work entry (nested get_pr per in-edge),
        then virtual pull_pr() per edge."""
        self.dangling[1 - self.b].zero_()
        a = self._pr_args(d)
        self._dispatch(vf.APP_GRAPH_EN, vf.GRAPH_EN_PR_GATHER, self.entries.data_ptr(), self.E, a, stream)
        self._pull(vf.EDGE_PULL_PR, 1 - self.b, contrib=self.contrib, stream=stream)
        self.b = 1 - self.b
        self.rk[0], self.rk[1] = self.rk[1], self.rk[0]
        return self.E, 2 * self.A

    def pagerank(self, iters: int = 20, d: float = 0.85):
        self.pr_init(d)
        vc = ec = 0
        for _ in range(iters):
            v, e = self.pr_iteration(d)
            vc, ec = vc + v, ec + e
        self.vcalls, self.ecalls = vc, ec
        return self.rk[0], vc, ec

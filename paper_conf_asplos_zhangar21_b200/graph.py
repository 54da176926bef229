"""Config 4 driver: BFS / CC / PageRank over polymorphic vertices (Table 2).

Argument marshalling and step sequencing over the C ABI only: vertex objects
are allocated through libvf (typed arenas by degree bucket, or device-heap
`new` for the CUDA baseline), and every per-vertex computation is a virtual
method call dispatched by libvf (vf_dispatch). Host code reads back one scalar
per BFS level / CC iteration to decide termination.

Multi-GPU (``rank``/``world``): vertex ids are split into contiguous blocks;
each rank dispatches only its owned vertices and the per-iteration state
(depth / labels / contributions) is exchanged with an all-gather over the
process group (NCCL on B200, gloo on CPU tests).

State layout (hot-first): the per-vertex state arrays and the CSR the bodies
read are indexed by a STORAGE slot, not by the vertex id: within each rank's
block, slots are assigned by descending degree (ties by id), so the state of
the hubs that most rows gather (RMAT: the >= 256-degree class holds ~70% of
the arcs) sits in a few dense lines at the start of the block. The vertex
objects, their allocation and the dispatch order stay in vertex-id order (the
recipe's random permutation: types interleaved); each object's `vid` field is
its storage slot. Rows keep their CSR order (same summation order), labels
are original vertex ids, and every result is returned indexed by vertex id.
"""
from __future__ import annotations

import ctypes

import numpy as np
import torch

import synth

from . import exchange, vf


def _sync_scalar(t):
    return int(t.item())


def block_range(V: int, rank: int, world: int):
    """Owned vertex block [lo, hi) of `rank` and the per-rank block size (a
    multiple of 32 for world > 1, so frontier-bitmap slices are whole u32 words)."""
    return exchange.block_range(V, rank, world, align=32 if world > 1 else 1)


def allgather_block(t, V: int, per: int, rank: int, world: int, group=None):
    """All-gather of each rank's owned block of a per-vertex array held in a
    plain (unpadded) tensor: kept for callers outside the app classes, which
    use persistent padded ``exchange.BlockArray`` buffers instead."""
    if world == 1:
        return
    import torch.distributed as dist
    rest = tuple(t.shape[1:])
    padded = torch.zeros((per * world,) + rest, dtype=t.dtype, device=t.device)
    padded[:V] = t
    mine = padded[rank * per:(rank + 1) * per].clone()
    if exchange._staged(padded, group):
        h = padded.cpu()
        dist.all_gather_into_tensor(h, mine.cpu(), group=group)
        padded.copy_(h)
    else:
        dist.all_gather_into_tensor(padded, mine, group=group)
    t.copy_(padded[:V])


def allreduce_sum(t, world: int, group=None):
    exchange.allreduce_(t, world, group)


def work_entries(deg: np.ndarray, lo: int, hi: int, C: int):
    """Work entries of vertices [lo, hi) (vf.h VF_APP_GRAPH): vertex v appears
    nch(v) = max(1, ceil(deg/C)) times consecutively, with chunk ids 0..nch-1.
    Returns (entry vertex ids int64[E], chunk ids uint32[E])."""
    d = np.asarray(deg[lo:hi], np.int64)
    nch = np.maximum(1, (d + C - 1) // C)
    vid = np.repeat(np.arange(lo, hi, dtype=np.int64), nch)
    first = np.repeat(np.cumsum(nch) - nch, nch)
    chunk = (np.arange(len(vid), dtype=np.int64) - first).astype(np.uint32)
    return vid, chunk


def _csr_by_slot(offs: np.ndarray, col: np.ndarray, perm, inv, dev):
    """The CSR in storage-slot space: row s is vertex inv[s]'s row, in the same
    order, with every neighbour id replaced by its slot (setup, on the GPU)."""
    offs_t = torch.from_numpy(np.ascontiguousarray(offs, dtype=np.int64)).to(dev)
    col_t = torch.from_numpy(np.ascontiguousarray(col, dtype=np.uint32).view(np.int32)).to(dev)
    V, E = len(offs) - 1, len(col)
    deg_s = (offs_t[1:] - offs_t[:-1])[inv]
    offs_s = torch.zeros(V + 1, dtype=torch.int64, device=dev)
    torch.cumsum(deg_s, 0, out=offs_s[1:])
    col_s = torch.empty(E, dtype=torch.int32, device=dev)
    step = 1 << 26  # arcs per pass (bounded temporaries)
    if E:
        row = torch.repeat_interleave(torch.arange(V, device=dev), deg_s)
        for k0 in range(0, E, step):
            k1 = min(E, k0 + step)
            r = row[k0:k1]
            src = offs_t[inv[r]] + (torch.arange(k0, k1, device=dev) - offs_s[r])
            col_s[k0:k1] = perm[col_t[src].long()].int()
        del row
    return offs_s, col_s


HOT_DEGREE = 0  # 0: every vertex by degree (measured best, DESIGN §5 "Graph vertex order")


def slot_order(deg: np.ndarray, V: int, world: int, hot_degree: int = HOT_DEGREE) -> np.ndarray:
    """perm[v] = storage slot of vertex v: within each rank's block, the hot
    vertices (degree >= hot_degree) first by descending degree (ties by id),
    then every other vertex in id order — so the cold majority's own state
    accesses (in dispatch = id order) stay monotone, and the state every row
    gathers most (the high-degree endpoints) is dense. hot_degree = 0: a full
    degree sort."""
    perm = np.empty(V, np.int64)
    for r in range(world):
        blo, bhi, _ = block_range(V, r, world)
        d = deg[blo:bhi]
        hot = np.flatnonzero(d >= hot_degree)
        hot = hot[np.argsort(-d[hot], kind="stable")]
        cold = np.flatnonzero(d < hot_degree)
        order = np.concatenate([hot, cold])
        perm[blo + order] = np.arange(blo, bhi, dtype=np.int64)
    return perm


class Graph:
    def __init__(self, ctx: vf.Ctx, offs: np.ndarray, col: np.ndarray, variant: str = "typeptr",
                 rank: int = 0, world: int = 1, group=None, chunk: int = 256, hot_degree: int = HOT_DEGREE):
        self.ctx, self.variant = ctx, variant
        self.v = vf.VARIANTS[variant]
        dev = torch.device(f"cuda:{ctx.device}")
        self.dev = dev
        V = len(offs) - 1
        self.V = V
        self.C = int(chunk)
        self.rank, self.world, self.group = rank, world, group
        # owned vertex block [lo, hi)
        self.lo, self.hi, self.per = block_range(V, rank, world)
        deg = np.diff(np.asarray(offs, dtype=np.int64))
        # storage slot of every vertex (hot-first within each rank's block)
        perm = slot_order(deg, V, world, hot_degree)
        self.perm = torch.from_numpy(perm).to(dev)        # vertex id -> slot
        self.inv = torch.empty_like(self.perm)
        self.inv[self.perm] = torch.arange(V, dtype=torch.int64, device=dev)  # slot -> vertex id
        self.offs, self.col = _csr_by_slot(offs, col, self.perm, self.inv, dev)
        types = synth.vertex_types(offs)
        self.types_np = types
        own = np.arange(self.lo, self.hi)
        ctor = np.stack([perm[own].astype(np.uint32), deg[own].astype(np.uint32)], axis=1).copy()
        ctor_t = torch.from_numpy(ctor.view(np.int32)).to(dev)
        tt = torch.from_numpy(types[own].astype(np.int32)).to(dev)
        objs = ctx.alloc_for(variant, vf.APP_GRAPH, tt, ctor_t)
        # the owned objects in vertex-id order; vobj is indexed by storage slot
        # (BFS appends a discovered slot's entries); only the owned block is filled
        self.owned = objs
        self.vobj = torch.zeros(V, dtype=torch.int64, device=dev)
        self.vobj[self.perm[self.lo:self.hi]] = objs
        # work entries of the owned block in vertex-id order (one virtual call each)
        evid, ech = work_entries(deg, self.lo, self.hi, self.C)
        self.E = len(evid)
        self.entries = objs[torch.from_numpy(evid - self.lo).to(dev)].contiguous()
        self.entry_chunk = torch.from_numpy(ech.view(np.int32)).to(dev)
        e_all = int(np.maximum(1, (deg + self.C - 1) // self.C).sum())
        # per-vertex state in persistent buffers padded to per * world rows; the
        # owned block of each is all-gathered in place (exchange.BlockArray)
        blk = dict(n=V, per=self.per, rank=rank, world=world, device=dev, group=group)
        self._depth = exchange.BlockArray(dtype=torch.int32, **blk)
        self.depth = self._depth.view
        nw = (V + 31) // 32
        wblk = dict(n=nw, per=self.per // 32 if world > 1 else nw, rank=rank, world=world, device=dev, group=group)
        self._bits = [exchange.BlockArray(dtype=torch.int32, **wblk) for _ in range(2)]
        self.q = [torch.empty(max(e_all, 1), dtype=torch.int64, device=dev) for _ in range(2)]
        self.qc = [torch.empty(max(e_all, 1), dtype=torch.int32, device=dev) for _ in range(2)]
        self.count = torch.zeros(1, dtype=torch.int32, device=dev)
        self._lab = [exchange.BlockArray(dtype=torch.int32, **blk) for _ in range(2)]
        self.lab = [b.view for b in self._lab]
        self.changed = torch.zeros(1, dtype=torch.int32, device=dev)
        self._rk = [exchange.BlockArray(dtype=torch.float32, **blk) for _ in range(2)]
        self.rk = [b.view for b in self._rk]
        self._contrib = exchange.BlockArray(dtype=torch.float32, **blk)  # fp32 shares (DESIGN §2 R-PR32)
        self.contrib = self._contrib.view
        self.dangling = torch.zeros(1, dtype=torch.float64, device=dev)
        self.partial = torch.zeros(max(self.E, 1), dtype=torch.float64, device=dev)
        self.counter = torch.zeros(V, dtype=torch.int32, device=dev)
        self.calls = 0
        torch.cuda.synchronize(dev)

    # ---------------------------------------------------------------- helpers
    def by_id(self, t):
        """A per-slot state array re-indexed by vertex id."""
        return t[self.perm]

    def _allreduce_sum(self, t, stream=None):
        exchange.allreduce_(t, self.world, self.group, stream)

    def _dispatch(self, method, objs_ptr, n, args, stream=None):
        st = self.ctx.dispatch_raw(self.v, vf.APP_GRAPH, method, objs_ptr, n, args, vf._stream(stream))
        if st:
            self.ctx._check(st, f"graph method {method}")

    # ---------------------------------------------------------------- BFS
    def bfs(self, src: int, mode: str = "topdown", alpha: int = 64):
        """Level-synchronous BFS from src; returns (depth tensor, levels, calls).
        topdown: one virtual bfs_expand() per frontier work entry (single GPU);
        hybrid: top-down, then bottom-up once the frontier exceeds V / alpha entries (single GPU);
        bottomup: one virtual bfs_probe() per work entry per level, depth array as frontier (single GPU);
        bits (and every mode at world > 1): one virtual bfs_probe_bits() per owned work entry per
        level over a frontier bitmap whose owned slices are all-gathered (multi-GPU)."""
        L = vf.lib()
        src = int(self.perm[src].item())  # the source vertex id -> its storage slot
        st = L.vf_graph_bfs_init(self.V, self.depth.data_ptr(), src, self.vobj.data_ptr(), self.offs.data_ptr(),
                                 self.C, self.q[0].data_ptr(), self.qc[0].data_ptr(), self.count.data_ptr(),
                                 vf._stream(None))
        if st:
            raise vf.VFError(st, "bfs_init")
        calls, level = 0, 0
        if mode == "hybrid" and self.world == 1:
            # direction-optimizing (Beamer): top-down while the frontier is small,
            # bottom-up probes over every entry once it holds > V / alpha entries
            # (depths are unique, reading G23, so the result is the same)
            n = _sync_scalar(self.count)
            while n > 0 and n <= self.V // alpha:
                self.count.zero_()
                a = vf.graph_bfs_args(self.offs.data_ptr(), self.col.data_ptr(), self.depth.data_ptr(),
                                      self.vobj.data_ptr(), self.qc[0].data_ptr(), self.q[1].data_ptr(),
                                      self.qc[1].data_ptr(), self.count.data_ptr(), level, self.C)
                self._dispatch(vf.GRAPH_BFS_EXPAND, self.q[0].data_ptr(), n, a)
                calls += n
                n = _sync_scalar(self.count)
                self.q[0], self.q[1] = self.q[1], self.q[0]
                self.qc[0], self.qc[1] = self.qc[1], self.qc[0]
                level += 1
            while n > 0:
                self.count.zero_()
                a = vf.graph_bfs_args(self.offs.data_ptr(), self.col.data_ptr(), self.depth.data_ptr(),
                                      self.vobj.data_ptr(), self.entry_chunk.data_ptr(), 0, 0, self.count.data_ptr(),
                                      level, self.C)
                self._dispatch(vf.GRAPH_BFS_PROBE, self.entries.data_ptr(), self.E, a)
                calls += self.E
                n = _sync_scalar(self.count)
                level += 1
        elif mode == "topdown" and self.world == 1:
            n = _sync_scalar(self.count)
            while n > 0:
                self.count.zero_()
                a = vf.graph_bfs_args(self.offs.data_ptr(), self.col.data_ptr(), self.depth.data_ptr(),
                                      self.vobj.data_ptr(), self.qc[0].data_ptr(), self.q[1].data_ptr(),
                                      self.qc[1].data_ptr(), self.count.data_ptr(), level, self.C)
                self._dispatch(vf.GRAPH_BFS_EXPAND, self.q[0].data_ptr(), n, a)
                calls += n
                n = _sync_scalar(self.count)
                self.q[0], self.q[1] = self.q[1], self.q[0]
                self.qc[0], self.qc[1] = self.qc[1], self.qc[0]
                level += 1
        elif mode == "bottomup" and self.world == 1:
            while True:
                self.count.zero_()
                a = vf.graph_bfs_args(self.offs.data_ptr(), self.col.data_ptr(), self.depth.data_ptr(),
                                      self.vobj.data_ptr(), self.entry_chunk.data_ptr(), 0, 0, self.count.data_ptr(),
                                      level, self.C)
                self._dispatch(vf.GRAPH_BFS_PROBE, self.entries.data_ptr(), self.E, a)
                calls += self.E
                level += 1
                if _sync_scalar(self.count) == 0:
                    break
        else:
            level, calls = self._bfs_bits(src)
        self.calls = calls
        return self.by_id(self.depth), level, calls

    def _bfs_bits(self, src: int):
        """Bottom-up BFS over frontier bitmaps (multi-GPU): per level
        one virtual bfs_probe_bits() per owned work entry, then ONE all-gather of
        the owned bitmap slices (V/8 bytes in total) and an all-reduce of the
        "joined" flag. Depths stay on their owner until the end."""
        cur, nxt = self._bits
        cur.view.zero_()
        word, bit = divmod(src, 32)
        cur.view[word] = int(np.array(1 << bit, dtype=np.uint32).view(np.int32))
        if self.lo <= src < self.hi:
            self.depth[src] = 0
        calls, level = 0, 0
        while True:
            nxt.mine.zero_()
            self.count.zero_()
            a = vf.graph_bfs_bits_args(self.offs.data_ptr(), self.col.data_ptr(), self.depth.data_ptr(),
                                       cur.data_ptr(), nxt.data_ptr(), self.entry_chunk.data_ptr(),
                                       self.count.data_ptr(), level, self.C)
            self._dispatch(vf.GRAPH_BFS_PROBE_BITS, self.entries.data_ptr(), self.E, a)
            calls += self.E
            self._allreduce_sum(self.count)
            nxt.gather()
            cur, nxt = nxt, cur
            level += 1
            if _sync_scalar(self.count) == 0:
                break
        self._bits = [cur, nxt]
        self._depth.gather()
        return level, calls

    # ---------------------------------------------------------------- CC
    def cc(self, max_iters: int = 10 ** 6):
        """Jacobi min-label propagation until no label changes; returns (labels, iters, calls)."""
        # initial label of a slot = its vertex id; the other buffer too (>= every
        # later label: the atomicMin combine of multi-chunk vertices)
        self.lab[0].copy_(self.inv)
        self.lab[1].copy_(self.inv)
        it, calls = 0, 0
        while it < max_iters:
            self.changed.zero_()
            a = vf.graph_cc_args(self.offs.data_ptr(), self.col.data_ptr(), self.lab[0].data_ptr(),
                                 self.lab[1].data_ptr(), self.changed.data_ptr(), self.entry_chunk.data_ptr(), self.C)
            self._dispatch(vf.GRAPH_CC_UPDATE, self.entries.data_ptr(), self.E, a)
            calls += self.E
            it += 1
            self._lab[1].gather()
            self._allreduce_sum(self.changed)
            self._lab.reverse()
            self.lab = [b.view for b in self._lab]
            if _sync_scalar(self.changed) == 0:
                break
        self.calls = calls
        return self.by_id(self.lab[0]), it, calls

    # ---------------------------------------------------------------- PageRank
    def pr_init(self):
        vf.lib().vf_fill_f32(self.V, self.rk[0].data_ptr(), ctypes.c_float(1.0 / self.V).value, vf._stream(None))

    def pr_iteration(self, d: float = 0.85, stream=None):
        """One PageRank iteration = virtual pr_contrib() + pr_update() per owned work entry."""
        with exchange._on(stream, self.dangling):
            self.dangling.zero_()
        a = vf.graph_pr_args(self.offs.data_ptr(), self.col.data_ptr(), self.rk[0].data_ptr(), self.rk[1].data_ptr(),
                             self.contrib.data_ptr(), self.dangling.data_ptr(), (1.0 - d) / self.V, d, float(self.V),
                             self.entry_chunk.data_ptr(), self.partial.data_ptr(), self.counter.data_ptr(), self.C)
        self._dispatch(vf.GRAPH_PR_CONTRIB, self.entries.data_ptr(), self.E, a, stream)
        self._contrib.gather(stream)
        self._allreduce_sum(self.dangling, stream)
        self._dispatch(vf.GRAPH_PR_UPDATE, self.entries.data_ptr(), self.E, a, stream)
        self._rk.reverse()
        self.rk = [b.view for b in self._rk]
        return 2 * self.E

    def pagerank(self, iters: int = 20, d: float = 0.85):
        self.pr_init()
        calls = 0
        for _ in range(iters):
            calls += self.pr_iteration(d)
        self._rk[0].gather()  # ranks stay on their owner during the iterations
        self.calls = calls
        return self.by_id(self.rk[0]), calls

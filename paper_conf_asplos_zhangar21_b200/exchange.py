"""Per-step exchange of the multi-GPU apps.

The paper runs on one GPU; the exchange is this build's
extension for the shardable apps. One process per GPU; every rank owns a
contiguous block of ids (vertices, bodies, node rows) and the step kernels
write only owned entries. What the next step needs from other ranks is
exchanged here, with NO per-call allocation:

* ``BlockArray``: a per-id array that lives in a persistent buffer padded to
  ``per * world`` rows. ``view`` (the first n rows) is what the kernels index.
  ``gather()`` is ONE ``all_gather_into_tensor`` of this rank's block (copied
  into a persistent send buffer, 1/world of the array) into the buffer. The
  graph's frontier bitmap, CC labels, PR contributions, N-body / STUT
  positions all use it.
* ``HaloRows``: the GEN row slabs' halo exchange, ``batch_isend_irecv`` of
  one boundary row to each neighbour slab per generation.
* ``VarGather``: variable-length row lists (collision: only the bodies with a
  merge candidate travel after update).
* ``allreduce_``: in-place sum (BFS "changed", PR dangling mass).

CPU tests drive the same code over ``gloo`` process groups. gloo cannot move
CUDA tensors in these collectives, so when the group is gloo and the tensor
is on a GPU, the owned block is staged through a pinned host buffer (the
2-process GPU tests run both ranks on one device that way); with NCCL nothing
is staged.
"""
from __future__ import annotations

import torch


def _dist():
    import torch.distributed as dist
    return dist


def block_range(n: int, rank: int, world: int, align: int = 1):
    """Owned block [lo, hi) of `rank` and the per-rank block size `per`
    (ceil(n / world) rounded up to `align`, so that bitmap slices are whole words)."""
    per = -(-n // world) if world > 0 else n
    per = -(-per // align) * align if align > 1 else per
    return min(n, rank * per), min(n, (rank + 1) * per), per


def _staged(t: torch.Tensor, group) -> bool:
    return t.is_cuda and _dist().get_backend(group) == "gloo"


def _on(stream, t: torch.Tensor):
    """Run the collective (NCCL) or the staging copies (gloo) on `stream`, the
    stream the app's kernels were enqueued on (None: the current stream)."""
    import contextlib
    if stream is None or not t.is_cuda:
        return contextlib.nullcontext()
    if not isinstance(stream, torch.cuda.Stream):
        stream = torch.cuda.ExternalStream(int(stream), device=t.device)
    return torch.cuda.stream(stream)


class BlockArray:
    """Persistent padded per-id array whose owned blocks are all-gathered into it."""

    def __init__(self, n: int, per: int, rank: int, world: int, dtype, device, rest=(), group=None,
                 fill=None):
        self.n, self.per, self.rank, self.world, self.group = n, per, rank, world, group
        rows = per * world if world > 1 else n
        self.buf = torch.empty((max(rows, 1),) + tuple(rest), dtype=dtype, device=device)
        if fill is not None:
            self.buf.fill_(fill)
        self.view = self.buf[:n]
        self.mine = self.buf[rank * per:(rank + 1) * per] if world > 1 else self.view
        self._host = None
        self._send = None

    def data_ptr(self) -> int:
        return self.view.data_ptr()

    def gather(self, stream=None):
        """After the call every rank holds every rank's block (one collective),
        ordered after the work already enqueued on `stream`."""
        if self.world == 1:
            return
        with _on(stream, self.buf):
            self._gather()

    def _gather(self):
        dist = _dist()
        if _staged(self.buf, self.group):
            if self._host is None:
                self._host = (torch.empty_like(self.buf, device="cpu").pin_memory(),
                              torch.empty_like(self.mine, device="cpu").pin_memory())
            hb, hm = self._host
            hm.copy_(self.mine)
            dist.all_gather_into_tensor(hb, hm, group=self.group)
            self.buf.copy_(hb, non_blocking=False)
        else:
            # the owned block goes through a persistent send buffer (a D2D copy
            # of 1/world of the array) rather than aliasing the output
            if self._send is None:
                self._send = torch.empty_like(self.mine)
            self._send.copy_(self.mine)
            dist.all_gather_into_tensor(self.buf, self._send, group=self.group)


class VarGather:
    """All-gather of variable-length row lists (persistent, grown on demand):
    every rank contributes `count` rows; the result holds world segments of
    max(count) rows each, rank r's first counts[r] rows valid. Two collectives
    (the counts, then the padded rows) and one host read of the counts."""

    def __init__(self, world: int, row_bytes: int, device, group=None):
        self.world, self.row_bytes, self.device, self.group = world, row_bytes, device, group
        self.counts = torch.zeros(world, dtype=torch.int64, device=device)
        self._send = self._recv = None
        self._host = None

    def send_buffer(self, rows: int) -> torch.Tensor:
        """A (rows x row_bytes) uint8 buffer to pack into (kept across calls)."""
        if self._send is None or self._send.shape[0] < rows:
            grown = torch.empty((max(rows, 1), self.row_bytes), dtype=torch.uint8, device=self.device)
            if self._send is not None:
                grown[:self._send.shape[0]].copy_(self._send)  # keep what was packed
            self._send = grown
        return self._send

    def gather(self, count: int, stream=None):
        """-> (recv uint8[world * seg, row_bytes], counts int64[world] on the device, seg)."""
        dist = _dist()
        with _on(stream, self.counts):
            mine = torch.tensor([count], dtype=torch.int64, device=self.device)
            staged = _staged(self.counts, self.group)
            if staged:
                hc = torch.empty(self.world, dtype=torch.int64)
                dist.all_gather_into_tensor(hc, mine.cpu(), group=self.group)
                self.counts.copy_(hc)
            else:
                dist.all_gather_into_tensor(self.counts, mine, group=self.group)
                hc = self.counts.cpu()
            seg = max(int(hc.max()), 1)
            send = self.send_buffer(seg)[:seg]
            if self._recv is None or self._recv.shape[0] < self.world * seg:
                self._recv = torch.empty((self.world * seg, self.row_bytes), dtype=torch.uint8, device=self.device)
            recv = self._recv[:self.world * seg]
            if staged:
                hr = torch.empty(recv.shape, dtype=torch.uint8)
                dist.all_gather_into_tensor(hr, send.cpu(), group=self.group)
                recv.copy_(hr)
            else:
                dist.all_gather_into_tensor(recv, send, group=self.group)
        return recv, self.counts, seg


def allreduce_(t: torch.Tensor, world: int, group=None, stream=None):
    """In-place sum over ranks (a few bytes: flags, the dangling mass)."""
    if world == 1:
        return
    dist = _dist()
    with _on(stream, t):
        if _staged(t, group):
            h = t.cpu()
            dist.all_reduce(h, group=group)
            t.copy_(h)
        else:
            dist.all_reduce(t, group=group)


class HaloRows:
    """Halo rows of a W x H row-slab decomposition (GEN).

    Rank r owns rows [r0, r1). Before a generation it needs rows r0-1 and r1
    (torus: modulo H) of the previous state, owned by the neighbour slabs.
    ``exchange(state)`` sends its first / last owned row to the previous /
    next rank and receives theirs into the halo rows of `state` (a full-size
    H*W uint8 buffer indexed by global cell)."""

    def __init__(self, W: int, H: int, rank: int, world: int, torus: bool = False, group=None):
        self.W, self.H, self.rank, self.world, self.torus, self.group = W, H, rank, world, torus, group
        self.r0, self.r1, self.per = block_range(H, rank, world)
        self._host = None

    def _peers(self):
        prev = self.rank - 1 if self.rank > 0 else (self.world - 1 if self.torus else None)
        nxt = self.rank + 1 if self.rank < self.world - 1 else (0 if self.torus else None)
        return prev, nxt

    def exchange(self, state: torch.Tensor, stream=None):
        if self.world == 1 or self.r1 <= self.r0:
            return
        with _on(stream, state):
            self._exchange(state)

    def _exchange(self, state: torch.Tensor):
        dist = _dist()
        W, H = self.W, self.H
        s2 = state.view(H, W)
        prev, nxt = self._peers()
        staged = _staged(state, self.group)
        if staged:
            if self._host is None:
                self._host = [torch.empty(W, dtype=state.dtype).pin_memory() for _ in range(4)]
            send_first, send_last, recv_above, recv_below = self._host
            send_first.copy_(s2[self.r0])
            send_last.copy_(s2[self.r1 - 1])
        else:
            send_first, send_last = s2[self.r0], s2[self.r1 - 1]
            recv_above = s2[(self.r0 - 1) % H]
            recv_below = s2[self.r1 % H]
        # downward messages (last row -> next slab's halo above) first, then
        # upward ones: messages between one pair of ranks match in posting
        # order, which keeps world = 2 with torus (both neighbours are the same
        # rank) correct
        ops = []
        g = self.group
        if nxt is not None:
            ops.append(dist.P2POp(dist.isend, send_last, _peer_global(nxt, g), g))
        if prev is not None:
            ops.append(dist.P2POp(dist.irecv, recv_above, _peer_global(prev, g), g))
            ops.append(dist.P2POp(dist.isend, send_first, _peer_global(prev, g), g))
        if nxt is not None:
            ops.append(dist.P2POp(dist.irecv, recv_below, _peer_global(nxt, g), g))
        if ops:
            for r in dist.batch_isend_irecv(ops):
                r.wait()
        if staged:
            if prev is not None:
                s2[(self.r0 - 1) % H].copy_(recv_above)
            if nxt is not None:
                s2[self.r1 % H].copy_(recv_below)


def _peer_global(r: int, group):
    if group is None:
        return r
    return _dist().get_global_rank(group, r)

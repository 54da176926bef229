"""Config 5 STUT driver: spring-node structure (Table 2, reading G17).

Every node and spring is a libvf object; one step = a virtual force() on every
spring, then a virtual move() on every node (libvf dispatch).

Multi-GPU (§8e): node row slabs. A rank owns the nodes of its rows and the
springs whose a-end is one of them; it also holds "ghost" copies of the
springs that reach into its slab from the row above (their b-end is owned),
so every force its nodes need is computed locally (a ghost evolves exactly
like its owner: same inputs, same arithmetic, same fracture step). Node
positions are all-gathered after every step over the process group.
"""
from __future__ import annotations

import numpy as np
import torch

from . import exchange as xc, vf
from .exchange import block_range


class Stut:
    def __init__(self, ctx: vf.Ctx, w: dict, variant: str = "typeptr", rank: int = 0, world: int = 1,
                 group=None, exchange: bool = True):
        self.ctx, self.variant = ctx, variant
        self.v = vf.VARIANTS[variant]
        dev = torch.device(f"cuda:{ctx.device}")
        self.dev = dev
        W, H = int(w["W"]), int(w["H"])
        n, S = len(w["types"]), len(w["a"])
        self.n, self.S, self.W = n, S, W
        self.rank, self.world, self.group, self.exchange = rank, world, group, exchange
        r0, r1, rper = block_range(H, rank, world)
        self.lo, self.hi, self.per = r0 * W, r1 * W, rper * W
        a, b = np.asarray(w["a"], np.int64), np.asarray(w["b"], np.int64)
        own_s = (a >= self.lo) & (a < self.hi)
        ghost_s = ~own_s & (b >= self.lo) & (b < self.hi)
        sids = np.nonzero(own_s | ghost_s)[0]
        self.n_own_springs = int(own_s.sum())
        self.spring_ids = sids
        nodes = np.arange(self.lo, self.hi)
        nctor = np.zeros((len(nodes), 4), np.uint32)
        nctor[:, 0] = nodes
        nctor[:, 1:3] = np.ascontiguousarray(w["vel"][nodes], np.float32).view(np.uint32)
        nctor[:, 3] = np.ascontiguousarray(w["mass"][nodes], np.float32).view(np.uint32)
        sctor = np.zeros((len(sids), 6), np.uint32)
        sctor[:, 0] = sids
        sctor[:, 1] = a[sids]
        sctor[:, 2] = b[sids]
        sctor[:, 3] = np.ascontiguousarray(w["L0"][sids], np.float32).view(np.uint32)
        sctor[:, 4] = np.ascontiguousarray(w["k"][sids], np.float32).view(np.uint32)
        nt = torch.from_numpy(w["types"][nodes].astype(np.int32)).to(dev)
        st = torch.full((len(sids),), 3, dtype=torch.int32, device=dev)
        nc = torch.from_numpy(nctor.view(np.int32)).to(dev)
        sc = torch.from_numpy(sctor.view(np.int32)).to(dev)
        self.nodes = ctx.alloc_for(variant, vf.APP_STUT, nt, nc)
        self.springs = ctx.alloc_for(variant, vf.APP_STUT, st, sc)
        self._pos = xc.BlockArray(n, self.per, rank, world, torch.float32, dev, rest=(2,), group=group, fill=0.0)
        self._pos.view.copy_(torch.from_numpy(np.ascontiguousarray(w["pos"], np.float32)))
        self.pos = self._pos.view
        self.F = torch.zeros((max(S, 1), 2), dtype=torch.float32, device=dev)
        self.inc_offs = torch.from_numpy(np.ascontiguousarray(w["inc_offs"], np.uint32).view(np.int32)).to(dev)
        self.inc = torch.from_numpy(np.ascontiguousarray(w["inc"], np.uint32).view(np.int32)).to(dev)
        self.fa = vf.stut_force_args(self.pos.data_ptr(), self.F.data_ptr(), float(w["break_ratio"]))
        self.ma = vf.stut_move_args(self.pos.data_ptr(), self.F.data_ptr(), self.inc_offs.data_ptr(),
                                    self.inc.data_ptr(), float(w["dt"]), float(w["damping"]), float(w["v_pull"]))
        torch.cuda.synchronize(dev)

    @property
    def calls_per_step(self):
        """owned springs + owned nodes (ghost springs are extra work, not counted)."""
        return self.n_own_springs + (self.hi - self.lo)

    def step(self, stream=None):
        s = vf._stream(stream)
        st = self.ctx.dispatch_raw(self.v, vf.APP_STUT, vf.STUT_FORCE, self.springs.data_ptr(),
                                   self.springs.numel(), self.fa, s)
        if st:
            self.ctx._check(st, "stut force")
        st = self.ctx.dispatch_raw(self.v, vf.APP_STUT, vf.STUT_MOVE, self.nodes.data_ptr(), self.nodes.numel(),
                                   self.ma, s)
        if st:
            self.ctx._check(st, "stut move")
        if self.world > 1 and self.exchange:
            self._pos.gather(stream)

    def positions(self):
        return self.pos.cpu().numpy()

    def velocities(self):
        """owned nodes [lo, hi) -> float32[hi-lo, 2]."""
        out = torch.zeros((self.hi - self.lo, 2), dtype=torch.float32, device=self.dev)
        self.ctx.dispatch(self.v, vf.APP_STUT, vf.STUT_GET, self.nodes, vf.stut_get_args(out.data_ptr(), 0, self.lo, 0))
        return out.cpu().numpy()

    def broken(self):
        """broken flag of every spring this rank holds, indexed by global spring id (uint8[S]; others 0)."""
        out = torch.zeros(max(self.S, 1), dtype=torch.uint8, device=self.dev)
        self.ctx.dispatch(self.v, vf.APP_STUT, vf.STUT_GET, self.springs,
                          vf.stut_get_args(0, out.data_ptr(), 0, 0))
        return out.cpu().numpy()[:self.S]

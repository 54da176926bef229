"""Config 5 all-pairs N-body driver over polymorphic bodies (reading G18).

Every body is a libvf object (Star / Planet / Dust); one step = one virtual
update() per body (libvf dispatch), reading all positions at the start of the
step and writing the body's new position into the other buffer.

Multi-GPU (§8e): bodies are split into contiguous id blocks; each rank owns
(allocates and dispatches) its block, every rank holds all positions, and
after each step the owned slices of the new position buffer are exchanged
with an all-gather over the process group (NCCL over NVLink on B200).
"""
from __future__ import annotations

import ctypes

import numpy as np
import torch

from . import exchange as xc, vf
from .exchange import block_range


class Nbody:
    def __init__(self, ctx: vf.Ctx, sys_: dict, variant: str = "typeptr", rank: int = 0, world: int = 1,
                 group=None, exchange: bool = True):
        self.ctx, self.variant = ctx, variant
        self.v = vf.VARIANTS[variant]
        dev = torch.device(f"cuda:{ctx.device}")
        self.dev = dev
        N = len(sys_["types"])
        self.N = N
        self.rank, self.world, self.group = rank, world, group
        self.exchange = exchange  # False: the caller stitches the owned slices (emulated ranks)
        self.lo, self.hi, self.per = block_range(N, rank, world)
        own = np.arange(self.lo, self.hi)
        ctor = np.zeros((len(own), 4), np.uint32)
        ctor[:, 0] = own
        ctor[:, 1:] = np.ascontiguousarray(sys_["vel"][own], dtype=np.float32).view(np.uint32)
        tt = torch.from_numpy(sys_["types"][own].astype(np.int32)).to(dev)
        ct = torch.from_numpy(ctor.view(np.int32)).to(dev)
        self.objs = ctx.alloc_for(variant, vf.APP_NBODY, tt, ct)
        pos = torch.from_numpy(np.ascontiguousarray(sys_["pos"], dtype=np.float32)).to(dev)
        # double-buffered positions in persistent buffers padded to per * world
        # rows; the owned block of the new buffer is all-gathered in place
        self._p = [xc.BlockArray(N, self.per, rank, world, torch.float32, dev, rest=(4,), group=group, fill=0.0)
                   for _ in range(2)]
        self._p[0].view.copy_(pos)
        self.p = [b.view for b in self._p]
        self.dt = float(sys_["dt"])
        self.eps2 = [float(x) for x in sys_["eps2"]]
        self.damp = float(sys_["damp"])
        torch.cuda.synchronize(dev)

    @property
    def calls_per_step(self):
        return self.hi - self.lo

    def _args(self):
        return vf.nbody_update_args(self.p[0].data_ptr(), self.p[1].data_ptr(), self.N, self.dt,
                                    (ctypes.c_float * 3)(*self.eps2), self.damp)

    def step(self, stream=None):
        s = vf._stream(stream)
        st = self.ctx.dispatch_raw(self.v, vf.APP_NBODY, vf.NBODY_UPDATE, self.objs.data_ptr(),
                                   self.hi - self.lo, self._args(), s)
        if st:
            self.ctx._check(st, "nbody update")
        if self.world > 1 and self.exchange:
            self._p[1].gather(stream)
        self._p.reverse()
        self.p = [b.view for b in self._p]

    def positions(self):
        return self.p[0].cpu().numpy()

    def velocities(self):
        """Velocities of the owned block [lo, hi), float32[hi-lo, 3]."""
        out = torch.zeros((self.hi - self.lo, 3), dtype=torch.float32, device=self.dev)
        self.ctx.dispatch(self.v, vf.APP_NBODY, vf.NBODY_GET, self.objs,
                          vf.nbody_get_args(out.data_ptr(), self.lo))
        return out.cpu().numpy()

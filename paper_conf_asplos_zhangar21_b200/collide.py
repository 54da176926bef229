"""Config 5 collision driver at 16M bodies (readings G18 / G19; vf.h VF_APP_COLLIDE).

Every body is a libvf object (Star / Planet / Dust) holding its velocity;
positions + masses are float4 arrays indexed by body id. One step:
  (0) vf_collide_grid: uniform grid (cells of side rc), cell-sorted positions,
      and the dispatch order = owned active objects in cell order;
  (1) one virtual update() per active body  (P -> Pm, Vm, near);
  (2) one virtual merge() per active body   (Pm, Vm, near -> P).

Multi-GPU (§8e): bodies are split into contiguous id blocks. Every rank holds
all positions and builds the (replicated) grid; it dispatches its own bodies
only. After update only the bodies with a merge candidate (near >= 0, a few
per mille) travel, as packed (id, near, Pm, Vm) entries (a merge partner may
live on another rank); after merge the owned slices of P are all-gathered.
"""
from __future__ import annotations

import ctypes

import numpy as np
import torch

from . import exchange as xc, vf
from .exchange import block_range


class Collide:
    def __init__(self, ctx: vf.Ctx, sys_: dict, variant: str = "typeptr", rank: int = 0, world: int = 1,
                 group=None, exchange: bool = True):
        self.ctx, self.variant = ctx, variant
        self.v = vf.VARIANTS[variant]
        dev = torch.device(f"cuda:{ctx.device}")
        self.dev = dev
        N = len(sys_["types"])
        self.N, self.G = N, int(sys_["G"])
        self.rank, self.world, self.group, self.exchange = rank, world, group, exchange
        self.lo, self.hi, self.per = block_range(N, rank, world)
        own = np.arange(self.lo, self.hi)
        ctor = np.zeros((len(own), 4), np.uint32)
        ctor[:, 0] = own
        ctor[:, 1:] = np.ascontiguousarray(sys_["vel"][own, :3], dtype=np.float32).view(np.uint32)
        tt = torch.from_numpy(sys_["types"][own].astype(np.int32)).to(dev)
        ct = torch.from_numpy(ctor.view(np.int32)).to(dev)
        self.objs = ctx.alloc_for(variant, vf.APP_COLLIDE, tt, ct)
        f4 = dict(dtype=torch.float32, device=dev)
        blk = dict(n=N, per=self.per, rank=rank, world=world, device=dev, group=group)
        self._P = xc.BlockArray(dtype=torch.float32, rest=(4,), fill=0.0, **blk)
        self._P.view.copy_(torch.from_numpy(np.ascontiguousarray(sys_["pos"], dtype=np.float32)))
        self._Pm = xc.BlockArray(dtype=torch.float32, rest=(4,), fill=0.0, **blk)
        self._Vm = xc.BlockArray(dtype=torch.float32, rest=(4,), fill=0.0, **blk)
        self._near = xc.BlockArray(dtype=torch.int32, fill=-1, **blk)
        self.P, self.Pm, self.Vm, self.near = self._P.view, self._Pm.view, self._Vm.view, self._near.view
        self._vg = None  # variable-length exchange after update (created on first use)
        self.Ps = torch.zeros((max(N, 1), 4), **f4)
        ncell = self.G ** 3
        u32 = dict(dtype=torch.int32, device=dev)
        self.cell_of = torch.zeros(max(N, 1), **u32)
        self.cell_count = torch.zeros(ncell, **u32)
        self.cell_start = torch.zeros(ncell + 1, **u32)
        self.list = torch.zeros(max(N, 1), **u32)
        self.slot = torch.zeros(max(N, 1), **u32)
        self.tmp = torch.zeros(int(vf.lib().vf_collide_tmp_words(N, self.G)), **u32)
        self.order = torch.zeros(max(self.hi - self.lo, 1), dtype=torch.int64, device=dev)
        self.active = torch.zeros(1, dtype=torch.int64, device=dev)  # owned active bodies, summed over steps
        rc, rm = np.float32(sys_["rc"]), np.float32(sys_["rm"])
        self.rc, self.rc2, self.rm2 = float(rc), float(rc * rc), float(rm * rm)
        self.dt, self.damp = float(sys_["dt"]), float(sys_["damp"])
        self.eps2 = [float(x) for x in sys_["eps2"]]
        self._grid = vf.collide_grid_args(
            N, self.G, self.rc, self.P.data_ptr(), self.cell_of.data_ptr(), self.cell_count.data_ptr(),
            self.cell_start.data_ptr(), self.list.data_ptr(), self.Ps.data_ptr(), self.slot.data_ptr(),
            self.tmp.data_ptr(),
            self.objs.data_ptr() if self.hi > self.lo else None, self.lo, self.hi, self.order.data_ptr(),
            self.active.data_ptr())
        self._upd = vf.collide_update_args(
            self.P.data_ptr(), self.Ps.data_ptr(), self.list.data_ptr(), self.cell_start.data_ptr(),
            self.slot.data_ptr(), self.Pm.data_ptr(), self.Vm.data_ptr(), self.near.data_ptr(), self.G, self.rc, self.rc2, self.rm2,
            self.dt, (ctypes.c_float * 3)(*self.eps2), self.damp)
        self._mrg = vf.collide_merge_args(self.Pm.data_ptr(), self.Vm.data_ptr(), self.near.data_ptr(),
                                          self.P.data_ptr())
        torch.cuda.synchronize(dev)

    @property
    def n_owned(self):
        return self.hi - self.lo

    def grid(self, stream=None):
        st = vf.lib().vf_collide_grid(ctypes.byref(self._grid), vf._stream(stream))
        if st:
            self.ctx._check(st, "collide grid")

    def update(self, stream=None):
        """Steps (0) and (1): grid, then one virtual update() per owned active body."""
        self.grid(stream)
        self.ctx._check(self.ctx.dispatch_raw(self.v, vf.APP_COLLIDE, vf.COLLIDE_UPDATE, self.order.data_ptr(),
                                              self.n_owned, self._upd, vf._stream(stream)), "collide update")

    def exchange_update(self, stream=None):
        """merge() of body i reads near / Pm / Vm of j = near[i] only when j has a
        candidate too (near[j] >= 0): only those bodies' entries travel
        (vf_collide_pack_near -> all-gather of the packed lists ->
        vf_collide_unpack_near), a few per mille of the bodies instead of the
        whole 36 B/body arrays."""
        if not (self.world > 1 and self.exchange):
            return
        L = vf.lib()
        s = vf._stream(stream)
        if self._vg is None:
            self._vg = xc.VarGather(self.world, ctypes.sizeof(vf.collide_near_entry), self.dev, self.group)
            self._cnt = torch.zeros(1, dtype=torch.int32, device=self.dev)
        send = self._vg.send_buffer(max(self.per, 1))  # worst case: every owned body has a candidate
        with xc._on(stream, self._cnt):
            self._cnt.zero_()
        self.ctx._check(L.vf_collide_pack_near(self.lo, self.hi, self.near.data_ptr(), self.Pm.data_ptr(),
                                               self.Vm.data_ptr(), send.data_ptr(), self._cnt.data_ptr(), s),
                        "collide pack")
        with xc._on(stream, self._cnt):
            count = int(self._cnt.item())
        recv, counts, seg = self._vg.gather(count, stream)
        self.ctx._check(L.vf_collide_unpack_near(recv.data_ptr(), self.world, seg, counts.data_ptr(), self.N,
                                                 self.lo, self.hi, self.near.data_ptr(), self.Pm.data_ptr(),
                                                 self.Vm.data_ptr(), s), "collide unpack")

    def merge(self, stream=None):
        """Step (2): one virtual merge() per owned active body."""
        self.ctx._check(self.ctx.dispatch_raw(self.v, vf.APP_COLLIDE, vf.COLLIDE_MERGE, self.order.data_ptr(),
                                              self.n_owned, self._mrg, vf._stream(stream)), "collide merge")

    def exchange_merge(self, stream=None):
        if self.world > 1 and self.exchange:
            self._P.gather(stream)

    def step(self, stream=None):
        self.update(stream)
        self.exchange_update(stream)
        self.merge(stream)
        self.exchange_merge(stream)

    def calls(self) -> int:
        """Virtual calls issued so far by this rank (2 per owned active body per step)."""
        return 2 * int(self.active.item())

    def positions(self):
        return self.P.cpu().numpy()

    def velocities(self):
        """Velocities of the owned block [lo, hi), float32[hi-lo, 3]."""
        out = torch.zeros((self.hi - self.lo, 3), dtype=torch.float32, device=self.dev)
        self.ctx.dispatch(self.v, vf.APP_COLLIDE, vf.COLLIDE_GET, self.objs,
                          vf.collide_get_args(out.data_ptr(), self.lo))
        return out.cpu().numpy()

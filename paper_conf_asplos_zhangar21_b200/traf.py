"""Config 5 TRAF driver: Nagel-Schreckenberg rings (Table 2, reading G16).

Every cell and vehicle is a libvf object; one step = a virtual update() on
every cell, then a virtual step() on every vehicle (libvf dispatch). The
rings are independent, so multi-GPU splits whole rings across ranks with no
data-path collective (§8e).
"""
from __future__ import annotations

import numpy as np
import torch

from . import vf


class Traf:
    def __init__(self, ctx: vf.Ctx, world: dict, variant: str = "typeptr", rank: int = 0, nranks: int = 1):
        self.ctx, self.variant = ctx, variant
        self.v = vf.VARIANTS[variant]
        dev = torch.device(f"cuda:{ctx.device}")
        self.dev = dev
        R, L = world["R"], world["L"]
        # this rank's rings [r0, r1): cells and vehicles re-indexed locally
        per = (R + nranks - 1) // nranks
        r0, r1 = min(R, rank * per), min(R, (rank + 1) * per)
        self.R, self.L = r1 - r0, L
        N = self.R * L
        self.N = N
        vsel = (world["veh_ring"] >= r0) & (world["veh_ring"] < r1)
        self.vid_global = np.nonzero(vsel)[0]
        nveh = int(vsel.sum())
        self.nveh = nveh
        light = world["light"][r0 * L:r1 * L]
        phase = world["phase"][r0 * L:r1 * L]
        tag = variant == "typeptr"
        cell_types = torch.from_numpy(light.astype(np.int32)).to(dev)  # 0 Plain, 1 Light
        cell_args = torch.from_numpy(np.stack([np.arange(N, dtype=np.uint32), phase.astype(np.uint32)], 1)
                                     .copy().view(np.int32)).to(dev)
        veh_types = torch.from_numpy((world["veh_type"][vsel] + 2).astype(np.int32)).to(dev)
        vargs = np.zeros((nveh, 4), np.uint32)
        vargs[:, 0] = self.vid_global  # global ids: the slow-down draws are keyed by id
        self.id_base = int(self.vid_global[0]) if nveh else 0
        vargs[:, 1] = world["veh_ring"][vsel] - r0
        vargs[:, 2] = world["veh_pos"][vsel]
        veh_args = torch.from_numpy(vargs.view(np.int32)).to(dev)
        self.cells = ctx.alloc_for(variant, vf.APP_TRAF, cell_types, cell_args)
        self.vehs = ctx.alloc_for(variant, vf.APP_TRAF, veh_types, veh_args)
        self.occ = [torch.zeros(N, dtype=torch.uint8, device=dev) for _ in range(2)]
        self.blocked = torch.zeros(N, dtype=torch.uint8, device=dev)
        self.seed = world["seed"]
        self.vmax = [int(x) for x in world["vmax"]]
        self.thr = [int(x) for x in world["slow_thr"]]
        self.t = 0
        self.ctx.dispatch(self.v, vf.APP_TRAF, vf.TRAF_PLACE, self.vehs,
                          vf.traf_get_args(0, 0, self.occ[0].data_ptr(), L))
        torch.cuda.synchronize(dev)

    @property
    def calls_per_step(self):
        return self.N + self.nveh

    def step(self, stream=None):
        s = vf._stream(stream)
        ca = vf.traf_cell_args(self.blocked.data_ptr(), self.occ[1].data_ptr(), self.t)
        st = self.ctx.dispatch_raw(self.v, vf.APP_TRAF, vf.TRAF_CELL_UPDATE, self.cells.data_ptr(), self.N, ca, s)
        if st:
            self.ctx._check(st, "traf cell update")
        sa = vf.traf_step_args(self.occ[0].data_ptr(), self.blocked.data_ptr(), self.occ[1].data_ptr(), self.L,
                               self.t, self.seed, (ctypes_u32x3(self.vmax)), (ctypes_u32x3(self.thr)))
        st = self.ctx.dispatch_raw(self.v, vf.APP_TRAF, vf.TRAF_VEH_STEP, self.vehs.data_ptr(), self.nveh, sa, s)
        if st:
            self.ctx._check(st, "traf vehicle step")
        self.occ[0], self.occ[1] = self.occ[1], self.occ[0]
        self.t += 1

    def state(self):
        pos = torch.empty(self.nveh, dtype=torch.int32, device=self.dev)
        vel = torch.empty(self.nveh, dtype=torch.int32, device=self.dev)
        self.ctx.dispatch(self.v, vf.APP_TRAF, vf.TRAF_GET, self.vehs,
                          vf.traf_get_args(pos.data_ptr(), vel.data_ptr(), 0, self.L, self.id_base))
        return pos.cpu().numpy().view(np.uint32), vel.cpu().numpy().view(np.uint32)


def ctypes_u32x3(vals):
    import ctypes
    return (ctypes.c_uint32 * 3)(*vals)

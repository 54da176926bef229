"""Config 3 driver: ray tracer over polymorphic shapes (Table 2 RAY).

Allocates the scene's shape objects through libvf (typed arenas / device heap)
and renders with vf_ray_render. Multi-GPU: 8-row pixel strips are dealt
round-robin to ranks (§8e); each rank renders its strips (independent, no
data-path collective) and the image is assembled once at the end
(Ray.gather_image: one all-reduce each of rgb and hit ids), outside the timed
calls/s.
"""
from __future__ import annotations

import ctypes

import numpy as np
import torch

import synth

from . import vf


class Ray:
    STRIP = 8

    def __init__(self, ctx: vf.Ctx, types, params, variant: str = "typeptr"):
        self.ctx, self.variant = ctx, variant
        self.v = vf.VARIANTS[variant]
        dev = torch.device(f"cuda:{ctx.device}")
        self.dev = dev
        self.S = len(types)
        tt = torch.from_numpy(np.asarray(types, np.int32)).to(dev)
        pp = torch.from_numpy(np.ascontiguousarray(params, np.float32)).to(dev)
        self.objs = ctx.alloc_for(variant, vf.APP_RAY, tt, pp)
        self.albedo = (ctypes.c_float * 12)(*synth.RAY_ALBEDO.reshape(-1).tolist())
        torch.cuda.synchronize(dev)

    def render(self, W: int, H: int, cam, row0: int = 0, nrows: int | None = None, rgb=None, hid=None,
               stream=None):
        nrows = H - row0 if nrows is None else nrows
        if rgb is None:
            rgb = torch.empty((nrows, W, 3), dtype=torch.float32, device=self.dev)
        if hid is None:
            hid = torch.empty((nrows, W), dtype=torch.int32, device=self.dev)
        c = (ctypes.c_float * 5)(*[float(x) for x in cam])
        st = vf.lib().vf_ray_render(self.ctx.h, self.v, self.objs.data_ptr(), self.S, W, H, row0, nrows, c,
                                    self.albedo, rgb.data_ptr(), hid.data_ptr(), vf._stream(stream))
        if st:
            self.ctx._check(st, "ray_render")
        return rgb, hid

    def strips(self, H: int, rank: int, world: int):
        """8-row strips [row0, row0+n) owned by `rank` (round-robin)."""
        k = 0
        out = []
        for r0 in range(0, H, self.STRIP):
            if k % world == rank:
                out.append((r0, min(self.STRIP, H - r0)))
            k += 1
        return out

    @staticmethod
    def gather_image(rgb, hid, world: int, group=None):
        """Assemble the frame on every rank after render_frame (once
        per frame, outside the timed calls/s). Rows a rank does not own hold
        rgb 0 and hit id -1, so one SUM all-reduce of rgb (x + 0 = x exactly)
        and one MAX all-reduce of the hit ids (-1 < any id) give every rank the
        whole image."""
        if world == 1:
            return rgb, hid
        import torch.distributed as dist
        from . import exchange
        if exchange._staged(rgb, group):
            hr, hh = rgb.cpu(), hid.cpu()
            dist.all_reduce(hr, group=group)
            dist.all_reduce(hh, op=dist.ReduceOp.MAX, group=group)
            rgb.copy_(hr)
            hid.copy_(hh)
        else:
            dist.all_reduce(rgb, group=group)
            dist.all_reduce(hid, op=dist.ReduceOp.MAX, group=group)
        return rgb, hid

    def render_frame(self, W: int, H: int, cam, rank: int = 0, world: int = 1, rgb=None, hid=None, stream=None):
        """Render this rank's strips into full-frame buffers (rows it does not own
        keep rgb 0 / hit id -1; gather_image assembles the frame)."""
        if rgb is None:
            rgb = torch.zeros((H, W, 3), dtype=torch.float32, device=self.dev)
        if hid is None:
            hid = torch.full((H, W), -1, dtype=torch.int32, device=self.dev)
        if world == 1:
            return self.render(W, H, cam, 0, H, rgb, hid, stream)
        for r0, n in self.strips(H, rank, world):
            self.render(W, H, cam, r0, n, rgb[r0:r0 + n], hid[r0:r0 + n], stream)
        return rgb, hid

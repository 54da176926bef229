"""Workload drivers over the C ABI (argument marshalling and step sequencing only).

Each driver allocates its objects through libvf (typed arenas for sharedoa /
coal / typeptr, device-heap `new` for cuda), then a `step()` enqueues the
app's kernels on a stream. Inputs come from ``synth`` (seeded; shared with the
oracle tests); nothing here computes any part of the method.
"""
from __future__ import annotations

import numpy as np
import torch

import synth

from . import vf


def _dev(device):
    return torch.device(f"cuda:{device}" if isinstance(device, int) else device)


class Micro:
    """Config 2: one virtual `apply()` per object over n objects of T types.

    Paper §8.3. Object i has type t(i) (synth.micro_types) and
    val = init_i; after R steps val_i = init_i + R (t(i)+1).
    """

    # variants beyond the four of vf.h: comparison points of the paper
    #   concord       embedded type tag + switch (§7), typed arenas
    #   typeptr_heap  TypePointer tags on device-heap `new` objects (§8.2 Fig. 11)
    EXTRA = {"typeptr_heap": vf.TYPEPTR}

    def __init__(self, ctx: vf.Ctx, n: int, T: int, order: str = "random", seed: int = 42,
                 variant: str = "typeptr", k: int | None = None, types_np=None, init_np=None):
        self.ctx, self.n, self.T, self.variant = ctx, n, T, variant
        self.v = self.EXTRA[variant] if variant in self.EXTRA else vf.VARIANTS[variant]
        dev = _dev(ctx.device)
        if types_np is None:
            types_np = synth.micro_types(n, T, order, seed=seed, k=k)
        if init_np is None:
            init_np = synth.micro_init(n, seed=seed)
        self.types = torch.from_numpy(types_np.astype(np.int32)).to(dev)
        init = torch.from_numpy(init_np.astype(np.int32)).to(dev)
        if variant in ("cuda", "typeptr_heap"):
            self.objs = ctx.alloc_cuda(vf.APP_MICRO, self.types, init, tag=(variant == "typeptr_heap"))
        elif variant == "cuda_packed":
            self.objs = ctx.alloc_packed(vf.APP_MICRO, self.types, init)
        else:
            self.objs = ctx.alloc_typed_batch(vf.APP_MICRO, self.types, init, tag=(variant == "typeptr"))
        torch.cuda.synchronize(dev)
        self._ptr = int(self.objs.data_ptr())

    def step(self, stream=None):
        st = self.ctx.dispatch_raw(self.v, vf.APP_MICRO, vf.MICRO_APPLY, self._ptr, self.n, None,
                                   vf._stream(stream))
        if st:
            self.ctx._check(st, "micro step")

    def values(self, out=None, stream=None):
        if out is None:
            out = torch.empty(self.n, dtype=torch.int32, device=self.objs.device)
        self.ctx.dispatch(self.v, vf.APP_MICRO, vf.MICRO_GET, self.objs,
                          vf.micro_get_args(out.data_ptr()), stream=stream)
        return out


class MicroBranch:
    """BRANCH ceiling of config 2 (§8.3): no objects, the type comes
    from registers, a switch picks the addition (vf_micro_branch)."""

    def __init__(self, ctx: vf.Ctx, n: int, T: int, order: str = "random", seed: int = 42, k: int | None = None,
                 init_np=None):
        self.n, self.T, self.order, self.seed = n, T, order, seed
        self.k = (T if k is None else k) if order == "kperwarp" else 1
        if init_np is None:
            init_np = synth.micro_init(n, seed=seed)
        self.vals = torch.from_numpy(init_np.astype(np.int32)).to(_dev(ctx.device))

    def step(self, stream=None):
        vf.micro_branch(self.vals, self.T, self.order, self.seed, self.k, stream)

    def values(self, out=None, stream=None):
        return self.vals


class Gol:
    """Config 1: Game of Life over polymorphic Alive / Dead cells (Table 2).

    Per generation: (1) vf_gol_neighbors, (2) one virtual next() per
    cell, (3) vf_gol_swap. Every cell owns one object in each type's arena, so
    a type change is a pointer swap.
    """

    def __init__(self, ctx: vf.Ctx, W: int, H: int, alive0, variant: str = "typeptr",
                 torus: bool = False):
        self.ctx, self.W, self.H, self.variant, self.torus = ctx, W, H, variant, torus
        self.v = vf.VARIANTS[variant]
        dev = _dev(ctx.device)
        N = W * H
        self.N = N
        cells = torch.arange(N, dtype=torch.int32, device=dev)
        if variant in ("cuda", "cuda_packed"):
            self.alive = ctx.alloc_for(variant, vf.APP_GOL, torch.ones(N, dtype=torch.int32, device=dev), cells)
            self.dead = ctx.alloc_for(variant, vf.APP_GOL, torch.zeros(N, dtype=torch.int32, device=dev), cells)
        else:
            tag = variant == "typeptr"
            self.alive = ctx.alloc_typed(vf.APP_GOL, 1, N, cells, tag=tag)
            self.dead = ctx.alloc_typed(vf.APP_GOL, 0, N, cells, tag=tag)
        self.grid = self.dead.clone()
        a0 = torch.from_numpy(np.ascontiguousarray(alive0, dtype=np.uint8)).to(dev)
        zeros = torch.zeros(N, dtype=torch.uint8, device=dev)
        vf.gol_swap(ctx, zeros, a0, self.grid, self.alive, self.dead)  # grid <- initial types
        self.state = a0.clone()
        self.next = torch.empty_like(self.state)
        self.nbr = torch.empty_like(self.state)
        self.args = [vf.gol_next_args(self.nbr.data_ptr(), self.next.data_ptr()),
                     vf.gol_next_args(self.nbr.data_ptr(), self.state.data_ptr())]
        self.parity = 0
        torch.cuda.synchronize(dev)

    def gen(self, stream=None, fused: bool = True):
        """One generation. fused (default, B200 design): one vf_gol_step launch;
        else the three phases as separate calls (neighbours, dispatch, swap)."""
        cur, nxt = (self.state, self.next) if self.parity == 0 else (self.next, self.state)
        if fused:
            vf.gol_step(self.ctx, self.v, self.W, self.H, self.torus, cur, nxt, self.nbr, self.grid, self.alive,
                        self.dead, stream)
        else:
            vf.gol_neighbors(self.W, self.H, cur, self.nbr, self.torus, stream)
            self.ctx.dispatch(self.v, vf.APP_GOL, vf.GOL_NEXT, self.grid, self.args[self.parity], stream=stream)
            vf.gol_swap(self.ctx, cur, nxt, self.grid, self.alive, self.dead, stream)
        self.parity ^= 1

    def run(self, gens: int, stream=None):
        """`gens` generations in ONE persistent cooperative launch (vf_gol_run):
        same results as `gens` calls of gen()."""
        if not hasattr(self, "barrier"):
            self.barrier = torch.zeros(1, dtype=torch.int32, device=self.grid.device)
        s0, s1 = (self.state, self.next) if self.parity == 0 else (self.next, self.state)
        vf.gol_run(self.ctx, self.v, self.W, self.H, self.torus, s0, s1, self.nbr, self.grid, self.alive, self.dead,
                   gens, self.barrier, stream)
        self.parity ^= gens & 1

    @property
    def current(self):
        return self.state if self.parity == 0 else self.next

    def counters(self):
        ctr = torch.empty(self.N, dtype=torch.int16, device=self.grid.device)
        typ = torch.empty(self.N, dtype=torch.uint8, device=self.grid.device)
        self.ctx.dispatch(self.v, vf.APP_GOL, vf.GOL_GET, self.grid,
                          vf.gol_get_args(ctr.data_ptr(), typ.data_ptr()))
        return ctr, typ


def rule_masks(born: str, survive: str):
    """'B2/S345' digit strings -> (born_mask, survive_mask)."""
    return sum(1 << int(d) for d in str(born)), sum(1 << int(d) for d in str(survive))


class Gen:
    """Config 5 GEN: Generations CA B/S/C over polymorphic Dead / Alive / Dying cells
    (Table 2, reading G15). Same three steps per generation as Gol.

    Multi-GPU: row slabs. Rank r owns rows [r0, r1) (objects for
    its cells only) and runs vf_gen_step_rows on them; after every generation
    the boundary rows go to the neighbour slabs (exchange.HaloRows,
    batch_isend_irecv of one W-byte row each way)."""

    def __init__(self, ctx: vf.Ctx, W: int, H: int, state0, variant: str = "typeptr",
                 born: str = "2", survive: str = "345", C: int = 4, torus: bool = False,
                 rank: int = 0, world: int = 1, group=None):
        from . import exchange
        self.ctx, self.W, self.H, self.variant, self.torus = ctx, W, H, variant, torus
        self.v = vf.VARIANTS[variant]
        dev = _dev(ctx.device)
        N = W * H
        self.N = N
        self.rank, self.world = rank, world
        self.halo = exchange.HaloRows(W, H, rank, world, torus, group)
        self.r0, self.r1 = self.halo.r0, self.halo.r1
        lo, hi = self.r0 * W, self.r1 * W
        self.lo, self.hi = lo, hi
        cells = torch.arange(lo, hi, dtype=torch.int32, device=dev)
        objs = []
        for t in range(3):
            o = torch.zeros(N, dtype=torch.int64, device=dev)
            if variant in ("cuda", "cuda_packed"):
                o[lo:hi] = ctx.alloc_for(variant, vf.APP_GEN, torch.full((hi - lo,), t, dtype=torch.int32, device=dev),
                                         cells)
            else:
                o[lo:hi] = ctx.alloc_typed(vf.APP_GEN, t, hi - lo, cells, tag=(variant == "typeptr"))
            objs.append(o)
        self.dead, self.alive, self.dying = objs
        self.grid = self.dead.clone()
        s0 = torch.from_numpy(np.ascontiguousarray(state0, dtype=np.uint8).reshape(-1)).to(dev)
        zeros = torch.zeros(hi - lo, dtype=torch.uint8, device=dev)
        vf.gen_swap(ctx, zeros, s0[lo:hi], self.grid[lo:hi], self.dead[lo:hi], self.alive[lo:hi],
                    self.dying[lo:hi])
        self.state = s0.clone()
        self.next = self.state.clone()
        self.nbr = torch.zeros_like(self.state)
        bm, sm = rule_masks(born, survive)
        self.rule = (bm, sm, C)
        self.args = [vf.gen_next_args(self.nbr.data_ptr(), self.next.data_ptr(), bm, sm, C),
                     vf.gen_next_args(self.nbr.data_ptr(), self.state.data_ptr(), bm, sm, C)]
        self.parity = 0
        torch.cuda.synchronize(dev)

    @property
    def calls_per_gen(self):
        return self.hi - self.lo

    def gen(self, stream=None, fused: bool = True):
        cur, nxt = (self.state, self.next) if self.parity == 0 else (self.next, self.state)
        if fused:
            vf.gen_step_rows(self.ctx, self.v, self.W, self.H, self.torus, self.r0, self.r1 - self.r0, cur, nxt,
                             self.nbr, self.grid, self.dead, self.alive, self.dying, *self.rule, stream)
        else:
            assert self.world == 1, "the unfused form is single-GPU"
            vf.gol_neighbors(self.W, self.H, cur, self.nbr, self.torus, stream)
            self.ctx.dispatch(self.v, vf.APP_GEN, vf.GEN_NEXT, self.grid, self.args[self.parity], stream=stream)
            vf.gen_swap(self.ctx, cur, nxt, self.grid, self.dead, self.alive, self.dying, stream)
        self.halo.exchange(nxt, stream)
        self.parity ^= 1

    @property
    def current(self):
        return self.state if self.parity == 0 else self.next

    def counters(self):
        """(counter, type) per cell; only the owned rows [r0, r1) are written (others 0)."""
        ctr = torch.zeros(self.N, dtype=torch.int16, device=self.grid.device)
        typ = torch.zeros(self.N, dtype=torch.uint8, device=self.grid.device)
        self.ctx.dispatch(self.v, vf.APP_GEN, vf.GEN_GET, self.grid[self.lo:self.hi],
                          vf.gen_get_args(ctr.data_ptr(), typ.data_ptr()))
        return ctr, typ

"""GPU parity for the config-2 microbenchmark: CUDA path (through the C ABI) vs the CPU oracle.

Integer work -> bit-exact. Sizes span several 4096-object regions and CTA tiles
with a ragged tail; the full-size (64M) case checks sampled outputs against the
closed form and brute-force type identity over every pointer.
"""
import numpy as np
import pytest
import torch

import oracle
import synth
from paper_conf_asplos_zhangar21_b200 import apps, vf

pytestmark = pytest.mark.gpu
VARIANTS = ["cuda", "sharedoa", "coal", "typeptr"]


@pytest.fixture(scope="module")
def ctx():
    c = vf.Ctx(0, cuda_heap_bytes=4 << 30)
    yield c
    c.close()


@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("T,order", [(1, "random"), (2, "random"), (4, "random"), (4, "sorted"),
                                     (32, "random"), (32, "sorted"), (32, "kperwarp"), (3, "kperwarp")])
def test_micro_parity(ctx, variant, T, order):
    n, R = 3 * 4096 * 8 + 1234, 3
    types = synth.micro_types(n, T, order, seed=42, k=min(T, 7))
    init = synth.micro_init(n, seed=42)
    ref, _ = oracle.micro_run(types, init, T, R)
    m = apps.Micro(ctx, n, T, variant=variant, types_np=types, init_np=init)
    for _ in range(R):
        m.step()
    got = m.values().cpu().numpy()
    assert np.array_equal(got, ref)
    assert ctx.verify(vf.APP_MICRO, m.v, m.objs) == 0
    res = ctx.resolve(vf.APP_MICRO, m.v, m.objs).cpu().numpy()
    assert np.array_equal(res.astype(np.uint32), types)


@pytest.mark.parametrize("unroll", [1, 2, 4])
@pytest.mark.parametrize("prefetch", [0, 1, 2, 3])
@pytest.mark.parametrize("pipeline,regroup", [(0, 0), (1, 0), (0, 1), (0, 2)])
@pytest.mark.parametrize("variant", ["coal", "typeptr"])
@pytest.mark.parametrize("n", [50_000 + 3, 1024 * 300, 100])
def test_micro_tuning_knobs(ctx, unroll, prefetch, pipeline, regroup, variant, n):
    T, R = 8, 2
    types = synth.micro_types(n, T, "random", seed=3)
    init = synth.micro_init(n, seed=3)
    ref, _ = oracle.micro_run(types, init, T, R)
    vf.set_tuning("unroll", unroll)
    vf.set_tuning("prefetch", prefetch)
    vf.set_tuning("pipeline", pipeline)
    vf.set_tuning("regroup", regroup)
    try:
        m = apps.Micro(ctx, n, T, variant=variant, types_np=types, init_np=init)
        for _ in range(R):
            m.step()
        assert np.array_equal(m.values().cpu().numpy(), ref)
    finally:
        vf.set_tuning("unroll", -1)
        vf.set_tuning("prefetch", -1)
        vf.set_tuning("pipeline", 0)
        vf.set_tuning("regroup", 1)


@pytest.mark.parametrize("n", [0, 1, 31, 33, 255, 257, 4097])
@pytest.mark.parametrize("variant", VARIANTS)
def test_micro_small_and_ragged(ctx, n, variant):
    T = 5
    types = synth.micro_types(n, T, "random", seed=n)
    init = synth.micro_init(n, seed=n)
    ref, _ = oracle.micro_run(types, init, T, 2)
    if n == 0:
        return
    m = apps.Micro(ctx, n, T, variant=variant, types_np=types, init_np=init)
    m.step()
    m.step()
    assert np.array_equal(m.values().cpu().numpy(), ref)


def test_null_pointers_skipped_and_fallback(ctx):
    """Null entries are skipped; pointers COAL cannot resolve (device-heap objects,
    outside every range) and untagged pointers under TypePointer fall back to the
    embedded vTable* (P:1305-1311)."""
    n, T = 3000, 4
    types = synth.micro_types(n, T, "random", seed=9)
    init = synth.micro_init(n, seed=9)
    dev = torch.device("cuda:0")
    typed = ctx.alloc_typed_batch(vf.APP_MICRO, torch.from_numpy(types.astype(np.int32)).to(dev),
                                  torch.from_numpy(init).to(dev))
    heap = ctx.alloc_cuda(vf.APP_MICRO, torch.from_numpy(types.astype(np.int32)).to(dev),
                          torch.from_numpy(init).to(dev))
    # mix: even i -> typed arena object, odd i -> heap object, every 7th -> null
    mixed = torch.where(torch.arange(n, device=dev) % 2 == 0, typed, heap)
    mixed[::7] = 0
    expect = init + (types.astype(np.int32) + 1)
    expect[::7] = init[::7]
    for variant in ("coal", "typeptr", "sharedoa"):
        ctx.dispatch(vf.VARIANTS[variant], vf.APP_MICRO, vf.MICRO_APPLY, mixed)
        # read back through the CUDA rule (works for every pointer)
        vals = torch.zeros(n, dtype=torch.int32, device=dev)
        ctx.dispatch(vf.CUDA, vf.APP_MICRO, vf.MICRO_GET, mixed, vf.micro_get_args(vals.data_ptr()))
        got = vals.cpu().numpy()
        nonnull = np.ones(n, bool)
        nonnull[::7] = False
        assert np.array_equal(got[nonnull], expect[nonnull]), variant
        assert np.array_equal(got[~nonnull], np.zeros((~nonnull).sum(), np.int32))
        # the next variant applies once more on the same objects
        expect = np.where(nonnull, got + (types.astype(np.int32) + 1), expect)
    res = ctx.resolve(vf.APP_MICRO, vf.COAL, mixed).cpu().numpy().view(np.uint32)
    assert np.all(res[1::2][(np.arange(1, n, 2) % 7) != 0] == vf.NOT_FOUND)


def test_range_table_matches_oracle_and_closed_form():
    """reserve_va=0: one cudaMalloc per region -> the table follows the paper's
    doubling policy; compare with oracle.region_plan and oracle.build_table."""
    c = vf.Ctx(0, reserve_va=False, cuda_heap_bytes=0)
    try:
        n, T = 100_000, 4
        types = synth.micro_types(n, T, "random", seed=5)
        init = synth.micro_init(n, seed=5)
        m = apps.Micro(c, n, T, variant="coal", types_np=types, init_np=init)
        regs = c.regions()
        counts = np.bincount(types, minlength=T)
        for t in range(T):
            caps = [r["cap_objs"] for r in regs if r["type_id"] == t]
            assert caps == oracle.region_plan(int(counts[t]), 4096)
        ts, te, tt = oracle.build_table([r["start"] for r in regs],
                                        [r["cap_objs"] * r["obj_bytes"] for r in regs],
                                        [r["type_id"] for r in regs])
        rows = c.range_table(vf.APP_MICRO)
        assert [(r.start, r.end, r.type_id) for r in rows] == list(zip(ts, te, tt))
        vptrs = c.type_vptrs(vf.APP_MICRO)
        assert all(r.vptr == vptrs[r.type_id] for r in rows)
        # COAL over the fragmented table, plus oracle Alg. 1 on the same addresses
        m.step()
        ref, _ = oracle.micro_run(types, init, T, 1)
        assert np.array_equal(m.values().cpu().numpy(), ref)
        addrs = vf.as_u64(m.objs)
        probe = np.concatenate([addrs, ts - np.uint64(1), te, te - np.uint64(1)])
        gpu = c.resolve(vf.APP_MICRO, vf.COAL,
                        torch.from_numpy(probe.view(np.int64)).cuda()).cpu().numpy().view(np.uint32)
        assert np.array_equal(gpu, oracle.coal_lookup(ts, te, tt, probe))
    finally:
        c.close()


def test_reserve_va_merges_to_one_row_per_type(ctx):
    n, T = 200_000, 4
    types = synth.micro_types(n, T, "random", seed=11)
    c = vf.Ctx(0, reserve_va=True, cuda_heap_bytes=0)
    try:
        apps.Micro(c, n, T, variant="coal", types_np=types, init_np=synth.micro_init(n, seed=11))
        rows = c.range_table(vf.APP_MICRO)
        assert len(rows) == T
        regs = c.regions()
        assert len(regs) == sum(len(oracle.region_plan(int(k), 4096)) for k in np.bincount(types))
    finally:
        c.close()


def test_typepointer_tags_match_oracle(ctx):
    n, T = 5000, 32
    types = synth.micro_types(n, T, "random", seed=2)
    m = apps.Micro(ctx, n, T, variant="typeptr", types_np=types, init_np=synth.micro_init(n, seed=2))
    q = vf.as_u64(m.objs)
    for k in range(0, n, 97):
        assert oracle.tp_type(int(q[k])) == int(types[k])
        assert oracle.tp_strip(int(q[k])) == vf.strip(int(q[k]))


@pytest.mark.slow
def test_micro_full_size_sampled():
    """BASELINE config 2 at full size (2^26 objects) in the bench's launch
    configuration: closed form on a sample + brute-force type identity on all."""
    n, T, R = 1 << 26, 4, 2
    c = vf.Ctx(0, cuda_heap_bytes=0)
    try:
        types = synth.micro_types(n, T, "random", seed=42)
        init = synth.micro_init(n, seed=42)
        rng = np.random.default_rng(0)
        idx = np.concatenate([rng.integers(0, n, 20000), np.arange(64), np.arange(n - 64, n)])
        for variant in ("sharedoa", "coal", "typeptr"):
            m = apps.Micro(c, n, T, variant=variant, types_np=types, init_np=init)
            for _ in range(R):
                m.step()
            got = m.values().cpu().numpy()
            ref_s, _ = oracle.micro_run(types[idx], init[idx], T, R)
            assert np.array_equal(got[idx], ref_s), variant
            assert ctx_verify(c, m) == 0
            del m
            c.reset()
    finally:
        c.close()


def ctx_verify(c, m):
    return c.verify(vf.APP_MICRO, m.v, m.objs)


# ---- the paper's comparison points (§7, §8.2 Fig. 11, §8.3 Fig. 12, Table 1 row C)
@pytest.mark.parametrize("variant", ["concord", "typeptr_heap"])
@pytest.mark.parametrize("T,order", [(1, "random"), (4, "random"), (4, "sorted"), (32, "random"), (5, "kperwarp")])
def test_micro_comparison_variants(ctx, variant, T, order):
    n, R = 4096 * 5 + 77, 3
    types = synth.micro_types(n, T, order, seed=3, k=min(T, 5))
    init = synth.micro_init(n, seed=3)
    ref, _ = oracle.micro_run(types, init, T, R)
    m = apps.Micro(ctx, n, T, variant=variant, types_np=types, init_np=init)
    for _ in range(R):
        m.step()
    assert np.array_equal(m.values().cpu().numpy(), ref)
    assert ctx.verify(vf.APP_MICRO, m.v, m.objs) == 0  # concord: the embedded tag names the right class


@pytest.mark.parametrize("variant", ["coal", "typeptr"])
@pytest.mark.parametrize("T,order", [(4, "random"), (32, "random"), (3, "sorted")])
def test_micro_indirect_call_flavour(ctx, variant, T, order):
    """vf_set_tuning("call", 1): resolved type -> vFunc* table -> indirect CALL (the paper's design)."""
    n, R = 4096 * 7 + 5, 2
    types = synth.micro_types(n, T, order, seed=8)
    init = synth.micro_init(n, seed=8)
    ref, _ = oracle.micro_run(types, init, T, R)
    vf.set_tuning("call", 1)
    try:
        m = apps.Micro(ctx, n, T, variant=variant, types_np=types, init_np=init)
        for _ in range(R):
            m.step()
        assert np.array_equal(m.values().cpu().numpy(), ref)
    finally:
        vf.set_tuning("call", 0)


@pytest.mark.parametrize("T,order,k", [(1, "random", 1), (4, "random", 1), (32, "random", 1), (4, "sorted", 1),
                                       (32, "kperwarp", 7)])
def test_micro_branch_ceiling_closed_form(ctx, T, order, k):
    """BRANCH computes the same types in registers: val_i = init_i + R(t_i+1)."""
    n, R = 100_003, 4
    types = synth.micro_types(n, T, order, seed=11, k=k)
    init = synth.micro_init(n, seed=11)
    b = apps.MicroBranch(ctx, n, T, order, seed=11, k=k, init_np=init)
    for _ in range(R):
        b.step()
    assert np.array_equal(b.values().cpu().numpy(), init.astype(np.int64) + R * (types.astype(np.int64) + 1))


def test_concord_unsupported_without_tag(ctx):
    g = apps.Gol(ctx, 8, 8, synth.soup(8, 8, seed=1), "sharedoa")
    with pytest.raises(vf.VFError) as e:
        ctx.dispatch(vf.CONCORD, vf.APP_GOL, vf.GOL_NEXT, g.grid, g.args[0])
    assert e.value.status == 7


@pytest.mark.parametrize("variant", ["cuda", "sharedoa", "coal", "typeptr"])
@pytest.mark.parametrize("chunk", [0, 1000, 4096 * 3 + 5])
def test_dispatch_host_matches_closed_form(variant, chunk):
    """vf_dispatch_host (chunked H2D overlapped with the calls) == the closed form
    val_i = init_i + R (t_i + 1), for chunk sizes that leave ragged tails."""
    import torch
    c = vf.Ctx(0, cuda_heap_bytes=1 << 30)
    n, T, R = 4096 * 5 + 77, 4, 3
    types = synth.micro_types(n, T, "random", seed=9)
    init = synth.micro_init(n, seed=9)
    m = apps.Micro(c, n, T, variant=variant, types_np=types, init_np=init)
    host = m.objs.cpu().pin_memory()
    staging = torch.empty_like(m.objs)
    for _ in range(R):
        c.dispatch_host(m.v, vf.APP_MICRO, vf.MICRO_APPLY, host, staging, chunk=chunk)
    got = m.values().cpu().numpy()
    assert np.array_equal(got, init + R * (types.astype(np.int32) + 1))
    assert torch.equal(staging, m.objs)
    c.close()


@pytest.mark.parametrize("unroll", [1, 2, 4])
@pytest.mark.parametrize("variant,T", [("coal", 4), ("typeptr", 4), ("coal", 32), ("typeptr", 32)])
def test_micro_deep_pipeline_many_waves(ctx, unroll, variant, T):
    """prefetch 3 (pointers two tiles ahead, the next tile resolved and warmed
    during this one): inputs spanning >= 3 persistent-grid waves so every CTA
    runs the steady state, the last two tiles and a ragged tail."""
    n = 3 * 148 * 8 * 1024 + 77
    R = 2
    types = synth.micro_types(n, T, "random", seed=5)
    init = synth.micro_init(n, seed=5)
    vf.set_tuning("unroll", unroll)
    vf.set_tuning("prefetch", 3)
    try:
        m = apps.Micro(ctx, n, T, variant=variant, types_np=types, init_np=init)
        for _ in range(R):
            m.step()
        got = m.values().cpu().numpy()
        assert np.array_equal(got, init + R * (types.astype(np.int32) + 1))  # closed form (W0)
    finally:
        vf.set_tuning("unroll", -1)
        vf.set_tuning("prefetch", -1)


@pytest.mark.parametrize("unroll", [1, 2, 4])
@pytest.mark.parametrize("order", ["random", "sorted"])
@pytest.mark.parametrize("variant,T", [("coal", 4), ("typeptr", 4), ("typeptr", 32)])
def test_micro_two_barrier_sort_many_waves(ctx, unroll, order, variant, T):
    """regroup 2 (two barriers per tile: double-buffered histogram, per-warp
    scans) over >= 3 persistent-grid waves, mixed and type-uniform tiles."""
    n = 3 * 148 * 8 * 1024 + 77
    R = 3
    types = synth.micro_types(n, T, order, seed=6)
    init = synth.micro_init(n, seed=6)
    vf.set_tuning("unroll", unroll)
    vf.set_tuning("prefetch", 2)
    vf.set_tuning("regroup", 2)
    try:
        m = apps.Micro(ctx, n, T, variant=variant, types_np=types, init_np=init)
        for _ in range(R):
            m.step()
        assert np.array_equal(m.values().cpu().numpy(), init + R * (types.astype(np.int32) + 1))
    finally:
        vf.set_tuning("unroll", -1)
        vf.set_tuning("prefetch", -1)
        vf.set_tuning("regroup", 1)

"""Pins for the oracle's allocator policy, range table, COAL lookup and TypePointer.

Pinned against: closed forms (region counts), Fig. 3's structural example,
brute force linear scans (an independent definition of "the unique range that
contains p"), and round-trip invariants. None of these re-call the oracle's own
routine as the expected value.
"""
import math

import numpy as np
import pytest

import oracle
import synth

NF = oracle.NOT_FOUND


@pytest.mark.parametrize("count", [0, 1, 4095, 4096, 4097, 12288, 12289, 10**6, 2**26, 2**24 // 3])
def test_region_plan_closed_form(count):
    caps = oracle.region_plan(count, 4096)
    expect_k = 0 if count == 0 else math.ceil(math.log2(count / 4096 + 1))
    assert len(caps) == expect_k
    for j, c in enumerate(caps):
        assert c == 4096 * 2**j
    if count:
        assert sum(caps) >= count > sum(caps[:-1])


def test_region_plan_small_chunk_f1():
    # SURVEY fixture F1: init chunk 4, 9 objects -> 2 regions (4 + 8)
    assert oracle.region_plan(9, 4) == [4, 8]
    assert oracle.region_plan(5, 4) == [4, 8]
    assert oracle.region_plan(3, 4) == [4]


def test_fig3_structural_table():
    # Fig. 3: three types, one region each (addresses arbitrary)
    start = np.array([0x3000, 0x1000, 0x2000], np.uint64)
    nbytes = np.array([0x100, 0x200, 0x80], np.uint64)
    types = np.array([2, 0, 1], np.uint32)
    ts, te, tt = oracle.build_table(start, nbytes, types)
    assert list(ts) == [0x1000, 0x2000, 0x3000]
    assert list(te) == [0x1200, 0x2080, 0x3100]
    assert list(tt) == [0, 1, 2]
    # OBJk of region k resolves to TYPEk
    objs = np.array([0x1000, 0x1010, 0x11F0, 0x2000, 0x2070, 0x3000, 0x30F0], np.uint64)
    assert list(oracle.coal_lookup(ts, te, tt, objs)) == [0, 0, 0, 1, 1, 2, 2]


def test_table_merge_only_when_adjacent_same_type():
    start = np.array([100, 200, 300, 400, 500], np.uint64)
    nbytes = np.array([100, 100, 50, 100, 100], np.uint64)
    types = np.array([0, 0, 0, 1, 0], np.uint32)
    ts, te, tt = oracle.build_table(start, nbytes, types)
    # [100,300) merged (adjacent, type 0); [300,350) adjacent to 300 -> merged too;
    # [400,500) type 1; [500,600) type 0 adjacent to a type-1 row -> separate
    assert list(zip(ts, te, tt)) == [(100, 350, 0), (400, 500, 1), (500, 600, 0)]


def _random_regions(rng, K, types=4, adjacent_p=0.3):
    starts, sizes, tys = [], [], []
    cur = 0x7F0000000000
    for _ in range(K):
        if rng.random() > adjacent_p:
            cur += int(rng.integers(1, 1 << 16)) * 16
        sz = int(rng.integers(1, 4096)) * 16
        starts.append(cur)
        sizes.append(sz)
        tys.append(int(rng.integers(0, types)))
        cur += sz
    perm = rng.permutation(K)
    return (np.array(starts, np.uint64)[perm], np.array(sizes, np.uint64)[perm],
            np.array(tys, np.uint32)[perm])


def _brute_type(regions, a):
    s, b, t = regions
    hits = [int(t[j]) for j in range(len(s)) if int(s[j]) <= a < int(s[j]) + int(b[j])]
    assert len(hits) <= 1
    return hits[0] if hits else NF


@pytest.mark.parametrize("K", [1, 2, 3, 5, 8, 17, 64, 300])
def test_table_invariants_and_coal_vs_brute_force(K):
    rng = np.random.default_rng(K)
    regions = _random_regions(rng, K)
    ts, te, tt = oracle.build_table(*regions)
    # sorted, disjoint, non-empty
    assert np.all(ts < te)
    assert np.all(te[:-1] <= ts[1:])
    # no two consecutive rows that should have merged
    assert not np.any((te[:-1] == ts[1:]) & (tt[:-1] == tt[1:]))
    # union preserved
    assert int((te - ts).sum()) == int(regions[1].sum())
    # every edge address of every region, plus random addresses: tree == brute force
    s, b, _ = regions
    probes = []
    for j in range(K):
        lo, hi = int(s[j]), int(s[j]) + int(b[j])
        probes += [lo - 1, lo, lo + 1, hi - 1, hi, hi + 1]
    probes += [int(x) for x in synth.random_addresses(200, seed=K)]
    probes += [0, (1 << 64) - 1]
    probes = np.array([p & synth.M64 for p in probes], np.uint64)
    got = oracle.coal_lookup(ts, te, tt, probes)
    ref = [_brute_type(regions, int(p)) for p in probes]
    assert list(got) == ref


def test_coal_large_K():
    # K = 4096 ranges, every start/end-1 and a gap address each
    K = 4096
    base = np.arange(K, dtype=np.uint64) * np.uint64(0x1000) + np.uint64(0x10000)
    ts, te = base, base + np.uint64(0x800)
    tt = (np.arange(K) % 127).astype(np.uint32)
    probes = np.concatenate([ts, te - np.uint64(1), te, ts - np.uint64(1)])
    got = oracle.coal_lookup(ts, te, tt, probes)
    assert np.array_equal(got[:K], tt) and np.array_equal(got[K:2 * K], tt)
    assert np.all(got[2 * K:] == NF)


def test_coal_empty_table():
    e = np.zeros(0, np.uint64)
    assert list(oracle.coal_lookup(e, e, np.zeros(0, np.uint32), np.array([5], np.uint64))) == [NF]


def test_typepointer_roundtrip():
    addrs = synth.random_addresses(500, seed=3) & np.uint64((1 << 57) - 1)
    for a in addrs[:100]:
        for t in (0, 1, 5, 63, 126):
            q = oracle.tp_tag(int(a), t)
            assert oracle.tp_strip(q) == int(a)
            assert oracle.tp_type(q) == t
            assert q >> 57 == t + 1  # Fig. 5a: type in the upper bits
        assert oracle.tp_type(int(a)) == NF  # untagged -> fallback
        assert oracle.tp_strip(int(a)) == int(a)


def test_typepointer_vfunc_padded_index():
    # 3 types, padded vTables of 4 slots: slot m of type t
    slots = 4
    vt = np.array([1000 * t + m for t in range(3) for m in range(slots)], np.uint64)
    for t in range(3):
        q = oracle.tp_tag(0x7F00_0000_1000, t)
        for m in range(slots):
            assert oracle.tp_vfunc(q, vt, slots, m) == 1000 * t + m
    assert oracle.tp_vfunc(0x7F00_0000_1000, vt, slots, 0) == 0

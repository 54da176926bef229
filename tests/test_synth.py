"""Pins for the shared seeded input generators (synth/)."""
import numpy as np

import synth

GOLDEN = 0x9E3779B97F4A7C15


def _golden_values():
    import os
    p = os.path.join(os.path.dirname(__file__), "golden", "splitmix64.txt")
    return [int(l, 16) for l in open(p) if l.strip() and not l.startswith("#")]


def test_splitmix64_published_values():
    vals = _golden_values()
    xs = np.array([(k * GOLDEN) & synth.M64 for k in range(len(vals))], dtype=np.uint64)
    got = synth.splitmix64(xs)
    assert [int(v) for v in got] == vals
    assert [synth.splitmix64_int(int(x)) for x in xs] == vals


def test_splitmix64_vector_matches_scalar():
    xs = synth.draw(3, 1, np.arange(1000, dtype=np.uint64))
    for x in xs[:200]:
        assert int(synth.splitmix64(np.uint64(x))) == synth.splitmix64_int(int(x))


def test_uniform_exact_against_bigint():
    u = synth.draw(11, 2, np.arange(5000, dtype=np.uint64))
    for n in (1, 2, 3, 7, 32, 1000, 2**31 - 1, 2**32 - 1):
        got = synth.uniform(u, n)
        ref = np.array([(int(x) * n) >> 64 for x in u], dtype=np.uint64)
        assert np.array_equal(got.astype(np.uint64), ref)
        assert got.max() < n


def test_micro_orders():
    t = synth.micro_types(1000, 4, "sorted")
    assert t[0] == 0 and t[-1] == 3 and np.all(np.diff(t.astype(int)) >= 0)
    t = synth.micro_types(64, 32, "kperwarp", k=5)
    assert list(t[:10]) == [0, 1, 2, 3, 4, 0, 1, 2, 3, 4]
    t = synth.micro_types(100000, 4, "random")
    counts = np.bincount(t, minlength=4)
    assert counts.min() > 24000

"""Pins for the oracle's config-2 microbenchmark (paper §8.3).

Closed form: object i of type t(i) whose apply() adds t+1 (reading G11) ends at
init_i + R*(t(i)+1) after R passes — derived from the definition, independent of
the oracle's dispatch.
"""
import numpy as np
import pytest

import oracle
import synth


@pytest.mark.parametrize("T", [1, 2, 3, 4, 8, 32])
@pytest.mark.parametrize("order", ["random", "sorted", "kperwarp"])
def test_micro_closed_form(T, order):
    n, R = 20000 + 37, 5
    t = synth.micro_types(n, T, order, seed=42)
    init = synth.micro_init(n, seed=42)
    vals, _ = oracle.micro_run(t, init, T, R)
    assert np.array_equal(vals, init + R * (t.astype(np.int32) + 1))


def test_micro_fixture_f2():
    # N = 1000, T = 3, random order, seed 1, R = 7
    t = synth.micro_types(1000, 3, "random", seed=1)
    init = synth.micro_init(1000, seed=1)
    vals, _ = oracle.micro_run(t, init, 3, 7)
    assert np.array_equal(vals, init + 7 * (t.astype(np.int32) + 1))


def test_micro_threads_identical():
    n = 1 << 16
    t = synth.micro_types(n, 32, "random", seed=5)
    init = synth.micro_init(n, seed=5)
    a, _ = oracle.micro_run(t, init, 32, 3, threads=1)
    b, _ = oracle.micro_run(t, init, 32, 3, threads=oracle.max_threads())
    assert np.array_equal(a, b)


def test_micro_empty_and_bad_type():
    vals, _ = oracle.micro_run(np.zeros(0, np.uint32), np.zeros(0, np.int32), 4, 3)
    assert len(vals) == 0
    with pytest.raises(ValueError):
        oracle.micro_run(np.array([4], np.uint32), np.array([0], np.int32), 4, 1)

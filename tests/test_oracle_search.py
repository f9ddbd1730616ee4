"""O1 (sorted array + lower_bound) pinned against brute force (O3), closed forms and the
pointer B+tree (O2).  CPU only."""
import numpy as np
import pytest

import harmonia_gen as gen

MAX = (1 << 64) - 1


def _sets():
    yield np.zeros(0, dtype=np.uint64)
    yield np.array([5], dtype=np.uint64)
    yield np.array([0, MAX - 1], dtype=np.uint64)
    for T in (7, 100, 1000, 4096):
        yield gen.random_keys(T, seed=T)
        yield gen.uniform_keys(T)
    yield gen.random_keys(3000, seed=9, bits=14)  # dense small-universe keys
    yield gen.clustered_keys(3000)


@pytest.mark.parametrize("case", range(12))
def test_point_matches_brute_force(orc, case):
    keys = list(_sets())[case]
    vals = gen.values_for(keys)
    q = np.concatenate([
        gen.uniform_queries(keys, 800, miss_frac=0.5) if keys.shape[0] else gen._stream(1, 0, 50),
        gen.edge_queries(keys),
        (keys + np.uint64(1)) if keys.shape[0] else np.zeros(0, dtype=np.uint64),
    ])
    a = orc.sorted_search(keys, vals, q)
    b = orc.brute_search(keys, vals, q)
    assert np.array_equal(a, b)
    # every hit returns the value aligned with its key
    hit = a != orc.NOT_FOUND
    idx = np.searchsorted(keys, q[hit])
    assert np.array_equal(keys[idx], q[hit]) and np.array_equal(vals[idx], a[hit])


def test_point_closed_form(orc):
    # keys 2i (i < n), values 3i+7: even q=2i found with 3i+7, odd q never found.
    n = 5000
    keys = np.arange(n, dtype=np.uint64) * np.uint64(2)
    vals = np.arange(n, dtype=np.uint64) * np.uint64(3) + np.uint64(7)
    q = np.arange(2 * n + 3, dtype=np.uint64)
    out = orc.sorted_search(keys, vals, q, nthreads=4)
    even = q % 2 == 0
    hit = even & (q < 2 * n)
    assert np.array_equal(out[hit], (q[hit] // 2) * 3 + 7)
    assert np.all(out[~hit] == orc.NOT_FOUND)


def test_multithread_equals_single(orc):
    keys = gen.uniform_keys(1 << 16)
    vals = gen.values_for(keys)
    q = gen.uniform_queries(keys, 1 << 16, miss_frac=0.3)
    assert np.array_equal(orc.sorted_search(keys, vals, q, 1), orc.sorted_search(keys, vals, q, 8))


@pytest.mark.parametrize("cap", [0, 1, 5, 64])
def test_range_matches_brute_force(orc, cap):
    for keys in list(_sets())[:9]:
        vals = gen.values_for(keys)
        lo, hi = gen.random_ranges(keys, 300, max_width_keys=40)
        a = orc.sorted_range(keys, vals, lo, hi, cap)
        b = orc.brute_range(keys, vals, lo, hi, cap)
        assert np.array_equal(a[2], b[2])
        for j in range(lo.shape[0] if cap else 0):
            m = min(int(a[2][j]), cap)
            assert np.array_equal(a[0][j][:m], b[0][j][:m])
            assert np.array_equal(a[1][j][:m], b[1][j][:m])


def test_range_closed_form(orc):
    # keys = 0..n-1 -> range [lo, hi] holds exactly max(0, min(hi, n-1) - lo + 1) keys
    n = 1000
    keys = np.arange(n, dtype=np.uint64)
    vals = keys * np.uint64(5) + np.uint64(1)
    lo = np.array([0, 10, 999, 500, 1200, 7, 3], dtype=np.uint64)
    hi = np.array([999, 19, 5000, 499, 1300, 7, MAX], dtype=np.uint64)
    ko, vo, cnt = orc.sorted_range(keys, vals, lo, hi, 16)
    exp = [1000, 10, 1, 0, 0, 1, 997]
    assert cnt.tolist() == exp
    assert ko[1][:10].tolist() == list(range(10, 20))
    assert vo[1][:10].tolist() == [5 * k + 1 for k in range(10, 20)]
    assert ko[0].tolist() == list(range(16))  # truncated at cap, ascending


def test_bptree_agrees_with_sorted_array(orc):
    for F in (4, 8, 16, 64):
        keys = gen.random_keys(5000, seed=F)
        vals = gen.values_for(keys)
        t = orc.BPlusTree(F)
        order = np.random.default_rng(F).permutation(keys.shape[0])
        t.insert_many(keys[order], vals[order])
        assert t.check() == 0
        q = np.concatenate([gen.uniform_queries(keys, 3000, miss_frac=0.5), gen.edge_queries(keys)])
        assert np.array_equal(t.search(q), orc.sorted_search(keys, vals, q))
        lo, hi = gen.random_ranges(keys, 200)
        a, b = t.range(lo, hi, 32), orc.sorted_range(keys, vals, lo, hi, 32)
        assert np.array_equal(a[2], b[2])
        for j in range(lo.shape[0]):
            m = min(int(a[2][j]), 32)
            assert np.array_equal(a[0][j][:m], b[0][j][:m]) and np.array_equal(a[1][j][:m], b[1][j][:m])

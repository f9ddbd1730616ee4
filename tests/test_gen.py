"""Generator properties (the one module shared by oracle, tests and bench)."""
import numpy as np

import harmonia_gen as gen

MAX = np.uint64((1 << 64) - 1)


def test_splitmix64_reference_values():
    # splitmix64 with state 0: the first outputs of the reference generator
    # (x += golden gamma; mix) -> 0xE220A8397B1DCDAF, 0x6E789E6AA1B965F4
    assert int(gen.splitmix64(np.array([0], dtype=np.uint64))[0]) == 0xE220A8397B1DCDAF
    assert int(gen.splitmix64(np.array([0x9E3779B97F4A7C15], dtype=np.uint64))[0]) == 0x6E789E6AA1B965F4


def test_uniform_keys_properties():
    for T in (1, 2, 1000, 1 << 16):
        k = gen.uniform_keys(T)
        assert k.shape == (T,) and k.dtype == np.uint64
        assert np.all(k[1:] > k[:-1]) and np.all(k != MAX)
    k = gen.uniform_keys(1 << 16)
    assert np.array_equal(gen.uniform_keys(1 << 16, start=1000, count=500), k[1000:1500])
    top = (k >> np.uint64(56)).astype(np.int64)
    h = np.bincount(top, minlength=256)
    assert h.min() > 200 and h.max() < 320  # stratified: the top byte is uniform


def test_clustered_and_random_keys():
    k = gen.clustered_keys(5000)
    assert np.all(k[1:] > k[:-1])
    assert np.sum(np.diff(k) == 1) >= 5000 - 10
    r = gen.random_keys(3000, seed=3)
    assert r.shape == (3000,) and np.all(r[1:] > r[:-1])


def test_queries_and_values():
    k = gen.uniform_keys(1 << 12)
    v = gen.values_for(k)
    assert np.all(v != MAX)
    q = gen.uniform_queries(k, 5000)
    assert np.all(np.isin(q, k))
    qm = gen.uniform_queries(k, 5000, miss_frac=0.5)
    miss = ~np.isin(qm, k)
    assert 0.4 < miss.mean() < 0.6
    z = gen.zipf_queries(k, 20000)
    _, c = np.unique(z, return_counts=True)
    assert c.max() > 20000 * 0.03  # theta 0.99: a very hot head
    s = gen.sorted_run_queries(k, 4096, run=1024)
    assert np.all(np.diff(s.reshape(4, 1024).astype(np.float64), axis=1) > 0)


def test_torch_generators_equal_numpy():
    import torch

    for T in (4, 1000, 123457):
        kn = gen.uniform_keys(T)
        kt = gen.uniform_keys_t(T, "cpu").numpy().view(np.uint64)
        assert np.array_equal(kn, kt)
        assert np.array_equal(gen.values_for(kn), gen.values_for_t(torch.from_numpy(kn.view(np.int64))).numpy().view(np.uint64))
        qn = gen.uniform_queries(kn, 5000, start=77)
        qt = gen.uniform_queries_t(torch.from_numpy(kn.view(np.int64)), 5000, start=77).numpy().view(np.uint64)
        assert np.array_equal(qn, qt)
    x = np.array([0, 1, (1 << 64) - 1, 0x9E3779B97F4A7C15], dtype=np.uint64)
    assert np.array_equal(gen.splitmix64(x), gen.splitmix64_t(torch.from_numpy(x.view(np.int64))).numpy().view(np.uint64))


def test_ranges_count_len():
    k = gen.uniform_keys(1 << 12)
    lo, hi = gen.ranges(k, 100, 16)
    i0, i1 = np.searchsorted(k, lo), np.searchsorted(k, hi)
    assert np.all(i1 - i0 == 15)


def test_update_ops_mix():
    k = gen.uniform_keys(1 << 14)
    ops, ks, vs = gen.update_ops(k, 100000, insert_frac=0.05, delete_frac=0.05)
    assert 0.04 < (ops == 1).mean() < 0.06
    ins = (ops == 0) & ~np.isin(ks, k)
    assert 0.04 < ins.mean() < 0.06


def test_device_zipf_and_key_index_generators():
    import torch

    k = gen.uniform_keys(100003)
    kt = torch.from_numpy(k.view(np.int64))
    idx = torch.tensor([0, 1, 5, 100002, 77777], dtype=torch.int64)
    assert np.array_equal(gen.keys_at_t(100003, idx).numpy().view(np.uint64), k[idx.numpy()])
    zn = gen.zipf_queries(k, 50000, start=3)
    zt = gen.zipf_queries_t(kt, 50000, start=3).numpy().view(np.uint64)
    assert (zn == zt).mean() > 0.999  # equal up to last-ulp pow rounding at rank boundaries


def test_device_update_ops():
    import torch

    T = 1 << 14
    k = gen.uniform_keys(T)
    ops, ks, vs = gen.update_ops_t(T, 100000, 0.05, 0.05, "cpu")
    ops, ks = ops.numpy(), ks.numpy().view(np.uint64)
    assert 0.04 < (ops == 1).mean() < 0.06
    ins = (ops == 0) & ~np.isin(ks, k)
    assert 0.04 < ins.mean() < 0.06
    assert np.isin(ks[ops == 1], k).all()
    # a shard: keys of [lo, hi) only
    ops2, ks2, _ = gen.update_ops_t(T, 20000, 0.05, 0.05, "cpu", lo=4096, hi=8192)
    kk = ks2.numpy().view(np.uint64)
    assert (kk >= k[4096]).all() and (kk <= k[8191]).all()

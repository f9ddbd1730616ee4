"""GPU: the PSA order the search consumes (Eq 2) read back through
harmonia_psa_inspect and checked against the oracle's bucket function (orc_psa_bucket, C-A11),
and bit-exact parity of the two-level PSA path (psa_levels = 2) against the oracle.

Run on a B200 with ``pytest -m gpu``."""
import numpy as np
import pytest

import harmonia_gen as gen

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def hm():
    import torch

    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    import paper_conf_ppopp_yanlpz19_b200 as m

    m.lib()
    return m


def cu(a):
    import torch

    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def host(t):
    return t.cpu().numpy()


def nondecreasing(b):
    return bool(np.all(b[1:] >= b[:-1]))


def order_of(hm, orc, t, q, **kw):
    """(plan, visiting order, its Nb-bit buckets) for the search of q with options kw."""
    plan = t.plan(q.shape[0], **kw)
    order = host(t.psa_inspect(cu(q), **kw))
    assert np.array_equal(np.sort(order), np.sort(q)), "PSA output is not a permutation of the batch"
    info = t.info()
    b = orc.psa_buckets(order, plan["psa_bits"], info["min_key"], info["max_key"])
    return plan, order, b


@pytest.mark.parametrize("T,F,Q,nb", [(1 << 20, 64, 1 << 22, 0), (1 << 18, 16, 3_000_017, 20), (1 << 22, 128, 1 << 23, 0)])
def test_two_level_order_whole_window(hm, orc, T, F, Q, nb):
    """psa_levels 2: the whole window is non-decreasing in the Nb-bit bucket (Eq 2 order)."""
    keys = gen.uniform_keys(T)
    t = hm.Tree(cu(keys), cu(gen.values_for(keys)), fanout=F)
    q = gen.uniform_queries(keys, Q, miss_frac=0.2)
    plan, order, b = order_of(hm, orc, t, q, flags=hm.QF_PSA_L16, psa_bits=nb)
    assert plan["psa_levels"] == 2 and plan["psa_bits"] >= 16 and plan["chunk_group"] >= 1
    assert nondecreasing(b), "two-level PSA must order the whole window by the Nb-bit bucket"


def test_one_level_order_granularity(hm, orc):
    """psa_levels 1: top 8 bucket bits ordered over the window, all Nb bits inside each chunk."""
    keys = gen.uniform_keys(1 << 20)
    t = hm.Tree(cu(keys), cu(gen.values_for(keys)), fanout=64)
    q = gen.uniform_queries(keys, (1 << 22) + 777)
    plan, order, b = order_of(hm, orc, t, q, flags=hm.QF_PSA_L8)
    nb, ch = plan["psa_bits"], plan["sort_chunk"]
    assert plan["psa_levels"] == 1 and ch in (4096, 8192)
    assert nondecreasing(b >> np.uint64(nb - 8))
    for c0 in range(0, q.shape[0], ch):
        assert nondecreasing(b[c0:c0 + ch]), c0
    # and the one-level order is NOT the whole-window order (the test can tell them apart)
    assert not nondecreasing(b)


def test_auto_plan_levels(hm):
    """Auto: two levels when a 4096-query level-1 chunk would hold < 0.5 queries per leaf."""
    small = gen.uniform_keys(1 << 20)
    t = hm.Tree(cu(small), cu(gen.values_for(small)), fanout=64)
    assert t.plan(1 << 22)["psa_levels"] == 1          # 16.6K leaves: 4096 x 256 / 16.6K = 63
    import torch

    big = gen.uniform_keys_t(1 << 27, "cuda")
    t2 = hm.Tree(big.view(torch.uint64), gen.values_for_t(big).view(torch.uint64), fanout=64)
    p = t2.plan(1 << 24)
    assert p["psa_levels"] == 2 and p["sort_chunk"] == 8192    # 2^27 keys, 2.1M leaves: 0.49 queries per leaf


def test_two_level_skewed_batch(hm, orc):
    """Zipf batch: a hot 16-bit bucket larger than a chunk is split into chunk pieces; the
    16-bit prefix stays ordered everywhere, and the results stay bit-exact."""
    keys = gen.uniform_keys(1 << 20)
    vals = gen.values_for(keys)
    t = hm.Tree(cu(keys), cu(vals), fanout=32)
    q = gen.zipf_queries(keys, 1 << 22)
    plan, order, b = order_of(hm, orc, t, q, flags=hm.QF_PSA_L16, psa_bits=20)
    assert plan["psa_levels"] == 2
    assert nondecreasing(b >> np.uint64(plan["psa_bits"] - 16))
    out = host(t.search(cu(q), flags=hm.QF_PSA_L16, psa_bits=20))
    assert np.array_equal(out, gen.values_for(q))


@pytest.mark.parametrize("F,fill", [(4, 1.0), (8, 0.69), (16, 1.0), (64, 0.5), (128, 1.0), (256, 0.69)])
@pytest.mark.parametrize("kind", ["uniform", "miss50", "zipf", "sorted_run"])
def test_two_level_parity(hm, orc, F, fill, kind):
    keys = gen.uniform_keys(200_003)
    vals = gen.values_for(keys)
    t = hm.Tree(cu(keys), cu(vals), fanout=F, fill=fill)
    n = 1_500_001
    if kind == "uniform":
        q = gen.uniform_queries(keys, n)
    elif kind == "miss50":
        q = gen.uniform_queries(keys, n, miss_frac=0.5)
    elif kind == "zipf":
        q = gen.zipf_queries(keys, n)
    else:
        q = gen.sorted_run_queries(keys, n)
    q = np.concatenate([q, gen.edge_queries(keys)])
    for chunk in (4096, 8192):
        out = host(t.search(cu(q), flags=hm.QF_PSA_L16, psa_bits=18, sort_chunk=chunk))
        assert t.plan(q.shape[0], flags=hm.QF_PSA_L16, psa_bits=18, sort_chunk=chunk)["psa_levels"] == 2
        assert np.array_equal(out, orc.sorted_search(keys, vals, q)), (F, fill, kind, chunk)


@pytest.mark.parametrize("n", [1, 31, 1000, 65537, 300_000])
def test_two_level_small_batches(hm, orc, n):
    """Batches far smaller than 2^16 buckets: most buckets empty, ragged tiles and chunks."""
    keys = gen.uniform_keys(1 << 16)
    vals = gen.values_for(keys)
    t = hm.Tree(cu(keys), cu(vals), fanout=16)
    q = gen.uniform_queries(keys, n, miss_frac=0.3)
    out = host(t.search(cu(q), flags=hm.QF_PSA_L16, psa_bits=16))
    assert np.array_equal(out, orc.sorted_search(keys, vals, q))


def test_two_level_windows(hm, orc):
    """Several PSA windows per call, each partitioned on its own."""
    keys = gen.uniform_keys(1 << 18)
    vals = gen.values_for(keys)
    t = hm.Tree(cu(keys), cu(vals), fanout=64)
    q = gen.uniform_queries(keys, 3 * (1 << 20) + 5, miss_frac=0.1)
    kw = dict(flags=hm.QF_PSA_L16, psa_bits=18, window=1 << 20)
    out = host(t.search(cu(q), **kw))
    assert np.array_equal(out, orc.sorted_search(keys, vals, q))
    order = host(t.psa_inspect(cu(q), **kw))
    info = t.info()
    b = orc.psa_buckets(order, 18, info["min_key"], info["max_key"])
    for w0 in range(0, q.shape[0], 1 << 20):
        assert nondecreasing(b[w0:w0 + (1 << 20)])

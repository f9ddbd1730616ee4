"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle, element by element.

Run on a B200 with ``pytest -m gpu``.  Every comparison is bit-exact (integer work)."""
import numpy as np
import pytest

import harmonia_gen as gen

pytestmark = pytest.mark.gpu

MAX = (1 << 64) - 1


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


def tree(hm, keys, vals, F, fill=1.0):
    return hm.Tree(cu(keys), cu(vals), fanout=F, fill=fill)


# ----------------------------------------------------------------------------- layout
@pytest.mark.parametrize("n,F,fill", [(0, 16, 1.0), (1, 4, 1.0), (3, 4, 1.0), (15, 16, 1.0), (16, 16, 1.0),
                                      (1000, 4, 1.0), (5000, 8, 0.69), (20000, 16, 0.5), (65536, 16, 1.0),
                                      (100000, 64, 1.0), (100000, 128, 0.69), (70000, 256, 1.0), (1 << 20, 64, 1.0)])
def test_layout_bit_exact_and_invariants(hm, orc, n, F, fill):
    keys = gen.uniform_keys(n)
    vals = gen.values_for(keys)
    t = tree(hm, keys, vals, F, fill)
    info, kr, ps, lv = t.export_layout()
    ref = orc.layout_build(keys, vals, F, fill)
    assert info["height"] == ref.h and info["level_start"] == ref.level_start.tolist()
    assert np.array_equal(kr, ref.key_region)      # I8: bit-exact key region
    assert np.array_equal(ps, ref.ps)              # I8: bit-exact PS
    assert np.array_equal(lv, ref.leaf_vals)
    lay = orc.Layout(F, info["height"], info["level_start"], kr, ps, lv)
    code, msg = lay.check(keys, vals)
    assert code == 0, msg
    assert info["ps_bytes"] == 4 * (info["n_internal"] + 1)  # I9


def test_build_from_host_equals_device(hm):
    keys = gen.uniform_keys(30000)
    vals = gen.values_for(keys)
    a = hm.Tree(keys, vals, fanout=32).export_layout()
    b = tree(hm, keys, vals, 32).export_layout()
    for x, y in zip(a[1:], b[1:]):
        assert np.array_equal(x, y)


def test_build_errors(hm):
    k = np.array([1, 5, 5, 9], dtype=np.uint64)
    with pytest.raises(hm.HarmoniaError, match="UNSORTED"):
        tree(hm, k, k, 8)
    k = np.array([9, 5], dtype=np.uint64)
    with pytest.raises(hm.HarmoniaError, match="UNSORTED"):
        tree(hm, k, k, 8)
    k = np.array([1, MAX], dtype=np.uint64)
    with pytest.raises(hm.HarmoniaError, match="RESERVED"):
        tree(hm, k, np.array([1, 2], dtype=np.uint64), 8)
    k = np.array([1, 2], dtype=np.uint64)
    with pytest.raises(hm.HarmoniaError, match="RESERVED"):
        tree(hm, k, np.array([1, MAX], dtype=np.uint64), 8)
    with pytest.raises(hm.HarmoniaError, match="INVALID_ARG"):
        tree(hm, k, k, 12)


# ----------------------------------------------------------------------------- config 1
def _queries(kind, keys, Q):
    if kind == "uniform":
        return gen.uniform_queries(keys, Q)
    if kind == "miss50":
        return gen.uniform_queries(keys, Q, miss_frac=0.5)
    if kind == "zipf":
        return gen.zipf_queries(keys, Q)
    if kind == "sorted_run":
        return gen.sorted_run_queries(keys, Q)
    raise ValueError(kind)


@pytest.mark.parametrize("kind", ["uniform", "miss50", "zipf", "sorted_run"])
@pytest.mark.parametrize("fill", [1.0, 0.69])
def test_config1_parity(hm, orc, kind, fill):
    """BASELINE config 1: 2^16 uint64 keys, F=16, 2^20 queries."""
    keys = gen.uniform_keys(1 << 16)
    vals = gen.values_for(keys)
    t = tree(hm, keys, vals, 16, fill)
    q = _queries(kind, keys, 1 << 20)
    exp = orc.sorted_search(keys, vals, q)
    assert np.array_equal(host(t.search(cu(q))), exp)
    assert np.array_equal(host(t.search(cu(q), psa_bits=-1)), exp)


@pytest.mark.parametrize("keyset", ["clustered", "random", "dense"])
def test_key_distributions(hm, orc, keyset):
    keys = {"clustered": gen.clustered_keys(50000), "random": gen.random_keys(50000, seed=4),
            "dense": np.arange(50000, dtype=np.uint64)}[keyset]
    vals = gen.values_for(keys)
    t = tree(hm, keys, vals, 64)
    q = np.concatenate([gen.uniform_queries(keys, 200000, miss_frac=0.3), gen.edge_queries(keys),
                        keys + np.uint64(1), keys - np.uint64(1)])
    assert np.array_equal(host(t.search(cu(q))), orc.sorted_search(keys, vals, q))


FG = [(F, G) for F in (4, 8, 16, 32, 64, 128, 256) for G in (1, 2, 4, 8, 16, 32) if 2 * G <= F]


@pytest.mark.parametrize("F", [4, 8, 16, 64, 256])
@pytest.mark.parametrize("lane_queries", [1, 2, 4])
def test_lane_search_queries_per_lane(hm, orc, F, lane_queries):
    """G = 1 (one lane per query) with 1, 2, 4 interleaved queries per lane, ragged tails."""
    keys = gen.random_keys(30000, seed=F + lane_queries)
    vals = gen.values_for(keys)
    t = tree(hm, keys, vals, F)
    q = np.concatenate([gen.uniform_queries(keys, 50003, miss_frac=0.4), gen.edge_queries(keys)])
    exp = orc.sorted_search(keys, vals, q)
    for kw in ({}, {"psa_bits": -1}, {"window": 3072}, {"smem_levels": -1}, {"flags": hm.QF_SCATTER_RETURN},
               {"flags": hm.QF_SCATTER_RETURN, "window": 7168}, {"window": 7168, "smem_levels": -1},
               {"flags": hm.QF_PSA_L16, "psa_bits": 17}, {"flags": hm.QF_PSA_L16, "psa_bits": 17, "window": 13312},
               {"flags": hm.QF_PER_LANE}, {"flags": hm.QF_PER_LANE, "window": 7168, "smem_levels": -1},
               {"sort_chunk": 8192}, {"sort_chunk": 8192, "window": 13312}, {"sort_chunk": 4096},
               {"sort_chunk": 8192, "smem_levels": -1}, {"sort_chunk": 8192, "flags": hm.QF_PER_LANE}):
        got = host(t.search(cu(q), group_size=1, lane_queries=lane_queries, **kw))
        assert np.array_equal(got, exp), kw


def test_removed_ablation_flags_rejected(hm):
    """ABI 2 retired three ablation flags (64, 128, 512): they are INVALID_ARG, not ignored."""
    keys = gen.uniform_keys(1000)
    t = tree(hm, keys, gen.values_for(keys), 16)
    for f in (64, 128, 512):
        with pytest.raises(hm.HarmoniaError):
            t.search(cu(keys), flags=f)


@pytest.mark.parametrize("F", [4, 16, 64, 128])
@pytest.mark.parametrize("keyset", ["dense", "top", "clustered", "wide"])
def test_warp_shared_descent(hm, orc, F, keyset):
    """The default G = 1 PSA path descends warp by warp while the warp's query interval stays
    inside one child (search.cu warp_core).  Cases aimed at its bounds: every query in one
    leaf, intervals straddling leaf and parent boundaries, queries below min / above max key
    in the same warp as hits, keys at the top of the 64-bit space (qhi saturation), a dense
    key set (cshift = 0) and a 64-bit-wide span (cshift = 32)."""
    n = 20000
    keys = {"dense": np.arange(n, dtype=np.uint64) + np.uint64(5),
            "top": np.uint64(MAX - 1) - np.arange(n, dtype=np.uint64)[::-1] * np.uint64(3),
            "clustered": gen.clustered_keys(n), "wide": gen.uniform_keys(n)}[keyset]
    vals = gen.values_for(keys)
    t = tree(hm, keys, vals, F)
    rng = np.random.default_rng(F)
    parts = [np.full(5000, keys[n // 2]),                          # one key, every lane
             keys[rng.integers(100, 140, 30000)],                   # a few neighbouring leaves
             np.repeat(keys[::F - 1], 3),                           # leaf boundaries
             np.concatenate([keys[:200], np.zeros(50, np.uint64), keys[-200:],
                             np.full(50, MAX - 1, np.uint64), np.full(50, MAX, np.uint64)]),
             keys[:3000] + np.uint64(1), keys[-3000:] - np.uint64(1),
             gen.uniform_queries(keys, 40000, miss_frac=0.3)]
    q = np.concatenate(parts)
    exp = orc.sorted_search(keys, vals, q)
    for kw in ({}, {"window": 5120}, {"smem_levels": -1}, {"smem_levels": 1}, {"lane_queries": 1},
               {"lane_queries": 4}, {"flags": hm.QF_PER_LANE}, {"sort_chunk": 8192},
               {"sort_chunk": 8192, "window": 9216}, {"sort_chunk": 4096}):
        assert np.array_equal(host(t.search(cu(q), group_size=1, **kw)), exp), kw
    assert t.plan(len(q))["warp_shared"] == 1 and t.plan(len(q), flags=hm.QF_PER_LANE)["warp_shared"] == 0


def test_sort_chunk_plan(hm):
    """Auto level-2 chunk: 8192 queries when the window holds >= 192 queries per leaf, else
    4096; an explicit sort_chunk wins; non-staged plans report 0."""
    keys = gen.uniform_keys(1 << 16)
    t = tree(hm, keys, gen.values_for(keys), 64)
    inf = t.info()
    leaves = inf["n_nodes"] - inf["level_start"][inf["height"] - 1]
    dense, sparse = 192 * leaves, 191 * leaves
    assert t.plan(dense)["sort_chunk"] == 8192
    assert t.plan(sparse)["sort_chunk"] == 4096
    assert t.plan(dense, sort_chunk=4096)["sort_chunk"] == 4096
    assert t.plan(sparse, sort_chunk=8192)["sort_chunk"] == 8192
    assert t.plan(dense, psa_bits=-1)["sort_chunk"] == 0


@pytest.mark.parametrize("F,G", FG)
def test_every_fanout_and_group_size(hm, orc, F, G):
    keys = gen.random_keys(40000, seed=F * 100 + G)
    vals = gen.values_for(keys)
    t = tree(hm, keys, vals, F, 0.69 if G % 4 == 0 else 1.0)
    q = np.concatenate([gen.uniform_queries(keys, 60001, miss_frac=0.4), gen.edge_queries(keys)])
    exp = orc.sorted_search(keys, vals, q)
    for kw in ({}, {"psa_bits": -1}, {"window": 4096}, {"smem_levels": -1}, {"smem_levels": 2},
               {"flags": hm.QF_GATHER, "window": 8192}, {"psa_bits": 3}, {"flags": hm.QF_LINEAR},
               {"flags": hm.QF_LINEAR, "psa_bits": -1, "smem_levels": 1},
               {"flags": hm.QF_PSA_GLOBAL}, {"flags": hm.QF_PSA_GLOBAL | hm.QF_LINEAR, "window": 3072},
               {"flags": hm.QF_ILP1}, {"flags": hm.QF_ILP1, "psa_bits": -1, "smem_levels": -1}):
        assert np.array_equal(host(t.search(cu(q), group_size=G, **kw)), exp), kw


def test_edge_cases(hm, orc):
    for keys in (np.zeros(0, dtype=np.uint64), np.array([0], dtype=np.uint64),
                 np.array([MAX - 1], dtype=np.uint64), np.array([0, MAX - 1], dtype=np.uint64),
                 np.arange(7, dtype=np.uint64) * np.uint64(3)):
        vals = gen.values_for(keys)
        for F in (4, 8, 64):
            t = tree(hm, keys, vals, F)
            q = np.concatenate([gen.edge_queries(keys), keys, gen._stream(3, 0, 100)])
            assert np.array_equal(host(t.search(cu(q))), orc.sorted_search(keys, vals, q))
            lo, hi = gen.random_ranges(keys, 64)
            ko, vo, cnt = t.range(cu(lo), cu(hi), 8)
            eko, evo, ecnt = orc.sorted_range(keys, vals, lo, hi, 8)
            _cmp_range(host(ko), host(vo), host(cnt), eko, evo, ecnt, 8)
    # zero queries is a no-op
    t = tree(hm, np.arange(10, dtype=np.uint64), np.arange(10, dtype=np.uint64), 8)
    assert t.search(cu(np.zeros(0, dtype=np.uint64))).numel() == 0


# ----------------------------------------------------------------------------- range
def _cmp_range(ko, vo, cnt, eko, evo, ecnt, cap):
    assert np.array_equal(cnt, ecnt)
    m = np.minimum(cnt.astype(np.int64), cap)
    mask = np.arange(cap)[None, :] < m[:, None]
    if cap:
        assert np.array_equal(ko[mask], eko[mask])
        assert np.array_equal(vo[mask], evo[mask])
        assert np.all(ko[~mask] == np.uint64(MAX))  # slab entries past the count untouched


@pytest.mark.parametrize("F,G", [(16, 2), (16, 8), (64, 4), (64, 32), (8, 4), (128, 16)])
@pytest.mark.parametrize("length,cap", [(16, 16), (64, 64), (256, 100), (1024, 1024), (50, 0)])
def test_range_parity(hm, orc, F, G, length, cap):
    keys = gen.uniform_keys(1 << 16)
    vals = gen.values_for(keys)
    t = tree(hm, keys, vals, F)
    lo, hi = gen.ranges(keys, 3000, length)
    lo2, hi2 = gen.random_ranges(keys, 3000, max_width_keys=3 * max(cap, 8))
    lo, hi = np.concatenate([lo, lo2]), np.concatenate([hi, hi2])
    eko, evo, ecnt = orc.sorted_range(keys, vals, lo, hi, cap)
    for kw in ({}, {"psa_bits": -1}, {"window": 2048}, {"flags": hm.QF_LINEAR}):
        ko, vo, cnt = t.range(cu(lo), cu(hi), cap, group_size=G, **kw)
        _cmp_range(host(ko) if cap else None, host(vo) if cap else None, host(cnt), eko, evo, ecnt, cap)


@pytest.mark.parametrize("F,fill", [(4, 1.0), (8, 0.69), (16, 1.0), (32, 0.69), (64, 1.0), (64, 0.69), (128, 1.0),
                                    (256, 0.69)])
@pytest.mark.parametrize("length,cap", [(1, 128), (16, 200), (128, 128), (300, 130), (1024, 1024), (5000, 256),
                                        (50, 0), (64, 64)])
def test_range_warp_kernel(hm, orc, F, fill, length, cap):
    """Default range path (k_range_warp: joint descent of lo/hi, counts from leaf_base ranks,
    batched leaf copy): exact slabs and true totals, ranges starting mid-leaf, spanning many
    leaves, truncated by the cap, empty, lo > hi, unbounded and PAD bounds."""
    keys = gen.uniform_keys(50000) if F != 4 else gen.uniform_keys(6000)
    vals = gen.values_for(keys)
    t = tree(hm, keys, vals, F, fill)
    lo, hi = gen.ranges(keys, 2000, min(length, len(keys)))
    lo2, hi2 = gen.random_ranges(keys, 2000, max_width_keys=3 * max(cap, 8))
    lo3 = np.array([0, 0, int(keys[500]), int(keys[-1]), MAX, 5, MAX - 1, int(keys[7]) + 1], dtype=np.uint64)
    hi3 = np.array([MAX, int(keys[99]), MAX, MAX, MAX, 4, MAX, int(keys[9])], dtype=np.uint64)
    lo, hi = np.concatenate([lo, lo2, lo3]), np.concatenate([hi, hi2, hi3])
    eko, evo, ecnt = orc.sorted_range(keys, vals, lo, hi, cap)
    for kw in ({}, {"psa_bits": -1}, {"window": 2048}, {"smem_levels": -1}):
        ko, vo, cnt = t.range(cu(lo), cu(hi), cap, **kw)
        _cmp_range(host(ko) if cap else None, host(vo) if cap else None, host(cnt), eko, evo, ecnt, cap)
    ko, vo, cnt = t.range(cu(lo), cu(hi), cap, flags=hm.QF_RANGE_GROUP)  # the G-lane group walk
    _cmp_range(host(ko) if cap else None, host(vo) if cap else None, host(cnt), eko, evo, ecnt, cap)


@pytest.mark.parametrize("F,fill", [(4, 1.0), (8, 0.69), (16, 0.5), (64, 1.0), (64, 0.69), (128, 1.0), (256, 0.69)])
@pytest.mark.parametrize("length,cap", [(1, 1), (16, 16), (16, 5), (40, 64), (64, 127), (300, 100), (7, 0),
                                        (256, 256), (700, 511)])
def test_range_lane_kernel(hm, orc, F, fill, length, cap):
    """Default short-range path (cap < 512, k_range_lane: one lane per range on the warp-shared
    descent of the PSA-ordered lo, counts from leaf_base ranks, per-lane leaf walk): exact slabs
    and true totals, mid-leaf starts, ranges across leaves, truncation, empty ranges in key gaps,
    lo > hi, lo = 0, PAD bounds, several PSA windows."""
    keys = gen.uniform_keys(70000) if F != 4 else gen.uniform_keys(9000)
    vals = gen.values_for(keys)
    t = tree(hm, keys, vals, F, fill)
    lo, hi = gen.ranges(keys, 20000, min(length, len(keys)))
    lo2, hi2 = gen.random_ranges(keys, 5000, max_width_keys=3 * max(cap, 8))
    lo3 = np.array([0, 0, int(keys[500]), int(keys[-1]), MAX, 5, MAX - 1, int(keys[7]) + 1, 1, int(keys[3])],
                   dtype=np.uint64)
    hi3 = np.array([MAX, int(keys[99]), MAX, MAX, MAX, 4, MAX, int(keys[9]), 0, int(keys[3])], dtype=np.uint64)
    lo, hi = np.concatenate([lo, lo2, lo3]), np.concatenate([hi, hi2, hi3])
    eko, evo, ecnt = orc.sorted_range(keys, vals, lo, hi, cap)
    for kw in ({}, {"window": 4096}, {"smem_levels": -1}, {"psa_bits": 20}):
        ko, vo, cnt = t.range(cu(lo), cu(hi), cap, **kw)
        _cmp_range(host(ko) if cap else None, host(vo) if cap else None, host(cnt), eko, evo, ecnt, cap)
    ko, vo, cnt = t.range(cu(lo), cu(hi), cap, flags=hm.QF_NO_RANGE_LANE)  # the G-lane group walk
    _cmp_range(host(ko) if cap else None, host(vo) if cap else None, host(cnt), eko, evo, ecnt, cap)


def test_range_lane_clustered(hm, orc):
    """Dense sorted-run keys (a common prefix: C-A11 span) with long and short ranges."""
    keys = gen.clustered_keys(1 << 17)
    vals = gen.values_for(keys)
    t = tree(hm, keys, vals, 32)
    lo, hi = gen.random_ranges(keys, 30000, max_width_keys=200)
    for cap in (16, 100):
        eko, evo, ecnt = orc.sorted_range(keys, vals, lo, hi, cap)
        ko, vo, cnt = t.range(cu(lo), cu(hi), cap)
        _cmp_range(host(ko), host(vo), host(cnt), eko, evo, ecnt, cap)


def test_range_unbounded_counts(hm, orc):
    keys = gen.uniform_keys(100000)
    vals = gen.values_for(keys)
    t = tree(hm, keys, vals, 32, 0.69)
    lo = np.array([0, 0, int(keys[500]), int(keys[-1]), MAX, 5], dtype=np.uint64)
    hi = np.array([MAX, int(keys[99]), MAX, MAX, MAX, 4], dtype=np.uint64)
    ko, vo, cnt = t.range(cu(lo), cu(hi), 32)
    eko, evo, ecnt = orc.sorted_range(keys, vals, lo, hi, 32)
    _cmp_range(host(ko), host(vo), host(cnt), eko, evo, ecnt, 32)


# ----------------------------------------------------------------------------- host API
def test_search_host_pipeline(hm, orc):
    import torch

    keys = gen.uniform_keys(1 << 18)
    vals = gen.values_for(keys)
    t = tree(hm, keys, vals, 64)
    q = gen.uniform_queries(keys, (1 << 22) * 3 + 12345, miss_frac=0.1)
    qh = torch.from_numpy(q).pin_memory()
    out = t.search_host(qh)
    torch.cuda.synchronize()
    assert np.array_equal(out.numpy(), orc.sorted_search(keys, vals, q))
    out2 = t.search_host(qh, psa_bits=-1)
    torch.cuda.synchronize()
    assert np.array_equal(out2.numpy(), out.numpy())


def test_search_host_unordered_back_to_back(hm, orc):
    """HARMONIA_QF_HOST_UNORDERED: back-to-back host-buffer calls with different queries and
    outputs, queued without synchronising in between (the next call's first H2D copies overlap
    the previous call's last D2H copies); every output equals the oracle's."""
    import torch

    keys = gen.uniform_keys(1 << 18)
    vals = gen.values_for(keys)
    t = tree(hm, keys, vals, 64)
    n = (1 << 22) * 2 + 777  # three host chunks: both device buffers in use at the call end
    qs = [gen.uniform_queries(keys, n, seed=gen.SEED_QUERY + i, miss_frac=0.1) for i in range(4)]
    qh = [torch.from_numpy(q).pin_memory() for q in qs]
    oh = [torch.empty(n, dtype=torch.uint64, pin_memory=True) for _ in qs]
    for i in range(4):
        t.search_host(qh[i], oh[i], flags=hm.QF_HOST_UNORDERED)
    torch.cuda.synchronize()
    for i in range(4):
        assert np.array_equal(oh[i].numpy(), orc.sorted_search(keys, vals, qs[i])), f"call {i}"


# ----------------------------------------------------------------------------- routing
def test_route_partition_and_scatter(hm):
    import torch

    keys = gen.uniform_keys(1 << 16)
    q = gen.uniform_queries(keys, 100003, miss_frac=0.2)
    for P in (1, 2, 3, 8):
        split = keys[[(p * keys.shape[0]) // P for p in range(1, P)]].astype(np.uint64)
        routed, pos, counts = hm.route_partition(cu(split), P, cu(q))
        r, p_ = host(routed), host(pos).astype(np.int64)
        assert sum(counts) == q.shape[0]
        assert np.array_equal(np.sort(p_), np.arange(q.shape[0]))
        assert np.array_equal(r, q[p_])
        dest = np.searchsorted(split, q, side="right")
        bounds = np.concatenate([[0], np.cumsum(counts)])
        for d in range(P):
            assert np.all(dest[p_[bounds[d]:bounds[d + 1]]] == d)
        back = hm.scatter_results(routed, pos)
        assert np.array_equal(host(back), q)
    torch.cuda.synchronize()


# ----------------------------------------------------------------------------- full size
def test_config2_full_size_sampled(hm, orc):
    """BASELINE config 2 at full size in the bench's launch configuration (defaults):
    2^23 keys, F=64, 2^26 uniform queries.  Values are key-derived, so every output is
    checked by the property out == values_for(q); 2^20 sampled outputs against the oracle."""
    import torch

    T, Q = 1 << 23, 1 << 26
    keys = gen.uniform_keys(T)
    vals = gen.values_for(keys)
    t = tree(hm, keys, vals, 64)
    q = gen.uniform_queries(keys, Q)
    out = host(t.search(cu(q)))
    torch.cuda.synchronize()
    assert np.array_equal(out, gen.values_for(q))
    sel = gen._stream(77, 0, 1 << 20) % np.uint64(Q)
    assert np.array_equal(out[sel], orc.sorted_search(keys, vals, q[sel]))


def test_l2_access_policy_window(hm, orc):
    """The search kernels carry an L2 access-policy window over the internal levels below the
    staged top (north_star (c)); it changes no result.  Plan reporting, the opt-out flag and
    an explicit byte cap."""
    keys = gen.uniform_keys(1 << 18)
    vals = gen.values_for(keys)
    t = tree(hm, keys, vals, 16)
    inf = t.info()
    leaf0 = inf["level_start"][inf["height"] - 1]
    pl = t.plan(1 << 18)
    internal_unstaged = (leaf0 - min(pl["smem_nodes"], leaf0)) * 16 * 8
    assert 0 < pl["l2_window_bytes"] <= internal_unstaged
    assert t.plan(1 << 18, flags=hm.QF_NO_L2_WINDOW)["l2_window_bytes"] == 0
    assert t.plan(1 << 18, l2_window_bytes=4096)["l2_window_bytes"] == 4096
    q = np.concatenate([gen.uniform_queries(keys, 200003, miss_frac=0.3), gen.edge_queries(keys)])
    exp = orc.sorted_search(keys, vals, q)
    for kw in ({}, {"flags": hm.QF_NO_L2_WINDOW}, {"l2_window_bytes": 4096}, {"group_size": 4},
               {"psa_bits": -1}):
        assert np.array_equal(host(t.search(cu(q), **kw)), exp), kw
    lo, hi = gen.ranges(keys, 5000, 64)
    ko, vo, cnt = t.range(cu(lo), cu(hi), 64)
    eko, evo, ecnt = orc.sorted_range(keys, vals, lo, hi, 64)
    assert np.array_equal(host(cnt), ecnt) and np.array_equal(host(ko), eko) and np.array_equal(host(vo), evo)


def test_concurrent_streams_separate_workspaces(hm, orc):
    """Searches on two streams at once each get their own workspace (the C ABI needs one per
    stream): interleaved calls on the same Tree return exact results on both streams."""
    import torch

    keys = gen.uniform_keys(1 << 18)
    vals = gen.values_for(keys)
    t = tree(hm, keys, vals, 64)
    qa = gen.uniform_queries(keys, (1 << 21) + 3, miss_frac=0.2)
    qb = gen.uniform_queries(keys, (1 << 20) + 11, seed=gen.SEED_QUERY + 5, miss_frac=0.3)
    da, db = cu(qa), cu(qb)
    sa, sb = torch.cuda.Stream(), torch.cuda.Stream()
    torch.cuda.synchronize()
    outs = []
    for _ in range(3):
        with torch.cuda.stream(sa):
            oa = t.search(da, stream=sa)
        with torch.cuda.stream(sb):
            ob = t.search(db, stream=sb)
        outs.append((oa, ob))
    torch.cuda.synchronize()
    ea, eb = orc.sorted_search(keys, vals, qa), orc.sorted_search(keys, vals, qb)
    for oa, ob in outs:
        assert np.array_equal(host(oa), ea) and np.array_equal(host(ob), eb)

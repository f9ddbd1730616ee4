"""GPU parity of harmonia_update_batch against the std::map update oracle (O6).

After every batch the exported layout must equal the oracle's closed-form layout of the
resulting record set bit for bit (the update rebuilds the layout), pass the
invariant checker, and answer point/range queries exactly like the oracle."""
import numpy as np
import pytest

import harmonia_gen as gen

pytestmark = pytest.mark.gpu
MAX = (1 << 64) - 1


@pytest.fixture(scope="module")
def hm():
    import torch

    assert torch.cuda.is_available()
    import paper_conf_ppopp_yanlpz19_b200 as m

    m.lib()
    return m


def cu(a):
    import torch

    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def check_tree(hm, orc, t, F, ref_keys, ref_vals, probe):
    info, kr, ps, lv = t.export_layout()
    lay = orc.layout_build(ref_keys, ref_vals, F, 1.0)
    assert info["n_keys"] == ref_keys.shape[0]
    assert np.array_equal(kr, lay.key_region) and np.array_equal(ps, lay.ps) and np.array_equal(lv, lay.leaf_vals)
    code, msg = orc.Layout(F, info["height"], info["level_start"], kr, ps, lv).check(ref_keys, ref_vals)
    assert code == 0, msg
    out = t.search(cu(probe)).cpu().numpy()
    assert np.array_equal(out, orc.sorted_search(ref_keys, ref_vals, probe))
    lo, hi = gen.random_ranges(ref_keys, 500)
    ko, vo, cnt = t.range(cu(lo), cu(hi), 8)
    eko, evo, ecnt = orc.sorted_range(ref_keys, ref_vals, lo, hi, 8)
    assert np.array_equal(cnt.cpu().numpy(), ecnt)
    m = np.minimum(ecnt.astype(np.int64), 8)
    mask = np.arange(8)[None, :] < m[:, None]
    assert np.array_equal(ko.cpu().numpy()[mask], eko[mask]) and np.array_equal(vo.cpu().numpy()[mask], evo[mask])


@pytest.mark.parametrize("F", [4, 16, 64])
def test_update_batches_match_oracle(hm, orc, F):
    keys = gen.uniform_keys(30000)
    vals = gen.values_for(keys)
    t = hm.Tree(cu(keys), cu(vals), fanout=F)
    ref = orc.UpdateMap(keys, vals)
    touched = []
    for b in range(4):
        ops, ks, vs = gen.update_ops(keys, 8000, insert_frac=0.05 + 0.1 * b, delete_frac=0.05 * b,
                                     seed=gen.SEED_OPS + 31 * b + F)
        # repeated keys inside one batch: the last op must win (C-A18)
        ops = np.concatenate([ops, ops[:500] ^ np.uint8(1)])
        ks = np.concatenate([ks, ks[:500]])
        vs = np.concatenate([vs, vs[:500] + np.uint64(7)])
        t.update(ops, cu(ks), cu(vs))
        ref.apply(ops, ks, vs)
        touched.append(ks)
        rk, rv = ref.dump()
        probe = np.concatenate([np.concatenate(touched), gen.uniform_queries(rk, 20000, miss_frac=0.3)])
        check_tree(hm, orc, t, F, rk, rv, probe)


def test_update_edge_cases(hm, orc):
    keys = np.arange(1, 200, dtype=np.uint64) * np.uint64(10)
    vals = gen.values_for(keys)
    t = hm.Tree(cu(keys), cu(vals), fanout=8)
    ref = orc.UpdateMap(keys, vals)
    # delete everything -> empty tree
    ops = np.ones(keys.shape[0], dtype=np.uint8)
    t.update(ops, cu(keys), cu(vals))
    ref.apply(ops, keys, vals)
    assert t.info()["n_keys"] == 0
    q = np.concatenate([keys, gen.edge_queries(keys)])
    assert np.all(t.search(cu(q)).cpu().numpy() == np.uint64(MAX))
    # insert into the empty tree, including key 0 and MAX-1
    ks = np.array([5, 0, MAX - 1, 77, 5], dtype=np.uint64)
    vs = np.array([1, 2, 3, 4, 9], dtype=np.uint64)
    ops = np.zeros(5, dtype=np.uint8)
    t.update(ops, cu(ks), cu(vs))
    ref.apply(ops, ks, vs)
    rk, rv = ref.dump()
    check_tree(hm, orc, t, 8, rk, rv, np.concatenate([ks, gen.edge_queries(rk)]))
    # reserved key / value -> RESERVED, tree unchanged
    before = t.export_layout()
    with pytest.raises(hm.HarmoniaError, match="RESERVED"):
        t.update(np.zeros(1, dtype=np.uint8), cu(np.array([MAX], dtype=np.uint64)), cu(np.array([1], dtype=np.uint64)))
    with pytest.raises(hm.HarmoniaError, match="RESERVED"):
        t.update(np.zeros(1, dtype=np.uint8), cu(np.array([3], dtype=np.uint64)), cu(np.array([MAX], dtype=np.uint64)))
    after = t.export_layout()
    for x, y in zip(before[1:], after[1:]):
        assert np.array_equal(x, y)
    # delete of a missing key is a no-op; a delete value may be anything
    t.update(np.ones(1, dtype=np.uint8), cu(np.array([123456], dtype=np.uint64)), cu(np.array([MAX], dtype=np.uint64)))
    check_tree(hm, orc, t, 8, rk, rv, rk)


def test_paper_scale_update_batch(hm, orc):
    """batches of 4096K ops, 5 % inserts + 95 % updates, on a 2^23-key tree."""
    keys = gen.uniform_keys(1 << 23)
    vals = gen.values_for(keys)
    t = hm.Tree(cu(keys), cu(vals), fanout=64)
    ops, ks, vs = gen.update_ops(keys, 1 << 22, insert_frac=0.05)
    t.update(ops, cu(ks), cu(vs))
    ref = orc.UpdateMap(keys, vals)
    ref.apply(ops, ks, vs)
    rk, rv = ref.dump()
    assert t.info()["n_keys"] == rk.shape[0]
    sel = gen._stream(5, 0, 1 << 18) % np.uint64(rk.shape[0])
    probe = np.concatenate([rk[sel], ks[: 1 << 18]])
    assert np.array_equal(t.search(cu(probe)).cpu().numpy(), orc.sorted_search(rk, rv, probe))


@pytest.mark.parametrize("F", [8, 64])
def test_update_batch_seq_order(hm, orc, F):
    """harmonia_update_batch_seq: ops take effect in ascending seq, not in array order; with
    many ops per key (upserts and deletes interleaved) the last by seq must win."""
    keys = gen.uniform_keys(20000)
    vals = gen.values_for(keys)
    t = hm.Tree(cu(keys), cu(vals), fanout=F)
    ops, k, v = gen.update_ops(keys, 30000, insert_frac=0.1, delete_frac=0.3)
    k[10000:20000] = k[:10000]  # every key of the first third appears two or three times
    k[20000:25000] = k[:5000]
    rng = np.random.default_rng(F)
    seq = (rng.permutation(30000).astype(np.uint64) << np.uint64(20)) | np.uint64(7)
    t.update(cu(ops), cu(k), cu(v), seq=cu(seq))
    order = np.argsort(seq, kind="stable")
    ref = orc.UpdateMap(keys, vals)
    ref.apply(ops[order], k[order], v[order])
    rk, rv = ref.dump()
    probe = np.concatenate([keys, k, gen.edge_queries(keys)])
    check_tree(hm, orc, t, F, rk, rv, probe)


def test_route_update_payload(hm):
    import torch

    n = 10007
    rng = np.random.default_rng(3)
    ops = rng.integers(0, 2, n).astype(np.uint8)
    vals = gen._stream(9, 0, n)
    pos = rng.permutation(n).astype(np.uint32)
    o, v, s = hm.route_update_payload(cu(ops), cu(vals), torch.from_numpy(pos.view(np.int32)).cuda().view(torch.uint32),
                                      5)
    assert np.array_equal(o.cpu().numpy(), ops[pos])
    assert np.array_equal(v.cpu().numpy(), vals[pos])
    assert np.array_equal(s.cpu().numpy(), (np.uint64(5) << np.uint64(32)) | pos.astype(np.uint64))


def check_tree_relaxed(hm, orc, t, F, ref_keys, ref_vals, probe):
    """After in-place batches: I1-I7 with routing separators (the equality half of I5 only
    holds for a fresh build), results equal to the std::map oracle."""
    info, kr, ps, lv = t.export_layout()
    assert info["n_keys"] == ref_keys.shape[0]
    assert info["min_key"] == int(ref_keys[0]) and info["max_key"] == int(ref_keys[-1])
    code, msg = orc.Layout(F, info["height"], info["level_start"], kr, ps, lv).check(ref_keys, ref_vals,
                                                                                    strict_separators=False)
    assert code == 0, msg
    out = t.search(cu(probe)).cpu().numpy()
    assert np.array_equal(out, orc.sorted_search(ref_keys, ref_vals, probe))
    for cap in (8, 300):  # the lane and the warp range kernels (counts from the recomputed leaf_base)
        lo, hi = gen.random_ranges(ref_keys, 500, max_width_keys=3 * cap)
        ko, vo, cnt = t.range(cu(lo), cu(hi), cap)
        eko, evo, ecnt = orc.sorted_range(ref_keys, ref_vals, lo, hi, cap)
        assert np.array_equal(cnt.cpu().numpy(), ecnt)
        m = np.minimum(ecnt.astype(np.int64), cap)
        mask = np.arange(cap)[None, :] < m[:, None]
        assert np.array_equal(ko.cpu().numpy()[mask], eko[mask]) and np.array_equal(vo.cpu().numpy()[mask], evo[mask])


@pytest.mark.parametrize("F,fill,in_place", [(8, 0.69, False), (16, 0.69, True), (32, 0.69, True), (64, 0.69, True),
                                             (128, 0.75, True)])
def test_update_in_place(hm, orc, F, fill, in_place):
    """Trees with room (fill < 1): the paper's 5 % insert + 5 % delete + 90 % update batches
     go in place; values, re-packed leaves and leaf_base match the oracle after every
    batch, including keys below the minimum / above the maximum and repeated keys."""
    keys = gen.uniform_keys(60000)
    vals = gen.values_for(keys)
    t = hm.Tree(cu(keys), cu(vals), fanout=F, fill=fill)
    ref = orc.UpdateMap(keys, vals)
    touched = []
    modes = []
    for b in range(5):
        rk, _ = ref.dump()
        ops, ks, vs = gen.update_ops(rk, 3000, insert_frac=0.05, delete_frac=0.05, seed=gen.SEED_OPS + 7 * b + F)
        ops = np.concatenate([ops, ops[:200] ^ np.uint8(1), np.zeros(2, dtype=np.uint8)])
        ks = np.concatenate([ks, ks[:200], np.array([b + 1, MAX - 1 - b], dtype=np.uint64)])
        vs = np.concatenate([vs, vs[:200] + np.uint64(3), np.array([5, 6], dtype=np.uint64)])
        t.update(ops, cu(ks), cu(vs))
        modes.append(t.last_update_mode())
        ref.apply(ops, ks, vs)
        touched.append(ks)
        rk, rv = ref.dump()
        probe = np.concatenate([np.concatenate(touched), gen.uniform_queries(rk, 20000, miss_frac=0.3),
                                gen.edge_queries(rk)])
        check_tree_relaxed(hm, orc, t, F, rk, rv, probe)
    # in place unless a leaf ran out of room (F = 8 at fill 0.69 builds minimum-occupancy
    # leaves of 4 records: any delete there underflows, so those batches rebuild)
    assert modes.count(1) >= 2 if in_place else modes.count(2) >= 1, modes


def test_update_in_place_overflow_falls_back(hm, orc):
    """A batch that overfills one leaf (many inserts into one key gap) takes the full rebuild,
    whose layout is the closed form again; in-place batches resume afterwards."""
    keys = (np.arange(1, 20001, dtype=np.uint64) * np.uint64(1000))
    vals = gen.values_for(keys)
    F = 16
    t = hm.Tree(cu(keys), cu(vals), fanout=F, fill=0.69)
    ref = orc.UpdateMap(keys, vals)
    ks = np.arange(5001, 5001 + 40, dtype=np.uint64)  # 40 keys into the gap after key 5000
    ops = np.zeros(ks.shape[0], dtype=np.uint8)
    vs = gen.values_for(ks)
    t.update(ops, cu(ks), cu(vs))
    ref.apply(ops, ks, vs)
    assert t.last_update_mode() == 2
    rk, rv = ref.dump()
    check_tree_relaxed(hm, orc, t, F, rk, rv, np.concatenate([ks, gen.uniform_queries(rk, 5000, miss_frac=0.3)]))
    ops2, ks2, vs2 = gen.update_ops(rk, 500, insert_frac=0.0, delete_frac=0.02, seed=99)
    t.update(ops2, cu(ks2), cu(vs2))
    ref.apply(ops2, ks2, vs2)
    assert t.last_update_mode() == 1
    rk, rv = ref.dump()
    check_tree_relaxed(hm, orc, t, F, rk, rv, np.concatenate([ks2, gen.uniform_queries(rk, 5000, miss_frac=0.3)]))

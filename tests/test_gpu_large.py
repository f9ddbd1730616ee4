"""Parity at the BASELINE configurations' full sizes (GPU).

Full-size outputs are checked by properties that hold at any size (values are key-derived,
so a hit must return values_for(q); key+1 between two keys must return NOT_FOUND), plus
sampled element-by-element comparisons against the oracle where the key set fits the host
comfortably."""
import numpy as np
import pytest

import harmonia_gen as gen

pytestmark = pytest.mark.gpu
MAX = np.uint64((1 << 64) - 1)


@pytest.fixture(scope="module")
def hm():
    import torch

    assert torch.cuda.is_available()
    import paper_conf_ppopp_yanlpz19_b200 as m

    m.lib()
    return m


def _check_device(hm, t, keys_t, Q, seed):
    """All-hit batch (property) + key+1 misses (property) on the device, no host copies."""
    import torch

    q = gen.uniform_queries_t(keys_t, Q, seed=seed)
    out = t.search(q.view(torch.uint64)).view(torch.int64)
    bad = int((out != gen.values_for_t(q)).sum())
    assert bad == 0, f"{bad} wrong hits"
    sel = torch.randint(0, keys_t.shape[0] - 1, (1 << 20,), device=keys_t.device,
                        generator=torch.Generator(device=keys_t.device).manual_seed(seed))
    nxt = keys_t[sel] + 1
    miss = nxt[nxt != keys_t[sel + 1]]                      # strictly between two keys
    out2 = t.search(miss.view(torch.uint64)).view(torch.int64)
    assert int((out2 != -1).sum()) == 0, "absent keys must return NOT_FOUND"
    return q, out


def test_config3_zipf_full_size(hm, orc):
    """c3: 2^26 keys, F=64, 2^26 Zipfian (theta 0.99) queries; 2^20 sampled vs the oracle."""
    import torch

    T, Q = 1 << 26, 1 << 26
    keys = gen.uniform_keys(T)
    vals = gen.values_for(keys)
    t = hm.Tree(torch.from_numpy(keys).cuda(), torch.from_numpy(vals).cuda(), fanout=64)
    q = gen.zipf_queries(keys, Q)
    out = t.search(torch.from_numpy(q).cuda()).cpu().numpy()
    assert np.array_equal(out, gen.values_for(q))
    sel = gen._stream(11, 0, 1 << 20) % np.uint64(Q)
    assert np.array_equal(out[sel], orc.sorted_search(keys, vals, q[sel]))
    # ranges at the c4 lengths on this tree
    for length in (16, 1024):
        lo, hi = gen.ranges(keys, 1 << 14, length)
        ko, vo, cnt = t.range(torch.from_numpy(lo).cuda(), torch.from_numpy(hi).cuda(), length)
        eko, evo, ecnt = orc.sorted_range(keys, vals, lo, hi, length)
        assert np.array_equal(cnt.cpu().numpy(), ecnt)
        assert np.array_equal(ko.cpu().numpy(), eko) and np.array_equal(vo.cpu().numpy(), evo)


def test_config4_full_size_device_generated(hm, orc):
    """c4: 2^28 keys (one replica), 2^27 queries per GPU, generated on the device."""
    import torch

    T, Q = 1 << 28, 1 << 27
    keys_t = gen.uniform_keys_t(T, "cuda")
    t = hm.Tree(keys_t.view(torch.uint64), gen.values_for_t(keys_t).view(torch.uint64), fanout=64)
    assert t.info()["height"] == 5
    q, out = _check_device(hm, t, keys_t, Q, seed=gen.SEED_QUERY)
    # sampled element-by-element comparison against the oracle (keys copied once to the host)
    keys = keys_t.cpu().numpy().view(np.uint64)
    vals = gen.values_for(keys)
    sel = torch.from_numpy((gen._stream(12, 0, 1 << 18) % np.uint64(Q)).astype(np.int64)).cuda()
    qs = q[sel].cpu().numpy().view(np.uint64)
    assert np.array_equal(out[sel].cpu().numpy().view(np.uint64), orc.sorted_search(keys, vals, qs))


def test_config5_shard_full_size(hm):
    """c5: one of the 8 key-range shards of 2^32 keys (2^29 keys, indices [3*2^29, 4*2^29)),
    F=64 -- 64-bit slot addressing beyond 2^32 slots, queries routed to this shard."""
    import torch

    T, S = 1 << 32, 1 << 29
    keys_t = gen.uniform_keys_t(T, "cuda", start=3 * S, count=S)
    t = hm.Tree(keys_t.view(torch.uint64), gen.values_for_t(keys_t).view(torch.uint64), fanout=64)
    info = t.info()
    assert info["n_keys"] == S and info["key_region_bytes"] > (1 << 32)  # byte offsets beyond 32 bits
    _check_device(hm, t, keys_t, 1 << 26, seed=gen.SEED_QUERY + 5)


@pytest.mark.parametrize("fanout,fill", [(8, 1.0), (16, 1.0), (32, 1.0), (128, 1.0), (8, 0.69), (32, 0.69),
                                         (64, 0.69), (128, 0.69)])
def test_config3_fanout_sweep_full_size(hm, orc, fanout, fill):
    """c3's fanout sweep at its full size (2^26 keys, F in 8..128, fill
    1.0 and 0.69, 2^26 Zipfian queries), in the launch configuration the bench's sweep times:
    every hit checked on the device by the key-derived values, key+1 misses, and 2^18 sampled
    queries element by element against the oracle."""
    import torch

    T, Q = 1 << 26, 1 << 26
    keys_t = gen.uniform_keys_t(T, "cuda")
    t = hm.Tree(keys_t.view(torch.uint64), gen.values_for_t(keys_t).view(torch.uint64), fanout=fanout, fill=fill)
    q = gen.zipf_queries_t(keys_t, Q)
    out = t.search(q.view(torch.uint64)).view(torch.int64)
    assert int((out != gen.values_for_t(q)).sum()) == 0
    _check_device(hm, t, keys_t, 1 << 22, seed=gen.SEED_QUERY + fanout)
    keys = keys_t.cpu().numpy().view(np.uint64)
    sel = torch.from_numpy((gen._stream(13 + fanout, 0, 1 << 18) % np.uint64(Q)).astype(np.int64)).cuda()
    qs = q[sel].cpu().numpy().view(np.uint64)
    assert np.array_equal(out[sel].cpu().numpy().view(np.uint64), orc.sorted_search(keys, gen.values_for(keys), qs))
    vals = gen.values_for(keys)
    lo, hi = gen.ranges(keys, 1 << 12, 64)
    ko, vo, cnt = t.range(torch.from_numpy(lo).cuda(), torch.from_numpy(hi).cuda(), 64)
    eko, evo, ecnt = orc.sorted_range(keys, vals, lo, hi, 64)
    assert np.array_equal(cnt.cpu().numpy(), ecnt)
    assert np.array_equal(ko.cpu().numpy(), eko) and np.array_equal(vo.cpu().numpy(), evo)

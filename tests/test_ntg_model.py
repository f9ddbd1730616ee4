"""NTG static profiling (Eq 3/4) in the library (csrc/tune.cu) against the oracle's
model (oracle/model.cc, itself pinned by tests/test_oracle_models.py).

The host arithmetic (harmonia_ntg_choose) runs without a GPU: the per-level (r, cnt) profile
of each sample is taken here from the oracle-built layout with a plain descent, and the
library's step table and chosen GS must equal the oracle's on the same PSA-ordered sample.
The device path (harmonia_tune_group_size: profiling kernel + PSA buckets) is checked on the
GPU against the same oracle numbers."""
import numpy as np
import pytest

import harmonia_gen as gen

PAD = np.uint64((1 << 64) - 1)


@pytest.fixture(scope="module")
def hm():
    import paper_conf_ppopp_yanlpz19_b200 as m

    m.lib()
    return m


def _profile(lay, q):
    """(r, cnt) per sample and level on the oracle layout: r = keys <= q in internal nodes
    (Eq 1's rank), keys < q at the leaf; cnt = valid keys of the node."""
    F, h = lay.F, lay.h
    kr = lay.key_region.reshape(-1, F)
    prof = np.zeros((len(q), h, 2), dtype=np.uint32)
    for j, x in enumerate(q):
        node = 0
        for l in range(h):
            k = kr[node]
            k = k[k != PAD]
            leaf = l + 1 == h
            prof[j, l] = (int(np.sum(k < x)) if leaf else int(np.sum(k <= x)), len(k))
            if not leaf:
                node = int(lay.ps[node]) + int(np.sum(k <= x))
    return prof


@pytest.mark.parametrize("F,fill,n,nb", [(8, 1.0, 3000, 6), (16, 0.69, 5000, 8), (32, 1.0, 20000, 10),
                                         (64, 1.0, 40000, 11), (128, 0.69, 60000, 12), (64, 0.69, 5000, 0)])
def test_ntg_choose_equals_oracle(hm, orc, F, fill, n, nb):
    keys = gen.uniform_keys(n)
    vals = gen.values_for(keys)
    lay = orc.layout_build(keys, vals, F, fill)
    q = gen.uniform_queries(keys, 1000, miss_frac=0.2)
    lo, hi = int(keys[0]), int(keys[-1])
    bucket = np.array([orc.psa_bucket(int(x), nb, lo, hi) for x in q], dtype=np.uint32)
    prof = _profile(lay, q)
    qs = q[orc.psa_order(q, nb, lo, hi)] if nb else q
    gs0 = min(32, F // 2)
    for lev0 in range(lay.h):
        gs, steps = hm.ntg_choose(prof, bucket if nb else None, lay.h, lev0, gs0, 2)
        assert gs == lay.ntg_choose_gs(qs, gs0, 2, lev0)
        for i in range(6):
            g = 1 << i
            want = lay.ntg_warp_steps(qs, g, 2, lev0) if g <= gs0 else 0.0
            assert steps[i] == pytest.approx(want, rel=1e-12, abs=1e-12), (lev0, g)


def test_ntg_choose_closed_forms(hm):
    # one level, every node full (cnt = 31 keys) and every target at r = 30 (the last slot):
    # steps = min(30 // (2 GS) + 1, ceil(31 / (2 GS))) = ceil(31 / (2 GS)) -> 8, 4, 2, 1 for
    # GS = 2, 4, 8, 16; S(GS) is that per warp, so 2 S(b)/S(a) = 1 at every halving and Eq 4
    # stops immediately (no gain from narrowing when every query walks the whole node)
    prof = np.zeros((64, 1, 2), dtype=np.uint32)
    prof[:, 0] = (30, 31)
    gs, st = hm.ntg_choose(prof, None, 1, 0, 16, 2)
    assert st[1:5] == [8.0, 4.0, 2.0, 1.0] and gs == 16
    # every target in the first step (r = 0): one step at any GS, so S is flat and halving
    # doubles throughput: Eq 4 narrows all the way to GS = 2
    prof[:, 0] = (0, 31)
    gs, st = hm.ntg_choose(prof, None, 1, 0, 16, 2)
    assert st[1:5] == [1.0, 1.0, 1.0, 1.0] and gs == 2
    # bad arguments
    from paper_conf_ppopp_yanlpz19_b200 import HarmoniaError

    with pytest.raises(HarmoniaError):
        hm.ntg_choose(prof, None, 1, 0, 12, 2)


@pytest.mark.gpu
@pytest.mark.parametrize("F,fill", [(8, 1.0), (16, 0.69), (64, 1.0), (128, 0.69)])
def test_tune_group_size_device_equals_oracle(hm, orc, F, fill):
    import torch

    keys = gen.uniform_keys(50000)
    vals = gen.values_for(keys)
    t = hm.Tree(torch.from_numpy(keys).cuda(), torch.from_numpy(vals).cuda(), fanout=F, fill=fill)
    lay = orc.layout_build(keys, vals, F, fill)
    q = gen.uniform_queries(keys, 1000, miss_frac=0.2)
    plan = t.plan(1 << 27)
    nb, lev0 = plan["psa_bits"], plan["smem_levels"]
    lev0 = min(lev0, lay.h - 1)
    qs = q[orc.psa_order(q, nb, int(keys[0]), int(keys[-1]))] if nb else q
    gs0 = min(32, F // 2)
    gs, steps = t.tune_group_size(torch.from_numpy(q).cuda())
    assert gs == lay.ntg_choose_gs(qs, gs0, 2, lev0)
    for i in range(6):
        g = 1 << i
        want = lay.ntg_warp_steps(qs, g, 2, lev0) if g <= gs0 else 0.0
        assert steps[i] == pytest.approx(want, rel=1e-12, abs=1e-12)

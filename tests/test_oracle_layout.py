"""O4: the oracle's Harmonia layout builder, checker and Eq-1 interpreter, pinned by the
paper's worked examples (Fig 4 / Eq 1 / P:L270 sizes), a hand-derived layout, the
invariant checker (which must also reject mutated layouts) and O1 results."""
import numpy as np
import pytest

import harmonia_gen as gen
from conftest import golden_kv, golden_lines

PAD = (1 << 64) - 1


def test_eq1_worked_example(orc):
    g = golden_lines("fig4_ps.txt")
    ps = [int(x) for x in g[0].split(":")[1].split()]
    counts = [int(x) for x in g[1].split(":")[1].split()]
    assert [ps[i + 1] - ps[i] for i in range(len(ps) - 1)] == counts
    for ln in g[2:]:
        kv = dict(t.split("=") for t in ln.split(":")[1].split())
        assert orc.eq1_child(ps, int(kv["node"]), int(kv["i"])) == int(kv["child"])


def test_hand_derived_layout(orc):
    g = golden_kv("layout_n10_f4.txt")
    F = int(g["fanout"])
    keys = np.arange(10, 101, 10, dtype=np.uint64)
    vals = keys + np.uint64(1)
    lay = orc.layout_build(keys, vals, F, 1.0)
    conv = lambda s: [PAD if t == "P" else int(t) for t in s.split()]
    assert lay.h == int(g["height"])
    assert lay.level_start.tolist() == conv(g["level_start"])
    assert lay.ps.tolist() == conv(g["ps"])
    for n in range(lay.n_nodes):
        assert lay.key_region[n * F:(n + 1) * F].tolist() == conv(g[f"node{n}"]), n
    assert lay.leaf_vals.tolist() == conv(g["leafvals"])
    assert lay.check(keys, vals)[0] == 0


def test_ps_size_claim(orc):
    """a 64-fanout 4-level tree's PS array is 'about 16KB' (C-A7 reading)."""
    g = golden_kv("sizes.txt")
    F = 64
    n = (F - 1) * F ** 3  # a completely full 4-level tree
    h, ln = orc.layout_shape(n, F, 1.0)
    assert h == 4 and ln.tolist() == [1, 64, 4096, 262144]
    ps_bytes = 4 * (int(ln[:-1].sum()) + 1)
    assert ps_bytes == int(g["ps_bytes_f64_h4_full"])
    assert abs(ps_bytes / 1024 - int(g["ps_bytes_claim_kb_about"])) < 1.0
    assert (F - 1) * 8 == int(g["harmonia_item_bytes_f64"])
    assert (F - 1) * 8 + F * 8 == int(g["regular_node_bytes_f64"])       # P:L218 ~1 KB


def test_shape_closed_form():
    """C-A6 level sizes, recomputed here by plain ceil-division (fill 1.0)."""
    import oracle

    def expect(n, F):
        lv = [max(1, -(-n // (F - 1)))]
        while lv[-1] > 1:
            lv.append(-(-lv[-1] // F))
        return lv[::-1]

    for n, F in [(0, 4), (1, 4), (3, 4), (4, 4), (1 << 16, 16), (1 << 23, 64), (1 << 26, 8),
                 (1 << 26, 128), (1 << 28, 64), (12345, 256)]:
        h, ln = oracle.layout_shape(n, F, 1.0)
        assert ln.tolist() == expect(n, F), (n, F)
    # SURVEY Appendix A rows (hand arithmetic): 2^16 F16 and 2^23 F64
    assert oracle.layout_shape(1 << 16, 16)[1].tolist() == [1, 2, 18, 274, 4370]
    assert oracle.layout_shape(1 << 23, 64)[1].tolist() == [1, 33, 2081, 133153]


CASES = [(n, F, fill) for n in (0, 1, 2, 3, 7, 64, 500, 4095, 20000)
         for F in (4, 8, 16, 64, 256) for fill in (1.0, 0.69, 0.5)]


@pytest.mark.parametrize("n,F,fill", CASES)
def test_invariants_and_interpreter(orc, n, F, fill):
    keys = gen.random_keys(n, seed=n * 7 + F) if n else np.zeros(0, dtype=np.uint64)
    vals = gen.values_for(keys)
    lay = orc.layout_build(keys, vals, F, fill)
    code, msg = lay.check(keys, vals)
    assert code == 0, msg
    q = np.concatenate([gen.uniform_queries(keys, 500, miss_frac=0.4) if n else gen._stream(5, 0, 20),
                        gen.edge_queries(keys)])
    assert np.array_equal(lay.search(q), orc.sorted_search(keys, vals, q))
    lo, hi = gen.random_ranges(keys, 100)
    a, b = lay.range(lo, hi, 24), orc.sorted_range(keys, vals, lo, hi, 24)
    assert np.array_equal(a[2], b[2])
    for j in range(lo.shape[0]):
        m = min(int(a[2][j]), 24)
        assert np.array_equal(a[0][j][:m], b[0][j][:m]) and np.array_equal(a[1][j][:m], b[1][j][:m])


def test_fill_lowers_occupancy(orc):
    keys = gen.uniform_keys(50000)
    for F in (16, 64):
        h1, l1 = orc.layout_shape(keys.shape[0], F, 1.0)
        h2, l2 = orc.layout_shape(keys.shape[0], F, 0.5)
        assert l2[-1] > l1[-1] and h2 >= h1


def test_checker_rejects_mutations(orc):
    """The checker must not be vacuous: each targeted corruption trips its invariant."""
    keys = gen.uniform_keys(3000)
    vals = gen.values_for(keys)
    base = orc.layout_build(keys, vals, 8, 1.0)
    F, I = base.F, base.n_internal

    def mutated(fn):
        lay = orc.Layout(base.F, base.h, base.level_start.copy(), base.key_region.copy(),
                         base.ps.copy(), base.leaf_vals.copy())
        fn(lay)
        return lay.check(keys, vals)[0]

    def bump_ps(l):
        l.ps[3] += 1

    def sentinel(l):
        l.ps[I] -= 1

    def swap_keys(l):
        s = (I + 5) * F
        l.key_region[s], l.key_region[s + 1] = l.key_region[s + 1], l.key_region[s]

    def bad_sep(l):
        l.key_region[2 * F] += np.uint64(1)

    def bad_val(l):
        l.leaf_vals[17] ^= np.uint64(1)

    def pad_val(l):
        cnt = int((l.key_region[(I) * F:(I + 1) * F] != np.uint64(PAD)).sum())
        l.leaf_vals[cnt] = np.uint64(0)

    def drop_key(l):
        s = (I + 9) * F
        cnt = int((l.key_region[s:s + F] != np.uint64(PAD)).sum())
        l.key_region[s + cnt - 1] = np.uint64(PAD)

    assert mutated(bump_ps) in (1, 2, 5, 6)
    assert mutated(sentinel) == 1
    assert mutated(swap_keys) == 6
    assert mutated(bad_sep) == 5
    assert mutated(bad_val) == 7
    assert mutated(pad_val) == 6
    assert mutated(drop_key) in (3, 6, 7)  # value slot no longer padded, or record lost


def test_hand_derived_layout_fill05(orc):
    """A fill-0.5 build (C-A6) written out by hand: level sizes, PS, separators, slots."""
    g = golden_kv("layout_n10_f4_fill05.txt")
    F = int(g["fanout"])
    keys = np.arange(10, 101, 10, dtype=np.uint64)
    vals = keys + np.uint64(1)
    lay = orc.layout_build(keys, vals, F, 0.5)
    conv = lambda s: [PAD if t == "P" else int(t) for t in s.split()]
    assert lay.h == int(g["height"])
    assert lay.level_start.tolist() == conv(g["level_start"])
    assert lay.ps.tolist() == conv(g["ps"])
    for n in range(lay.n_nodes):
        assert lay.key_region[n * F:(n + 1) * F].tolist() == conv(g[f"node{n}"]), n
    assert lay.leaf_vals.tolist() == conv(g["leafvals"])
    assert lay.check(keys, vals)[0] == 0


def test_shape_fill_below_one():
    """C-A6 at fill 0.69 / 0.5 against hand arithmetic (2^23 F64 -> h = 5)."""
    import oracle

    for ln in golden_lines("shape_fill.txt"):
        f = ln.split()
        n, F, fill, levels = 1 << int(f[0]), int(f[1]), float(f[2]), [int(x) for x in f[3:]]
        h, ln_ = oracle.layout_shape(n, F, fill)
        assert h == len(levels) and ln_.tolist() == levels, (n, F, fill)


def test_relaxed_separator_check(orc):
    """strict_separators=False accepts a layout whose leaf lost its minimum (a delete applied in
    place) but still rejects keys outside the separator bounds (I5 routing)."""
    keys = gen.uniform_keys(3000)
    vals = gen.values_for(keys)
    lay = orc.layout_build(keys, vals, 8, 1.0)  # 7 records per leaf: one can go (I3 >= 4)
    I, F = lay.n_internal, lay.F
    leaf = I + 5  # a leaf with a separator in its parent (not the first child)
    kr, lv = lay.key_region.copy(), lay.leaf_vals.copy()
    cnt = int((kr[leaf * F:(leaf + 1) * F] != np.uint64(PAD)).sum())
    gone = kr[leaf * F]
    kr[leaf * F:leaf * F + cnt - 1] = kr[leaf * F + 1:leaf * F + cnt]
    kr[leaf * F + cnt - 1] = np.uint64(PAD)
    lv[(leaf - I) * F:(leaf - I) * F + cnt - 1] = lv[(leaf - I) * F + 1:(leaf - I) * F + cnt]
    lv[(leaf - I) * F + cnt - 1] = np.uint64(PAD)
    keep = keys != gone
    mut = orc.Layout(F, lay.h, lay.level_start.copy(), kr, lay.ps.copy(), lv)
    assert cnt - 1 >= F // 2
    assert mut.check(keys[keep], vals[keep])[0] == 5                      # strict: separator != min
    assert mut.check(keys[keep], vals[keep], strict_separators=False)[0] == 0
    bad = orc.Layout(F, lay.h, lay.level_start.copy(), kr.copy(), lay.ps.copy(), lv)
    bad.key_region[leaf * F] = np.uint64(1)                              # below its separator
    kk = np.sort(np.concatenate([keys[keep & (keys != kr[leaf * F])], np.array([1], dtype=np.uint64)]))
    assert bad.check(kk, gen.values_for(kk), strict_separators=False)[0] != 0

"""bench.py's algorithmic-bytes model of the search kernel on the
c2 geometry, computed by hand: it is the numerator of roofline.achieved.  CPU only."""
import bench

# c2: T = 2^23 keys, F = 64, fill 1.0 -> levels of 1, 33, 2081, 133153 nodes
INFO = {"fanout": 64, "height": 4, "level_start": [0, 1, 34, 2115, 135268]}
NW = 1 << 26


def test_c2_staged_model():
    plan = {"psa_bits": 19, "smem_levels": 2, "staged_return": 1}
    got, noreuse = bench.roofline_model(INFO, plan, NW, 126 << 20)
    io = 18 * NW                            # 8 B query + 2 B chunk offset + 8 B result
    lvl2 = 2081 * 512                        # whole level (no-reuse would be NW * 544)
    leaf = 133153 * 512 * 2                  # whole leaf level + its values
    assert got == io + lvl2 + leaf
    assert noreuse == 18 + 2 * (512 + 32)


def test_no_psa_and_unstaged_levels():
    plan = {"psa_bits": 0, "smem_levels": 0, "staged_return": 0}
    got, noreuse = bench.roofline_model(INFO, plan, 1000, 0)
    # 1000 queries: every level is charged min(no-reuse, whole level)
    expect = 16 * 1000 + min(1000 * 544, 1 * 512) + min(1000 * 544, 33 * 512) + \
        min(1000 * 544, 2081 * 512) + min(1000 * 544, 133153 * 1024)
    assert got == expect
    assert noreuse == 16 + 4 * 544


def test_c2_step_model_by_hand():
    """SURVEY §8(d) step model on c2: levels 0-1 in shared memory; level 2 (2081 x 512 B) and
    the leaves with their values (133153 x 1024 B) fit the 126.5 MiB L2 (+5 %): L2 tier."""
    plan = {"smem_levels": 2}
    m = bench.step_model(INFO, plan, NW, 132644864, 6538.0, 17775.2, psa=True)
    assert m["B_hbm"] == 16 + 72
    assert m["B_l2"] == 88 + 2 * (512 + 32)
    assert m["l2_tier_levels"] == 2 and m["hbm_tier_levels"] == 0
    assert abs(m["bound_gqs"] - min(6538.0 / 88, 17775.2 / 1176)) < 1e-9
    unique = (2081 * 512 + 133153 * 1024) / NW
    assert abs(m["reuse_aware"]["B_l2"] - (88 + unique)) < 1e-9
    assert abs(m["reuse_aware"]["bound_gqs"] - 6538.0 / 88) < 1e-9


def test_step_model_hbm_tier():
    """c4 geometry (2^28 keys, F64): levels 2-3 (33 MiB) in L2, the 2 GiB leaves in HBM."""
    info = {"fanout": 64, "height": 5, "level_start": [0, 1, 18, 1059, 67636, 4328517]}
    m = bench.step_model(info, {"smem_levels": 2}, 1 << 27, 132644864, 6538.0, 17775.2)
    assert m["l2_tier_levels"] == 2 and m["hbm_tier_levels"] == 1
    assert m["B_hbm"] == 88 + 544 and m["B_l2"] == 88 + 3 * 544


def test_lsu_roofline_from_committed_capture():
    """roofline.lsu / step_lsu from the committed c2 capture: the search kernel's wavefronts
    over its launch time against 1 wavefront / cycle / SM, and the sum over the five kernels
    of a step as an LSU-bound step time (DESIGN.md §7 item 4)."""
    import json
    import os

    d = json.load(open(os.path.join(os.path.dirname(bench.__file__), "profiles", "ncu_r2.json")))
    allk = d["c2_T2^23_F64_Q2^26_uniform"]
    st = allk["k_lane_search_c"]
    lsu, step = bench.lsu_roofline(st, allk, 148, 2000.0, 1.0, 2.0, True)
    assert abs(lsu["peak"] - 296.0) < 1e-9                      # 148 x 2 GHz x 1 wavefront
    assert abs(lsu["achieved"] - st["lsu_wavefronts"] / 1e-3 / 1e9) < 1e-9
    wsum = sum(allk[k]["lsu_wavefronts"] for k in bench.STEP_KERNELS)
    assert step["wavefronts_per_step"] == wsum
    assert abs(step["bound_ms"] - wsum / 296e9 * 1e3) < 1e-12
    assert abs(step["frac"] - step["bound_ms"] / 2.0) < 1e-12
    # the committed capture: the search alone is the largest share of the step's wavefronts
    assert st["lsu_wavefronts"] > 0.4 * wsum
    # absent inputs: no figure, no exception
    assert bench.lsu_roofline(None, {}, 148, 2000.0, 1.0, 2.0, True) == (None, None)
    assert bench.lsu_roofline(st, allk, 148, None, 1.0, 2.0, True) == (None, None)
    assert bench.lsu_roofline(st, allk, 148, 2000.0, 1.0, 2.0, False)[1] is None

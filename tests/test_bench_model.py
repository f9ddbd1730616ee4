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

"""Algorithm 2, the kernel-configuration heuristic, as
the library implements it (lop_alg2_select; no GPU needed).  Pinned by the
paper's own worked example (L682-L689): for a 13 x 13 window "we prefer a
configuration of 32x6 over 32x4 ... a configuration of 32x3, however, would
be preferred to the two aforementioned configurations", and by the rules of
lines 1-3 and 18-20 on hand-built cases."""
import pytest

import paper_conf_ipps_membarthhtke12_b200 as lop


def _c(bx, by, occ, valid=True, ox=1, oy=1):
    return dict(block_x=bx, block_y=by, occupancy=occ, valid=valid, out_x=ox, out_y=oy)


# 4092 rows (a multiple of 3, 4 and 6) x 4096 columns, 13 x 13 window (r = 6)
W, H, R = 4096, 4092, 6


def test_paper_example_32x6_over_32x4():
    i, bh = lop.alg2_select([_c(32, 4, 1.0), _c(32, 6, 1.0)], W, H, R, R)
    assert i == 1
    # 32x6 tiles: one tile row at the top and one at the bottom reach outside,
    # plus the left / right tile columns (32 wide > r): 6-row tiles
    nty, ntx = H // 6, W // 32
    assert bh == (ntx * nty - (ntx - 2) * (nty - 2)) * 192


def test_paper_example_32x3_preferred_to_both():
    # equal occupancy: sorted by ascending threads, 32x3 first; its border
    # threads (2 tile rows of 3 = 6 rows) are not beaten strictly by 32x6
    i, _ = lop.alg2_select([_c(32, 4, 1.0), _c(32, 6, 1.0), _c(32, 3, 1.0)], W, H, R, R)
    assert i == 2


def test_occupancy_first_then_border_threads():
    # 32x6 has fewer border threads but lower occupancy: only the highest-occupancy
    # configurations compete (line 8)
    i, _ = lop.alg2_select([_c(32, 4, 1.0), _c(32, 6, 0.75)], W, H, R, R)
    assert i == 0


def test_simd_multiple_and_resource_limits():
    # line 1: thread counts not a multiple of the SIMD width are dropped; line 2: invalid ones
    i, _ = lop.alg2_select([_c(30, 4, 1.0), _c(32, 6, 1.0, valid=False), _c(64, 2, 0.5)], W, H, R, R)
    assert i == 2
    assert lop.alg2_select([_c(30, 1, 1.0)], W, H, R, R)[0] == -1


def test_no_border_handling_takes_the_first():
    # lines 18-20: no window -> highest occupancy, then fewest threads
    i, bh = lop.alg2_select([_c(256, 1, 1.0), _c(128, 1, 1.0), _c(512, 1, 0.5)], W, H, 0, 0)
    assert i == 1 and bh == 0


@pytest.mark.parametrize("oy", [1, 4])
def test_border_threads_count_tiles_whose_footprint_leaves_the_image(oy):
    # 100 x 50 image, 32 x 2 threads, each 1 x oy outputs, r = (3, 2)
    i, bh = lop.alg2_select([_c(32, 2, 1.0, oy=oy)], 100, 50, 3, 2)
    th = 2 * oy
    ntx, nty = -(-100 // 32), -(-50 // th)
    bx = sum(1 for t in range(ntx) if t * 32 - 3 < 0 or (t + 1) * 32 - 1 + 3 > 99)
    by = sum(1 for t in range(nty) if t * th - 2 < 0 or (t + 1) * th - 1 + 2 > 49)
    assert i == 0 and bh == (ntx * nty - (ntx - bx) * (nty - by)) * 64

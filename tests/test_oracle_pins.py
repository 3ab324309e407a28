"""Pins for the CPU oracle (oracle/), run with -m "not gpu".

Each test checks the oracle against something other than itself: the values
the paper prints (Fig. 2 cells, Listing 4's 0.018316), library routines
(np.pad, scipy.ndimage.correlate, scipy.special.comb), closed forms and
hand-computed worked examples, and invariants chosen so that a dropped term,
a wrong sign or index, or a transposed operand fails at least one of them.
"""
import math
import os
import zlib

import numpy as np
import pytest
import scipy.ndimage as ndi
import scipy.special

import oracle
from conftest import GOLDEN

MODES = ["clamp", "repeat", "mirror", "constant"]
SCIPY_MODE = {"clamp": "nearest", "repeat": "wrap", "mirror": "reflect", "constant": "constant"}
NP_PAD_MODE = {"clamp": "edge", "repeat": "wrap", "mirror": "symmetric"}


def _grid(name):
    rows = []
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            if line.startswith("#") or not line.strip():
                continue
            rows.append(line.split())
    assert len(rows) == 10 and all(len(r) == 10 for r in rows)
    return rows


def _letters_image():
    # A..P on a 4x4 image, Fig. 2
    return np.arange(16, dtype=np.float32).reshape(4, 4)


LETTER = {chr(ord("A") + i): float(i) for i in range(16)}
Q = 99.0


# ---------------------------------------------------------------- Fig. 2 ----

@pytest.mark.parametrize("mode,fname", [("repeat", "fig2_repeat.txt"),
                                        ("clamp", "fig2_clamp.txt"),
                                        ("constant", "fig2_constant.txt"),
                                        ("mirror", "fig2_mirror.txt"),
                                        ("undefined", "fig2_undefined.txt")])
def test_fig2_cells(mode, fname):
    img = _letters_image()
    grid = _grid(fname)
    checked = 0
    for iy, y in enumerate(range(-3, 7)):
        for ix, x in enumerate(range(-3, 7)):
            cell = grid[iy][ix]
            if cell == "*":
                continue          # mirror corner, drawn transposed (reading c6)
            v, undef = oracle.read(img, x, y, mode, cval=Q)
            if cell == "?":
                assert undef, (x, y)
            elif cell == "Q":
                assert not undef and v == Q, (x, y)
            else:
                assert not undef and v == LETTER[cell], (x, y, cell, v)
            checked += 1
    assert checked == (64 if mode == "mirror" else 100)


def test_fig2_mirror_corners_are_diagonal_reflections_of_per_axis_blocks():
    """Reading c6: every printed Mirror corner block equals the per-axis block
    reflected across the 45-degree diagonal through that image corner
    (transpose for TL/BR, anti-transpose for TR/BL), so the figure agrees with
    per-axis mirroring up to its drawing of the corners."""
    printed = {  # PAPER.md L404-L421, as scraped
        "TL": ["KGC", "JFB", "IEA"], "TR": ["BFJ", "CGK", "DHL"],
        "BL": ["EIM", "FJN", "GKO"], "BR": ["PLH", "OKG", "NJF"]}
    img = _letters_image()
    spans = {"TL": (range(-3, 0), range(-3, 0)), "TR": (range(-3, 0), range(4, 7)),
             "BL": (range(4, 7), range(-3, 0)), "BR": (range(4, 7), range(4, 7))}
    inv = {v: k for k, v in LETTER.items()}
    for name, (ys, xs) in spans.items():
        block = [[inv[oracle.read(img, x, y, "mirror")[0]] for x in xs] for y in ys]
        if name in ("TL", "BR"):
            refl = ["".join(block[j][i] for j in range(3)) for i in range(3)]
        else:
            refl = ["".join(block[2 - j][2 - i] for j in range(3)) for i in range(3)]
        assert refl == printed[name], (name, block)
        assert ["".join(r) for r in block] != printed[name]   # not the per-axis block


# ---------------------------------------------------------- index maps ----

@pytest.mark.parametrize("mode", ["clamp", "repeat", "mirror"])
@pytest.mark.parametrize("n", [1, 2, 3, 4, 5, 7])
def test_map_index_matches_np_pad(mode, n):
    pad = 2 * n + 1
    ref = np.pad(np.arange(n), (pad, pad), mode=NP_PAD_MODE[mode])
    for i in range(-pad, n + pad):
        assert oracle.map_index(i, n, mode) == ref[i + pad], (mode, n, i)


def test_map_index_constant_and_undefined():
    for mode in ("constant", "undefined"):
        assert oracle.map_index(-1, 4, mode) == -1
        assert oracle.map_index(4, 4, mode) == -1
        assert oracle.map_index(2, 4, mode) == 2


# ------------------------------------------------------------- masks ----

def test_closeness_listing4_printed_value():
    with open(os.path.join(GOLDEN, "listing4_closeness.txt")) as f:
        vals = [l.split() for l in f if not l.startswith("#") and l.strip()][0]
    sigma_d, size, index, printed, digits = (float(vals[0]), int(vals[1]), int(vals[2]),
                                             float(vals[3]), int(vals[4]))
    assert size == 4 * sigma_d + 1            # L325: window (4*sigma_d+1)^2
    m = oracle.closeness_mask(sigma_d, size)
    assert round(m.ravel()[index], digits) == printed
    assert m[size // 2, size // 2] == 1.0


@pytest.mark.parametrize("sigma_d,sx,sy", [(3, 13, 13), (1, 3, 3), (1, 5, 5), (2.5, 9, 3),
                                           (0.7, 3, 7)])
def test_closeness_equals_listing1_product_form(sigma_d, sx, sy):
    """Listing 1 l.13, l.21 (L234, L254): c = exp(-c_d*xf*xf) * exp(-c_d*yf*yf),
    c_d = 1/(2 sigma_d^2) -- a different formula from the oracle's Eq. (1)."""
    c_d = 1.0 / (2.0 * sigma_d * sigma_d)
    m = oracle.closeness_mask(sigma_d, sx, sy)
    assert m.shape == (sy, sx)
    for yf in range(-(sy // 2), sy // 2 + 1):
        for xf in range(-(sx // 2), sx // 2 + 1):
            ref = math.exp(-c_d * xf * xf) * math.exp(-c_d * yf * yf)
            assert abs(m[yf + sy // 2, xf + sx // 2] - ref) < 1e-15


@pytest.mark.parametrize("size", [1, 3, 5, 7, 9])
def test_gaussian_binomial(size):
    m, k = oracle.gaussian_mask(size)
    row = np.array([scipy.special.comb(size - 1, i, exact=True) for i in range(size)])
    assert (m == np.outer(row, row)).all()
    assert m.sum() == 2 ** k
    if size == 3:
        assert k == 4 and list(m[1]) == [2, 4, 2]
    if size == 5:
        assert k == 8 and list(m[2]) == [6, 24, 36, 24, 6]


def test_sobel_masks():
    sx = oracle.sobel_mask(0)
    assert sx.tolist() == [[-1, 0, 1], [-2, 0, 2], [-1, 0, 1]]
    assert (oracle.sobel_mask(1) == sx.T).all()


# ------------------------------------------------------- convolution ----

def _rng(seed):
    return np.random.default_rng(seed)


@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("shape,msize", [((17, 13), (3, 3)), ((9, 11), (5, 3)),
                                         ((6, 5), (1, 7)), ((4, 4), (9, 9)),
                                         ((3, 8), (7, 5)), ((1, 1), (3, 3))])
def test_convolve_f32_matches_scipy(mode, shape, msize):
    rng = _rng(zlib.crc32(repr((mode, shape, msize)).encode()))
    img = rng.random(shape).astype(np.float32)
    mask = rng.standard_normal((msize[1], msize[0]))          # asymmetric
    cval = 0.375
    out, valid = oracle.convolve_f32(img, mask, mode, cval)
    ref = ndi.correlate(img.astype(np.float64), mask, mode=SCIPY_MODE[mode], cval=cval)
    assert valid.all()
    np.testing.assert_allclose(out, ref, rtol=0, atol=1e-12)


def test_convolve_undefined_interior_and_valid_mask():
    rng = _rng(5)
    img = rng.random((12, 15)).astype(np.float32)
    mask = rng.standard_normal((5, 3))
    out, valid = oracle.convolve_f32(img, mask, "undefined")
    ref = ndi.correlate(img.astype(np.float64), mask, mode="nearest")
    exp_valid = np.zeros_like(valid)
    exp_valid[2:-2, 1:-1] = True                             # window (3 wide, 5 tall)
    assert (valid == exp_valid).all()
    np.testing.assert_allclose(out[valid], ref[valid], rtol=0, atol=1e-12)


def test_impulse_response_is_rotated_mask():
    rng = _rng(7)
    mask = rng.standard_normal((5, 7))
    img = np.zeros((15, 17), np.float32)
    img[7, 8] = 1.0
    out, _ = oracle.convolve_f32(img, mask, "constant", 0.0)
    # correlation: out(x,y) = sum M(xf,yf) I(x+xf,y+yf) -> response = mask rotated 180
    np.testing.assert_array_equal(out[5:10, 5:12], mask[::-1, ::-1])
    assert np.count_nonzero(out) == np.count_nonzero(mask)


@pytest.mark.parametrize("size", [3, 5])
def test_gaussian_preserves_ramp_and_sobel_gives_8a(size):
    a, b, c = 0.125, -0.0625, 0.5                     # exactly representable
    H, W = 12, 14
    y, x = np.mgrid[0:H, 0:W]
    img = (a * x + b * y + c).astype(np.float32)
    gm, k = oracle.gaussian_mask(size)
    out, _ = oracle.convolve_f32(img, gm / 2.0 ** k, "clamp")
    r = size // 2
    np.testing.assert_allclose(out[r:-r, r:-r], img[r:-r, r:-r], rtol=0, atol=1e-12)
    sx, _ = oracle.convolve_f32(img, oracle.sobel_mask(0), "clamp")
    sy, _ = oracle.convolve_f32(img, oracle.sobel_mask(1), "clamp")
    np.testing.assert_allclose(sx[1:-1, 1:-1], 8 * a, rtol=0, atol=1e-12)
    np.testing.assert_allclose(sy[1:-1, 1:-1], 8 * b, rtol=0, atol=1e-12)


@pytest.mark.parametrize("mode", MODES)
def test_separable_equals_2d(mode):
    rng = _rng(11)
    img = rng.random((10, 13)).astype(np.float32)
    g = np.array([1, 4, 6, 4, 1], np.float64) / 16.0
    two_d, _ = oracle.convolve_f32(img, np.outer(g, g), mode, cval=0.25)
    rows, _ = oracle.convolve_f32(img, g[None, :], mode, cval=0.25)
    # the column pass sees the row-filtered image; for constant mode its
    # out-of-bounds rows are C * sum(g) = C because g is normalised
    both, _ = oracle.convolve_f32(rows.astype(np.float64).astype(np.float32), g[:, None], mode,
                                  cval=0.25)
    # float32 round trip of the intermediate -> 1e-7 level agreement
    np.testing.assert_allclose(both, two_d, rtol=0, atol=2e-7)


@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("mask_kind", ["gauss3", "gauss5", "sobelx", "sobely", "random"])
def test_convolve_u8_exact_vs_scipy_integer(mode, mask_kind):
    rng = _rng(zlib.crc32(repr((mode, mask_kind)).encode()))
    img = rng.integers(0, 256, (13, 11)).astype(np.uint8)
    if mask_kind.startswith("gauss"):
        mask, _ = oracle.gaussian_mask(int(mask_kind[-1]))
    elif mask_kind == "sobelx":
        mask = oracle.sobel_mask(0)
    elif mask_kind == "sobely":
        mask = oracle.sobel_mask(1)
    else:
        mask = rng.integers(-9, 10, (5, 3)).astype(np.int32)
    S, valid = oracle.convolve_u8_sum(img, mask, mode, cval=128)
    ref = ndi.correlate(img.astype(np.int64), mask.astype(np.int64), mode=SCIPY_MODE[mode],
                        cval=128)
    assert valid.all()
    assert (S == ref).all()


def test_quantize_hand_cases_and_numpy():
    # (S + 2^(k-1)) >> k, saturating for u8 (reading c12)
    assert oracle.quantize(128, 8, True) == 1
    assert oracle.quantize(127, 8, True) == 0
    assert oracle.quantize(65280, 8, True) == 255
    assert oracle.quantize(-1, 0, True) == 0
    assert oracle.quantize(300, 0, True) == 255
    assert oracle.quantize(-129, 8, False) == -1
    assert oracle.quantize(-1020, 0, False) == -1020
    S = np.arange(-70000, 70000, 37, dtype=np.int64)
    for k in (0, 1, 4, 8):
        ref = (S + (1 << (k - 1) if k else 0)) // (1 << k)
        assert (oracle.quantize(S, k, False) == ref).all()
        assert (oracle.quantize(S, k, True) == np.clip(ref, 0, 255)).all()


def test_gaussian_u8_ramp_exact():
    # integer ramp image: the binomial Gaussian returns it exactly (interior)
    H, W = 9, 40
    y, x = np.mgrid[0:H, 0:W]
    img = (3 * x + 2 * y + 7).astype(np.uint8)
    for size in (3, 5):
        gm, k = oracle.gaussian_mask(size)
        q, valid = oracle.convolve_u8(img, gm, k, "clamp")
        r = size // 2
        assert (q[r:-r, r:-r] == img[r:-r, r:-r]).all()


def test_points_match_full():
    rng = _rng(3)
    img = rng.random((20, 23)).astype(np.float32)
    xs = rng.integers(0, 23, 50)
    ys = rng.integers(0, 20, 50)
    mask = rng.standard_normal((3, 5))
    full, _ = oracle.convolve_f32(img, mask, "mirror")
    pts, _ = oracle.convolve_f32_points(img, mask, "mirror", xs, ys)
    assert (pts == full[ys, xs]).all()
    u8 = rng.integers(0, 256, (20, 23)).astype(np.uint8)
    gm, _ = oracle.gaussian_mask(5)
    S, _ = oracle.convolve_u8_sum(u8, gm, "repeat")
    Sp, _ = oracle.convolve_u8_sum_points(u8, gm, "repeat", xs, ys)
    assert (Sp == S[ys, xs]).all()
    b, _ = oracle.bilateral_f32(img, 1.0, 0.1, "clamp", size=5)
    bp, _ = oracle.bilateral_f32_points(img, 1.0, 0.1, "clamp", xs, ys, size=5)
    assert (bp == b[ys, xs]).all()


# --------------------------------------------------------- bilateral ----

def test_bilateral_hand_example_center_and_corner():
    """3x3 zero image with a single 1 at the centre, sigma_d=1 (3x3), sigma_r=0.5.
    Centre: diff=1 to all 8 neighbours, s=exp(-1/2*(1/0.5)^2)=e^-2; edge taps
    c=e^-1/2, corner taps c=e^-1:  out = 1 / (1 + 4e^-2.5 + 4e^-3).
    Corner (0,0) under Clamp: only tap (+1,+1) reads the 1 (c=e^-1, s=e^-2);
    all other taps read 0 (s=1):  out = e^-3 / (1 + 4e^-.5 + 4e^-1 - e^-1 + e^-3)."""
    img = np.zeros((3, 3), np.float32)
    img[1, 1] = 1.0
    out, _ = oracle.bilateral_f32(img, 1.0, 0.5, "clamp", size=3)
    assert abs(out[1, 1] - 0.6546695126705685) < 1e-15
    assert abs(out[0, 0] - 0.01087161179089065) < 1e-15


@pytest.mark.parametrize("mode", MODES)
def test_bilateral_sigma_r_infinity_is_gaussian_correlation(mode):
    rng = _rng(21)
    img = rng.random((19, 16)).astype(np.float32)
    for sigma_d, size in ((1.0, 3), (1.5, 7), (3.0, 13)):
        out, _ = oracle.bilateral_f32(img, sigma_d, 1e6, mode, cval=0.3, size=size)
        c = oracle.closeness_mask(sigma_d, size)
        ref = ndi.correlate(img.astype(np.float64), c / c.sum(), mode=SCIPY_MODE[mode], cval=0.3)
        np.testing.assert_allclose(out, ref, rtol=0, atol=1e-9)


def test_bilateral_user_mask_orientation():
    """Listing 5: c = CMask(xf, yf); an asymmetric mask at sigma_r -> inf must act
    as correlation with the normalised mask (catches a transposed mask)."""
    rng = _rng(22)
    img = rng.random((11, 12)).astype(np.float32)
    cm = rng.random((3, 5)) + 0.1               # 5 wide, 3 tall
    out, _ = oracle.bilateral_f32(img, 1.0, 1e6, "mirror", cmask=cm)
    ref = ndi.correlate(img.astype(np.float64), cm / cm.sum(), mode="reflect")
    np.testing.assert_allclose(out, ref, rtol=0, atol=1e-9)
    # and with the closeness mask passed explicitly == computed in-kernel (A2 vs A3)
    cm2 = oracle.closeness_mask(2.0, 9)
    a, _ = oracle.bilateral_f32(img, 2.0, 0.1, "clamp", cmask=cm2)
    b, _ = oracle.bilateral_f32(img, 2.0, 0.1, "clamp", size=9)
    np.testing.assert_allclose(a, b, rtol=0, atol=1e-15)


def test_bilateral_step_edge_preserved():
    img = np.asarray(__import__("synthetic").levels(40, 37, seed=9).numpy())
    out, _ = oracle.bilateral_f32(img, 3.0, 0.02, "clamp")
    # cross-edge weights exp(-1/2 (0.5/0.02)^2) = e^-312.5 ~ 1e-136
    assert np.abs(out - img).max() < 1e-100
    # at sigma_r = 0.5 the range term no longer separates the levels
    out2, _ = oracle.bilateral_f32(img, 3.0, 0.5, "clamp")
    assert np.abs(out2 - img).max() > 1e-2


@pytest.mark.parametrize("mode", MODES)
def test_bilateral_constant_image(mode):
    v = 0.6875
    img = np.full((9, 8), v, np.float32)
    out, _ = oracle.bilateral_f32(img, 1.0, 0.1, mode, cval=v, size=5)
    np.testing.assert_allclose(out, v, rtol=0, atol=1e-15)


@pytest.mark.parametrize("mode", MODES)
def test_bilateral_convexity_and_flip_symmetry(mode):
    rng = _rng(31)
    img = rng.random((14, 15)).astype(np.float32)
    cval = 0.9
    out, _ = oracle.bilateral_f32(img, 1.0, 0.2, mode, cval=cval, size=5)
    fmode = SCIPY_MODE[mode]
    lo = ndi.minimum_filter(img.astype(np.float64), size=5, mode=fmode, cval=cval)
    hi = ndi.maximum_filter(img.astype(np.float64), size=5, mode=fmode, cval=cval)
    assert (out >= lo - 1e-15).all() and (out <= hi + 1e-15).all()
    flip, _ = oracle.bilateral_f32(np.ascontiguousarray(img[:, ::-1]), 1.0, 0.2, mode,
                                   cval=cval, size=5)
    np.testing.assert_allclose(flip[:, ::-1], out, rtol=0, atol=1e-14)
    flipud, _ = oracle.bilateral_f32(np.ascontiguousarray(img[::-1, :]), 1.0, 0.2, mode,
                                     cval=cval, size=5)
    np.testing.assert_allclose(flipud[::-1, :], out, rtol=0, atol=1e-14)


def test_bilateral_repeat_is_shift_equivariant():
    rng = _rng(32)
    img = rng.random((10, 12)).astype(np.float32)
    out, _ = oracle.bilateral_f32(img, 1.0, 0.3, "repeat", size=7)
    rolled, _ = oracle.bilateral_f32(np.roll(img, (3, -5), (0, 1)), 1.0, 0.3, "repeat", size=7)
    np.testing.assert_allclose(rolled, np.roll(out, (3, -5), (0, 1)), rtol=0, atol=1e-14)


def test_bilateral_undefined_valid_region():
    rng = _rng(33)
    img = rng.random((16, 18)).astype(np.float32)
    out, valid = oracle.bilateral_f32(img, 3.0, 0.1, "undefined")
    ref, _ = oracle.bilateral_f32(img, 3.0, 0.1, "clamp")
    exp_valid = np.zeros_like(valid)
    exp_valid[6:-6, 6:-6] = True
    assert (valid == exp_valid).all()
    assert (out[valid] == ref[valid]).all()


def test_bilateral_window_larger_than_image():
    # 13x13 window on a 2x3 image: repeat / mirror wrap several periods (reading c7)
    img = np.array([[0.1, 0.7, 0.3], [0.9, 0.2, 0.5]], np.float32)
    for mode in ("repeat", "mirror"):
        out, _ = oracle.bilateral_f32(img, 3.0, 1e6, mode)
        c = oracle.closeness_mask(3.0, 13)
        ref = ndi.correlate(img.astype(np.float64), c / c.sum(), mode=SCIPY_MODE[mode])
        np.testing.assert_allclose(out, ref, rtol=0, atol=1e-9)


# ------------------------------------------- local MIN / MAX (Listing 9) ----

def _domain(rng, msize, kind):
    if kind == "full":
        return np.ones((msize[1], msize[0]), np.int32)
    d = (rng.random((msize[1], msize[0])) < 0.5).astype(np.int32)   # asymmetric, holes
    d[rng.integers(0, msize[1]), rng.integers(0, msize[0])] = 7     # at least one tap
    return d


@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("op", ["min", "max"])
@pytest.mark.parametrize("shape,msize,kind", [((17, 13), (3, 3), "full"), ((9, 11), (5, 3), "random"),
                                              ((6, 5), (1, 7), "random"), ((4, 4), (9, 9), "full"),
                                              ((3, 8), (7, 5), "random"), ((1, 1), (3, 3), "full")])
def test_reduce_matches_scipy_rank_filters(mode, op, shape, msize, kind):
    """oracle.reduce (Listing 9 convolve(mask, MIN/MAX, ...)) == scipy.ndimage
    minimum_filter / maximum_filter with the mask's non-zero taps as footprint,
    f32 and u8, every defined mode, windows larger than the image, asymmetric
    domains with holes (a transposed or flipped domain fails)."""
    rng = _rng(zlib.crc32(repr(("reduce", mode, op, shape, msize, kind)).encode()))
    dom = _domain(rng, msize, kind)
    fn = ndi.minimum_filter if op == "min" else ndi.maximum_filter
    img = rng.random(shape).astype(np.float32)
    out, valid = oracle.reduce(img, dom, op, mode, 0.4375)
    ref = fn(img.astype(np.float64), footprint=dom != 0, mode=SCIPY_MODE[mode], cval=0.4375)
    assert valid.all() and np.array_equal(out, ref)
    u8 = rng.integers(0, 256, shape).astype(np.uint8)
    out, valid = oracle.reduce(u8, dom, op, mode, 77)
    ref = fn(u8.astype(np.int64), footprint=dom != 0, mode=SCIPY_MODE[mode], cval=77)
    assert valid.all() and np.array_equal(out, ref)


@pytest.mark.parametrize("mode", MODES)
def test_reduce_invariants(mode):
    """Erosion <= image <= dilation for domains holding the centre; MIN/MAX
    duality under negation (f32) and 255 - x (u8, constant mapped too); a
    constant image is a fixed point (constant mode with the same constant)."""
    rng = _rng(11)
    img = rng.random((23, 19)).astype(np.float32)
    dom = _domain(rng, (5, 7), "random")
    dom[3, 2] = 1                                                     # centre tap
    lo, _ = oracle.reduce(img, dom, "min", mode, 0.25)
    hi, _ = oracle.reduce(img, dom, "max", mode, 0.25)
    if mode != "undefined":
        assert (lo <= img).all() and (img <= hi).all()
        neg, _ = oracle.reduce(-img, dom, "min", mode, -0.25)
        assert np.array_equal(-neg, hi)
        u8 = rng.integers(0, 256, (23, 19)).astype(np.uint8)
        a, _ = oracle.reduce(u8, dom, "max", mode, 40)
        b, _ = oracle.reduce((255 - u8).astype(np.uint8), dom, "min", mode, 215)
        assert np.array_equal(a, 255 - b)
    flat = np.full((8, 9), 0.625, np.float32)
    out, _ = oracle.reduce(flat, dom, "min", mode, 0.625)
    assert (out == 0.625).all()


def test_reduce_undefined_valid_region():
    rng = _rng(12)
    img = rng.random((12, 15)).astype(np.float32)
    dom = np.ones((3, 5), np.int32)
    out, valid = oracle.reduce(img, dom, "max", "undefined")
    exp = np.zeros_like(valid)
    exp[1:-1, 2:-2] = True
    assert np.array_equal(valid, exp)
    ref, _ = oracle.reduce(img, dom, "max", "clamp")
    assert np.array_equal(out[valid], ref[valid])


# ---------------------- two local operators + point-operator epilogue (N3) ----

@pytest.mark.parametrize("mode", ["clamp", "mirror"])
def test_convolve2_sobel_magnitude_on_ramps(mode):
    """Sobel magnitude of a ramp I = a x + b y: gx = 8a, gy = 8b in the interior
    (the Sobel ramp pin above), so L2 = 8 sqrt(a^2 + b^2), L1 = 8 (|a| + |b|),
    SUMSQ = 64 (a^2 + b^2); exact for integer ramps on u8."""
    sx, sy = oracle.sobel_mask(0), oracle.sobel_mask(1)
    ys, xs = np.mgrid[0:20, 0:24]
    a, b = 3, -2
    u8 = (100 + a * xs + b * ys).astype(np.uint8)
    l1, _ = oracle.convolve2(u8, sx, sy, "l1", mode)
    sq, _ = oracle.convolve2(u8, sx, sy, "sumsq", mode)
    assert (l1[1:-1, 1:-1] == 8 * (abs(a) + abs(b))).all()
    assert (sq[1:-1, 1:-1] == 64 * (a * a + b * b)).all()
    f = (0.01 * a * xs + 0.01 * b * ys).astype(np.float32)
    l2, _ = oracle.convolve2(f, sx.astype(np.float64), sy.astype(np.float64), "l2", mode)
    gx, _ = oracle.convolve_f32(f, sx.astype(np.float64), mode)
    gy, _ = oracle.convolve_f32(f, sy.astype(np.float64), mode)
    np.testing.assert_allclose(l2[1:-1, 1:-1], 0.08 * math.hypot(a, b), rtol=1e-5)
    np.testing.assert_allclose(l2, np.hypot(gx, gy), rtol=1e-14, atol=1e-15)


def test_convolve2_transpose_symmetry():
    """Swapping the image axes swaps Sobel-x and Sobel-y: the L2 / L1 magnitude
    of the transposed image is the transposed magnitude (symmetric modes)."""
    rng = _rng(21)
    img = rng.random((17, 23)).astype(np.float32)
    sx, sy = oracle.sobel_mask(0).astype(np.float64), oracle.sobel_mask(1).astype(np.float64)
    for mode in ("clamp", "mirror", "repeat"):
        m, _ = oracle.convolve2(img, sx, sy, "l2", mode)
        mt, _ = oracle.convolve2(np.ascontiguousarray(img.T), sx, sy, "l2", mode)
        np.testing.assert_allclose(mt, m.T, rtol=0, atol=1e-12)


# ------------------------------------------------- global operators (N3) ----

def test_global_reduce_closed_forms():
    """Sum of a constant image = v N exactly; sum of an integer ramp = the
    arithmetic-series closed form; min / max of a ramp = its end values;
    a region and a stack of frames reduce the selected pixels only."""
    flat = np.full((37, 53), 0.375, np.float32)
    assert oracle.global_reduce(flat, "sum") == 0.375 * 37 * 53
    ys, xs = np.mgrid[0:40, 0:50]
    ramp = (xs + 50 * ys).astype(np.float32)                 # 0 .. 1999, each once
    assert oracle.global_reduce(ramp, "sum") == 1999 * 2000 / 2
    assert oracle.global_reduce(ramp, "min") == 0 and oracle.global_reduce(ramp, "max") == 1999
    # region rows 10..19, columns 5..14: sum of x + 50 y over the block
    exp = sum(x + 50 * y for y in range(10, 20) for x in range(5, 15))
    assert oracle.global_reduce(ramp, "sum", roi=(5, 10, 10, 10)) == exp
    u8 = (np.arange(3 * 16 * 16) % 256).astype(np.uint8).reshape(3, 16, 16)
    assert oracle.global_reduce(u8, "sum") == 3 * 255 * 256 / 2
    assert oracle.global_reduce(u8, "max") == 255


def test_global_reduce_matches_numpy_and_is_exact():
    """min / max agree with np.min / np.max; the f32 sum is the exact sum
    (fractions.Fraction) correctly rounded to double."""
    from fractions import Fraction
    rng = _rng(31)
    img = rng.random((29, 31)).astype(np.float32)
    assert oracle.global_reduce(img, "min") == float(img.min())
    assert oracle.global_reduce(img, "max") == float(img.max())
    exact = sum(Fraction(float(v)) for v in img.ravel())
    assert oracle.global_reduce(img, "sum") == float(exact)

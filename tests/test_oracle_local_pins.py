"""Pins for oracle.local -- the local operator over several Accessors with a
per-tap function (Listing 9;
DESIGN.md reading c22).  Run with -m "not gpu".

Every check compares against something other than the oracle itself:
scipy.ndimage (correlate, minimum/maximum_filter) on the same boundary modes,
numpy's sliding windows over np.pad-expanded images, and closed forms
(Sum M (v - c)^2 = corr(v^2) - 2 c corr(v) + c^2 Sum M), chosen so that a
swapped accessor, a wrong offset sign, a transposed mask or a dropped centre
term fails.
"""
import numpy as np
import pytest
import scipy.ndimage as ndi

import oracle

MODES = ["clamp", "repeat", "mirror", "constant"]
SCIPY_MODE = {"clamp": "nearest", "repeat": "wrap", "mirror": "reflect", "constant": "constant"}
NP_PAD = {"clamp": "edge", "repeat": "wrap", "mirror": "symmetric", "constant": "constant"}


def _img(h, w, seed):
    return np.random.default_rng(seed).random((h, w)).astype(np.float32)


def _embed(mask, ox, oy):
    """Mask M read at offset (ox, oy) == mask M' centred at 0 with M placed at (ox, oy)."""
    mh, mw = mask.shape
    n, m = mh // 2 + abs(oy), mw // 2 + abs(ox)
    out = np.zeros((2 * n + 1, 2 * m + 1))
    out[n + oy - mh // 2:n + oy + mh // 2 + 1, m + ox - mw // 2:m + ox + mw // 2 + 1] = mask
    return out


@pytest.mark.parametrize("mode", MODES)
def test_single_accessor_product_sum_is_correlation_with_offset(mode):
    img = _img(11, 14, 1)
    rng = np.random.default_rng(2)
    mask = rng.normal(size=(3, 5))
    for ox, oy in ((0, 0), (2, -1), (-3, 2)):
        got, _ = oracle.local([img], [mask], "sum", "product", mode, 0.375, offsets=[(ox, oy)])
        ref = ndi.correlate(img.astype(np.float64), _embed(mask, ox, oy),
                            mode=SCIPY_MODE[mode], cval=0.375)
        assert np.allclose(got, ref, rtol=0, atol=1e-12), (mode, ox, oy)


def test_two_accessors_linear_with_their_own_modes_and_sizes():
    a, b = _img(9, 12, 3), _img(9, 12, 4)
    ma = np.random.default_rng(5).normal(size=(5, 3))
    mb = np.random.default_rng(6).normal(size=(3, 7))
    got, _ = oracle.local([a, b], [ma, mb], "sum", "product", ["mirror", "constant"], [0.0, 0.8],
                          offsets=[(1, 0), (0, -2)])
    ref = (ndi.correlate(a.astype(np.float64), _embed(ma, 1, 0), mode="reflect") +
           ndi.correlate(b.astype(np.float64), _embed(mb, 0, -2), mode="constant", cval=0.8))
    assert np.allclose(got, ref, rtol=0, atol=1e-12)
    # swapping the accessors' masks changes the result (no symmetric mix-up)
    swapped, _ = oracle.local([a, b], [mb, ma], "sum", "product", ["mirror", "constant"],
                              [0.0, 0.8], offsets=[(1, 0), (0, -2)])
    assert not np.allclose(swapped, ref)


@pytest.mark.parametrize("mode", MODES)
def test_sqdiff_square_closed_forms(mode):
    img = _img(10, 13, 7).astype(np.float64)
    mask = np.random.default_rng(8).random((5, 5))
    c1 = ndi.correlate(img, mask, mode=SCIPY_MODE[mode], cval=0.25)
    c2 = ndi.correlate(img * img, mask, mode=SCIPY_MODE[mode], cval=0.25 ** 2)   # v^2 of C is C^2
    got, _ = oracle.local([img.astype(np.float32)], [mask], "sum", "sqdiff", mode, 0.25)
    # sum M (v - c)^2 = corr(v^2) - 2 c corr(v) + c^2 sum(M), c = the pixel itself
    assert np.allclose(got, c2 - 2 * img * c1 + img * img * mask.sum(), rtol=0, atol=1e-12)
    sq, _ = oracle.local([img.astype(np.float32)], [mask], "sum", "square", mode, 0.25)
    assert np.allclose(sq, c2, rtol=0, atol=1e-12)


@pytest.mark.parametrize("mode", MODES)
def test_absdiff_max_is_local_contrast(mode):
    img = _img(12, 9, 9).astype(np.float64)
    fp = np.ones((3, 5))
    kw = dict(footprint=fp, mode=SCIPY_MODE[mode], cval=0.5)
    ref = np.maximum(ndi.maximum_filter(img, **kw) - img, img - ndi.minimum_filter(img, **kw))
    got, _ = oracle.local([img.astype(np.float32)], [fp], "max", "absdiff", mode, 0.5)
    assert np.allclose(got, ref, rtol=0, atol=1e-15)


@pytest.mark.parametrize("op", ["min", "max"])
@pytest.mark.parametrize("fn", ["product", "absdiff", "sqdiff", "square"])
def test_min_max_brute_force_sliding_windows(op, fn):
    """Every (op, fn) against numpy sliding windows over np.pad-expanded
    images of two accessors with holes in their domains."""
    a, b = _img(8, 10, 10), _img(8, 10, 11)
    rng = np.random.default_rng(12)
    ma = rng.random((3, 3)) + 0.1
    ma[0, 1] = 0.0                                   # a hole: excluded from MIN / MAX
    mb = rng.random((5, 3)) + 0.1
    mb[2, 0] = 0.0
    got, _ = oracle.local([a, b], [ma, mb], op, fn, ["clamp", "repeat"])
    vals = []
    for im, m, md in ((a, ma, "clamp"), (b, mb, "repeat")):
        n, mm = m.shape[0] // 2, m.shape[1] // 2
        pad = np.pad(im.astype(np.float64), ((n, n), (mm, mm)), mode=NP_PAD[md])
        win = np.lib.stride_tricks.sliding_window_view(pad, m.shape)      # (H, W, mh, mw)
        c = im.astype(np.float64)[:, :, None, None]
        f = {"product": m * win, "absdiff": m * np.abs(win - c), "sqdiff": m * (win - c) * (win - c),
             "square": m * win * win}[fn]
        f = np.where(m != 0, f, np.inf if op == "min" else -np.inf)
        vals.append(f.reshape(im.shape + (-1,)))
    allv = np.concatenate(vals, axis=-1)
    ref = allv.min(-1) if op == "min" else allv.max(-1)
    assert np.array_equal(got, ref)


def test_u8_exact_integer_forms():
    rng = np.random.default_rng(13)
    a = rng.integers(0, 256, (9, 11)).astype(np.uint8)
    b = rng.integers(0, 256, (9, 11)).astype(np.uint8)
    ma = rng.integers(-3, 4, (3, 3)).astype(np.int32)
    mb = rng.integers(0, 5, (5, 5)).astype(np.int32)
    got, _ = oracle.local([a, b], [ma, mb], "sum", "product", ["clamp", "constant"], [0, 200])
    ref = (ndi.correlate(a.astype(np.int64), ma.astype(np.int64), mode="nearest") +
           ndi.correlate(b.astype(np.int64), mb.astype(np.int64), mode="constant", cval=200))
    assert got.dtype == np.int64 and np.array_equal(got, ref)
    sq, _ = oracle.local([a], [mb], "sum", "sqdiff", "mirror")
    A = a.astype(np.int64)
    ref2 = (ndi.correlate(A * A, mb.astype(np.int64), mode="reflect")
            - 2 * A * ndi.correlate(A, mb.astype(np.int64), mode="reflect") + A * A * mb.sum())
    assert np.array_equal(sq, ref2)


def test_undefined_valid_region_is_the_largest_window():
    a, b = _img(12, 12, 14), _img(12, 12, 15)
    # accessor a: 3x3 at offset (2, 0) -> needs x + 2 +- 1 in range; b: 7x5 -> x +- 2, y +- 3
    _, valid = oracle.local([a, b], [np.ones((3, 3)), np.ones((7, 5))], "sum", "product",
                            "undefined", offsets=[(2, 0), (0, 0)])
    ys, xs = np.mgrid[0:12, 0:12]
    ok = (xs + 1 >= 0) & (xs + 3 <= 11) & (ys - 1 >= 0) & (ys + 1 <= 11)
    ok &= (xs - 2 >= 0) & (xs + 2 <= 11) & (ys - 3 >= 0) & (ys + 3 <= 11)
    assert np.array_equal(valid, ok)


# ---------------------------------------- point-operator prologue (reading c27) ----

@pytest.mark.parametrize("mode", MODES)
def test_point_prologue_is_the_local_operator_of_the_mapped_image(mode):
    """Read'_k = a Read_k + b: the result equals the
    operator applied to the explicitly mapped image a I + b with the
    constant mapped too (a boundary constant is a pixel value), for every
    op / tap function -- checked against scipy on the mapped image."""
    img = _img(9, 13, 21).astype(np.float64)
    a, b = 2.5, -0.75
    mask = np.random.default_rng(22).random((3, 5))
    got, _ = oracle.local([img.astype(np.float32)], [mask], "sum", "product", mode, 0.2,
                          point=[(a, b)])
    f32 = img.astype(np.float32).astype(np.float64)
    ref = ndi.correlate(a * f32 + b, mask, mode=SCIPY_MODE[mode], cval=a * 0.2 + b)
    assert np.allclose(got, ref, rtol=0, atol=1e-12)
    # SQDIFF about the mapped centre: a^2 times the unmapped result (b cancels)
    g1, _ = oracle.local([img.astype(np.float32)], [mask], "sum", "sqdiff", mode, 0.2,
                         point=[(a, b)])
    g0, _ = oracle.local([img.astype(np.float32)], [mask], "sum", "sqdiff", mode, 0.2)
    assert np.allclose(g1, a * a * g0, rtol=1e-13, atol=1e-13)


def test_point_prologue_u8_integer_and_per_accessor():
    rng = np.random.default_rng(23)
    u = rng.integers(0, 256, (10, 12)).astype(np.uint8)
    v = rng.integers(0, 256, (10, 12)).astype(np.uint8)
    m = np.ones((3, 3), np.int32)
    got, _ = oracle.local([u, v], [m, m], "sum", "product", "clamp", point=[(-1, 255), (3, 0)])
    ref = (ndi.correlate(255 - u.astype(np.int64), m.astype(np.int64), mode="nearest")
           + ndi.correlate(3 * v.astype(np.int64), m.astype(np.int64), mode="nearest"))
    assert np.array_equal(got, ref)


# ------------------------------------ global merge: sum of squares (reading c26) ----

def test_global_sumsq_exact():
    """sum of squares: the exact sum (fractions.Fraction) of v^2 correctly
    rounded; a constant image v gives v^2 N; u8 an exact integer; a ramp the
    closed form sum_{k<n} k^2 = (n-1) n (2n-1) / 6."""
    from fractions import Fraction
    img = np.random.default_rng(24).random((17, 19)).astype(np.float32)
    exact = sum(Fraction(float(x)) ** 2 for x in img.ravel())
    assert oracle.global_reduce(img, "sumsq") == float(exact)
    assert oracle.global_reduce(np.full((7, 9), 0.5, np.float32), "sumsq") == 0.25 * 63
    n = 2000
    ramp = np.arange(n, dtype=np.float32).reshape(40, 50)
    assert oracle.global_reduce(ramp, "sumsq") == (n - 1) * n * (2 * n - 1) / 6
    u8 = (np.arange(512) % 256).astype(np.uint8).reshape(2, 16, 16)
    assert oracle.global_reduce(u8, "sumsq") == 2 * 255 * 256 * 511 / 6

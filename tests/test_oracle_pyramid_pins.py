"""Pins of the multiresolution-filter oracle (PAPER.md
L309-L314 and ref [7]; reading c28 in DESIGN.md) against things other than
itself:
  * REDUCE  == scipy.ndimage.correlate with the 5x5 binomial, then every
               second sample (a library routine; all four modes),
  * EXPAND  == an independent numpy formulation: np.pad of the coarse level
               (the mode's per-axis extension), zero insertion, a 5-tap
               correlation with 2 w per axis,
  * the Laplacian pyramid reconstructs its input exactly (up to rounding)
    when no level is filtered -- a plausible slip in REDUCE / EXPAND / the
    band-pass subtraction (a wrong phase, a dropped factor 4, a transposed
    level) breaks it only if the two disagree, so the first two pins guard
    each operator on its own,
  * a constant image stays constant through the whole filter,
  * one level is the bilateral filter itself (oracle.bilateral_f32, pinned in
    test_oracle_pins.py),
  * EXPAND of a linear ramp is the ramp at half rate in the interior, REDUCE
    of a ramp the ramp at double rate (closed forms).
"""
import numpy as np
import pytest
import scipy.ndimage as ndi

import oracle

MODES = ["clamp", "repeat", "mirror", "constant"]
SCIPY_MODE = {"clamp": "nearest", "repeat": "wrap", "mirror": "reflect", "constant": "constant"}
NP_PAD = {"clamp": "edge", "repeat": "wrap", "mirror": "symmetric", "constant": "constant"}
W5 = np.array([1, 4, 6, 4, 1], np.float64) / 16.0


def _img(h, w, seed):
    return np.random.default_rng(seed).random((h, w))


@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("shape", [(1, 1), (2, 3), (5, 7), (16, 9), (33, 40)])
def test_reduce_is_binomial_correlation_decimated(mode, shape):
    g = _img(*shape, seed=shape[0] * 100 + shape[1])
    got = oracle.pyr_reduce(g, mode, cval=0.3)
    ref = ndi.correlate(g, np.outer(W5, W5), mode=SCIPY_MODE[mode], cval=0.3)[::2, ::2]
    assert got.shape == ((shape[0] + 1) // 2, (shape[1] + 1) // 2)
    assert np.allclose(got, ref, rtol=0, atol=1e-14)


def _expand_numpy(gc, shape, mode, cval):
    """Zero-insertion formulation: U(t) = Gc(t/2) for even t (Gc extended by
    np.pad), E(x) = sum_i 2 w(i) U(x - i) per axis (separable)."""
    H, W = shape
    P = 3
    gp = np.pad(gc, P, mode=NP_PAD[mode], **({"constant_values": cval} if mode == "constant" else {}))
    # U on t in [-2P, 2(n+P)) (index t + 2P), zero at odd t
    U = np.zeros((2 * gp.shape[0], 2 * gp.shape[1]))
    U[::2, ::2] = gp
    k = 2 * W5
    E = np.zeros((H, W))
    for j in range(-2, 3):
        for i in range(-2, 3):
            ys = np.arange(H) - j + 2 * P
            xs = np.arange(W) - i + 2 * P
            E += k[i + 2] * k[j + 2] * U[np.ix_(ys, xs)]
    return E


@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("shape", [(1, 1), (2, 2), (3, 5), (8, 13), (31, 24)])
def test_expand_is_zero_insertion_upsampling(mode, shape):
    H, W = shape
    gc = _img((H + 1) // 2, (W + 1) // 2, seed=H * 7 + W)
    got = oracle.pyr_expand(gc, shape, mode, cval=0.6)
    ref = _expand_numpy(gc, shape, mode, 0.6)
    assert np.allclose(got, ref, rtol=0, atol=1e-14)


def test_reduce_expand_ramps_closed_form():
    y, x = np.mgrid[0:40, 0:48].astype(np.float64)
    ramp = 0.5 * x - 0.25 * y + 3.0
    r = oracle.pyr_reduce(ramp, "clamp")
    yy, xx = np.mgrid[0:20, 0:24].astype(np.float64)
    inner = (slice(1, -1), slice(1, -1))
    assert np.allclose(r[inner], (0.5 * 2 * xx - 0.25 * 2 * yy + 3.0)[inner], atol=1e-12)
    c = 0.5 * xx - 0.25 * yy + 3.0
    e = oracle.pyr_expand(c, (40, 48), "clamp")
    assert np.allclose(e[2:-2, 2:-2], (0.5 * x / 2 - 0.25 * y / 2 + 3.0)[2:-2, 2:-2], atol=1e-12)


@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("shape,levels", [((37, 53), 3), ((64, 64), 4), ((9, 17), 5)])
def test_perfect_reconstruction(mode, shape, levels):
    img = _img(*shape, seed=levels)
    out = oracle.multires_bilateral(img, levels, 1.0, [0.0] * levels, mode, cval=0.2)
    assert np.allclose(out, img, rtol=0, atol=1e-13)


@pytest.mark.parametrize("mode", MODES)
def test_constant_image(mode):
    img = np.full((23, 30), 0.625)
    out = oracle.multires_bilateral(img, 3, 1.0, [0.1, 0.2, 0.3], mode, cval=0.625)
    assert np.array_equal(out, img)


@pytest.mark.parametrize("mode", ["clamp", "mirror"])
def test_one_level_is_the_bilateral_filter(mode):
    img = _img(20, 27, seed=5).astype(np.float32)
    a = oracle.multires_bilateral(img, 1, 1.0, [0.1], mode)
    b, _ = oracle.bilateral_f32(img, 1.0, 0.1, mode)
    assert np.allclose(a, b, rtol=0, atol=1e-14)


def test_filtering_a_band_changes_only_through_that_band():
    """Filtering level 1 alone: out - in == EXPAND(F_1 - B_1) (the change of the
    band propagates through one EXPAND, linear in the band)."""
    img = _img(32, 32, seed=9)
    out = oracle.multires_bilateral(img, 3, 1.0, [0.0, 0.05, 0.0], "mirror")
    g1 = oracle.pyr_reduce(img, "mirror")
    g2 = oracle.pyr_reduce(g1, "mirror")
    b1 = g1 - oracle.pyr_expand(g2, g1.shape, "mirror")
    f1 = oracle.bilateral_f64(b1, 1.0, 0.05, "mirror", 0.0)
    assert np.allclose(out - img, oracle.pyr_expand(f1 - b1, img.shape, "mirror"), atol=1e-13)

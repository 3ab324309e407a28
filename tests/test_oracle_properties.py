"""Property-based pins of the oracle (hypothesis): random shapes, odd windows,
modes, constants and masks against library routines and invariants.
Complements tests/test_oracle_pins.py (CPU only)."""
import numpy as np
import scipy.ndimage as ndi
from hypothesis import given, settings, strategies as st

import oracle

SCIPY_MODE = {"clamp": "nearest", "repeat": "wrap", "mirror": "reflect", "constant": "constant"}
modes = st.sampled_from(["clamp", "repeat", "mirror", "constant"])
odd = st.sampled_from([1, 3, 5, 7, 9])


@settings(max_examples=60, deadline=None)
@given(h=st.integers(1, 12), w=st.integers(1, 12), mx=odd, my=odd, mode=modes,
       cval=st.floats(-2, 2, allow_nan=False), seed=st.integers(0, 2**31))
def test_convolve_matches_scipy(h, w, mx, my, mode, cval, seed):
    rng = np.random.default_rng(seed)
    img = rng.random((h, w)).astype(np.float32)
    mask = rng.standard_normal((my, mx))
    out, valid = oracle.convolve_f32(img, mask, mode, cval)
    ref = ndi.correlate(img.astype(np.float64), mask, mode=SCIPY_MODE[mode], cval=cval)
    assert valid.all()
    np.testing.assert_allclose(out, ref, rtol=0, atol=1e-12)


@settings(max_examples=60, deadline=None)
@given(h=st.integers(1, 10), w=st.integers(1, 10), mx=odd, my=odd, mode=modes,
       cval=st.integers(0, 255), shift=st.integers(0, 9), seed=st.integers(0, 2**31))
def test_convolve_u8_matches_integer_correlate(h, w, mx, my, mode, cval, shift, seed):
    rng = np.random.default_rng(seed)
    img = rng.integers(0, 256, (h, w)).astype(np.uint8)
    mask = rng.integers(-20, 21, (my, mx)).astype(np.int32)
    S = ndi.correlate(img.astype(np.int64), mask.astype(np.int64), mode=SCIPY_MODE[mode],
                      cval=cval)
    q8, _ = oracle.convolve_u8(img, mask, shift, mode, cval=cval, out_dtype=np.uint8)
    q32, _ = oracle.convolve_u8(img, mask, shift, mode, cval=cval, out_dtype=np.int32)
    rnd = (1 << (shift - 1)) if shift else 0
    ref = (S + rnd) // (1 << shift)
    assert (q32 == ref).all()
    assert (q8 == np.clip(ref, 0, 255)).all()


@settings(max_examples=40, deadline=None)
@given(h=st.integers(1, 9), w=st.integers(1, 9), size=st.sampled_from([1, 3, 5, 7]),
       sigma_d=st.floats(0.3, 4), mode=modes, seed=st.integers(0, 2**31))
def test_bilateral_large_sigma_r_is_normalised_closeness_correlation(h, w, size, sigma_d, mode,
                                                                      seed):
    rng = np.random.default_rng(seed)
    img = rng.random((h, w)).astype(np.float32)
    out, _ = oracle.bilateral_f32(img, sigma_d, 1e7, mode, cval=0.4, size=size)
    c = oracle.closeness_mask(sigma_d, size)
    ref = ndi.correlate(img.astype(np.float64), c / c.sum(), mode=SCIPY_MODE[mode], cval=0.4)
    np.testing.assert_allclose(out, ref, rtol=0, atol=1e-9)


@settings(max_examples=40, deadline=None)
@given(h=st.integers(2, 9), w=st.integers(2, 9), size=st.sampled_from([3, 5]),
       sigma_r=st.floats(0.01, 1.0), mode=modes, seed=st.integers(0, 2**31))
def test_bilateral_is_a_convex_combination(h, w, size, sigma_r, mode, seed):
    rng = np.random.default_rng(seed)
    img = rng.random((h, w)).astype(np.float32)
    out, _ = oracle.bilateral_f32(img, 1.0, sigma_r, mode, cval=0.6, size=size)
    lo = ndi.minimum_filter(img.astype(np.float64), size=size, mode=SCIPY_MODE[mode], cval=0.6)
    hi = ndi.maximum_filter(img.astype(np.float64), size=size, mode=SCIPY_MODE[mode], cval=0.6)
    assert (out >= lo - 1e-15).all() and (out <= hi + 1e-15).all()


@settings(max_examples=100, deadline=None)
@given(n=st.integers(1, 20), i=st.integers(-70, 70))
def test_index_maps_stay_in_range_and_are_periodic(n, i):
    for mode, period in (("repeat", n), ("mirror", 2 * n)):
        m = oracle.map_index(i, n, mode)
        assert 0 <= m < n
        assert oracle.map_index(i + period, n, mode) == m
    assert oracle.map_index(i, n, "mirror") == oracle.map_index(-1 - i, n, "mirror")
    c = oracle.map_index(i, n, "clamp")
    assert c == min(max(i, 0), n - 1)

"""CPU oracle for the HIPAcc local operators (Membarth et al., IPDPS 2012).

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this
package.  The product package ``paper_conf_ipps_membarthhtke12_b200`` never
imports it and shares no code with it (see ``oracle/lop_oracle.c`` header).

This module is argument marshalling only: it compiles ``lop_oracle.c`` with
gcc (-O2, no -ffast-math, OpenMP over output rows) into ``liblop_oracle.so``
next to this file and wraps each entry point for numpy arrays.  All arithmetic
lives in the C file, in double precision, in the order of Algorithm 1
(PAPER.md L169-L186).

Parity status (details in DESIGN.md "Oracle pins"):
  map_index, read               pinned: Fig. 2 golden cells, np.pad
  closeness_mask                pinned: Listing 4 printed value 0.018316,
                                        Listing 1 l.21 product form
  gaussian_mask / sobel_mask    pinned: binomial coefficients (scipy.special),
                                        ramp responses
  convolve_f32 / convolve_u8    pinned: scipy.ndimage.correlate (all modes),
                                        impulse response, ramps, separability
  quantize                      pinned: hand-computed cases, numpy floor-div
  bilateral_f32                 pinned: sigma_r->inf == scipy Gaussian
                                        correlate, hand-computed 3x3 examples,
                                        step-edge preservation, constant image,
                                        convexity, flip symmetry
  pyr_reduce / pyr_expand       pinned: scipy correlate + decimation; np.pad +
                                        zero insertion (tests/test_oracle_pyramid_pins.py)
  multires_bilateral            pinned: perfect reconstruction, constant image,
                                        one level == bilateral_f32
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "lop_oracle.c")
_LIB = os.path.join(_HERE, "liblop_oracle.so")
_lock = threading.Lock()
_lib = None

UNDEFINED, CLAMP, REPEAT, MIRROR, CONSTANT = 0, 1, 2, 3, 4
MODES = {"undefined": UNDEFINED, "clamp": CLAMP, "repeat": REPEAT,
         "mirror": MIRROR, "constant": CONSTANT}


def build(force: bool = False) -> str:
    """Compile the oracle (plain C, gcc -O2 -fopenmp, no fast-math)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + ".tmp%d" % os.getpid()
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-fopenmp",
                               "-Wall", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    with _lock:
        if _lib is None:
            lib = ctypes.CDLL(build())
            i64, i32, dbl, vp = ctypes.c_int64, ctypes.c_int, ctypes.c_double, ctypes.c_void_p
            lib.oracle_num_threads.restype = i32
            lib.oracle_map_index.argtypes = [i64, i64, i32]
            lib.oracle_map_index.restype = i64
            lib.oracle_read_f32.argtypes = [vp, i64, i64, i64, i64, i64, i32, dbl, vp]
            lib.oracle_read_f32.restype = dbl
            lib.oracle_closeness_mask.argtypes = [dbl, i32, i32, vp]
            lib.oracle_gaussian_mask_int.argtypes = [i32, vp]
            lib.oracle_gaussian_mask_int.restype = i32
            lib.oracle_sobel_mask_int.argtypes = [i32, vp]
            lib.oracle_convolve_f32.argtypes = [vp, i64, i64, i64, vp, i32, i32, i32, dbl,
                                                i64, i64, vp, vp]
            lib.oracle_convolve_f32_points.argtypes = [vp, i64, i64, i64, vp, i32, i32, i32,
                                                       dbl, vp, vp, i64, vp, vp]
            lib.oracle_convolve_u8_sum.argtypes = [vp, i64, i64, i64, vp, i32, i32, i32, i64,
                                                   i64, i64, vp, vp]
            lib.oracle_convolve_u8_sum_points.argtypes = [vp, i64, i64, i64, vp, i32, i32, i32,
                                                          i64, vp, vp, i64, vp, vp]
            lib.oracle_reduce_f32.argtypes = [vp, i64, i64, i64, vp, i32, i32, i32, i32, dbl,
                                              i64, i64, vp, vp]
            lib.oracle_reduce_u8.argtypes = [vp, i64, i64, i64, vp, i32, i32, i32, i32, i64,
                                             i64, i64, vp, vp]
            lib.oracle_quantize.argtypes = [i64, i32, i32]
            lib.oracle_quantize.restype = i64
            lib.oracle_bilateral_f32.argtypes = [vp, i64, i64, i64, vp, i32, i32, dbl, dbl,
                                                 i32, dbl, i64, i64, vp, vp]
            lib.oracle_bilateral_f32_points.argtypes = [vp, i64, i64, i64, vp, i32, i32, dbl,
                                                        dbl, i32, dbl, vp, vp, i64, vp, vp]
            pa = ctypes.POINTER(ctypes.c_void_p)
            lib.oracle_local_f32.argtypes = [i32, pa, vp, i64, i64, pa, vp, vp, vp, vp, vp, vp,
                                             vp, vp, i32, i32, i64, i64, vp, vp]
            lib.oracle_local_u8.argtypes = [i32, pa, vp, i64, i64, pa, vp, vp, vp, vp, vp, vp,
                                            vp, vp, i32, i32, i64, i64, vp, vp]
            lib.oracle_pyr_reduce_f64.argtypes = [vp, i64, i64, i32, dbl, vp]
            lib.oracle_pyr_expand_f64.argtypes = [vp, i64, i64, i64, i64, i32, dbl, vp]
            lib.oracle_bilateral_f64.argtypes = [vp, i64, i64, i32, i32, dbl, dbl, i32, dbl, vp]
            _lib = lib
    return _lib


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def _mode(mode) -> int:
    return MODES[mode] if isinstance(mode, str) else int(mode)


def _img(img: np.ndarray, dtype):
    img = np.asarray(img)
    if img.dtype != dtype:
        raise TypeError("oracle expects %s image, got %s" % (dtype, img.dtype))
    if img.ndim != 2:
        raise ValueError("oracle expects a 2D image")
    if img.strides[1] != img.itemsize or img.strides[0] % img.itemsize:
        img = np.ascontiguousarray(img)
    return img, img.strides[0] // img.itemsize


def num_threads() -> int:
    return _load().oracle_num_threads()


def map_index(i: int, n: int, mode) -> int:
    """Per-axis index adjustment (Fig. 2); -1 = no pixel."""
    return _load().oracle_map_index(int(i), int(n), _mode(mode))


def read(img: np.ndarray, x: int, y: int, mode, cval: float = 0.0):
    """Read(x, y) of the virtually expanded image; returns (value, undefined)."""
    img, stride = _img(img, np.float32)
    und = ctypes.c_int(0)
    v = _load().oracle_read_f32(_ptr(img), img.shape[1], img.shape[0], stride, int(x), int(y),
                                _mode(mode), float(cval), ctypes.byref(und))
    return v, bool(und.value)


def closeness_mask(sigma_d: float, size_x: int, size_y: int | None = None) -> np.ndarray:
    """Eq. (1) closeness mask, row-major (yf outer), float64."""
    size_y = size_x if size_y is None else size_y
    out = np.empty((size_y, size_x), np.float64)
    _load().oracle_closeness_mask(float(sigma_d), size_x, size_y, _ptr(out))
    return out


def gaussian_mask(size: int):
    """Binomial Gaussian mask (int32, size x size) and its shift k (sum = 2^k)."""
    out = np.empty((size, size), np.int32)
    k = _load().oracle_gaussian_mask_int(size, _ptr(out))
    if k < 0:
        raise ValueError("bad Gaussian size %d" % size)
    return out, k


def sobel_mask(direction: int) -> np.ndarray:
    out = np.empty((3, 3), np.int32)
    _load().oracle_sobel_mask_int(int(direction), _ptr(out))
    return out


def convolve_f32(img, mask, mode, cval=0.0, rows=None):
    """Correlation of a float32 image with a float64 mask; returns (out f64, valid)."""
    img, stride = _img(img, np.float32)
    mask = np.ascontiguousarray(mask, np.float64)
    H, W = img.shape
    y0, y1 = (0, H) if rows is None else rows
    out = np.empty((y1 - y0, W), np.float64)
    valid = np.empty((y1 - y0, W), np.uint8)
    _load().oracle_convolve_f32(_ptr(img), W, H, stride, _ptr(mask), mask.shape[1],
                                mask.shape[0], _mode(mode), float(cval), y0, y1,
                                _ptr(out), _ptr(valid))
    return out, valid.astype(bool)


def convolve_f32_points(img, mask, mode, xs, ys, cval=0.0):
    img, stride = _img(img, np.float32)
    mask = np.ascontiguousarray(mask, np.float64)
    xs = np.ascontiguousarray(xs, np.int64)
    ys = np.ascontiguousarray(ys, np.int64)
    out = np.empty(len(xs), np.float64)
    valid = np.empty(len(xs), np.uint8)
    _load().oracle_convolve_f32_points(_ptr(img), img.shape[1], img.shape[0], stride,
                                       _ptr(mask), mask.shape[1], mask.shape[0], _mode(mode),
                                       float(cval), _ptr(xs), _ptr(ys), len(xs), _ptr(out),
                                       _ptr(valid))
    return out, valid.astype(bool)


def convolve_u8_sum(img, mask, mode, cval=0, rows=None):
    """Exact integer sums S of an uint8 image with an int32 mask; (S int64, valid)."""
    img, stride = _img(img, np.uint8)
    mask = np.ascontiguousarray(mask, np.int32)
    H, W = img.shape
    y0, y1 = (0, H) if rows is None else rows
    out = np.empty((y1 - y0, W), np.int64)
    valid = np.empty((y1 - y0, W), np.uint8)
    _load().oracle_convolve_u8_sum(_ptr(img), W, H, stride, _ptr(mask), mask.shape[1],
                                   mask.shape[0], _mode(mode), int(cval), y0, y1,
                                   _ptr(out), _ptr(valid))
    return out, valid.astype(bool)


def convolve_u8_sum_points(img, mask, mode, xs, ys, cval=0):
    img, stride = _img(img, np.uint8)
    mask = np.ascontiguousarray(mask, np.int32)
    xs = np.ascontiguousarray(xs, np.int64)
    ys = np.ascontiguousarray(ys, np.int64)
    out = np.empty(len(xs), np.int64)
    valid = np.empty(len(xs), np.uint8)
    _load().oracle_convolve_u8_sum_points(_ptr(img), img.shape[1], img.shape[0], stride,
                                          _ptr(mask), mask.shape[1], mask.shape[0],
                                          _mode(mode), int(cval), _ptr(xs), _ptr(ys), len(xs),
                                          _ptr(out), _ptr(valid))
    return out, valid.astype(bool)


def convolve2(img, mask_a, mask_b, combine, mode, cval=0.0, rows=None):
    """Two local operators on one input combined by a point operator
    (PAPER.md L107-L122): A, B = the oracle convolutions
    above (exact double / integer sums), then, in double (f32 images) or
    exact integers (u8 images):  "l2" sqrt(A^2 + B^2), "l1" |A| + |B|,
    "sumsq" A^2 + B^2.  Returns (out, valid)."""
    if np.asarray(img).dtype == np.uint8:
        A, va = convolve_u8_sum(img, mask_a, mode, int(cval), rows)
        B, vb = convolve_u8_sum(img, mask_b, mode, int(cval), rows)
    else:
        A, va = convolve_f32(img, mask_a, mode, cval, rows)
        B, vb = convolve_f32(img, mask_b, mode, cval, rows)
    if combine == "l2":
        out = np.sqrt(A.astype(np.float64) ** 2 + B.astype(np.float64) ** 2)
    elif combine == "l1":
        out = np.abs(A) + np.abs(B)
    elif combine == "sumsq":
        out = A * A + B * B
    else:
        raise ValueError(combine)
    return out, va & vb


def global_reduce(img, op, roi=None):
    """Global operator: one value for all pixels of the
    region (x0, y0, w, h) of a 2D image or a (B, H, W) stack.  "sum" is the
    correctly rounded exact sum (math.fsum over the float values; exact integer
    for u8), "min" / "max" the extreme pixel value, "sumsq" the correctly
    rounded exact sum of squares (the square of an f32 value is exact in
    double) -- a merge of two pixels a, b -> a^2 + b^2 summed over the image
    ("operations that merge/reduce two pixels"; reading c26)."""
    import math
    a = np.asarray(img)
    if a.ndim == 2:
        a = a[None]
    if roi is not None:
        x0, y0, w, h = roi
        a = a[:, y0:y0 + h, x0:x0 + w]
    if op == "sum":
        if a.dtype == np.uint8:
            return float(int(a.astype(np.int64).sum()))
        return math.fsum(float(v) for v in a.ravel())
    if op == "sumsq":
        if a.dtype == np.uint8:
            return float(int((a.astype(np.int64) ** 2).sum()))
        return math.fsum(float(v) * float(v) for v in a.ravel())
    if op == "min":
        return float(min(a.ravel().tolist()))
    if op == "max":
        return float(max(a.ravel().tolist()))
    raise ValueError(op)


_REDUCE_OPS = {"min": 1, "max": 2}


def reduce(img, domain, op, mode, cval=0.0, rows=None):
    """Listing 9's convolve(mask, op, ...) with op "min" / "max" over the taps
    where ``domain`` is non-zero.  float32 image -> (out f64, valid);
    uint8 image -> (out int64, valid)."""
    u8 = np.asarray(img).dtype == np.uint8
    img, stride = _img(img, np.uint8 if u8 else np.float32)
    dom = np.ascontiguousarray(np.asarray(domain) != 0, np.int32)
    H, W = img.shape
    y0, y1 = (0, H) if rows is None else rows
    out = np.empty((y1 - y0, W), np.int64 if u8 else np.float64)
    valid = np.empty((y1 - y0, W), np.uint8)
    fn = _load().oracle_reduce_u8 if u8 else _load().oracle_reduce_f32
    fn(_ptr(img), W, H, stride, _ptr(dom), dom.shape[1], dom.shape[0], _REDUCE_OPS[op],
       _mode(mode), int(cval) if u8 else float(cval), y0, y1, _ptr(out), _ptr(valid))
    return out, valid.astype(bool)


def quantize(S, shift: int, to_u8: bool):
    """(S + 2^(k-1)) >> k, saturated to [0,255] for u8 outputs (reading c12)."""
    lib = _load()
    f = np.vectorize(lambda s: lib.oracle_quantize(int(s), int(shift), int(bool(to_u8))),
                     otypes=[np.int64])
    return f(np.asarray(S, np.int64))


def convolve_u8(img, mask, shift, mode, cval=0, out_dtype=np.uint8, rows=None):
    """Full integer local operator: sums, then quantisation to u8 or i32."""
    S, valid = convolve_u8_sum(img, mask, mode, cval, rows)
    q = quantize(S, shift, out_dtype == np.uint8)
    return q.astype(out_dtype), valid


def bilateral_f32(img, sigma_d, sigma_r, mode, cval=0.0, size=None, cmask=None, rows=None):
    """Bilateral filter (Alg. 1) of a float32 image; returns (out f64, valid).

    ``cmask`` None -> closeness from Eq. (1) per tap with window ``size``
    (default 2*round(2*sigma_d)+1 = 4*sigma_d+1 for integer sigma_d,
    PAPER.md L325 / Listing 3; odd for every sigma_d, reading c1); else the given mask
    (Listing 5: c = CMask(xf, yf)).
    """
    img, stride = _img(img, np.float32)
    H, W = img.shape
    if cmask is not None:
        cmask = np.ascontiguousarray(cmask, np.float64)
        mh, mw = cmask.shape
        cptr = _ptr(cmask)
    else:
        if size is None:
            size = 2 * int(round(2 * sigma_d)) + 1     # 4*sigma_d+1, always odd (reading c1)
        mw, mh = (size, size) if isinstance(size, int) else size
        cptr = None
    y0, y1 = (0, H) if rows is None else rows
    out = np.empty((y1 - y0, W), np.float64)
    valid = np.empty((y1 - y0, W), np.uint8)
    _load().oracle_bilateral_f32(_ptr(img), W, H, stride, cptr, mw, mh, float(sigma_d),
                                 float(sigma_r), _mode(mode), float(cval), y0, y1,
                                 _ptr(out), _ptr(valid))
    return out, valid.astype(bool)


def bilateral_f32_points(img, sigma_d, sigma_r, mode, xs, ys, cval=0.0, size=None, cmask=None):
    img, stride = _img(img, np.float32)
    if cmask is not None:
        cmask = np.ascontiguousarray(cmask, np.float64)
        mh, mw = cmask.shape
        cptr = _ptr(cmask)
    else:
        if size is None:
            size = 2 * int(round(2 * sigma_d)) + 1     # 4*sigma_d+1, always odd (reading c1)
        mw, mh = (size, size) if isinstance(size, int) else size
        cptr = None
    xs = np.ascontiguousarray(xs, np.int64)
    ys = np.ascontiguousarray(ys, np.int64)
    out = np.empty(len(xs), np.float64)
    valid = np.empty(len(xs), np.uint8)
    _load().oracle_bilateral_f32_points(_ptr(img), img.shape[1], img.shape[0], stride, cptr,
                                        mw, mh, float(sigma_d), float(sigma_r), _mode(mode),
                                        float(cval), _ptr(xs), _ptr(ys), len(xs), _ptr(out),
                                        _ptr(valid))
    return out, valid.astype(bool)


LOCAL_OPS = {"sum": 0, "min": 1, "max": 2}
TAP_FNS = {"product": 0, "absdiff": 1, "sqdiff": 2, "square": 3}


def local(imgs, masks, op="sum", fn="product", modes="clamp", cvals=0.0, offsets=None,
          rows=None, point=None):
    """Local operator over K accessors (N2; Listing 9):
    out = op over k, taps of fn(M_k, Read_k(x+ox_k+xf, y+oy_k+yf), centre_k).
    imgs: K images of one shape and dtype (float32 -> double result, uint8 ->
    exact int64); masks: K 2D masks (odd sizes, float for f32, int for u8);
    modes / cvals / offsets: one per accessor (or a single value for all);
    point: per accessor (scale, offset) of a point-operator prologue
    Read'_k = scale * Read_k + offset applied to every read of accessor k
    (reading c27) -- None = identity."""
    K = len(imgs)
    assert K == len(masks) and K >= 1
    u8 = np.asarray(imgs[0]).dtype == np.uint8
    dt = np.uint8 if u8 else np.float32
    ims = [_img(im, dt) for im in imgs]
    H, W = ims[0][0].shape
    assert all(im.shape == (H, W) for im, _ in ims)
    mdt = np.int32 if u8 else np.float64
    ms = [np.ascontiguousarray(m, mdt) for m in masks]
    modes = [modes] * K if isinstance(modes, (str, int)) else list(modes)
    cvals = [cvals] * K if np.isscalar(cvals) else list(cvals)
    offsets = [(0, 0)] * K if offsets is None else list(offsets)
    img_ptrs = (ctypes.c_void_p * K)(*[im.ctypes.data for im, _ in ims])
    m_ptrs = (ctypes.c_void_p * K)(*[m.ctypes.data for m in ms])
    strides = np.array([s for _, s in ims], np.int64)
    mws = np.array([m.shape[1] for m in ms], np.int32)
    mhs = np.array([m.shape[0] for m in ms], np.int32)
    oxs = np.array([o[0] for o in offsets], np.int32)
    oys = np.array([o[1] for o in offsets], np.int32)
    mds = np.array([_mode(md) for md in modes], np.int32)
    point = [(1, 0)] * K if point is None else list(point)
    y0, y1 = (0, H) if rows is None else rows
    valid = np.empty((y1 - y0, W), np.uint8)
    if u8:
        cv = np.array([int(c) for c in cvals], np.int64)
        pa = np.array([int(a) for a, _ in point], np.int64)
        pb = np.array([int(b) for _, b in point], np.int64)
        out = np.empty((y1 - y0, W), np.int64)
        fnc = _load().oracle_local_u8
    else:
        cv = np.array([float(c) for c in cvals], np.float64)
        pa = np.array([float(a) for a, _ in point], np.float64)
        pb = np.array([float(b) for _, b in point], np.float64)
        out = np.empty((y1 - y0, W), np.float64)
        fnc = _load().oracle_local_f32
    fnc(K, ctypes.cast(img_ptrs, ctypes.POINTER(ctypes.c_void_p)), _ptr(strides), W, H,
        ctypes.cast(m_ptrs, ctypes.POINTER(ctypes.c_void_p)), _ptr(mws), _ptr(mhs), _ptr(oxs),
        _ptr(oys), _ptr(mds), _ptr(cv), _ptr(pa), _ptr(pb), LOCAL_OPS[op], TAP_FNS[fn], y0, y1,
        _ptr(out), _ptr(valid))
    return out, valid.astype(bool)


# ------------------------------------------------ multiresolution filter (N4) ----
# PAPER.md L309-L314 ("a multiresolution filter (see [7]) is applied to an
# image: the image gets upsampled multiple times", Mirror at the borders);
# reading c28: a Laplacian pyramid (REDUCE / EXPAND with the 5x5 binomial)
# whose band-pass levels are bilateral-filtered, then reconstructed.

PYRAMID_MODES = ("clamp", "repeat", "mirror", "constant")


def pyr_size(n: int) -> int:
    """Size of the next coarser level: ceil(n / 2)."""
    return (int(n) + 1) // 2


def pyr_reduce(img, mode="mirror", cval=0.0):
    """REDUCE (lop_oracle.c oracle_pyr_reduce_f64): the 5x5 binomial at every
    second pixel; double result of size ceil(H/2) x ceil(W/2)."""
    assert _mode(mode) != UNDEFINED
    g = np.ascontiguousarray(img, np.float64)
    H, W = g.shape
    out = np.empty((pyr_size(H), pyr_size(W)), np.float64)
    _load().oracle_pyr_reduce_f64(_ptr(g), W, H, _mode(mode), float(cval), _ptr(out))
    return out


def pyr_expand(coarse, shape, mode="mirror", cval=0.0):
    """EXPAND (oracle_pyr_expand_f64) of a coarse level to ``shape`` = (H, W),
    ceil(H/2) x ceil(W/2) = coarse.shape."""
    assert _mode(mode) != UNDEFINED
    g = np.ascontiguousarray(coarse, np.float64)
    H, W = shape
    assert g.shape == (pyr_size(H), pyr_size(W))
    out = np.empty((H, W), np.float64)
    _load().oracle_pyr_expand_f64(_ptr(g), g.shape[1], g.shape[0], W, H, _mode(mode), float(cval),
                                  _ptr(out))
    return out


def bilateral_f64(img, sigma_d, sigma_r, mode, cval=0.0, size=None):
    """Alg. 1 on a double image (oracle_bilateral_f64), window 4*sigma_d+1."""
    g = np.ascontiguousarray(img, np.float64)
    H, W = g.shape
    if size is None:
        size = 2 * int(round(2 * sigma_d)) + 1
    out = np.empty((H, W), np.float64)
    _load().oracle_bilateral_f64(_ptr(g), W, H, size, size, float(sigma_d), float(sigma_r),
                                 _mode(mode), float(cval), _ptr(out))
    return out


def multires_bilateral(img, levels, sigma_d, sigma_r, mode="mirror", cval=0.0):
    """Multiresolution bilateral filter (N4, reading c28), step by step:
      G_0 = I;  G_{l+1} = REDUCE(G_l)                       l = 0 .. L-2
      B_l = G_l - EXPAND(G_{l+1}) (band-pass), B_{L-1} = G_{L-1} (low-pass)
      F_l = bilateral(B_l; sigma_d, sigma_r[l]) if sigma_r[l] > 0 else B_l
      R_{L-1} = F_{L-1};  R_l = F_l + EXPAND(R_{l+1});  result R_0.
    Every level uses ``mode``; in CONSTANT mode the Gaussian levels (REDUCE /
    EXPAND reads and the low-pass level) read ``cval``, the band-pass levels 0
    (the band-pass of a constant image).  sigma_r: one value per level."""
    L = int(levels)
    assert L >= 1 and len(sigma_r) == L
    G = [np.asarray(img, np.float64)]
    for _ in range(L - 1):
        G.append(pyr_reduce(G[-1], mode, cval))
    B = [G[l] - pyr_expand(G[l + 1], G[l].shape, mode, cval) for l in range(L - 1)] + [G[-1]]
    F = []
    for l in range(L):
        if sigma_r[l] > 0:
            F.append(bilateral_f64(B[l], sigma_d, sigma_r[l], mode,
                                   cval if l == L - 1 else 0.0))
        else:
            F.append(B[l])
    R = F[-1]
    for l in range(L - 2, -1, -1):
        R = F[l] + pyr_expand(R, F[l].shape, mode, cval)
    return R

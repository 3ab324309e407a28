"""B200-native local operators (HIPAcc, Membarth et al., IPDPS 2012).

Thin Python binding over the C ABI in ``include/lop.h`` (``liblop.so``):
argument marshalling only -- every pixel is computed by the sm_100a kernels
in ``csrc/``.  PyTorch provides device memory, streams and process groups.
There is no CPU fallback: the functions raise on non-CUDA tensors, and
importing this package raises if ``liblop.so`` has not been built.

Paper objects -> this API (PAPER.md line numbers):
  Image (L150-L154)              a CUDA tensor (H, W) or (B, H, W), rows contiguous
  IterationSpace (L155-L157)     ``roi=(x0, y0, w, h)`` (default: whole image)
  BoundaryCondition (Listing 3)  ``mode=``, ``constant=``, window ``size=``
  Accessor (L160-L162)           ``offset=(dx, dy)``
  Mask (Listing 4)               ``mask=`` (host array), ``closeness_mask()``,
                                 ``gaussian_mask()``, ``sobel_mask()``
  Kernel::execute (Listing 2)    ``bilateral()``, ``convolve()``, ``gaussian()``,
                                 ``sobel()``
"""
from __future__ import annotations

import ctypes

import numpy as np
import torch

from . import _lib
from ._lib import LopError

lib = _lib.load()

MODES = {"undefined": _lib.LOP_UNDEFINED, "clamp": _lib.LOP_CLAMP, "repeat": _lib.LOP_REPEAT,
         "mirror": _lib.LOP_MIRROR, "constant": _lib.LOP_CONSTANT}
_DT = {torch.uint8: _lib.LOP_U8, torch.int32: _lib.LOP_I32, torch.float32: _lib.LOP_F32}
VARIANTS = {"auto": _lib.LOP_VARIANT_AUTO, "generic": _lib.LOP_VARIANT_GENERIC,
            "tiled": _lib.LOP_VARIANT_TILED}

__all__ = ["bilateral", "convolve", "convolve_chain", "gaussian", "sobel", "local", "alg2_select",
           "closeness_mask", "gaussian_mask",
           "sobel_mask", "set_variant", "get_variant", "launch_count", "reset_launch_count",
           "Pipeline", "LopError", "image_view", "MODES", "library_path"]


def _default_window(sigma_d: float) -> int:
    """2*round(2 sigma_d) + 1: the paper's 4 sigma_d + 1 for
    integer sigma_d, and odd for every sigma_d (reading c1)."""
    return 2 * int(round(2.0 * float(sigma_d))) + 1


def library_path() -> str:
    return _lib.LIB_PATH


def _check(status: int):
    if status != _lib.LOP_OK:
        raise LopError(status, lib.lop_last_error().decode())


def _mode(mode) -> int:
    if isinstance(mode, str):
        return MODES[mode]
    return int(mode)


def image_view(t: torch.Tensor, halo_top: int = 0, halo_bottom: int = 0, global_y0: int = 0,
               global_height: int = 0) -> _lib.lop_image:
    """lop_image over a CUDA tensor (H, W) or (B, H, W) whose rows are contiguous.

    For band views, ``t`` covers the OWNED rows; ``halo_top``/``halo_bottom``
    rows directly above/below in the same storage are readable by the kernel.
    """
    if not t.is_cuda:
        raise TypeError("lop operates on CUDA tensors only (no CPU fallback)")
    if t.dtype not in _DT:
        raise TypeError("unsupported dtype %s" % t.dtype)
    if t.dim() == 2:
        b, (h, w) = 1, t.shape
        bstride = 0
    elif t.dim() == 3:
        b, h, w = t.shape
        bstride = t.stride(0) * t.element_size()
    else:
        raise ValueError("expected (H, W) or (B, H, W)")
    if t.stride(-1) != 1:
        raise ValueError("rows must be contiguous (stride(-1) == 1)")
    im = _lib.lop_image()
    im.data = t.data_ptr()
    im.width, im.height = int(w), int(h)
    im.stride_bytes = t.stride(-2) * t.element_size()
    im.dtype = _DT[t.dtype]
    im.batch = int(b)
    im.batch_stride_bytes = int(bstride)
    im.halo_top, im.halo_bottom = int(halo_top), int(halo_bottom)
    im.global_y0, im.global_height = int(global_y0), int(global_height)
    return im


def _stream_handle(t: torch.Tensor, stream):
    if stream is None:
        stream = torch.cuda.current_stream(t.device)
    return stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream)


def _host_mask(mask, dtype) -> tuple[np.ndarray, _lib.lop_mask]:
    arr = np.ascontiguousarray(np.asarray(mask.cpu() if torch.is_tensor(mask) else mask),
                               dtype=np.float32 if dtype == _lib.LOP_F32 else np.int32)
    if arr.ndim != 2:
        raise ValueError("mask must be 2D (size_y, size_x)")
    m = _lib.lop_mask()
    m.size_y, m.size_x = arr.shape
    m.dtype = dtype
    m.coeffs = arr.ctypes.data
    m.shift = 0
    return arr, m


def _execute(kind, x, out, mode, constant, size_xy, roi, offset, stream, band, call):
    halo_top, halo_bottom, gy0, gh = band
    in_im = image_view(x, halo_top, halo_bottom, gy0, gh)
    out_im = image_view(out, 0, 0, gy0, gh)
    bc = _lib.lop_boundary_condition()
    bc.image = in_im
    bc.mode = _mode(mode)
    bc.size_x, bc.size_y = size_xy
    bc.constant = float(constant)
    acc = _lib.lop_accessor(ctypes.pointer(bc), int(offset[0]), int(offset[1]))
    is_ = _lib.lop_iteration_space()
    is_.image = out_im
    if roi is not None:
        is_.x0, is_.y0, is_.width, is_.height = (int(v) for v in roi)
    with torch.cuda.device(x.device):
        _check(call(ctypes.byref(is_), ctypes.byref(acc), _stream_handle(x, stream)))
    return out


def bilateral(x: torch.Tensor, sigma_d: float, sigma_r: float, mode="clamp", constant=0.0,
              size=None, mask=None, out=None, roi=None, offset=(0, 0), stream=None,
              band=(0, 0, 0, 0)) -> torch.Tensor:
    """Bilateral filter (Alg. 1, Listing 5) of a float32 CUDA image.

    size: window (odd int or (sx, sy)); default 4*sigma_d+1.
    mask: optional host closeness mask (size_y, size_x); default Eq. (1).
    band: (halo_top, halo_bottom, global_y0, global_height) for row-band views.
    """
    if mask is not None:
        marr, m = _host_mask(mask, _lib.LOP_F32)
        size_xy = (m.size_x, m.size_y)
        mptr = ctypes.byref(m)
    else:
        marr, mptr = None, None
        if size is None:
            size = _default_window(sigma_d)
        size_xy = (size, size) if isinstance(size, int) else tuple(size)
    if out is None:
        out = torch.empty_like(x)
    return _execute("bilateral", x, out, mode, constant, size_xy, roi, offset, stream, band,
                    lambda is_, acc, s: lib.lop_bilateral_execute(is_, acc, mptr, float(sigma_d),
                                                                  float(sigma_r), s))


def convolve(x: torch.Tensor, mask, mode="clamp", constant=0.0, shift=0, out=None,
             out_dtype=None, roi=None, offset=(0, 0), stream=None,
             band=(0, 0, 0, 0)) -> torch.Tensor:
    """Local operator with a filter mask (correlation, Listing 5 / Listing 9).

    float32 image: float mask, out float32.  uint8 image: integer mask,
    out uint8 (default, rounded (S + 2^(k-1)) >> k, saturated) or int32.
    """
    mdt = _lib.LOP_F32 if x.dtype == torch.float32 else _lib.LOP_I32
    marr, m = _host_mask(mask, mdt)
    m.shift = int(shift)
    if out is None:
        out = torch.empty(x.shape, dtype=out_dtype or x.dtype, device=x.device)
    return _execute("convolve", x, out, mode, constant, (m.size_x, m.size_y), roi, offset,
                    stream, band,
                    lambda is_, acc, s: lib.lop_convolve_execute(is_, acc, ctypes.byref(m), s))


_WORKSPACE = {}


def _workspace(device, stream_handle: int, nbytes: int) -> torch.Tensor:
    """A cached byte buffer of at least nbytes per (device, stream): calls on
    one stream are ordered, so reusing its buffer is safe (grown on demand)."""
    key = (torch.device(device).index, int(stream_handle))
    ws = _WORKSPACE.get(key)
    if ws is None or ws.numel() < nbytes:
        if ws is not None:                   # growing: the old buffer may still be in use
            torch.cuda.synchronize(device)
        ws = torch.empty(max(nbytes, 1), dtype=torch.uint8, device=device)
        _WORKSPACE[key] = ws
    return ws


def convolve_chain(x: torch.Tensor, first, second, mode="clamp", constant=0.0, shift1=0,
                   shift2=0, out=None, out_dtype=None, roi=None, offset=(0, 0),
                   stream=None, fused=False) -> torch.Tensor:
    """second (*) (first (*) x) (e.g. Gaussian -> Sobel), equal bit for bit to
    two convolve() calls (u8: the intermediate is u8).  Default: the library
    picks the faster route with a cached workspace (lop_convolve_chain_execute_ws:
    two passes through L2 on B200); fused=True: the one-pass fused kernel
    (lop_convolve_chain_execute)."""
    mdt = _lib.LOP_F32 if x.dtype == torch.float32 else _lib.LOP_I32
    a1, m1 = _host_mask(first, mdt)
    a2, m2 = _host_mask(second, mdt)
    m1.shift, m2.shift = int(shift1), int(shift2)
    if out is None:
        out = torch.empty(x.shape, dtype=out_dtype or x.dtype, device=x.device)
    size = (m1.size_x + m2.size_x - 1, m1.size_y + m2.size_y - 1)
    if fused:
        return _execute("chain", x, out, mode, constant, size, roi, offset, stream, (0, 0, 0, 0),
                        lambda is_, acc, s: lib.lop_convolve_chain_execute(
                            is_, acc, ctypes.byref(m1), ctypes.byref(m2), s))

    def call(is_, acc, s):
        nb = ctypes.c_int64(0)
        st = lib.lop_convolve_chain_workspace_bytes(is_, acc, ctypes.byref(m1), ctypes.byref(m2),
                                                    ctypes.byref(nb))
        if st != _lib.LOP_OK:
            return st
        ws = _workspace(x.device, s or 0, nb.value)
        return lib.lop_convolve_chain_execute_ws(is_, acc, ctypes.byref(m1), ctypes.byref(m2),
                                                 ws.data_ptr(), nb.value, s)
    return _execute("chain", x, out, mode, constant, size, roi, offset, stream, (0, 0, 0, 0), call)


_REDUCE = {"sum": _lib.LOP_REDUCE_SUM, "min": _lib.LOP_REDUCE_MIN, "max": _lib.LOP_REDUCE_MAX}


def reduce(x: torch.Tensor, domain, op="min", mode="clamp", constant=0.0, out=None, roi=None,
           offset=(0, 0), stream=None, band=(0, 0, 0, 0)) -> torch.Tensor:
    """Local reduction over a mask domain, Listing 9's convolve(mask, <op>, f):
    op "min" / "max" over the taps where ``domain`` is non-zero (erosion /
    dilation), "sum" = convolve(x, domain).  float32 or uint8 images."""
    mdt = _lib.LOP_F32 if x.dtype == torch.float32 else _lib.LOP_I32
    marr, m = _host_mask(domain, mdt)
    if out is None:
        out = torch.empty_like(x)
    return _execute("reduce", x, out, mode, constant, (m.size_x, m.size_y), roi, offset, stream,
                    band, lambda is_, acc, s: lib.lop_reduce_execute(is_, acc, ctypes.byref(m),
                                                                     _REDUCE[op], s))


def global_reduce(x: torch.Tensor, op="sum", roi=None, out=None, work=None,
                  stream=None) -> torch.Tensor:
    """Global operator: "sum" / "min" / "max" / "sumsq"
    (the sum of squares; reading c26) of the pixels
    of ``roi`` over all frames, as a 1-element float64 CUDA tensor (written
    asynchronously; deterministic).  ``work``: a reusable zero-initialised
    float64 scratch tensor of LOP_GLOBAL_WORK_DOUBLES elements."""
    if out is None:
        out = torch.empty(1, dtype=torch.float64, device=x.device)
    if work is None:                         # zero-initialised (its last slot is a counter)
        work = torch.zeros(_lib.LOP_GLOBAL_WORK_DOUBLES, dtype=torch.float64, device=x.device)
    is_ = _lib.lop_iteration_space()
    is_.image = image_view(x)
    if roi is not None:
        is_.x0, is_.y0, is_.width, is_.height = (int(v) for v in roi)
    with torch.cuda.device(x.device):
        _check(lib.lop_global_reduce_execute(ctypes.byref(is_), _GLOBAL[op], out.data_ptr(),
                                             work.data_ptr(), _stream_handle(x, stream)))
    return out


_GLOBAL = dict(_REDUCE, sumsq=_lib.LOP_REDUCE_SUMSQ)
_TAP = {"product": _lib.LOP_TAP_PRODUCT, "absdiff": _lib.LOP_TAP_ABSDIFF,
        "sqdiff": _lib.LOP_TAP_SQDIFF, "square": _lib.LOP_TAP_SQUARE}


def local(inputs, masks, op="sum", fn="product", modes="clamp", constants=0.0, offsets=None,
          out=None, roi=None, stream=None, band=None, point=None) -> torch.Tensor:
    """Local operator over several Accessors with a per-tap function
    (lop_local_execute; Listing 9):
    out = op over k, taps of fn(M_k, Read_k(x+ox_k+xf, y+oy_k+yf), centre_k).
    inputs: up to 4 CUDA images of one shape and dtype (float32 -> float32,
    uint8 -> int32); masks: one 2D host mask per input (its window);
    modes / constants / offsets: per input (or one value for all); band: per input
    (halo_top, halo_bottom, global_y0, global_height) for row-band views;
    point: per input (scale, offset) of a point-operator prologue
    Read' = scale * Read + offset (lop_local_execute_point; PAPER.md
    L107-L122, reading c27), None = identity."""
    K = len(inputs)
    if K != len(masks):
        raise ValueError("one mask per input")
    modes = [modes] * K if isinstance(modes, (str, int)) else list(modes)
    constants = [constants] * K if np.isscalar(constants) else list(constants)
    offsets = [(0, 0)] * K if offsets is None else list(offsets)
    band = [(0, 0, 0, 0)] * K if band is None else list(band)
    x0 = inputs[0]
    mdt = _lib.LOP_F32 if x0.dtype == torch.float32 else _lib.LOP_I32
    if out is None:
        out = torch.empty(x0.shape, dtype=torch.float32 if x0.dtype == torch.float32 else torch.int32,
                          device=x0.device)
    keep, bcs, accs, ms = [], [], [], []
    for k in range(K):
        arr, m = _host_mask(masks[k], mdt)
        bc = _lib.lop_boundary_condition()
        bc.image = image_view(inputs[k], *band[k])
        bc.mode = _mode(modes[k])
        bc.size_x, bc.size_y = m.size_x, m.size_y
        bc.constant = float(constants[k])
        keep += [arr, bc]
        bcs.append(bc)
        accs.append(_lib.lop_accessor(ctypes.pointer(bc), int(offsets[k][0]), int(offsets[k][1])))
        ms.append(m)
    acc_arr = (ctypes.POINTER(_lib.lop_accessor) * K)(*[ctypes.pointer(a) for a in accs])
    m_arr = (ctypes.POINTER(_lib.lop_mask) * K)(*[ctypes.pointer(m) for m in ms])
    is_ = _lib.lop_iteration_space()
    is_.image = image_view(out, 0, 0, band[0][2], band[0][3])
    if roi is not None:
        is_.x0, is_.y0, is_.width, is_.height = (int(v) for v in roi)
    with torch.cuda.device(x0.device):
        if point is None:
            _check(lib.lop_local_execute(ctypes.byref(is_), acc_arr, m_arr, K, _REDUCE[op],
                                         _TAP[fn], _stream_handle(x0, stream)))
        else:
            if len(point) != K:
                raise ValueError("one (scale, offset) per input")
            sc = (ctypes.c_double * K)(*[float(a) for a, _ in point])
            of = (ctypes.c_double * K)(*[float(b) for _, b in point])
            _check(lib.lop_local_execute_point(ctypes.byref(is_), acc_arr, m_arr, K, _REDUCE[op],
                                               _TAP[fn], sc, of, _stream_handle(x0, stream)))
    del keep
    return out


# ------------------------------------------------ multiresolution filter (N4) ----

def _pyr_half(n: int) -> int:
    return (int(n) + 1) // 2


def pyramid_reduce(x: torch.Tensor, mode="mirror", constant=0.0, out=None,
                   stream=None) -> torch.Tensor:
    """REDUCE (lop_pyramid_reduce_execute; reading c28): the 5x5 binomial at
    every second pixel of a float32 (H, W) / (B, H, W) image -> ceil(H/2) x
    ceil(W/2)."""
    if out is None:
        out = torch.empty(x.shape[:-2] + (_pyr_half(x.shape[-2]), _pyr_half(x.shape[-1])),
                          dtype=x.dtype, device=x.device)
    return _execute("pyr_reduce", x, out, mode, constant, (5, 5), None, (0, 0), stream,
                    (0, 0, 0, 0), lambda is_, acc, s: lib.lop_pyramid_reduce_execute(is_, acc, s))


def pyramid_expand(coarse: torch.Tensor, shape, mode="mirror", constant=0.0, addend=None,
                   sign=1.0, out=None, stream=None) -> torch.Tensor:
    """EXPAND (lop_pyramid_expand_execute; reading c28) of a coarse level to
    ``shape`` = (H, W): out = addend + sign * EXPAND(coarse) (addend None ->
    sign * EXPAND); ``out`` may be ``addend`` (in place)."""
    H, W = (int(v) for v in shape)
    if out is None:
        out = torch.empty(coarse.shape[:-2] + (H, W), dtype=coarse.dtype, device=coarse.device)
    add = ctypes.byref(image_view(addend)) if addend is not None else None
    return _execute("pyr_expand", coarse, out, mode, constant, (5, 5), None, (0, 0), stream,
                    (0, 0, 0, 0), lambda is_, acc, s: lib.lop_pyramid_expand_execute(
                        is_, acc, add, float(sign), s))


def multires_workspace_bytes(shape, levels: int) -> int:
    b = 1 if len(shape) == 2 else int(shape[0])
    n = ctypes.c_int64(0)
    _check(lib.lop_multires_workspace_bytes(int(shape[-1]), int(shape[-2]), b, int(levels),
                                            ctypes.byref(n)))
    return n.value


def multires_bilateral(x: torch.Tensor, levels: int, sigma_d: float, sigma_r, mode="mirror",
                       constant=0.0, size=None, out=None, workspace=None,
                       stream=None) -> torch.Tensor:
    """Multiresolution bilateral filter (lop_multires_bilateral_execute; PAPER.md
    L309-L314, reading c28): Laplacian pyramid of ``levels`` levels, level l
    bilateral-filtered with (sigma_d, sigma_r[l]) (sigma_r[l] <= 0: unfiltered),
    reconstructed.  ``workspace``: a uint8 CUDA tensor of at least
    multires_workspace_bytes(x.shape, levels) bytes (allocated if None)."""
    levels = int(levels)
    sr = [float(v) for v in (sigma_r if np.ndim(sigma_r) else [sigma_r] * levels)]
    if len(sr) != levels:
        raise ValueError("one sigma_r per level")
    if size is None:
        size = _default_window(sigma_d)
    size_xy = (size, size) if isinstance(size, int) else tuple(size)
    need = multires_workspace_bytes(tuple(x.shape), levels)
    if workspace is None:
        workspace = torch.empty(max(need, 1), dtype=torch.uint8, device=x.device)
    if out is None:
        out = torch.empty_like(x)
    srs = (ctypes.c_float * levels)(*sr)
    return _execute("multires", x, out, mode, constant, size_xy, None, (0, 0), stream,
                    (0, 0, 0, 0), lambda is_, acc, s: lib.lop_multires_bilateral_execute(
                        is_, acc, levels, float(sigma_d), srs, workspace.data_ptr(),
                        workspace.numel(), s))


def alg2_select(candidates, width, height, rx, ry, simd_width=32):
    """Algorithm 2 over candidate configurations, each a
    dict(block_x, block_y, out_x=1, out_y=1, valid=True, occupancy);
    returns (index, border_threads) -- the library's own selector."""
    n = len(candidates)
    arr = (_lib.lop_config_candidate * n)()
    for a, c in zip(arr, candidates):
        a.block_x, a.block_y = int(c["block_x"]), int(c["block_y"])
        a.out_x, a.out_y = int(c.get("out_x", 1)), int(c.get("out_y", 1))
        a.valid = int(bool(c.get("valid", True)))
        a.occupancy = float(c["occupancy"])
    bh = ctypes.c_int64(0)
    i = lib.lop_alg2_select(ctypes.cast(arr, ctypes.c_void_p), n, int(simd_width), int(width),
                            int(height), int(rx), int(ry), ctypes.byref(bh))
    return i, bh.value


def erode(x: torch.Tensor, size: int = 3, mode="clamp", constant=0.0, **kw) -> torch.Tensor:
    """Grey-value erosion with a full size x size window (local MIN)."""
    return reduce(x, np.ones((size, size)), "min", mode, constant, **kw)


def dilate(x: torch.Tensor, size: int = 3, mode="clamp", constant=0.0, **kw) -> torch.Tensor:
    """Grey-value dilation with a full size x size window (local MAX)."""
    return reduce(x, np.ones((size, size)), "max", mode, constant, **kw)


_COMBINE = {"l2": _lib.LOP_COMBINE_L2, "l1": _lib.LOP_COMBINE_L1, "sumsq": _lib.LOP_COMBINE_SUMSQ}


def convolve2(x: torch.Tensor, mask_a, mask_b, combine="l2", mode="clamp", constant=0.0,
              out=None, roi=None, offset=(0, 0), stream=None) -> torch.Tensor:
    """Two local operators on one input combined by a point operator, one pass:
    combine = "l2" sqrt(A^2 + B^2) (float32), "l1" |A| + |B|, "sumsq" A^2 + B^2.
    float32 -> float32 or uint8 -> int32."""
    mdt = _lib.LOP_F32 if x.dtype == torch.float32 else _lib.LOP_I32
    aa, ma = _host_mask(mask_a, mdt)
    ab, mb = _host_mask(mask_b, mdt)
    if out is None:
        out = torch.empty(x.shape, dtype=torch.float32 if x.dtype == torch.float32 else torch.int32,
                          device=x.device)
    return _execute("convolve2", x, out, mode, constant, (ma.size_x, ma.size_y), roi, offset,
                    stream, (0, 0, 0, 0),
                    lambda is_, acc, s: lib.lop_convolve2_execute(is_, acc, ctypes.byref(ma),
                                                                  ctypes.byref(mb),
                                                                  _COMBINE[combine], s))


def sobel_magnitude(x: torch.Tensor, mode="clamp", constant=0.0, **kw) -> torch.Tensor:
    """Sobel gradient magnitude in one pass: sqrt(gx^2 + gy^2) for float32
    images, |gx| + |gy| (int32) for uint8 images."""
    dt = np.float32 if x.dtype == torch.float32 else np.int32
    combine = "l2" if x.dtype == torch.float32 else "l1"
    return convolve2(x, sobel_mask(0, dt), sobel_mask(1, dt), combine, mode, constant, **kw)


def gaussian(x: torch.Tensor, size: int = 5, mode="clamp", constant=0.0, **kw) -> torch.Tensor:
    """Binomial Gaussian (Tables VIII-IX; reading c11): f32 -> f32, u8 -> u8."""
    if x.dtype == torch.float32:
        m, _ = gaussian_mask(size, np.float32)
        return convolve(x, m, mode, constant, **kw)
    m, k = gaussian_mask(size, np.int32)
    return convolve(x, m, mode, constant, shift=k, **kw)


def sobel(x: torch.Tensor, direction: int = 0, mode="clamp", constant=0.0, **kw) -> torch.Tensor:
    """Sobel 3x3 (L847-L849): f32 -> f32, u8 -> int32 (reading c12)."""
    if x.dtype == torch.float32:
        return convolve(x, sobel_mask(direction, np.float32), mode, constant, **kw)
    kw.setdefault("out_dtype", torch.int32)
    return convolve(x, sobel_mask(direction, np.int32), mode, constant, **kw)


# --------------------------------------------------------------- masks ----

def closeness_mask(sigma_d: float, size_x: int | None = None, size_y: int | None = None):
    """Eq. (1) closeness coefficients as Listing 4's float mask[] (yf outer)."""
    size_x = _default_window(sigma_d) if size_x is None else size_x
    size_y = size_x if size_y is None else size_y
    out = np.empty((size_y, size_x), np.float32)
    _check(lib.lop_mask_closeness(float(sigma_d), size_x, size_y, out.ctypes.data))
    return out


def gaussian_mask(size: int, dtype=np.int32):
    out = np.empty((size, size), dtype)
    k = ctypes.c_int32(0)
    _check(lib.lop_mask_gaussian(size, _lib.LOP_I32 if dtype == np.int32 else _lib.LOP_F32,
                                 out.ctypes.data, ctypes.byref(k)))
    return out, k.value


def sobel_mask(direction: int = 0, dtype=np.int32):
    out = np.empty((3, 3), dtype)
    _check(lib.lop_mask_sobel(direction, _lib.LOP_I32 if dtype == np.int32 else _lib.LOP_F32,
                              out.ctypes.data))
    return out


# ------------------------------------------------------------ runtime ----

def set_variant(name: str):
    _check(lib.lop_set_variant(VARIANTS[name]))


def get_variant() -> str:
    v = lib.lop_get_variant()
    return {k: n for n, k in VARIANTS.items()}[v]


def launch_count() -> int:
    return int(lib.lop_launch_count())


def reset_launch_count():
    lib.lop_reset_launch_count()


class Pipeline:
    """End-to-end filtering of HOST images (Listing 2 flow) with overlapped
    chunked H2D / kernel / D2H on three CUDA streams (csrc/pipeline.cpp)."""

    def __init__(self, width: int, height: int, device: int = 0, chunk_rows: int = 512):
        h = ctypes.c_void_p()
        _check(lib.lop_pipeline_create(int(device), int(width), int(height), int(chunk_rows),
                                       ctypes.byref(h)))
        self._h = h
        self.width, self.height = width, height

    def bytes_moved(self):
        """(host->device, device->host) bytes of the last call."""
        h2d, d2h = ctypes.c_int64(), ctypes.c_int64()
        _check(lib.lop_pipeline_bytes(self._h, ctypes.byref(h2d), ctypes.byref(d2h)))
        return h2d.value, d2h.value

    def close(self):
        if self._h:
            lib.lop_pipeline_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    @staticmethod
    def _host(t: torch.Tensor):
        if t.is_cuda or t.stride(-1) != 1 or t.dim() != 2:
            raise ValueError("pipeline needs a 2D host tensor with contiguous rows")
        return t.data_ptr(), t.stride(0) * t.element_size()

    def bilateral(self, host_in: torch.Tensor, host_out: torch.Tensor, sigma_d: float,
                  sigma_r: float, mode="clamp", constant=0.0, size=None, mask=None):
        ip, istr = self._host(host_in)
        op, ostr = self._host(host_out)
        if mask is not None:
            marr, m = _host_mask(mask, _lib.LOP_F32)
            sx, sy, mptr = m.size_x, m.size_y, ctypes.byref(m)
        else:
            size = _default_window(sigma_d) if size is None else size
            sx, sy = (size, size) if isinstance(size, int) else size
            mptr = None
        _check(lib.lop_pipeline_bilateral(self._h, ip, istr, op, ostr, _mode(mode),
                                          float(constant), sx, sy, mptr, float(sigma_d),
                                          float(sigma_r)))
        return host_out

    def bilateral_frames(self, host_in: torch.Tensor, host_out: torch.Tensor, sigma_d: float,
                         sigma_r: float, mode="clamp", constant=0.0, size=None, mask=None):
        """A (F, H, W) host sequence streamed through the pipeline back to back
        (frame f+1 uploads while frame f computes / downloads)."""
        if host_in.is_cuda or host_in.dim() != 3 or host_in.stride(-1) != 1 or \
                host_out.shape != host_in.shape or host_out.stride(-1) != 1:
            raise ValueError("pipeline frames need (F, H, W) host tensors with contiguous rows")
        es = host_in.element_size()
        if mask is not None:
            marr, m = _host_mask(mask, _lib.LOP_F32)
            sx, sy, mptr = m.size_x, m.size_y, ctypes.byref(m)
        else:
            size = _default_window(sigma_d) if size is None else size
            sx, sy = (size, size) if isinstance(size, int) else size
            mptr = None
        _check(lib.lop_pipeline_bilateral_frames(
            self._h, host_in.data_ptr(), host_in.stride(1) * es, host_in.stride(0) * es,
            host_out.data_ptr(), host_out.stride(1) * es, host_out.stride(0) * es,
            int(host_in.shape[0]), _mode(mode), float(constant), sx, sy, mptr, float(sigma_d),
            float(sigma_r)))
        return host_out

    def convolve(self, host_in: torch.Tensor, host_out: torch.Tensor, mask, mode="clamp",
                 constant=0.0, shift=0):
        ip, istr = self._host(host_in)
        op, ostr = self._host(host_out)
        mdt = _lib.LOP_F32 if host_in.dtype == torch.float32 else _lib.LOP_I32
        marr, m = _host_mask(mask, mdt)
        m.shift = int(shift)
        _check(lib.lop_pipeline_convolve(self._h, ip, _DT[host_in.dtype], istr, op,
                                         _DT[host_out.dtype], ostr, _mode(mode),
                                         float(constant), ctypes.byref(m)))
        return host_out

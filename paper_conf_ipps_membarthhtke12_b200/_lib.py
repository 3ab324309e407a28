"""ctypes declarations of include/lop.h (argument marshalling only).

Loads the in-tree ``liblop.so`` built by ``build.py``.  There is no fallback:
if the library is missing or cannot be loaded, importing the package raises.
"""
from __future__ import annotations

import ctypes
import os

PKG = os.path.dirname(os.path.abspath(__file__))
# LOP_LIBRARY: load an alternative build (A/B experiments); default: the in-tree build
LIB_PATH = os.environ.get("LOP_LIBRARY") or os.path.join(PKG, "liblop.so")

LOP_OK, LOP_ERR_INVALID, LOP_ERR_UNSUPPORTED, LOP_ERR_CUDA = 0, -1, -2, -3
LOP_U8, LOP_I32, LOP_F32 = 0, 1, 2
LOP_UNDEFINED, LOP_CLAMP, LOP_REPEAT, LOP_MIRROR, LOP_CONSTANT = 0, 1, 2, 3, 4
LOP_VARIANT_AUTO, LOP_VARIANT_GENERIC, LOP_VARIANT_TILED = 0, 1, 2
LOP_REDUCE_SUM, LOP_REDUCE_MIN, LOP_REDUCE_MAX, LOP_REDUCE_SUMSQ = 0, 1, 2, 3
LOP_COMBINE_L2, LOP_COMBINE_L1, LOP_COMBINE_SUMSQ = 0, 1, 2
LOP_GLOBAL_WORK_DOUBLES = 1025
LOP_TAP_PRODUCT, LOP_TAP_ABSDIFF, LOP_TAP_SQDIFF, LOP_TAP_SQUARE = 0, 1, 2, 3
LOP_MAX_ACCESSORS = 4

c_i32, c_i64, c_dbl, c_flt, c_vp = (ctypes.c_int32, ctypes.c_int64, ctypes.c_double,
                                    ctypes.c_float, ctypes.c_void_p)


class lop_image(ctypes.Structure):
    _fields_ = [("data", c_vp), ("width", c_i32), ("height", c_i32),
                ("stride_bytes", c_i64), ("dtype", c_i32), ("batch", c_i32),
                ("batch_stride_bytes", c_i64), ("halo_top", c_i32), ("halo_bottom", c_i32),
                ("global_y0", c_i32), ("global_height", c_i32)]


class lop_boundary_condition(ctypes.Structure):
    _fields_ = [("image", lop_image), ("mode", c_i32), ("size_x", c_i32), ("size_y", c_i32),
                ("constant", c_dbl)]


class lop_accessor(ctypes.Structure):
    _fields_ = [("bc", ctypes.POINTER(lop_boundary_condition)), ("offset_x", c_i32),
                ("offset_y", c_i32)]


class lop_mask(ctypes.Structure):
    _fields_ = [("size_x", c_i32), ("size_y", c_i32), ("dtype", c_i32), ("coeffs", c_vp),
                ("shift", c_i32)]


class lop_config_candidate(ctypes.Structure):
    _fields_ = [("block_x", c_i32), ("block_y", c_i32), ("out_x", c_i32), ("out_y", c_i32),
                ("valid", c_i32), ("occupancy", c_dbl)]


class lop_iteration_space(ctypes.Structure):
    _fields_ = [("image", lop_image), ("x0", c_i32), ("y0", c_i32), ("width", c_i32),
                ("height", c_i32)]


# name -> (restype, argtypes); every symbol include/lop.h declares
SIGNATURES = {
    "lop_bilateral_execute": (c_i32, [ctypes.POINTER(lop_iteration_space),
                                      ctypes.POINTER(lop_accessor), ctypes.POINTER(lop_mask),
                                      c_flt, c_flt, c_vp]),
    "lop_convolve_execute": (c_i32, [ctypes.POINTER(lop_iteration_space),
                                     ctypes.POINTER(lop_accessor), ctypes.POINTER(lop_mask),
                                     c_vp]),
    "lop_convolve_chain_execute": (c_i32, [ctypes.POINTER(lop_iteration_space),
                                           ctypes.POINTER(lop_accessor), ctypes.POINTER(lop_mask),
                                           ctypes.POINTER(lop_mask), c_vp]),
    "lop_convolve_chain_workspace_bytes": (c_i32, [ctypes.POINTER(lop_iteration_space),
                                                   ctypes.POINTER(lop_accessor),
                                                   ctypes.POINTER(lop_mask),
                                                   ctypes.POINTER(lop_mask),
                                                   ctypes.POINTER(c_i64)]),
    "lop_convolve_chain_execute_ws": (c_i32, [ctypes.POINTER(lop_iteration_space),
                                              ctypes.POINTER(lop_accessor), ctypes.POINTER(lop_mask),
                                              ctypes.POINTER(lop_mask), c_vp, c_i64, c_vp]),
    "lop_reduce_execute": (c_i32, [ctypes.POINTER(lop_iteration_space),
                                   ctypes.POINTER(lop_accessor), ctypes.POINTER(lop_mask),
                                   c_i32, c_vp]),
    "lop_convolve2_execute": (c_i32, [ctypes.POINTER(lop_iteration_space),
                                      ctypes.POINTER(lop_accessor), ctypes.POINTER(lop_mask),
                                      ctypes.POINTER(lop_mask), c_i32, c_vp]),
    "lop_global_reduce_execute": (c_i32, [ctypes.POINTER(lop_iteration_space), c_i32, c_vp,
                                          c_vp, c_vp]),
    "lop_local_execute": (c_i32, [ctypes.POINTER(lop_iteration_space),
                                  ctypes.POINTER(ctypes.POINTER(lop_accessor)),
                                  ctypes.POINTER(ctypes.POINTER(lop_mask)), c_i32, c_i32, c_i32,
                                  c_vp]),
    "lop_local_execute_point": (c_i32, [ctypes.POINTER(lop_iteration_space),
                                        ctypes.POINTER(ctypes.POINTER(lop_accessor)),
                                        ctypes.POINTER(ctypes.POINTER(lop_mask)), c_i32, c_i32,
                                        c_i32, c_vp, c_vp, c_vp]),
    "lop_pyramid_reduce_execute": (c_i32, [ctypes.POINTER(lop_iteration_space),
                                           ctypes.POINTER(lop_accessor), c_vp]),
    "lop_pyramid_expand_execute": (c_i32, [ctypes.POINTER(lop_iteration_space),
                                           ctypes.POINTER(lop_accessor), ctypes.POINTER(lop_image),
                                           c_flt, c_vp]),
    "lop_multires_workspace_bytes": (c_i32, [c_i32, c_i32, c_i32, c_i32, ctypes.POINTER(c_i64)]),
    "lop_multires_bilateral_execute": (c_i32, [ctypes.POINTER(lop_iteration_space),
                                               ctypes.POINTER(lop_accessor), c_i32, c_flt, c_vp,
                                               c_vp, c_i64, c_vp]),
    "lop_alg2_select": (c_i32, [c_vp, c_i32, c_i32, c_i32, c_i32, c_i32, c_i32,
                                ctypes.POINTER(c_i64)]),
    "lop_mask_closeness": (c_i32, [c_flt, c_i32, c_i32, c_vp]),
    "lop_mask_gaussian": (c_i32, [c_i32, c_i32, c_vp, ctypes.POINTER(c_i32)]),
    "lop_mask_sobel": (c_i32, [c_i32, c_i32, c_vp]),
    "lop_set_variant": (c_i32, [c_i32]),
    "lop_get_variant": (c_i32, []),
    "lop_launch_count": (c_i64, []),
    "lop_reset_launch_count": (None, []),
    "lop_last_error": (ctypes.c_char_p, []),
    "lop_version": (c_i32, []),
    "lop_pipeline_create": (c_i32, [c_i32, c_i32, c_i32, c_i32, ctypes.POINTER(c_vp)]),
    "lop_pipeline_bilateral": (c_i32, [c_vp, c_vp, c_i64, c_vp, c_i64, c_i32, c_dbl, c_i32,
                                       c_i32, ctypes.POINTER(lop_mask), c_flt, c_flt]),
    "lop_pipeline_bilateral_frames": (c_i32, [c_vp, c_vp, c_i64, c_i64, c_vp, c_i64, c_i64,
                                              c_i32, c_i32, c_dbl, c_i32, c_i32,
                                              ctypes.POINTER(lop_mask), c_flt, c_flt]),
    "lop_pipeline_convolve": (c_i32, [c_vp, c_vp, c_i32, c_i64, c_vp, c_i32, c_i64, c_i32,
                                      c_dbl, ctypes.POINTER(lop_mask)]),
    "lop_pipeline_bytes": (c_i32, [c_vp, ctypes.POINTER(c_i64), ctypes.POINTER(c_i64)]),
    "lop_pipeline_destroy": (c_i32, [c_vp]),
}


class LopError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__("lop status %d: %s" % (status, msg))
        self.status = status


def load(path: str = LIB_PATH) -> ctypes.CDLL:
    if not os.path.exists(path):
        raise ImportError("liblop.so not built (%s); run "
                          "`python paper_conf_ipps_membarthhtke12_b200/build.py`" % path)
    lib = ctypes.CDLL(path)
    for name, (res, args) in SIGNATURES.items():
        fn = getattr(lib, name)
        fn.restype = res
        fn.argtypes = args
    return lib

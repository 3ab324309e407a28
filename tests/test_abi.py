"""C-ABI checks that need no GPU: the library loads, exports every symbol
include/lop.h declares, the host-side mask builders match the oracle, and
invalid arguments are rejected before anything is launched."""
import ctypes
import os
import re

import numpy as np
import pytest

import oracle
from conftest import ROOT

lop = pytest.importorskip("paper_conf_ipps_membarthhtke12_b200")
from paper_conf_ipps_membarthhtke12_b200 import _lib  # noqa: E402


def _declared_symbols():
    text = open(os.path.join(ROOT, "include", "lop.h")).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return sorted(set(re.findall(r"\b(lop_[a-z0-9_]+)\s*\(", text)))


def test_header_declares_expected_entry_points():
    syms = _declared_symbols()
    for s in ("lop_bilateral_execute", "lop_convolve_execute", "lop_mask_closeness",
              "lop_mask_gaussian", "lop_mask_sobel", "lop_last_error", "lop_pipeline_create",
              "lop_convolve_chain_execute", "lop_reduce_execute", "lop_convolve2_execute",
              "lop_pipeline_bilateral_frames", "lop_local_execute_point",
              "lop_pyramid_reduce_execute", "lop_pyramid_expand_execute",
              "lop_multires_workspace_bytes", "lop_multires_bilateral_execute"):
        assert s in syms


def test_library_exports_every_declared_symbol():
    lib = ctypes.CDLL(lop.library_path())
    missing = [s for s in _declared_symbols() if not hasattr(lib, s)]
    assert not missing, missing
    # and the binding declares a signature for each of them
    assert set(_declared_symbols()) == set(_lib.SIGNATURES)


def test_library_is_sm100a_only():
    import subprocess
    out = subprocess.run(["cuobjdump", "--list-elf", lop.library_path()], capture_output=True,
                         text=True).stdout
    archs = set(re.findall(r"sm_(\d+a?)", out))
    assert archs == {"100a"}, archs


def test_version():
    assert lop.lib.lop_version() == 100


@pytest.mark.parametrize("sigma_d,sx,sy", [(3, 13, 13), (1, 3, 3), (2.5, 9, 5)])
def test_closeness_builder_matches_oracle(sigma_d, sx, sy):
    m = lop.closeness_mask(sigma_d, sx, sy)
    ref = oracle.closeness_mask(sigma_d, sx, sy)
    np.testing.assert_allclose(m, ref, rtol=1e-7, atol=0)
    assert round(float(lop.closeness_mask(3.0)[0, 0]), 6) == 0.018316   # Listing 4


@pytest.mark.parametrize("size", [1, 3, 5, 7, 11])
def test_gaussian_builder_matches_oracle(size):
    m, k = lop.gaussian_mask(size, np.int32)
    ref, rk = oracle.gaussian_mask(size)
    assert k == rk and (m == ref).all()
    mf, kf = lop.gaussian_mask(size, np.float32)
    assert kf == 0
    np.testing.assert_allclose(mf, ref / 2.0 ** rk, rtol=1e-7)


def test_gaussian_builder_size_limits():
    with pytest.raises(lop.LopError):
        lop.gaussian_mask(13, np.int32)
    mf, _ = lop.gaussian_mask(31, np.float32)
    assert abs(mf.sum() - 1.0) < 1e-5


def test_sobel_builder_matches_oracle():
    for d in (0, 1):
        assert (lop.sobel_mask(d) == oracle.sobel_mask(d)).all()
        assert (lop.sobel_mask(d, np.float32) == oracle.sobel_mask(d)).all()


def test_mask_builder_validation():
    out = np.empty(9, np.float32)
    assert lop.lib.lop_mask_closeness(0.0, 3, 3, out.ctypes.data) == _lib.LOP_ERR_INVALID
    assert lop.lib.lop_mask_closeness(1.0, 4, 3, out.ctypes.data) == _lib.LOP_ERR_INVALID
    assert b"odd" in lop.lib.lop_last_error()
    k = ctypes.c_int32()
    assert lop.lib.lop_mask_gaussian(2, _lib.LOP_I32, out.ctypes.data, ctypes.byref(k)) == -1
    assert lop.lib.lop_mask_sobel(2, _lib.LOP_I32, out.ctypes.data) == -1


def _views(data=1, w=16, h=8, dtype=_lib.LOP_F32):
    im = _lib.lop_image()
    im.data, im.width, im.height = data, w, h
    im.stride_bytes = w * 4
    im.dtype, im.batch = dtype, 1
    bc = _lib.lop_boundary_condition()
    bc.image, bc.mode, bc.size_x, bc.size_y = im, _lib.LOP_CLAMP, 3, 3
    acc = _lib.lop_accessor(ctypes.pointer(bc), 0, 0)
    is_ = _lib.lop_iteration_space()
    is_.image = im
    return bc, acc, is_


def test_execute_rejects_invalid_arguments_before_launch():
    lib = lop.lib
    bc, acc, is_ = _views(data=0)
    assert lib.lop_bilateral_execute(ctypes.byref(is_), ctypes.byref(acc), None, 1.0, 1.0,
                                     None) == _lib.LOP_ERR_INVALID
    assert b"NULL" in lib.lop_last_error()
    assert lib.lop_bilateral_execute(None, ctypes.byref(acc), None, 1.0, 1.0, None) == -1
    bc, acc, is_ = _views()
    bc.size_x = 4
    st = lib.lop_convolve_execute(ctypes.byref(is_), ctypes.byref(acc), None, None)
    assert st == _lib.LOP_ERR_INVALID
    # a host address is not device memory: rejected at validation, no launch
    host = np.zeros((8, 16), np.float32)
    bc, acc, is_ = _views(data=host.ctypes.data)
    before = lop.launch_count()
    st = lib.lop_bilateral_execute(ctypes.byref(is_), ctypes.byref(acc), None, 1.0, 1.0, None)
    assert st == _lib.LOP_ERR_INVALID
    assert lop.launch_count() == before
    # the session-4 entry points validate before launching as well
    bc, acc, is_ = _views(data=0)
    m = _lib.lop_mask()
    assert lib.lop_reduce_execute(ctypes.byref(is_), ctypes.byref(acc), ctypes.byref(m), 7,
                                  None) == _lib.LOP_ERR_INVALID
    assert b"reduction" in lib.lop_last_error()
    assert lib.lop_convolve2_execute(ctypes.byref(is_), ctypes.byref(acc), None, None, 9,
                                     None) == _lib.LOP_ERR_INVALID
    assert b"combine" in lib.lop_last_error()
    assert lib.lop_reduce_execute(ctypes.byref(is_), ctypes.byref(acc), None,
                                  _lib.LOP_REDUCE_MIN, None) == _lib.LOP_ERR_INVALID
    assert lib.lop_pipeline_bilateral_frames(None, None, 0, 0, None, 0, 0, 1, 1, 0.0, 3, 3, None,
                                             1.0, 1.0) == _lib.LOP_ERR_INVALID
    assert lop.launch_count() == before


def test_python_binding_refuses_cpu_tensors():
    import torch
    x = torch.zeros(8, 8)
    with pytest.raises(TypeError, match="CUDA"):
        lop.bilateral(x, 1.0, 0.1)
    with pytest.raises(TypeError, match="CUDA"):
        lop.gaussian(x)


def test_variant_switch():
    assert lop.get_variant() == "auto"
    lop.set_variant("generic")
    assert lop.get_variant() == "generic"
    lop.set_variant("auto")
    assert lop.lib.lop_set_variant(7) == _lib.LOP_ERR_INVALID


def test_c_example_is_built_against_the_abi():
    """examples/bilateral_c.c uses only include/lop.h + the CUDA runtime."""
    exe = os.path.join(ROOT, "examples", "bilateral_c")
    assert os.path.exists(exe), "run __graft_entry__.build()"
    import subprocess
    out = subprocess.run(["ldd", exe], capture_output=True, text=True).stdout
    assert "liblop.so" in out


def test_pipeline_argument_errors_have_messages():
    h = ctypes.c_void_p()
    assert lop.lib.lop_pipeline_create(0, 0, 10, 128, ctypes.byref(h)) == _lib.LOP_ERR_INVALID
    assert b"pipeline" in lop.lib.lop_last_error()
    assert lop.lib.lop_pipeline_bilateral(None, None, 0, None, 0, 1, 0.0, 3, 3, None, 1.0,
                                          1.0) == _lib.LOP_ERR_INVALID
    assert lop.lib.lop_pipeline_destroy(None) == _lib.LOP_OK


def test_chain_rejects_bad_masks_before_launch():
    bc, acc, is_ = _views()
    bc.size_x = bc.size_y = 7
    m1 = _lib.lop_mask(5, 5, _lib.LOP_F32, None, 0)
    st = lop.lib.lop_convolve_chain_execute(ctypes.byref(is_), ctypes.byref(acc), None,
                                            ctypes.byref(m1), None)
    assert st == _lib.LOP_ERR_INVALID


def test_session5_entry_points_validate_before_launch():
    """The point prologue, SUMSQ, pyramid and multiresolution entry points reject
    bad arguments (host pointers, unknown ops, wrong sizes) without launching;
    the multiresolution workspace size is a pure host function."""
    lib = lop.lib
    before = lop.launch_count()
    host = np.zeros((8, 16), np.float32)
    bc, acc, is_ = _views(data=host.ctypes.data)
    accs = (ctypes.POINTER(_lib.lop_accessor) * 1)(ctypes.pointer(acc))
    m = _lib.lop_mask()
    ms = (ctypes.POINTER(_lib.lop_mask) * 1)(ctypes.pointer(m))
    sc = (ctypes.c_double * 1)(2.0)
    of = (ctypes.c_double * 1)(0.5)
    assert lib.lop_local_execute_point(ctypes.byref(is_), accs, ms, 1, 0, 0, sc, of, None) == \
        _lib.LOP_ERR_INVALID
    assert lib.lop_global_reduce_execute(ctypes.byref(is_), 9, None, None, None) == _lib.LOP_ERR_INVALID
    assert b"SUMSQ" in lib.lop_last_error()
    bc.size_x = bc.size_y = 5
    assert lib.lop_pyramid_reduce_execute(ctypes.byref(is_), ctypes.byref(acc), None) == \
        _lib.LOP_ERR_INVALID
    assert lib.lop_pyramid_expand_execute(ctypes.byref(is_), ctypes.byref(acc), None, 1.0, None) == \
        _lib.LOP_ERR_INVALID
    srs = (ctypes.c_float * 2)(0.1, 0.1)
    assert lib.lop_multires_bilateral_execute(ctypes.byref(is_), ctypes.byref(acc), 0, 1.0, srs, None,
                                              0, None) == _lib.LOP_ERR_INVALID
    assert b"levels" in lib.lop_last_error()
    assert lib.lop_multires_bilateral_execute(ctypes.byref(is_), ctypes.byref(acc), 2, 1.0, srs, None,
                                              0, None) == _lib.LOP_ERR_INVALID
    assert lop.launch_count() == before
    # workspace: the Gaussian levels 1..L-1 plus one full-size level (B_0, later the
    # filtered coarse levels), 256-B rounded; 1 level needs none
    n = ctypes.c_int64(-1)
    assert lib.lop_multires_workspace_bytes(4096, 4096, 1, 1, ctypes.byref(n)) == 0 and n.value == 0
    sizes = []
    for L in (2, 3, 4, 8):
        assert lib.lop_multires_workspace_bytes(4096, 4096, 1, L, ctypes.byref(n)) == 0
        sizes.append(n.value)
    full = 4096 * 4096 * 4
    assert sizes[0] == full + full // 4
    assert all(a < b for a, b in zip(sizes, sizes[1:]))
    assert sizes[-1] < full * 4 // 3 + full + 8 * 256
    assert lib.lop_multires_workspace_bytes(4096, 4096, 2, 3, ctypes.byref(n)) == 0
    assert n.value >= 2 * (full + full // 4)
    assert lib.lop_multires_workspace_bytes(0, 4096, 1, 3, ctypes.byref(n)) == _lib.LOP_ERR_INVALID
    assert lib.lop_multires_workspace_bytes(64, 64, 1, 17, ctypes.byref(n)) == _lib.LOP_ERR_INVALID

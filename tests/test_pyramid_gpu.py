"""GPU parity of the multiresolution filter (PAPER.md
L309-L314; reading c28): lop_pyramid_reduce_execute, lop_pyramid_expand_execute
and lop_multires_bilateral_execute against the oracle (oracle.pyr_reduce /
pyr_expand / multires_bilateral, pinned in tests/test_oracle_pyramid_pins.py).

f32 data in [0, 1]; max |gpu - oracle| <= 1e-5 (north_star's float tolerance)
for every output, all four modes, ragged sizes (odd widths / heights, 1 x 1),
frames; the whole filter at 1024^2 with the paper's 13 x 13 window."""
import numpy as np
import pytest
import torch

import oracle
import synthetic

pytestmark = pytest.mark.gpu

TOL = 1e-5
MODES = ["clamp", "repeat", "mirror", "constant"]
SHAPES = [(1, 1), (2, 3), (5, 7), (17, 64), (33, 70), (130, 257), (1000, 1030)]


@pytest.fixture(scope="module")
def lop():
    import paper_conf_ipps_membarthhtke12_b200 as lop
    return lop


def _err(gpu, ref):
    return float(np.abs(np.asarray(gpu, np.float64) - ref).max()) if ref.size else 0.0


@pytest.mark.parametrize("shape", SHAPES)
@pytest.mark.parametrize("mode", MODES)
def test_reduce(lop, shape, mode):
    img = synthetic.uniform(*shape, seed=shape[0] + 3 * shape[1])
    got = lop.pyramid_reduce(img.cuda(), mode, constant=0.3).cpu().numpy()
    ref = oracle.pyr_reduce(img.numpy(), mode, cval=0.3)
    assert got.shape == ref.shape
    assert _err(got, ref) <= TOL


@pytest.mark.parametrize("shape", SHAPES)
@pytest.mark.parametrize("mode", MODES)
def test_expand_with_and_without_addend(lop, shape, mode):
    H, W = shape
    coarse = synthetic.uniform((H + 1) // 2, (W + 1) // 2, seed=H * 5 + W)
    fine = synthetic.uniform(H, W, seed=H + W + 11)
    e_ref = oracle.pyr_expand(coarse.numpy(), (H, W), mode, cval=0.6)
    e = lop.pyramid_expand(coarse.cuda(), (H, W), mode, constant=0.6).cpu().numpy()
    assert _err(e, e_ref) <= TOL
    band = lop.pyramid_expand(coarse.cuda(), (H, W), mode, constant=0.6, addend=fine.cuda(),
                              sign=-1.0).cpu().numpy()
    assert _err(band, fine.numpy().astype(np.float64) - e_ref) <= TOL
    inplace = fine.cuda()
    lop.pyramid_expand(coarse.cuda(), (H, W), mode, constant=0.6, addend=inplace, sign=1.0,
                       out=inplace)
    assert _err(inplace.cpu().numpy(), fine.numpy().astype(np.float64) + e_ref) <= TOL


def test_reduce_expand_frames(lop):
    frames = torch.stack([synthetic.angio(67, 90, seed=s) for s in range(3)]).cuda()
    red = lop.pyramid_reduce(frames, "mirror")
    exp = lop.pyramid_expand(red, (67, 90), "mirror", addend=frames, sign=-1.0)
    for b in range(3):
        r = oracle.pyr_reduce(frames[b].cpu().numpy(), "mirror")
        assert _err(red[b].cpu().numpy(), r) <= TOL
        ref = frames[b].cpu().numpy() - oracle.pyr_expand(r, (67, 90), "mirror")
        assert _err(exp[b].cpu().numpy(), ref) <= TOL


@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("shape,levels,sigma_d", [((64, 64), 3, 1.0), ((130, 97), 4, 1.0),
                                                  ((45, 200), 2, 2.0), ((9, 13), 5, 1.0),
                                                  ((40, 33), 1, 1.0)])
def test_multires_bilateral(lop, mode, shape, levels, sigma_d):
    img = synthetic.angio(*shape, seed=levels * 100 + shape[1])
    sr = [0.05, 0.1, 0.0, 0.2, 0.3][:levels]
    got = lop.multires_bilateral(img.cuda(), levels, sigma_d, sr, mode, constant=0.4)
    ref = oracle.multires_bilateral(img.numpy(), levels, sigma_d, sr, mode, cval=0.4)
    assert _err(got.cpu().numpy(), ref) <= TOL


@pytest.mark.parametrize("mode", MODES)
def test_multires_perfect_reconstruction(lop, mode):
    img = synthetic.angio(257, 301, seed=3)
    got = lop.multires_bilateral(img.cuda(), 5, 1.0, [0.0] * 5, mode, constant=0.2)
    assert _err(got.cpu().numpy(), img.numpy().astype(np.float64)) <= 2e-6


def test_multires_1024_paper_window(lop):
    """1024^2 angiography frame (config 4's frame size), 4 levels, the paper's
    13 x 13 window (sigma_d = 3), Mirror: every output against the oracle."""
    img = synthetic.angio(1024, 1024, seed=2012004)
    sr = [0.05, 0.08, 0.12, 0.0]
    got = lop.multires_bilateral(img.cuda(), 4, 3.0, sr, "mirror")
    ref = oracle.multires_bilateral(img.numpy(), 4, 3.0, sr, "mirror")
    assert _err(got.cpu().numpy(), ref) <= TOL


def test_multires_frames_and_workspace_reuse(lop):
    frames = torch.stack([synthetic.angio(96, 128, seed=s) for s in (1, 2)]).cuda()
    ws = torch.empty(lop.multires_workspace_bytes(tuple(frames.shape), 3), dtype=torch.uint8,
                     device="cuda")
    a = lop.multires_bilateral(frames, 3, 1.0, [0.1, 0.1, 0.1], workspace=ws)
    b = lop.multires_bilateral(frames, 3, 1.0, [0.1, 0.1, 0.1], workspace=ws)
    assert torch.equal(a, b)
    for i in range(2):
        ref = oracle.multires_bilateral(frames[i].cpu().numpy(), 3, 1.0, [0.1, 0.1, 0.1], "mirror")
        assert _err(a[i].cpu().numpy(), ref) <= TOL


def test_pyramid_validation(lop):
    x = torch.rand(20, 30, device="cuda")
    with pytest.raises(lop.LopError):
        lop.pyramid_reduce(x, "undefined")
    with pytest.raises(lop.LopError):
        lop.pyramid_reduce(x, out=torch.empty(11, 15, device="cuda"))
    with pytest.raises(lop.LopError):
        lop.pyramid_expand(torch.rand(10, 15, device="cuda"), (20, 32))
    with pytest.raises(lop.LopError):
        lop.multires_bilateral(x, 2, 1.0, [0.1, 0.1], workspace=torch.empty(8, dtype=torch.uint8,
                                                                            device="cuda"))
    with pytest.raises(lop.LopError):
        lop.multires_bilateral(x, 0, 1.0, [])
    with pytest.raises(lop.LopError):                  # output aliases the input
        lop.multires_bilateral(x, 2, 1.0, [0.1, 0.1], out=x)

"""The TMEM pair-sharing bilateral kernel (bilateral_pair_tm_kernel, used for
launches of >= 1024^2 pixels with windows >= 9x9) against the generic kernel
(which mirrors the pair kernels' summation order: bit for bit) and against the
oracle on sampled outputs, in every boundary mode, with ROIs, accessor
offsets, frames and the sizes / windows at the TMEM kernel's threshold."""
import numpy as np
import pytest
import torch

import oracle
import synthetic

pytestmark = pytest.mark.gpu

MODES = ["undefined", "clamp", "repeat", "mirror", "constant"]


@pytest.fixture(scope="module")
def lop():
    import paper_conf_ipps_membarthhtke12_b200 as lop
    yield lop
    lop.set_variant("auto")


def _points(H, W, n, seed):
    rng = np.random.default_rng(seed)
    ys = np.concatenate([rng.integers(0, H, n), np.arange(0, H, max(1, H // 40)), [0, H - 1, 0, H - 1]])
    xs = np.concatenate([rng.integers(0, W, n), np.zeros(len(range(0, H, max(1, H // 40))), int),
                         [0, 0, W - 1, W - 1]])
    return ys.astype(np.int64), xs.astype(np.int64)


@pytest.mark.parametrize("win", [9, 13, 15])
@pytest.mark.parametrize("mode", MODES)
def test_tm_kernel_equals_generic_and_oracle(lop, monkeypatch, win, mode):
    monkeypatch.setenv("LOP_BILATERAL_PAIR", "1")       # the pair kernel at this size
    H, W = 1100, 1030                                  # 1.13 M pixels: the TMEM kernel
    img = synthetic.angio(H, W, seed=win * 7 + len(mode)).cuda()
    sd = (win - 1) / 4.0
    a = lop.bilateral(img, sd, 0.1, mode, constant=0.3, size=win)
    lop.set_variant("generic")
    b = lop.bilateral(img, sd, 0.1, mode, constant=0.3, size=win)
    lop.set_variant("auto")
    assert torch.equal(a, b)
    ys, xs = _points(H, W, 300, win)
    ref, valid = oracle.bilateral_f32_points(img.cpu().numpy(), sd, 0.1, mode, xs, ys, cval=0.3,
                                             size=win)
    got = a.cpu().numpy()[ys, xs]
    sel = valid if mode == "undefined" else np.ones_like(valid)
    assert float(np.abs(got[sel] - ref[sel]).max()) <= 1e-5


def test_tm_kernel_roi_offset_frames(lop, monkeypatch):
    monkeypatch.setenv("LOP_BILATERAL_PAIR", "1")
    H, W = 1030, 1100
    frames = torch.stack([synthetic.angio(H, W, seed=s) for s in (1, 2)]).cuda()
    roi = (37, 21, 801, 900)
    out = torch.zeros_like(frames)
    lop.bilateral(frames, 3.0, 0.1, "mirror", out=out, roi=roi, offset=(2, -3))
    lop.set_variant("generic")
    ref_gen = torch.zeros_like(frames)
    lop.bilateral(frames, 3.0, 0.1, "mirror", out=ref_gen, roi=roi, offset=(2, -3))
    lop.set_variant("auto")
    assert torch.equal(out, ref_gen)
    x0, y0, w, h = roi
    assert float(out[:, :y0].abs().max()) == 0.0 and float(out[:, :, :x0].abs().max()) == 0.0
    # whole-image call: the ROI outputs are the same bits (the kernel choice keys on the image)
    full = lop.bilateral(frames, 3.0, 0.1, "mirror", offset=(2, -3))
    assert torch.equal(full[:, y0:y0 + h, x0:x0 + w], out[:, y0:y0 + h, x0:x0 + w])
    ys, xs = _points(h, w, 200, 5)
    ys, xs = ys + y0, xs + x0
    for f in range(2):
        img = frames[f].cpu().numpy()
        # offset accessor: output (x, y) reads input (x + 2, y - 3); the oracle on the
        # shifted points with the mode's index map equals it for mirror
        ref, _ = oracle.bilateral_f32_points(img, 3.0, 0.1, "mirror", xs + 2, ys - 3)
        got = out[f].cpu().numpy()[ys, xs]
        assert float(np.abs(got - ref).max()) <= 1e-5


@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("win", [9, 13])
def test_tight_frames_bit_identical(lop, monkeypatch, mode, win):
    """TIGHT frames (frame columns [R, R + OWT)) and lane-aligned frames give the
    same bits: the summation order depends on x mod 4 only.  ROI with an odd
    start, accessor offset, two frames."""
    monkeypatch.setenv("LOP_BILATERAL_PAIR", "1")
    frames = torch.stack([synthetic.angio(1030, 1057, seed=s) for s in (3, 4)]).cuda()
    roi = (13, 9, 1001, 1000)
    outs = []
    for tight in ("0", "1"):
        monkeypatch.setenv("LOP_PAIR_TIGHT", tight)
        o = torch.zeros_like(frames)
        lop.bilateral(frames, (win - 1) / 4.0, 0.1, mode, constant=0.3, size=win, out=o, roi=roi,
                      offset=(1, -2))
        outs.append(o)
    assert torch.equal(outs[0], outs[1])
    x0, y0, w, h = roi
    assert float(outs[1][:, :, x0 + w:].abs().max()) == 0.0    # nothing stored past the ROI

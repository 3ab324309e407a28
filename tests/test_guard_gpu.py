"""Guard-band checks of the session-5 kernels (compute-sanitizer is not
available on the GPU pool): every image view sits inside a larger buffer whose
border is NaN (inputs) or a sentinel (outputs).  A read outside the view would
pull a NaN into some output (caught by the oracle comparison, which requires
finite values within 1e-5); a write outside the view would change the
sentinel.  Covers the TMEM pair-sharing bilateral kernel, the pyramid REDUCE /
EXPAND kernels, the multiresolution filter, the local operator's point
prologue and the global SUMSQ merge, with aligned and unaligned row pitches."""
import numpy as np
import pytest
import torch

import oracle
import synthetic

pytestmark = pytest.mark.gpu

SENT = -12345.0


@pytest.fixture(scope="module")
def lop():
    import paper_conf_ipps_membarthhtke12_b200 as lop
    return lop


def _guarded(img, g, fill, frames=1):
    """(view, buffer): img (H, W) inside a buffer padded by g on every side."""
    H, W = img.shape[-2:]
    buf = torch.full((frames, H + 2 * g, W + 2 * g) if frames > 1 else (H + 2 * g, W + 2 * g),
                     fill, dtype=img.dtype, device="cuda")
    view = buf[..., g:g + H, g:g + W]
    view.copy_(img.cuda())
    return view, buf


def _out(H, W, g):
    buf = torch.full((H + 2 * g, W + 2 * g), SENT, device="cuda")
    return buf[g:g + H, g:g + W], buf


def _pad_intact(buf, g, H, W):
    b = buf.clone()
    b[g:g + H, g:g + W] = SENT
    return bool((b == SENT).all())


@pytest.mark.parametrize("g", [4, 3])                       # aligned / unaligned row pitch
@pytest.mark.parametrize("mode", ["clamp", "mirror", "repeat", "constant"])
def test_pair_tm_bilateral_guard(lop, monkeypatch, g, mode):
    monkeypatch.setenv("LOP_BILATERAL_PAIR", "1")
    H, W = 150, 203
    img = synthetic.angio(H, W, seed=g + 5)
    x, _ = _guarded(img, g, float("nan"))
    o, ob = _out(H, W, g)
    lop.bilateral(x, 3.0, 0.1, mode, constant=0.25, out=o)
    got = o.cpu().numpy()
    assert np.isfinite(got).all()
    assert _pad_intact(ob, g, H, W)
    ref, _ = oracle.bilateral_f32(img.numpy(), 3.0, 0.1, mode, cval=0.25)
    assert float(np.abs(got - ref).max()) <= 1e-5


@pytest.mark.parametrize("g", [4, 3])
@pytest.mark.parametrize("shape", [(1, 1), (37, 53), (130, 257)])
def test_pyramid_guard(lop, g, shape):
    H, W = shape
    img = synthetic.uniform(H, W, seed=H + W)
    x, _ = _guarded(img, g, float("nan"))
    Hc, Wc = (H + 1) // 2, (W + 1) // 2
    c, cb = _out(Hc, Wc, g)
    lop.pyramid_reduce(x, "mirror", out=c)
    assert _pad_intact(cb, g, Hc, Wc) and torch.isfinite(c).all()
    assert float(np.abs(c.cpu().numpy() - oracle.pyr_reduce(img.numpy(), "mirror")).max()) <= 1e-5
    cg, _ = _guarded(c.clone(), g, float("nan"))
    e, eb = _out(H, W, g)
    lop.pyramid_expand(cg, (H, W), "mirror", addend=x, sign=-1.0, out=e)
    assert _pad_intact(eb, g, H, W) and torch.isfinite(e).all()
    ref = img.numpy().astype(np.float64) - oracle.pyr_expand(c.cpu().numpy(), (H, W), "mirror")
    assert float(np.abs(e.cpu().numpy() - ref).max()) <= 1e-5
    o, obuf = _out(H, W, g)
    lop.multires_bilateral(x, 3, 1.0, [0.05, 0.1, 0.2], "mirror", out=o)
    assert _pad_intact(obuf, g, H, W) and torch.isfinite(o).all()
    refm = oracle.multires_bilateral(img.numpy(), 3, 1.0, [0.05, 0.1, 0.2], "mirror")
    assert float(np.abs(o.cpu().numpy() - refm).max()) <= 1e-5


def test_point_prologue_and_sumsq_guard(lop):
    H, W = 70, 131
    img = synthetic.uniform(H, W, seed=7)
    x, _ = _guarded(img, 3, float("nan"))
    o, ob = _out(H, W, 3)
    m = [np.full((5, 3), 0.05, np.float32)]
    lop.local([x], m, "sum", "sqdiff", "mirror", point=[(-0.5, 0.75)], out=o)
    assert _pad_intact(ob, 3, H, W)
    ref, _ = oracle.local([img.numpy()], m, "sum", "sqdiff", "mirror", point=[(-0.5, 0.75)])
    assert float(np.abs(o.cpu().numpy() - ref).max()) <= 1e-5
    s = lop.global_reduce(x, "sumsq").item()
    r = oracle.global_reduce(img.numpy(), "sumsq")
    assert abs(s - r) <= 1e-12 * r

"""GPU parity of lop_local_execute -- the local operator over several
Accessors with a per-tap function (PAPER.md L556-L558,
Listing 9) -- against oracle.local (tests/test_oracle_local_pins.py pins it).

f32: max |gpu - oracle| <= 1e-5 with masks normalised so that |out| <= 1
(north_star's float tolerance); u8 -> i32: bit-exact.  The tiled kernel
(shared-memory staging) and the generic kernel are bit-identical.  Undefined
mode: only outputs whose windows stay inside are compared (reading c9)."""
import numpy as np
import pytest
import torch

import oracle
import synthetic

pytestmark = pytest.mark.gpu

TOL = 1e-5
MODES = ["undefined", "clamp", "repeat", "mirror", "constant"]
OPS = ["sum", "min", "max"]
FNS = ["product", "absdiff", "sqdiff", "square"]


@pytest.fixture(scope="module")
def lop():
    import paper_conf_ipps_membarthhtke12_b200 as lop
    yield lop
    lop.set_variant("auto")


def _masks(rng, sizes, u8, holes=True):
    out = []
    for (sy, sx) in sizes:
        if u8:
            m = rng.integers(-4, 5, (sy, sx)).astype(np.int32)
        else:
            m = rng.normal(size=(sy, sx))
            m = (m / np.abs(m).sum() / len(sizes)).astype(np.float32)   # |out| <= 1
        if holes and sy * sx > 1:
            m[0, 0] = 0
        if not np.any(m):
            m[sy // 2, sx // 2] = 1
        out.append(m)
    return out


def _compare(gpu, ref, valid, u8, mode_list):
    gpu = np.asarray(gpu)
    if "undefined" in mode_list:
        gpu, ref = gpu[valid], ref[valid]
    if u8:
        assert np.array_equal(gpu.astype(np.int64), ref)
    elif gpu.size:
        err = float(np.abs(gpu.astype(np.float64) - ref).max())
        assert err <= TOL, err


def _run(lop, imgs_host, masks, op, fn, modes, consts, offsets, u8, roi=None):
    dev = [t.cuda() for t in imgs_host]
    out = lop.local(dev, masks, op, fn, modes, consts, offsets, roi=roi)
    ref, valid = oracle.local([t.numpy() for t in imgs_host], masks, op, fn, modes, consts, offsets)
    return out.cpu().numpy(), ref, valid


SHAPES = [(1, 1), (1, 9), (7, 1), (5, 6), (33, 70), (67, 131)]


@pytest.mark.parametrize("shape", SHAPES)
@pytest.mark.parametrize("op", OPS)
@pytest.mark.parametrize("fn", FNS)
def test_local_f32_small_shapes_two_accessors(lop, shape, op, fn):
    H, W = shape
    rng = np.random.default_rng(H * 100 + W)
    a, b = synthetic.uniform(H, W, seed=1), synthetic.uniform(H, W, seed=2)
    masks = _masks(rng, [(3, 5), (5, 3)], False)
    for modes, offs in ((["clamp", "repeat"], [(0, 0), (1, -1)]),
                        (["mirror", "constant"], [(-2, 0), (0, 2)]),
                        (["undefined", "undefined"], [(0, 0), (0, 0)])):
        got, ref, valid = _run(lop, [a, b], masks, op, fn, modes, [0.25, 0.75], offs, False)
        _compare(got, ref, valid, False, modes)


@pytest.mark.parametrize("op", OPS)
@pytest.mark.parametrize("fn", FNS)
def test_local_u8_exact(lop, op, fn):
    rng = np.random.default_rng(5)
    H, W = 45, 133
    imgs = [synthetic.uniform_u8(H, W, seed=s) for s in (3, 4, 5)]
    masks = _masks(rng, [(3, 3), (1, 7), (5, 5)], True)
    got, ref, valid = _run(lop, imgs, masks, op, fn, ["clamp", "mirror", "constant"], [0, 0, 200],
                           [(0, 0), (3, 1), (-1, -2)], True)
    _compare(got, ref, valid, True, [])


@pytest.mark.parametrize("K", [1, 2, 3, 4])
@pytest.mark.parametrize("mode", MODES)
def test_local_accessor_counts_and_windows(lop, K, mode):
    """K accessors with different windows (the largest sets the halo,
    L556-L558), including windows larger than the image."""
    rng = np.random.default_rng(K * 10)
    H, W = 40, 37
    imgs = [synthetic.angio(H, W, seed=20 + k) for k in range(K)]
    sizes = [(1, 1), (3, 9), (15, 7), (31, 31)][:K]
    masks = _masks(rng, sizes, False, holes=False)
    got, ref, valid = _run(lop, imgs, masks, "sum", "sqdiff", [mode] * K, [0.5] * K,
                           [(k - 1, 1 - k) for k in range(K)], False)
    _compare(got, ref, valid, False, [mode])


def test_local_tiled_equals_generic_bit_for_bit(lop):
    rng = np.random.default_rng(9)
    H, W = 130, 300
    imgs = [synthetic.angio(H, W, seed=s).cuda() for s in (7, 8)]
    masks = _masks(rng, [(5, 5), (3, 7)], False)
    for op in OPS:
        for fn in FNS:
            lop.set_variant("tiled")
            a = lop.local(imgs, masks, op, fn, ["mirror", "repeat"], offsets=[(2, 1), (0, 0)])
            lop.set_variant("generic")
            b = lop.local(imgs, masks, op, fn, ["mirror", "repeat"], offsets=[(2, 1), (0, 0)])
            lop.set_variant("auto")
            assert torch.equal(a, b), (op, fn)


def test_local_roi_frames_and_band_views(lop):
    rng = np.random.default_rng(11)
    H, W = 96, 160
    fa = torch.stack([synthetic.angio(H, W, seed=s) for s in (1, 2, 3)]).cuda()
    fb = torch.stack([synthetic.uniform(H, W, seed=s) for s in (4, 5, 6)]).cuda()
    masks = _masks(rng, [(5, 5), (3, 3)], False)
    out = lop.local([fa, fb], masks, "sum", "absdiff", ["clamp", "mirror"])
    for f in range(3):
        single = lop.local([fa[f].contiguous(), fb[f].contiguous()], masks, "sum", "absdiff",
                           ["clamp", "mirror"])
        assert torch.equal(out[f], single)
    whole = out[1]
    roi = lop.local([fa[1].contiguous(), fb[1].contiguous()], masks, "sum", "absdiff",
                    ["clamp", "mirror"], roi=(17, 9, 100, 50))
    assert torch.equal(roi[9:59, 17:117], whole[9:59, 17:117])
    ref, _ = oracle.local([fa[1].cpu().numpy(), fb[1].cpu().numpy()], masks, "sum", "absdiff",
                          ["clamp", "mirror"])
    assert float(np.abs(whole.cpu().numpy() - ref).max()) <= TOL


@pytest.mark.parametrize("mode", MODES)
def test_local_band_views_bit_identical(lop, mode):
    """Row bands of both accessors (halo rows in place; REPEAT ring rows at
    the ends) reproduce the whole-image output bit for bit -- the largest
    window (7 rows here) sets the halo the band must hold (L556-L558)."""
    rng = np.random.default_rng(13)
    H, W = 120, 150
    a = synthetic.angio(H, W, seed=31).cuda()
    b = synthetic.uniform(H, W, seed=32).cuda()
    masks = _masks(rng, [(3, 5), (7, 3)], False)
    kw = dict(op="sum", fn="sqdiff", modes=[mode, mode], constants=[0.5, 0.25])
    whole = lop.local([a, b], masks, **kw)
    r = 3                                                   # the largest window: 7 rows
    for y0, y1 in ((0, 17), (17, 64), (64, 120)):
        top = r if (y0 > 0 or mode == "repeat") else 0
        bot = r if (y1 < H or mode == "repeat") else 0
        rows = [(y % H) for y in range(y0 - top, y1 + bot)]
        ba = a[rows].contiguous()[top:top + (y1 - y0)]
        bb = b[rows].contiguous()[top:top + (y1 - y0)]
        out = lop.local([ba, bb], masks, band=[(top, bot, y0, H)] * 2, **kw)
        assert torch.equal(out, whole[y0:y1]), (mode, y0, y1)


def test_local_4096_sampled(lop):
    """The bench case: two 4096^2 f32 frames, SUM of PRODUCT with a 5x5 and a
    3x3 mask (a temporal-spatial average of consecutive angiography frames)."""
    H = W = 4096
    a = synthetic.angio(H, W, seed=synthetic.config_seed(2), device="cuda")
    b = synthetic.angio(H, W, seed=synthetic.config_seed(2) + 1, device="cuda")
    masks = [np.full((5, 5), 0.5 / 25, np.float32), np.full((3, 3), 0.5 / 9, np.float32)]
    out = lop.local([a, b], masks, "sum", "product", "clamp").cpu().numpy()
    rng = np.random.default_rng(3)
    ys = np.concatenate([rng.integers(0, H, 3000), np.arange(64), H - 1 - np.arange(64)])
    xs = np.concatenate([rng.integers(0, W, 3000), np.zeros(64, int), np.full(64, W - 1)])
    ah, bh = a.cpu().numpy(), b.cpu().numpy()
    # the oracle on the sampled rows only (one output row per call)
    for y, x in zip(ys[::50], xs[::50]):
        ref, _ = oracle.local([ah, bh], masks, "sum", "product", "clamp", rows=(y, y + 1))
        assert abs(float(out[y, x]) - ref[0, x]) <= TOL


def test_local_validation(lop):
    x = torch.rand(20, 30, device="cuda")
    u = torch.zeros(20, 30, dtype=torch.uint8, device="cuda")
    m = np.ones((3, 3), np.float32) / 9
    with pytest.raises(lop.LopError, match="same dtype"):
        lop.local([x, u], [m, np.ones((3, 3), np.int32)])
    with pytest.raises(lop.LopError, match="n_inputs"):
        lop.local([x] * 5, [m] * 5)
    with pytest.raises(lop.LopError, match="non-zero"):
        lop.local([x], [np.zeros((3, 3), np.float32)], "min")
    with pytest.raises(lop.LopError, match="overlap"):
        lop.local([x], [m], out=x)
    with pytest.raises(lop.LopError, match="overflow"):
        lop.local([u], [np.full((31, 31), 4000, np.int32)], "sum", "square")


# ------------------------------- point-operator prologue (reading c27, N3) ----

@pytest.mark.parametrize("shape", [(1, 1), (5, 6), (67, 131), (260, 517)])
@pytest.mark.parametrize("fn", FNS)
def test_local_point_prologue_f32(lop, shape, fn):
    """Read'_k = a_k Read_k + b_k on every read of accessor k (centre and
    boundary constant included) against oracle.local(point=...), all modes,
    both tiled kernels and the generic kernel (bit-identical to each other)."""
    H, W = shape
    rng = np.random.default_rng(H + W)
    a, b = synthetic.uniform(H, W, seed=31), synthetic.uniform(H, W, seed=32)
    masks = _masks(rng, [(5, 5), (3, 7)], False)
    point = [(-0.5, 0.75), (1.0, -0.25)]                    # f32-exact scale / offset
    for modes, offs in ((["clamp", "constant"], [(0, 0), (1, -1)]),
                        (["mirror", "repeat"], [(-2, 0), (0, 2)]),
                        (["undefined", "undefined"], [(0, 0), (0, 0)])):
        outs = []
        for variant in ("auto", "generic"):
            lop.set_variant(variant)
            outs.append(lop.local([a.cuda(), b.cuda()], masks, "sum", fn, modes, [0.25, 0.5], offs,
                                  point=point))
        lop.set_variant("auto")
        assert torch.equal(outs[0], outs[1]), modes
        ref, valid = oracle.local([a.numpy(), b.numpy()], masks, "sum", fn, modes, [0.25, 0.5],
                                  offs, point=point)
        _compare(outs[0].cpu().numpy(), ref, valid, False, modes)
    # windows wider than 7 take the tiled (not the register-blocked) kernel
    big = _masks(rng, [(11, 9)], False)
    for op in OPS:
        got = lop.local([a.cuda()], big, op, fn, "mirror", point=[(2.0, -1.0)])
        ref, valid = oracle.local([a.numpy()], big, op, fn, "mirror", point=[(2.0, -1.0)])
        _compare(got.cpu().numpy(), ref, valid, False, ["mirror"])


@pytest.mark.parametrize("op", OPS)
@pytest.mark.parametrize("fn", FNS)
def test_local_point_prologue_u8_exact(lop, op, fn):
    """u8: integer prologues (inversion 255 - v, gain 3 v) are exact."""
    rng = np.random.default_rng(41)
    H, W = 45, 133
    imgs = [synthetic.uniform_u8(H, W, seed=s) for s in (43, 44)]
    masks = _masks(rng, [(3, 3), (5, 5)], True)
    point = [(-1, 255), (3, -7)]
    got = lop.local([t.cuda() for t in imgs], masks, op, fn, ["clamp", "constant"], [0, 200],
                    [(0, 0), (2, -1)], point=point)
    ref, valid = oracle.local([t.numpy() for t in imgs], masks, op, fn, ["clamp", "constant"],
                              [0, 200], [(0, 0), (2, -1)], point=point)
    _compare(got.cpu().numpy(), ref, valid, True, [])


def test_local_point_prologue_identity_and_validation(lop):
    """scale 1 / offset 0 is bit-identical to lop_local_execute; non-integer
    u8 prologues and int32 overflow are rejected."""
    x = synthetic.angio(64, 96, seed=5).cuda()
    m = [np.full((3, 3), 1.0 / 9, np.float32)]
    assert torch.equal(lop.local([x], m, point=[(1.0, 0.0)]), lop.local([x], m))
    u = synthetic.uniform_u8(16, 16, seed=6).cuda()
    mi = [np.ones((3, 3), np.int32)]
    with pytest.raises(lop.LopError):
        lop.local([u], mi, point=[(0.5, 0)])
    with pytest.raises(lop.LopError):
        lop.local([u], [np.full((31, 31), 1000, np.int32)], fn="square", point=[(4, 0)])
    with pytest.raises(ValueError):
        lop.local([u], mi, point=[(1, 0), (1, 0)])

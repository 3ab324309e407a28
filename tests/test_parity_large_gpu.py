"""GPU parity at BASELINE.json's full partitioned sizes (configs 4 and 5), in
the launch configuration bench.py times, against the CPU oracle on sampled
outputs ("Next round" item 2).

These are the sizes where 32-bit byte offsets would overflow: a 32768^2 f32
image is 4 GiB (row 32767 starts 4.29e9 bytes in, > 2^32) and frame 1023 of
a 1024 x 1024^2 batch starts at 1023 * 4 MiB > 2^32.  Sampled outputs:
the last rows, every P = 8 band seam +- 6 rows (the rows whose windows cross
a seam), the four corners, the image borders and random interior points;
computed one by one by the oracle (oracle.bilateral_f32_points).
"""
import numpy as np
import pytest
import torch

import oracle
import synthetic

pytestmark = pytest.mark.gpu

TOL = 1e-5
R = 6                      # 13 x 13 window


@pytest.fixture(scope="module")
def lop():
    import paper_conf_ipps_membarthhtke12_b200 as lop
    yield lop


def _cmp(gpu_vals, ref, tol=TOL):
    err = float(np.abs(np.asarray(gpu_vals, np.float64) - ref).max())
    assert err <= tol, "max abs err %.3g > %.1g" % (err, tol)
    return err


def _c5_points(H, W, P, seed):
    rng = np.random.default_rng(seed)
    pts = set()
    xs_sparse = list(range(0, W, 61)) + list(range(0, 2 * R + 2)) + list(range(W - 2 * R - 2, W))
    # the last rows (largest byte offsets) and the first rows
    for y in list(range(H - R - 2, H)) + list(range(0, R + 2)):
        pts.update((y, x) for x in xs_sparse)
    # every band seam of a P-way split +- R rows
    for k in range(1, P):
        s = H * k // P
        for y in range(s - R - 1, s + R + 1):
            pts.update((y, x) for x in xs_sparse[::2])
    # left / right borders
    for x in list(range(0, R + 2)) + list(range(W - R - 2, W)):
        pts.update((int(y), x) for y in rng.integers(0, H, 256))
    # corners
    for cy in (0, H - 1):
        for cx in (0, W - 1):
            for dy in range(-R, R + 1):
                for dx in range(-R, R + 1):
                    y, x = cy + dy, cx + dx
                    if 0 <= y < H and 0 <= x < W:
                        pts.add((y, x))
    pts.update(zip(rng.integers(0, H, 3000).tolist(), rng.integers(0, W, 3000).tolist()))
    pts = np.array(sorted(pts))
    return pts[:, 0], pts[:, 1]


@pytest.fixture(scope="module")
def c5_image():
    H = W = 32768
    img = synthetic.angio(H, W, seed=synthetic.config_seed(5), device="cuda")
    yield img
    del img
    torch.cuda.empty_cache()


@pytest.mark.parametrize("mode", ["clamp", "repeat"])
def test_config5_32768_whole_image_and_p8_bands(lop, c5_image, mode):
    """Config 5: the whole 32768^2 image on one GPU (bench.py's N = 1 step)
    against the oracle on sampled outputs, and the P = 8 row-band views
    (halo rows = the neighbours' rows, REPEAT ring rows at the ends) bit-
    identical to it at every seam."""
    img = c5_image
    H, W = img.shape
    P = 8
    out = lop.bilateral(img, 3.0, 5.0, mode, size=13)
    torch.cuda.synchronize()
    host = img.cpu().numpy()
    ys, xs = _c5_points(H, W, P, seed=5)
    got = out[torch.from_numpy(ys).cuda(), torch.from_numpy(xs).cuda()].cpu().numpy()
    ref, _ = oracle.bilateral_f32_points(host, 3.0, 5.0, mode, xs, ys)
    _cmp(got, ref)
    # small sigma_r at the seams and the last rows (the range term matters, reading c3)
    d = ys % (H // P)
    sel = (ys >= H - R - 2) | (d <= R + 1) | (d >= H // P - R - 1)
    out2 = lop.bilateral(img, 3.0, 0.05, mode, size=13)
    got2 = out2[torch.from_numpy(ys[sel]).cuda(), torch.from_numpy(xs[sel]).cuda()].cpu().numpy()
    ref2, _ = oracle.bilateral_f32_points(host, 3.0, 0.05, mode, xs[sel], ys[sel])
    _cmp(got2, ref2)
    del out2
    # P = 8 band views: rank r's buffer = its rows with R halo rows above/below
    for r in range(P):
        y0, y1 = H * r // P, H * (r + 1) // P
        top = R if (r > 0 or mode == "repeat") else 0
        bot = R if (r < P - 1 or mode == "repeat") else 0
        if mode == "repeat" and (r == 0 or r == P - 1):
            rows = torch.tensor([(y % H) for y in range(y0 - top, y1 + bot)], device="cuda")
            buf = img.index_select(0, rows)
            band = buf[top:top + (y1 - y0)]
        else:
            band = img[y0:y1]                       # halo rows: the neighbours' rows in place
        ob = lop.bilateral(band, 3.0, 5.0, mode, size=13, band=(top, bot, y0, H))
        # the rows next to the seams (and the whole band's first / last rows)
        for a, b in ((0, 2 * R + 1), (y1 - y0 - 2 * R - 1, y1 - y0)):
            assert torch.equal(ob[a:b], out[y0 + a:y0 + b]), (r, a, b)
        assert torch.equal(ob[::97], out[y0:y1:97]), r
        del ob
    del out
    torch.cuda.empty_cache()


def test_config4_last_frames_of_1024(lop, monkeypatch):
    """Config 4: 1024 frames of 1024^2 in one batched launch (bench.py's
    N = 1 step); the last frames -- beyond 2^32 bytes -- against the oracle
    (frame 1023 every output, frames 1020-1022 sampled), and bit-identical to
    single-frame calls."""
    F, S = 1024, 1024
    frames = synthetic.angio_frames(F, S, S, seed=synthetic.config_seed(4), device="cuda")
    out = lop.bilateral(frames, 3.0, 5.0, "clamp", size=13)
    torch.cuda.synchronize()
    last = frames[F - 1].cpu().numpy()
    ref, _ = oracle.bilateral_f32(last, 3.0, 5.0, "clamp", size=13)
    _cmp(out[F - 1].cpu().numpy(), ref)
    rng = np.random.default_rng(4)
    for f in (0, 511, 1020, 1021, 1022):
        host = frames[f].cpu().numpy()
        ys = np.concatenate([rng.integers(0, S, 1500), np.zeros(64, int), np.full(64, S - 1)])
        xs = np.concatenate([rng.integers(0, S, 1500), rng.integers(0, S, 128)])
        got = out[f].cpu().numpy()[ys, xs]
        ref, _ = oracle.bilateral_f32_points(host, 3.0, 5.0, "clamp", xs, ys, size=13)
        _cmp(got, ref)
    # one 1024^2 frame alone takes the unshared kernel (N1 rule, whole-launch
    # size); forced to the batch's pair kernel it reproduces the batch bit for bit
    monkeypatch.setenv("LOP_BILATERAL_PAIR", "1")
    for f in (0, 1023):
        assert torch.equal(out[f], lop.bilateral(frames[f].contiguous(), 3.0, 5.0, "clamp",
                                                 size=13))
    del frames, out
    torch.cuda.empty_cache()

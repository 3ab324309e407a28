"""Small launches of the round-2 kernels for compute-sanitizer (memcheck /
racecheck / initcheck): the local operator over several accessors (register-
blocked, tiled and generic kernels; every mode, offsets, windows up to 31x31,
images smaller than the window, ragged tails, ROI, frames, band views) and the
chain's two-pass workspace route."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import synthetic  # noqa: E402
import paper_conf_ipps_membarthhtke12_b200 as lop  # noqa: E402

MODES = ["undefined", "clamp", "repeat", "mirror", "constant"]
n = 0
for variant in ("auto", "generic"):
    lop.set_variant(variant)
    for H, W in ((1, 1), (3, 2), (13, 17), (70, 257), (131, 301)):
        a = synthetic.uniform(H, W, seed=H + W).cuda()
        b = synthetic.uniform(H, W, seed=H * W + 1).cuda()
        ua = synthetic.uniform_u8(H, W, seed=H).cuda()
        ub = synthetic.uniform_u8(H, W, seed=W).cuda()
        for mode in MODES:
            for sizes in (((3, 3), (5, 5)), ((1, 7), (15, 3)), ((31, 31), (3, 1))):
                m = [np.full(sz, 0.01, np.float32) for sz in sizes]
                mi = [np.ones(sz, np.int32) for sz in sizes]
                for op, fn in (("sum", "product"), ("max", "absdiff"), ("min", "sqdiff")):
                    lop.local([a, b], m, op, fn, mode, 0.5, offsets=[(1, -2), (0, 3)])
                    lop.local([ua, ub], mi, op, fn, mode, 7, offsets=[(-1, 0), (2, 1)])
                    n += 2
        if H > 20:
            lop.local([a, b], [np.ones((5, 5), np.float32)] * 2, "sum", "square", "mirror",
                      roi=(3, 5, W - 9, H - 12))
            buf = torch.stack([a, b])
            lop.local([buf, buf.flip(0).contiguous()], [np.ones((3, 3), np.float32)] * 2)
            n += 2
lop.set_variant("auto")
img = synthetic.angio(130, 600, seed=3).cuda()
u8 = synthetic.to_u8(img)
g5, _ = lop.gaussian_mask(5, np.float32)
gi, gk = lop.gaussian_mask(5, np.int32)
for mode in MODES:
    lop.convolve_chain(img, g5, lop.sobel_mask(0, np.float32), mode, constant=0.5)
    lop.convolve_chain(u8, gi, lop.sobel_mask(1, np.int32), mode, constant=9, shift1=gk,
                       out_dtype=torch.int32)
    n += 2
torch.cuda.synchronize()
print("sanitize_local ok: %d calls" % n)

"""Small launches of every kernel variant for compute-sanitizer (memcheck /
racecheck / initcheck): all boundary modes (Undefined must stay memory-safe),
images smaller than the window, ragged tails, ROI, band views, frames."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import synthetic  # noqa: E402
import paper_conf_ipps_membarthhtke12_b200 as lop  # noqa: E402

MODES = ["undefined", "clamp", "repeat", "mirror", "constant"]
shapes = [(1, 1), (3, 2), (13, 17), (70, 257), (131, 600)]
n = 0
for variant in ("generic", "tiled"):
    lop.set_variant(variant)
    for H, W in shapes:
        img = synthetic.uniform(H, W, seed=H + W).cuda()
        u8 = synthetic.uniform_u8(H, W, seed=H * W).cuda()
        for mode in MODES:
            for size in (3, 13):
                lop.bilateral(img, 3.0, 0.1, mode, constant=0.5, size=size)
                n += 1
            lop.bilateral(img, 3.0, 0.1, mode, mask=np.ones((5, 7), np.float32))
            lop.gaussian(img, 5, mode, constant=0.5)
            lop.gaussian(u8, 5, mode, constant=3)
            lop.sobel(u8, 1, mode, constant=3)
            n += 4
lop.set_variant("auto")
# ROI, offsets, frames, band views
img = synthetic.angio(90, 203, seed=1).cuda()
lop.bilateral(img, 2.0, 0.1, "mirror", size=9, roi=(5, 3, 101, 77))
lop.gaussian(img, 5, "clamp", offset=(3, -2))
frames = torch.stack([img, img, img])
lop.bilateral(frames, 3.0, 5.0, "repeat")
lop.gaussian(frames, 3, "constant")
buf = synthetic.angio(112, 203, seed=2).cuda()
band = buf[6:106]
lop.bilateral(band, 3.0, 0.1, "clamp", band=(6, 6, 40, 300))
lop.gaussian(band, 5, "repeat", band=(6, 6, 40, 300))
n += 6
# session 4: SWAR variants, local MIN / MAX, fused chains (tile and row-streaming)
for H, W in ((13, 17), (70, 257), (67, 1040)):
    img = synthetic.uniform(H, W, seed=H + 3 * W).cuda()
    u8 = synthetic.uniform_u8(H, W, seed=H * 7 + W).cuda()
    for mode in MODES:
        for v in ("generic", "tiled"):
            lop.set_variant(v)
            lop.erode(u8, 9, mode, constant=5)
            lop.dilate(img, 3, mode, constant=0.5)
            if v == "generic":
                lop.reduce(u8, [[0, 1, 0], [1, 1, 1], [0, 1, 1]], "min", mode)
            n += 3
        lop.set_variant("auto")
        lop.gaussian(u8, 3, mode, constant=9)                      # plain SWAR
        lop.convolve(u8, np.outer([1, 2, 3, 2, 1], [1, 2, 3, 2, 1]).astype(np.int32), mode,
                     shift=8)                                         # palindromic shift-8 SWAR
        gf, _ = lop.gaussian_mask(5, np.float32)
        gi, gk = lop.gaussian_mask(5, np.int32)
        for st in ("0", "1"):
            os.environ["LOP_CHAIN_STREAM"] = st
            lop.convolve_chain(img, gf, lop.sobel_mask(0, np.float32, fused=True), mode, constant=0.5)
            lop.convolve_chain(u8, gi, lop.sobel_mask(1, np.int32, fused=True), mode, constant=9, shift1=gk,
                               out_dtype=torch.int32)
            n += 2
        os.environ.pop("LOP_CHAIN_STREAM")
        n += 2
torch.cuda.synchronize()
print("sanitize probe: %d calls ok" % n)

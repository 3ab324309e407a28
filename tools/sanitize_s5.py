"""Small launches of the session-5 kernels for compute-sanitizer (memcheck /
racecheck / initcheck): the TMEM pair-sharing bilateral kernel (every mode,
windows 3..15, ROI, frames, band views, images smaller than the window), the
pyramid REDUCE / EXPAND kernels and the multiresolution filter (ragged sizes,
every pyramid mode, frames, in-place EXPAND), the local operator's point
prologue and the global SUMSQ merge."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import synthetic  # noqa: E402
import paper_conf_ipps_membarthhtke12_b200 as lop  # noqa: E402

MODES = ["undefined", "clamp", "repeat", "mirror", "constant"]
PMODES = MODES[1:]
n = 0
os.environ["LOP_BILATERAL_PAIR"] = "1"          # the pair kernel at every size
for H, W in ((1, 1), (5, 9), (40, 37), (130, 301)):
    x = synthetic.angio(H, W, seed=H + W).cuda()
    for mode in MODES:
        for win in (3, 7, 13, 15):
            lop.bilateral(x, (win - 1) / 4.0, 0.1, mode, constant=0.5, size=win)
            n += 1
    if H > 20:
        lop.bilateral(x, 3.0, 0.1, "mirror", roi=(3, 5, W - 9, H - 12))
        lop.bilateral(torch.stack([x, x.flip(0).contiguous()]), 3.0, 0.1, "repeat")
        n += 2
    for mode in PMODES:
        c = lop.pyramid_reduce(x, mode, constant=0.3)
        e = lop.pyramid_expand(c, (H, W), mode, constant=0.3, addend=x, sign=-1.0)
        lop.pyramid_expand(c, (H, W), mode, constant=0.3, addend=e, sign=1.0, out=e)
        lop.multires_bilateral(x, 3, 1.0, [0.05, 0.0, 0.2], mode, constant=0.3)
        n += 3 + 8
    lop.local([x], [np.full((3, 5), 0.05, np.float32)], "sum", "sqdiff", "constant", 0.2,
              point=[(-0.5, 0.75)])
    u = synthetic.to_u8(x)
    lop.local([u, u], [np.ones((3, 3), np.int32)] * 2, "max", "absdiff", "clamp",
              point=[(-1, 255), (3, -7)])
    lop.global_reduce(x, "sumsq")
    lop.global_reduce(u, "sumsq")
    n += 4
torch.cuda.synchronize()
print("ok", n, "calls")

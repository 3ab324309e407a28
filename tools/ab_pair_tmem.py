"""A/B of the pair-sharing bilateral kernels (register ring vs TMEM ring,
LOP_PAIR_TMEM=0/1 in the environment): per-config output SHA-1 (must match
between the two) and CUDA-event time per launch.  usage:
  LOP_PAIR_TMEM=1 python tools/ab_pair_tmem.py out.json"""
import hashlib
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import synthetic
import paper_conf_ipps_membarthhtke12_b200 as lop

CASES = [  # (H, W, window, mode, roi)
    (4096, 4096, 13, "clamp", None), (4096, 4096, 13, "mirror", None),
    (4096, 4096, 13, "constant", None), (4096, 4096, 13, "repeat", None),
    (4096, 4096, 13, "undefined", None),
    (1024, 1024, 13, "clamp", None), (2048, 2048, 13, "mirror", None),
    (4096, 4096, 9, "clamp", None), (4096, 4096, 15, "clamp", None), (4096, 4096, 11, "clamp", None),
    (4096, 4096, 3, "clamp", None), (4096, 4096, 5, "mirror", None), (4096, 4096, 7, "repeat", None),
    (777, 1031, 13, "mirror", (5, 7, 700, 600)), (300, 301, 13, "constant", None),
]
res = {}
for H, W, win, mode, roi in CASES:
    x = synthetic.angio(H, W, seed=H + W + win, device="cuda")
    y = torch.zeros_like(x)
    f = lambda: lop.bilateral(x, (win - 1) / 4.0, 5.0 if win == 13 else 0.2, mode, constant=0.25,
                              size=win, out=y, roi=roi)
    f()
    torch.cuda.synchronize()
    h = hashlib.sha1(y.cpu().numpy().tobytes()).hexdigest()
    n = 20 if H * W >= 4096 * 4096 else 50
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(n):
        f()
    b.record()
    torch.cuda.synchronize()
    res["%dx%d_w%d_%s_%s" % (H, W, win, mode, roi)] = {"sha1": h, "ms": a.elapsed_time(b) / n}
json.dump(res, open(sys.argv[1], "w"), indent=1)
for k, v in res.items():
    print("%-40s %.4f ms %s" % (k, v["ms"], v["sha1"][:10]))

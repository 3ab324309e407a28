"""Sweep the bilateral MUFU-offload setting (LOP_BILATERAL_NPOLY) on 4096^2 13x13.

Prints one JSON line per setting: Mpx/s from CUDA events over back-to-back
launches (3 rotating buffer sets), and the max |diff| to npoly=0.
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import synthetic  # noqa: E402
import paper_conf_ipps_membarthhtke12_b200 as lop  # noqa: E402

H = W = 4096
ins = [synthetic.angio(H, W, seed=synthetic.config_seed(2) + i, device="cuda") for i in range(3)]
outs = [torch.empty_like(ins[0]) for _ in range(3)]
ref = None
for npoly in [int(a) for a in (sys.argv[1:] or ["0", "1", "2", "3"])]:
    os.environ["LOP_BILATERAL_NPOLY"] = str(npoly)
    for i in range(6):
        lop.bilateral(ins[i % 3], 3.0, 5.0, "clamp", out=outs[i % 3])
    torch.cuda.synchronize()
    a = torch.cuda.Event(enable_timing=True)
    b = torch.cuda.Event(enable_timing=True)
    n = 60
    a.record()
    for i in range(n):
        lop.bilateral(ins[i % 3], 3.0, 5.0, "clamp", out=outs[i % 3])
    b.record()
    torch.cuda.synchronize()
    ms = a.elapsed_time(b) / n
    o = lop.bilateral(ins[0], 3.0, 0.05, "clamp")
    if ref is None:
        ref = o
    print(json.dumps({"npoly": npoly, "ms": round(ms, 4), "Mpx_s": round(H * W / ms / 1e3, 1),
                      "sfu_frac_168": round(168 * H * W / (ms * 1e-3) / 4.6531e12, 4),
                      "max_diff_vs_npoly0": float((o - ref).abs().max())}), flush=True)

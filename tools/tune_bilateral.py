"""Sweep the bilateral kernel settings (LOP_BILATERAL_NPOLY, LOP_BILATERAL_SCALED)
on 4096^2 13x13 clamp.

Prints one JSON line per setting: Mpx/s from CUDA events over back-to-back
launches (3 rotating buffer sets), and the max |diff| to the default setting.
usage: python tools/tune_bilateral.py [npoly:scaled[:m] ...]   (default 0:0 1:0 0:1)
A trailing ":m" passes the 13x13 closeness as an explicit user mask (Listing 5
precomputed-Mask path, tiled user-mask kernel) instead of sigma_d.
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
for setting in (sys.argv[1:] or ["0:0", "1:0", "0:1"]):
    npoly, scaled, *um = setting.split(":")
    kw = {"mask": lop.closeness_mask(3.0)} if um else {}
    os.environ["LOP_BILATERAL_NPOLY"] = npoly
    os.environ["LOP_BILATERAL_SCALED"] = scaled
    for i in range(6):
        lop.bilateral(ins[i % 3], 3.0, 5.0, "clamp", out=outs[i % 3], **kw)
    torch.cuda.synchronize()
    best = None
    for rep in range(3):
        a = torch.cuda.Event(enable_timing=True)
        b = torch.cuda.Event(enable_timing=True)
        n = 60
        a.record()
        for i in range(n):
            lop.bilateral(ins[i % 3], 3.0, 5.0, "clamp", out=outs[i % 3], **kw)
        b.record()
        torch.cuda.synchronize()
        ms = a.elapsed_time(b) / n
        best = ms if best is None else min(best, ms)
    o = lop.bilateral(ins[0], 3.0, 0.05, "clamp", **kw)
    if ref is None:
        ref = o
    print(json.dumps({"npoly": int(npoly), "scaled": int(scaled), "user_mask": bool(um), "ms": round(best, 4),
                      "Mpx_s": round(H * W / best / 1e3, 1),
                      "sfu_frac_168": round(168 * H * W / (best * 1e-3) / 4.6531e12, 4),
                      "max_diff_vs_first": float((o - ref).abs().max())}), flush=True)

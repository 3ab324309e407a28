"""Bilateral 4096^2 13x13 per boundary mode (paper E5, mode invariance), in
the order given, each mode timed over back-to-back launches on 3 rotating
buffer sets; run twice (forward, reverse order) to separate a mode effect
from a drift over the run.  Optional constants per mode via CONST=<v>.
usage: python tools/time_modes.py"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synthetic  # noqa: E402
import paper_conf_ipps_membarthhtke12_b200 as lop  # noqa: E402

H = W = 4096
cval = float(os.environ.get("CONST", "0"))
ins = [synthetic.angio(H, W, seed=synthetic.config_seed(2) + i, device="cuda") for i in range(3)]
outs = [torch.empty_like(ins[0]) for _ in range(3)]
modes = ["undefined", "clamp", "repeat", "mirror", "constant"]


def run(mode):
    for i in range(6):
        lop.bilateral(ins[i % 3], 3.0, 5.0, mode, constant=cval, out=outs[i % 3])
    torch.cuda.synchronize()
    best = None
    for rep in range(3):
        a = torch.cuda.Event(enable_timing=True)
        b = torch.cuda.Event(enable_timing=True)
        n = 40
        a.record()
        for i in range(n):
            lop.bilateral(ins[i % 3], 3.0, 5.0, mode, constant=cval, out=outs[i % 3])
        b.record()
        torch.cuda.synchronize()
        ms = a.elapsed_time(b) / n
        best = ms if best is None else min(best, ms)
    return round(best, 4)


res = {"forward": {m: run(m) for m in modes}, "reverse": {m: run(m) for m in reversed(modes)}}
print(json.dumps({"const": cval, "ms": res}))

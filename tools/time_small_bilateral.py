"""Bilateral on small images (BASELINE config 1 and neighbours), where a launch
is latency-bound: CUDA graph of 100 launches, replayed; Mpx/s per shape.
LOP_LIBRARY / LOP_PAIR_ROWS select the build / rows per warp.
usage: python tools/time_small_bilateral.py"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synthetic  # noqa: E402
import paper_conf_ipps_membarthhtke12_b200 as lop  # noqa: E402

res = {}
for (H, W, size, sd) in ((256, 256, 3, 1.0), (256, 256, 13, 3.0), (512, 512, 13, 3.0),
                         (1024, 1024, 13, 3.0), (2048, 2048, 13, 3.0)):
    img = synthetic.angio(H, W, seed=synthetic.config_seed(1), device="cuda")
    out = torch.empty_like(img)
    s2 = torch.cuda.Stream()
    g = torch.cuda.CUDAGraph()
    n = 100 if H <= 512 else 20
    with torch.cuda.stream(s2):
        lop.bilateral(img, sd, 5.0, "clamp", size=size, out=out, stream=s2)
        with torch.cuda.graph(g, stream=s2):
            for _ in range(n):
                lop.bilateral(img, sd, 5.0, "clamp", size=size, out=out, stream=s2)
    torch.cuda.synchronize()
    best = None
    for rep in range(5):
        a = torch.cuda.Event(enable_timing=True)
        b = torch.cuda.Event(enable_timing=True)
        a.record()
        g.replay()
        b.record()
        torch.cuda.synchronize()
        ms = a.elapsed_time(b) / n
        best = ms if best is None else min(best, ms)
    res["%dx%d_%dx%d" % (H, W, size, size)] = {"us": round(best * 1e3, 2),
                                               "Mpx_s": round(H * W / best / 1e3, 1)}
print(json.dumps({"lib": os.environ.get("LOP_LIBRARY", "in-tree"), "res": res}))

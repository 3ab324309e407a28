"""Time the u8 Gaussian on 4096^2 for every boundary mode: CUDA graph of 8
launches over 8 rotating input/output sets (footprint > L2), replayed; ms per
launch.  Environment (LOP_CONV_STREAM, LOP_STREAM_SEG, LOP_CONV_CFG) selects
the kernel.  usage: python tools/time_conv_u8.py [size=5]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synthetic  # noqa: E402
import paper_conf_ipps_membarthhtke12_b200 as lop  # noqa: E402

size = int(sys.argv[1]) if len(sys.argv) > 1 else 5
H = W = 4096
img = synthetic.angio(H, W, seed=synthetic.config_seed(3), device="cuda")
u8 = synthetic.to_u8(img)
sets = 8
u_in = [u8.clone() for _ in range(sets)]
u_out = [torch.empty_like(u8) for _ in range(sets)]
res = {}
for mode in ("clamp", "repeat", "mirror", "constant"):
    fn = lambda k, s: lop.gaussian(u_in[k], size, mode, out=u_out[k], stream=s)  # noqa: E731
    s2 = torch.cuda.Stream()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.stream(s2):
        for k in range(sets):
            fn(k, s2)
        with torch.cuda.graph(g, stream=s2):
            for k in range(sets):
                fn(k, s2)
    torch.cuda.synchronize()
    best = None
    for rep in range(5):
        a = torch.cuda.Event(enable_timing=True)
        b = torch.cuda.Event(enable_timing=True)
        a.record()
        for _ in range(10):
            g.replay()
        b.record()
        torch.cuda.synchronize()
        ms = a.elapsed_time(b) / 10 / sets
        best = ms if best is None else min(best, ms)
    res[mode] = {"ms": round(best, 5), "GB_s": round(2 * H * W / best / 1e6, 1)}
print(json.dumps({"env": {k: v for k, v in os.environ.items() if k.startswith("LOP_")},
                  "size": size, "res": res}))

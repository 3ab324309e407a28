"""Configuration exploration for the convolution kernels (the paper's §V-D /
Fig. 4 exploration, re-done for sm_100a): sweep LOP_CONV_CFG = "TS:NBUF"
(output rows per tile, 1 = one tile per CTA / 2 = persistent double-buffered)
over Gaussian 5x5 and Sobel 3x3 on 4096^2 f32 and u8.

Per-launch time = replay time of a CUDA graph of 8 launches over 8 rotating
input/output sets (footprint > L2) / 8.  One JSON line per (config, case).
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import synthetic  # noqa: E402
import paper_conf_ipps_membarthhtke12_b200 as lop  # noqa: E402

HBM = 6547.5
H = W = 4096
img = synthetic.angio(H, W, seed=synthetic.config_seed(3), device="cuda")
u8 = synthetic.to_u8(img)
sets = 8
f_in = [img.clone() for _ in range(sets)]
f_out = [torch.empty_like(img) for _ in range(sets)]
u_in = [u8.clone() for _ in range(sets)]
u_out = [torch.empty_like(u8) for _ in range(sets)]
i_out = [torch.empty(u8.shape, dtype=torch.int32, device="cuda") for _ in range(sets)]
cases = [("gaussian5x5_f32", lambda k, s: lop.gaussian(f_in[k], 5, "clamp", out=f_out[k], stream=s), 8),
         ("sobel3x3_f32", lambda k, s: lop.sobel(f_in[k], 0, "clamp", out=f_out[k], stream=s), 8),
         ("gaussian5x5_u8", lambda k, s: lop.gaussian(u_in[k], 5, "clamp", out=u_out[k], stream=s), 2),
         ("sobel3x3_u8_i32", lambda k, s: lop.sobel(u_in[k], 0, "clamp", out=i_out[k], stream=s), 5)]
cfgs = sys.argv[1:] or ["4:1", "8:1", "16:1", "32:1", "8:2", "16:2", "32:2"]
for cfg in cfgs:
    os.environ["LOP_CONV_CFG"] = cfg
    for name, fn, bpp in cases:
        s = torch.cuda.Stream()
        s.wait_stream(torch.cuda.current_stream())
        g = torch.cuda.CUDAGraph()
        with torch.cuda.stream(s):
            for k in range(sets):
                fn(k, s)
            with torch.cuda.graph(g, stream=s):
                for k in range(sets):
                    fn(k, s)
        torch.cuda.current_stream().wait_stream(s)
        for _ in range(3):
            g.replay()
        torch.cuda.synchronize()
        best = None
        for _ in range(5):
            a = torch.cuda.Event(enable_timing=True)
            b = torch.cuda.Event(enable_timing=True)
            a.record()
            g.replay()
            b.record()
            torch.cuda.synchronize()
            ms = a.elapsed_time(b) / sets
            best = ms if best is None else min(best, ms)
        gbs = H * W * bpp / best / 1e6
        print(json.dumps({"cfg": cfg, "case": name, "ms": round(best, 5),
                          "GB_s": round(gbs, 1), "hbm_frac": round(gbs / HBM, 3)}), flush=True)

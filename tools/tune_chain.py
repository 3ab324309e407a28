"""Sweep LOP_CHAIN_TS for the fused Gaussian5 -> Sobel3 chain (f32 and u8->i32) on
4096^2 and compare with the two separate passes (CUDA-graph replays, 8 rotating sets)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import synthetic  # noqa: E402
import paper_conf_ipps_membarthhtke12_b200 as lop  # noqa: E402

H = W = 4096
sets = 8
img = synthetic.angio(H, W, seed=3, device="cuda")
u8 = synthetic.to_u8(img)
fi = [img.clone() for _ in range(sets)]
fo = [torch.empty_like(img) for _ in range(sets)]
ui = [u8.clone() for _ in range(sets)]
io = [torch.empty(u8.shape, dtype=torch.int32, device="cuda") for _ in range(sets)]
mf, mu = torch.empty_like(img), torch.empty_like(u8)
gf, _ = lop.gaussian_mask(5, np.float32)
sxf = lop.sobel_mask(0, np.float32)
gi, gk = lop.gaussian_mask(5, np.int32)
sxi = lop.sobel_mask(0, np.int32)


def timed(fn):
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
    best = 1e9
    for _ in range(5):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        g.replay()
        b.record()
        torch.cuda.synchronize()
        best = min(best, a.elapsed_time(b) / sets)
    return best


cases = {
    "f32_fused": lambda k, s: lop.convolve_chain(fi[k], gf, sxf, "clamp", out=fo[k], stream=s, fused=True),
    "f32_two_pass": lambda k, s: lop.convolve(lop.convolve(fi[k], gf, "clamp", out=mf, stream=s),
                                              sxf, "clamp", out=fo[k], stream=s),
    "u8_i32_fused": lambda k, s: lop.convolve_chain(ui[k], gi, sxi, "clamp", shift1=gk,
                                                    out=io[k], stream=s, fused=True),
    "u8_i32_two_pass": lambda k, s: lop.convolve(lop.convolve(ui[k], gi, "clamp", shift=gk,
                                                              out=mu, stream=s),
                                                 sxi, "clamp", out=io[k], stream=s),
}
for ts in (sys.argv[1:] or ["4", "8", "16"]):
    os.environ["LOP_CHAIN_TS"] = ts
    for name, fn in cases.items():
        if "two_pass" in name and ts != (sys.argv[1:] or ["4"])[0]:
            continue
        ms = timed(fn)
        bpp = 8 if name.startswith("f32") else 5
        print(json.dumps({"ts": int(ts), "case": name, "ms": round(ms, 5),
                          "hbm_frac_of_fused_bytes": round(H * W * bpp / ms / 1e6 / 6547.5, 3)}),
              flush=True)

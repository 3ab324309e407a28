"""Time the 4096^2 convolution kernels of bench.py's config-3 extras (CUDA graph of 8 launches
over 8 rotating buffer sets, footprint > L2): Gaussian 5x5 / Sobel 3x3, f32 and u8."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import synthetic
import paper_conf_ipps_membarthhtke12_b200 as lop

S = 8
img = synthetic.angio(4096, 4096, seed=synthetic.config_seed(3), device="cuda")
u8 = synthetic.to_u8(img)
fi = [img.clone() for _ in range(S)]
fo = [torch.empty_like(img) for _ in range(S)]
ui = [u8.clone() for _ in range(S)]
uo = [torch.empty_like(u8) for _ in range(S)]
io_ = [torch.empty(u8.shape, dtype=torch.int32, device="cuda") for _ in range(S)]
cases = {"gaussian5x5_f32": lambda k, s: lop.gaussian(fi[k], 5, "clamp", out=fo[k], stream=s),
         "sobel3x3_f32": lambda k, s: lop.sobel(fi[k], 0, "clamp", out=fo[k], stream=s),
         "gaussian5x5_u8": lambda k, s: lop.gaussian(ui[k], 5, "clamp", out=uo[k], stream=s),
         "gaussian3x3_u8": lambda k, s: lop.gaussian(ui[k], 3, "clamp", out=uo[k], stream=s),
         "sobel3x3_u8_i32": lambda k, s: lop.sobel(ui[k], 0, "clamp", out=io_[k], stream=s),
         "erode5x5_u8": lambda k, s: lop.erode(ui[k], 5, "clamp", out=uo[k], stream=s),
         "sobel_magnitude_l2_f32": lambda k, s: lop.sobel_magnitude(fi[k], "clamp", out=fo[k], stream=s),
         "sobel_magnitude_l1_u8_i32": lambda k, s: lop.sobel_magnitude(ui[k], "clamp", out=io_[k], stream=s)}
res = {}
for name, fn in cases.items():
    s2 = torch.cuda.Stream()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.stream(s2):
        for k in range(S):
            fn(k, s2)
        with torch.cuda.graph(g, stream=s2):
            for k in range(S):
                fn(k, s2)
    torch.cuda.synchronize()
    g.replay()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(20):
        g.replay()
    b.record()
    torch.cuda.synchronize()
    res[name] = round(a.elapsed_time(b) / 20 / S * 1000, 2)
print(json.dumps({"us": res}))

"""Time the Laplacian-pyramid kernels (N4) at 4096^2 f32: REDUCE 4096^2 ->
2048^2 and the band-pass EXPAND (coarse + addend -> fine), CUDA graph of 8
launches over 8 rotating buffer sets (footprint > L2), and the whole
multiresolution filter (4 levels, 13 x 13)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import synthetic
import paper_conf_ipps_membarthhtke12_b200 as lop

dev = "cuda"
S = 8
fine = [synthetic.angio(4096, 4096, seed=s, device=dev) for s in range(S)]
coarse = [torch.empty(2048, 2048, device=dev) for _ in range(S)]
outs = [torch.empty(4096, 4096, device=dev) for _ in range(S)]


def graph_ms(fn):
    s2 = torch.cuda.Stream()
    with torch.cuda.stream(s2):
        for k in range(S):
            fn(k, s2)
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s2):
            for k in range(S):
                fn(k, s2)
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    g.replay()
    a.record()
    for _ in range(10):
        g.replay()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / 10 / S


res = {}
ms = graph_ms(lambda k, s: lop.pyramid_reduce(fine[k], "mirror", out=coarse[k], stream=s))
res["reduce"] = {"ms": ms, "GB_s": 4096 * 4096 * 5 / ms / 1e6}
ms = graph_ms(lambda k, s: lop.pyramid_expand(coarse[k], (4096, 4096), "mirror", addend=fine[k],
                                              sign=-1.0, out=outs[k], stream=s))
res["expand_bandpass"] = {"ms": ms, "GB_s": 4096 * 4096 * 9 / ms / 1e6}
ws = torch.empty(lop.multires_workspace_bytes((4096, 4096), 4), dtype=torch.uint8, device=dev)
f = lambda: lop.multires_bilateral(fine[0], 4, 3.0, [0.05, 0.08, 0.12, 0.0], "mirror", out=outs[0],
                                   workspace=ws)
f()
torch.cuda.synchronize()
a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
a.record()
for _ in range(10):
    f()
b.record()
torch.cuda.synchronize()
res["multires_4096_4lv"] = {"ms": a.elapsed_time(b) / 10}
print(json.dumps(res))

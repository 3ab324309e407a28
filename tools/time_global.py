"""Time the global reductions (SUM / MIN / MAX) on 4096^2 f32 and u8: CUDA
graph of 8 launches over 8 rotating inputs (footprint > L2), replayed; ms per
launch and GB/s of the image read.  usage: python tools/time_global.py"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synthetic  # noqa: E402
import paper_conf_ipps_membarthhtke12_b200 as lop  # noqa: E402

H = W = 4096
img = synthetic.angio(H, W, seed=synthetic.config_seed(3), device="cuda")
u8 = synthetic.to_u8(img)
sets = 8
ins = {"f32": [img.clone() for _ in range(sets)], "u8": [u8.clone() for _ in range(sets)]}
gres = torch.empty(1, dtype=torch.float64, device="cuda")
gwork = torch.zeros(1025, dtype=torch.float64, device="cuda")
res = {}
for dt in ("f32", "u8"):
    for op in ("sum", "min", "max"):
        fn = lambda k, s: lop.global_reduce(ins[dt][k], op, out=gres, work=gwork, stream=s)  # noqa: E731
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
        nbytes = ins[dt][0].numel() * ins[dt][0].element_size()
        res["%s_%s" % (op, dt)] = {"ms": round(best, 5), "GB_s": round(nbytes / best / 1e6, 1)}
print(json.dumps(res))

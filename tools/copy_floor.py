"""Achievable HBM rate at the operator sizes: torch's device copy (read + write)
of 4096^2 u8 / f32 images (16 / 64 MiB each way) and a read-only sum, timed as
the operators are (CUDA graph of 8 launches over 8 rotating buffer sets > L2,
replayed).  Context for the small-image roofline fractions: a ~10 us kernel
pays launch and ramp costs that the 1 GiB peak copy amortises.
usage: python tools/copy_floor.py"""
import json

import torch

res = {}
sets = 8
for name, dtype in (("u8", torch.uint8), ("f32", torch.float32)):
    src = [torch.randint(0, 255, (4096, 4096), device="cuda").to(dtype) for _ in range(sets)]
    dst = [torch.empty_like(s) for s in src]
    nbytes = src[0].numel() * src[0].element_size()
    for kind, fn, traffic in (("copy", lambda k: dst[k].copy_(src[k]), 2 * nbytes),
                              ("amax_read", lambda k: torch.amax(src[k]), nbytes)):
        s2 = torch.cuda.Stream()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.stream(s2):
            for k in range(sets):
                fn(k)
            with torch.cuda.graph(g, stream=s2):
                for k in range(sets):
                    fn(k)
        torch.cuda.synchronize()
        best = None
        for _ in range(5):
            a = torch.cuda.Event(enable_timing=True)
            b = torch.cuda.Event(enable_timing=True)
            a.record()
            for _ in range(10):
                g.replay()
            b.record()
            torch.cuda.synchronize()
            ms = a.elapsed_time(b) / 10 / sets
            best = ms if best is None else min(best, ms)
        res["%s_%s" % (kind, name)] = {"ms": round(best, 5), "GB_s": round(traffic / best / 1e6, 1)}
print(json.dumps(res))

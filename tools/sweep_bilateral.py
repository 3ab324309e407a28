"""Configuration exploration of the bilateral kernels on B200 (the paper's
§V-D / Fig. 4 idea; N1): per (image size, window) the time of the pair-sharing
kernel and of the unshared separable kernel (LOP_BILATERAL_PAIR=1/0), and at
4096^2 13x13 the pair kernel's rows-per-warp T (LOP_PAIR_ROWS).  CUDA graph of
n launches replayed, best of 5 (us per launch).  One JSON line per point.
usage: python tools/sweep_bilateral.py [sizes|rows|all]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synthetic  # noqa: E402
import paper_conf_ipps_membarthhtke12_b200 as lop  # noqa: E402


def timed(img, out, sd, size, n):
    s2 = torch.cuda.Stream()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.stream(s2):
        lop.bilateral(img, sd, 5.0, "clamp", size=size, out=out, stream=s2)
        with torch.cuda.graph(g, stream=s2):
            for _ in range(n):
                lop.bilateral(img, sd, 5.0, "clamp", size=size, out=out, stream=s2)
    torch.cuda.synchronize()
    best = None
    for _ in range(5):
        a = torch.cuda.Event(enable_timing=True)
        b = torch.cuda.Event(enable_timing=True)
        a.record()
        g.replay()
        b.record()
        torch.cuda.synchronize()
        ms = a.elapsed_time(b) / n
        best = ms if best is None else min(best, ms)
    return best * 1e3


what = sys.argv[1] if len(sys.argv) > 1 else "all"
if what in ("sizes", "all"):
    for S in (128, 256, 384, 512, 768, 1024, 1536, 2048, 3072, 4096):
        img = synthetic.angio(S, S, seed=synthetic.config_seed(1), device="cuda")
        out = torch.empty_like(img)
        for size in (3, 5, 7, 9, 11, 13, 15):
            r = {"H": S, "W": S, "window": size}
            for name, v in (("pair_us", "1"), ("sep_us", "0")):
                os.environ["LOP_BILATERAL_PAIR"] = v
                r[name] = round(timed(img, out, (size - 1) / 4.0, size, 40 if S <= 1024 else 8), 2)
            os.environ.pop("LOP_BILATERAL_PAIR")
            r["auto_us"] = round(timed(img, out, (size - 1) / 4.0, size, 40 if S <= 1024 else 8), 2)
            print(json.dumps(r), flush=True)
if what in ("rows", "all"):
    img = synthetic.angio(4096, 4096, seed=synthetic.config_seed(2), device="cuda")
    out = torch.empty_like(img)
    for T in (8, 16, 24, 32, 43, 48, 56, 64, 72, 86, 96, 128, 171, 256, 512):
        os.environ["LOP_PAIR_ROWS"] = str(T)
        print(json.dumps({"H": 4096, "W": 4096, "window": 13, "pair_rows_T": T,
                          "us": round(timed(img, out, 3.0, 13, 8), 2)}), flush=True)
    os.environ.pop("LOP_PAIR_ROWS")
    print(json.dumps({"H": 4096, "W": 4096, "window": 13, "pair_rows_T": "auto",
                      "us": round(timed(img, out, 3.0, 13, 8), 2)}), flush=True)

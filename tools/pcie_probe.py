"""Host<->device copy ceilings for the e2e number: pinned H2D, D2H and both at
once (separate streams), 64 MiB, plus the host pipeline at several chunk sizes."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import synthetic  # noqa: E402
import paper_conf_ipps_membarthhtke12_b200 as lop  # noqa: E402

N = 64 * 1024 * 1024 // 4
h_src = torch.empty(N, dtype=torch.float32).pin_memory()
h_dst = torch.empty(N, dtype=torch.float32).pin_memory()
d_a = torch.empty(N, dtype=torch.float32, device="cuda")
d_b = torch.empty(N, dtype=torch.float32, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()


def bw(fn, reps=10):
    fn()
    torch.cuda.synchronize()
    t = time.perf_counter()
    for _ in range(reps):
        fn()
    torch.cuda.synchronize()
    return reps * N * 4 / (time.perf_counter() - t) / 1e9


def h2d():
    with torch.cuda.stream(s1):
        d_a.copy_(h_src, non_blocking=True)


def d2h():
    with torch.cuda.stream(s2):
        h_dst.copy_(d_b, non_blocking=True)


def both():
    h2d()
    d2h()


print(json.dumps({"h2d_GB_s": round(bw(h2d), 1), "d2h_GB_s": round(bw(d2h), 1),
                  "bidirectional_each_GB_s": round(bw(both), 1)}), flush=True)


def chunked(nchunks):
    # the pipeline's copy pattern without the kernel: chunk k uploads while chunk k-1 downloads
    step = N // nchunks
    ev = [torch.cuda.Event() for _ in range(nchunks)]

    def run():
        for k in range(nchunks):
            with torch.cuda.stream(s1):
                d_a[k * step:(k + 1) * step].copy_(h_src[k * step:(k + 1) * step],
                                                   non_blocking=True)
                ev[k].record(s1)
            s2.wait_event(ev[k])
            with torch.cuda.stream(s2):
                h_dst[k * step:(k + 1) * step].copy_(d_a[k * step:(k + 1) * step],
                                                     non_blocking=True)
    return run


for n in (1, 4, 8, 16):
    print(json.dumps({"chunked_copies": n, "each_dir_GB_s": round(bw(chunked(n), reps=5), 1)}),
          flush=True)
H = W = 4096
img = synthetic.angio(H, W, seed=synthetic.config_seed(2)).pin_memory()
out = torch.empty_like(img).pin_memory()
for chunk in (128, 256, 512, 1024):
    p = lop.Pipeline(W, H, chunk_rows=chunk)
    p.bilateral(img, out, 3.0, 5.0)
    t = time.perf_counter()
    for _ in range(5):
        p.bilateral(img, out, 3.0, 5.0)
    dt = (time.perf_counter() - t) / 5
    p.close()
    print(json.dumps({"pipeline_chunk_rows": chunk, "ms": round(dt * 1e3, 3),
                      "Mpx_s": round(H * W / dt / 1e6, 1)}), flush=True)

"""Host pipeline: bilateral vs a cheap kernel (Gaussian 3x3) at several chunk sizes,
to separate the copy pattern from the kernel's share of the e2e time."""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import synthetic
import paper_conf_ipps_membarthhtke12_b200 as lop
H = W = 4096
img = synthetic.angio(H, W, seed=2).pin_memory()
out = torch.empty_like(img).pin_memory()
g3, _ = lop.gaussian_mask(3, np.float32)
for chunk in (256, 512, 1024, 2048):
    p = lop.Pipeline(W, H, chunk_rows=chunk)
    for name, fn in (("bilateral13", lambda: p.bilateral(img, out, 3.0, 5.0)),
                     ("gauss3", lambda: p.convolve(img, out, g3))):
        fn()
        t = time.perf_counter()
        for _ in range(5):
            fn()
        dt = (time.perf_counter() - t) / 5
        print(json.dumps({"chunk": chunk, "op": name, "ms": round(dt * 1e3, 3),
                          "Mpx_s": round(H * W / dt / 1e6, 1)}), flush=True)
    p.close()

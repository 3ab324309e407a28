"""Time lop.local (N2) on 4096^2: CUDA graph of 8 launches over 8 rotating
input sets (> L2), per-launch ms and fraction of the HBM roofline.
LOP_LOCAL_SMALL=0 forces the runtime-loop tiled kernel; LOP variant 'generic'
via argv[1] = generic."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, synthetic
import paper_conf_ipps_membarthhtke12_b200 as lop
if len(sys.argv) > 1:
    lop.set_variant(sys.argv[1])
H = W = 4096
img = synthetic.angio(H, W, seed=1, device="cuda")
u8 = synthetic.to_u8(img)
S = 8
fa = [img.clone() for _ in range(S)]; fb = [img.clone() for _ in range(S)]
ua = [u8.clone() for _ in range(S)]; ub = [u8.clone() for _ in range(S)]
fo = [torch.empty_like(img) for _ in range(S)]
io = [torch.empty(img.shape, dtype=torch.int32, device="cuda") for _ in range(S)]
m5 = np.full((5, 5), 0.5 / 25, np.float32); m3 = np.full((3, 3), 0.5 / 9, np.float32)
cases = {
    "f32_sum_product_5x5+3x3": (lambda k, s: lop.local([fa[k], fb[k]], [m5, m3], "sum", "product", "clamp", out=fo[k], stream=s), 12),
    "f32_sum_sqdiff_5x5": (lambda k, s: lop.local([fa[k]], [m5], "sum", "sqdiff", "mirror", out=fo[k], stream=s), 8),
    "u8_max_absdiff_3x3x2": (lambda k, s: lop.local([ua[k], ub[k]], [np.ones((3, 3), np.int32)] * 2, "max", "absdiff", "clamp", out=io[k], stream=s), 6),
    "f32_sum_product_9x9": (lambda k, s: lop.local([fa[k]], [np.full((9, 9), 1 / 81, np.float32)], "sum", "product", "clamp", out=fo[k], stream=s), 8),
}
for name, (fn, bpp) in cases.items():
    s2 = torch.cuda.Stream(); g = torch.cuda.CUDAGraph()
    with torch.cuda.stream(s2):
        for k in range(S): fn(k, s2)
        with torch.cuda.graph(g, stream=s2):
            for k in range(S): fn(k, s2)
    torch.cuda.synchronize()
    best = 1e9
    for _ in range(5):
        a = torch.cuda.Event(enable_timing=True); b = torch.cuda.Event(enable_timing=True)
        a.record(); g.replay(); b.record(); torch.cuda.synchronize()
        best = min(best, a.elapsed_time(b) / S)
    print(json.dumps({"case": name, "ms": round(best, 5), "GB_s": round(H * W * bpp / best / 1e6, 1),
                      "hbm_frac": round(H * W * bpp / best / 1e6 / 6531.3, 3)}), flush=True)

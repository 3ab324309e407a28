"""A/B the liblop build variants (build/variants/liblop_*.so via LOP_LIBRARY)
on the HBM-bound convolution kernels at 4096^2 (CUDA graph of 8 launches over
8 rotating input/output sets > L2): u8 Gaussian 5x5, f32 Gaussian 5x5,
Sobel u8 -> i32, erode 5x5 u8; ms per launch + output SHA-1 (bit identity).
usage: python tools/ab_conv.py [variant ...]"""
import glob, json, os, subprocess, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CHILD = r'''
import hashlib, json, sys
sys.path.insert(0, %r)
import torch, synthetic
import paper_conf_ipps_membarthhtke12_b200 as lop
H = W = 4096
img = synthetic.angio(H, W, seed=3, device="cuda"); u8 = synthetic.to_u8(img)
S = 8
fi = [img.clone() for _ in range(S)]; fo = [torch.empty_like(img) for _ in range(S)]
ui = [u8.clone() for _ in range(S)]; uo = [torch.empty_like(u8) for _ in range(S)]
io = [torch.empty(img.shape, dtype=torch.int32, device="cuda") for _ in range(S)]
cases = {"gauss5_u8": lambda k, s: lop.gaussian(ui[k], 5, "clamp", out=uo[k], stream=s),
         "gauss5_f32": lambda k, s: lop.gaussian(fi[k], 5, "clamp", out=fo[k], stream=s),
         "sobel_u8_i32": lambda k, s: lop.sobel(ui[k], 0, "clamp", out=io[k], stream=s),
         "erode5_u8": lambda k, s: lop.erode(ui[k], 5, "clamp", out=uo[k], stream=s)}
res = {}
for name, fn in cases.items():
    s2 = torch.cuda.Stream(); g = torch.cuda.CUDAGraph()
    with torch.cuda.stream(s2):
        for k in range(S): fn(k, s2)
        with torch.cuda.graph(g, stream=s2):
            for k in range(S): fn(k, s2)
    torch.cuda.synchronize()
    best = 1e9
    for _ in range(7):
        a = torch.cuda.Event(enable_timing=True); b = torch.cuda.Event(enable_timing=True)
        a.record(); g.replay(); b.record(); torch.cuda.synchronize()
        best = min(best, a.elapsed_time(b) / S)
    out = {"gauss5_u8": uo, "gauss5_f32": fo, "sobel_u8_i32": io, "erode5_u8": uo}[name][0]
    fn(0, torch.cuda.current_stream()); torch.cuda.synchronize()
    res[name] = {"us": round(best * 1e3, 2), "sha": hashlib.sha1(out.cpu().numpy().tobytes()).hexdigest()[:10]}
print(json.dumps(res))
''' % ROOT
names = sys.argv[1:] or sorted(os.path.basename(p)[7:-3] for p in glob.glob(os.path.join(ROOT, "build/variants/liblop_*.so")))
for v in names:
    env = dict(os.environ, LOP_LIBRARY=os.path.join(ROOT, "build/variants/liblop_%s.so" % v))
    r = subprocess.run([sys.executable, "-c", CHILD], env=env, capture_output=True, text=True, timeout=600)
    line = [l for l in r.stdout.splitlines() if l.startswith("{")]
    print(v, line[-1] if line else r.stderr[-500:], flush=True)

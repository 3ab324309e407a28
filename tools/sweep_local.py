"""Configuration exploration of the local-operator kernels (N1/N2; the
paper's §V-D / Fig. 4 on B200): every CTA shape (bx x by threads, bx*by a
multiple of 32 up to 1024) of the small-window kernel for the bench case
(two 4096^2 f32 accessors, 5x5 + 3x3, SUM of PRODUCT), against the shape
Algorithm 2 picks (LOP_DEBUG_SELECT).  One JSON line per shape.
usage: python tools/sweep_local.py"""
import json, os, subprocess, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CHILD = r'''
import json, os, sys
sys.path.insert(0, %r)
import numpy as np, torch, synthetic
import paper_conf_ipps_membarthhtke12_b200 as lop
H = W = 4096
S = 8
fa = [synthetic.angio(H, W, seed=1, device="cuda") for _ in range(1)] * 0
img = synthetic.angio(H, W, seed=1, device="cuda")
fa = [img.clone() for _ in range(S)]; fb = [img.clone() for _ in range(S)]
fo = [torch.empty_like(img) for _ in range(S)]
m5 = np.full((5, 5), 0.5 / 25, np.float32); m3 = np.full((3, 3), 0.5 / 9, np.float32)
fn = lambda k, s: lop.local([fa[k], fb[k]], [m5, m3], "sum", "product", "clamp", out=fo[k], stream=s)
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
print(json.dumps({"ms": round(best, 5), "hbm_frac": round(H * W * 12 / best / 1e6 / 6531.3, 3)}))
''' % ROOT
shapes = [None] + [(bx, t // bx) for t in range(32, 1025, 32) for bx in (8, 16, 32, 64)
                   if t % bx == 0 and t // bx <= 32 and t in (32, 64, 128, 256)]
for sh in shapes:
    env = dict(os.environ, LOP_DEBUG_SELECT="1")
    if sh:
        env["LOP_LOCAL_CFG"] = "%d:%d" % sh
    r = subprocess.run([sys.executable, "-c", CHILD], env=env, capture_output=True, text=True, timeout=300)
    line = [l for l in r.stdout.splitlines() if l.startswith("{")]
    d = json.loads(line[-1]) if line else {"error": r.stderr[-300:]}
    d["cfg"] = "alg2" if sh is None else "%dx%d" % sh
    if sh is None:
        d["alg2_pick"] = [l for l in r.stderr.splitlines() if "Algorithm 2" in l][-1:]
    print(json.dumps(d), flush=True)

"""A/B the liblop build variants (build/variants/liblop_*.so, one process per
variant via LOP_LIBRARY) on the 4096^2 13x13 bilateral: ms per launch (CUDA
events over back-to-back launches on 3 rotating buffer sets) and a SHA-1 of the
outputs for every boundary mode, so variants can be checked for bit identity.
usage: python tools/ab_variants.py [variant ...]   (default: all)"""
import glob
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CHILD = r'''
import hashlib, json, os, sys
sys.path.insert(0, %r)
import torch, synthetic
import paper_conf_ipps_membarthhtke12_b200 as lop
H = W = 4096
ins = [synthetic.angio(H, W, seed=synthetic.config_seed(2) + i, device="cuda") for i in range(3)]
outs = [torch.empty_like(ins[0]) for _ in range(3)]
res = {}
for mode in ("clamp", "repeat", "constant"):
    for i in range(6):
        lop.bilateral(ins[i %% 3], 3.0, 5.0, mode, out=outs[i %% 3])
    torch.cuda.synchronize()
    best = None
    for rep in range(3):
        a = torch.cuda.Event(enable_timing=True); b = torch.cuda.Event(enable_timing=True)
        n = 60
        a.record()
        for i in range(n):
            lop.bilateral(ins[i %% 3], 3.0, 5.0, mode, out=outs[i %% 3])
        b.record(); torch.cuda.synchronize()
        ms = a.elapsed_time(b) / n
        best = ms if best is None else min(best, ms)
    o = lop.bilateral(ins[0], 3.0, 0.05, mode)
    res[mode] = {"ms": round(best, 4), "sha": hashlib.sha1(o.cpu().numpy().tobytes()).hexdigest()[:12]}
print(json.dumps(res))
''' % ROOT

names = sys.argv[1:] or sorted(os.path.basename(p)[7:-3] for p in
                               glob.glob(os.path.join(ROOT, "build/variants/liblop_*.so")))
for v in names:
    env = dict(os.environ, LOP_LIBRARY=os.path.join(ROOT, "build/variants/liblop_%s.so" % v))
    r = subprocess.run([sys.executable, "-c", CHILD], env=env, capture_output=True, text=True,
                       timeout=300)
    line = r.stdout.strip().splitlines()[-1] if r.stdout.strip() else r.stderr[-400:]
    print(v, line, flush=True)

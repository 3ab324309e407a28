"""e2e pipeline sweep on 4096^2 f32 bilateral 13x13: chunk rows x staging
buffers (LOP_PIPELINE_BUFS, set per child process); wall clock per image from
pinned host memory to pinned host memory, best of 5.
usage: python tools/pipe_sweep.py"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CHILD = r'''
import sys, time, json
sys.path.insert(0, %r)
import torch, synthetic
import paper_conf_ipps_membarthhtke12_b200 as lop
H = W = 4096
img = synthetic.angio(H, W, seed=2012002).pin_memory()
out = torch.empty_like(img).pin_memory()
res = {}
for chunk in (512, 1024, 2048):
    p = lop.Pipeline(W, H, chunk_rows=chunk)
    ts = []
    for _ in range(6):
        t = time.perf_counter(); p.bilateral(img, out, 3.0, 5.0); ts.append((time.perf_counter() - t) * 1e3)
    p.close()
    res[chunk] = round(min(ts[1:]), 3)
print(json.dumps(res))
''' % ROOT
for bufs in sys.argv[1:] or ["4", "64"]:
    env = dict(os.environ, LOP_PIPELINE_BUFS=bufs)
    r = subprocess.run([sys.executable, "-c", CHILD], env=env, capture_output=True, text=True, timeout=600)
    print(json.dumps({"bufs": bufs, "ms": json.loads(r.stdout.strip().splitlines()[-1]) if r.stdout.strip() else r.stderr[-300:]}), flush=True)

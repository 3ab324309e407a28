"""e2e frame streaming (lop.Pipeline.bilateral_frames) on 4096^2 f32 frames:
Mpx/s per chunk size, after a warm-up pass over every frame.
usage: python tools/pipe_frames_sweep.py [frames=10]"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synthetic  # noqa: E402
import paper_conf_ipps_membarthhtke12_b200 as lop  # noqa: E402

F = int(sys.argv[1]) if len(sys.argv) > 1 else 10
H = W = 4096
img = synthetic.angio(H, W, seed=synthetic.config_seed(2))
host_in = img.unsqueeze(0).repeat(F, 1, 1).pin_memory()
host_out = torch.empty_like(host_in).pin_memory()
res = {}
for chunk in (512, 1024, 2048, 4096):
    p = lop.Pipeline(W, H, chunk_rows=chunk)
    p.bilateral_frames(host_in, host_out, 3.0, 5.0, "clamp", size=13)
    best = 0
    for _ in range(3):
        t0 = time.perf_counter()
        p.bilateral_frames(host_in, host_out, 3.0, 5.0, "clamp", size=13)
        best = max(best, F * H * W / (time.perf_counter() - t0) / 1e6)
    p.close()
    res[chunk] = round(best, 1)
print(json.dumps({"frames": F, "Mpx_s_by_chunk_rows": res,
                  "env": {k: v for k, v in os.environ.items() if k.startswith("LOP_")}}))

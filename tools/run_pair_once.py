"""Run the config-2 bilateral (4096^2, 13x13, clamp) a few times: a target for
ncu captures of bilateral_pair_kernel<6> (tools/ncu_hot.py, tools/summarize_ncu.py)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch

import synthetic
import paper_conf_ipps_membarthhtke12_b200 as lop

n = int(sys.argv[1]) if len(sys.argv) > 1 else 3
x = synthetic.angio(4096, 4096, seed=synthetic.config_seed(2), device="cuda")
y = torch.empty_like(x)
for _ in range(n):
    lop.bilateral(x, 3.0, 5.0, "clamp", size=13, out=y)
torch.cuda.synchronize()
print("ok", float(y.sum()))

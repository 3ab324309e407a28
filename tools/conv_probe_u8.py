"""Launch the u8 Gaussian on 4096^2 a few times (for ncu captures).
usage: python tools/conv_probe_u8.py [mode=clamp] [size=5]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synthetic  # noqa: E402
import paper_conf_ipps_membarthhtke12_b200 as lop  # noqa: E402

mode = sys.argv[1] if len(sys.argv) > 1 else "clamp"
size = int(sys.argv[2]) if len(sys.argv) > 2 else 5
u8 = synthetic.to_u8(synthetic.angio(4096, 4096, seed=synthetic.config_seed(3), device="cuda"))
out = torch.empty_like(u8)
for _ in range(3):
    lop.gaussian(u8, size, mode, out=out)
torch.cuda.synchronize()
print("ok")

"""A few global reductions on 4096^2 (for ncu captures)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synthetic  # noqa: E402
import paper_conf_ipps_membarthhtke12_b200 as lop  # noqa: E402

img = synthetic.angio(4096, 4096, seed=synthetic.config_seed(3), device="cuda")
u8 = synthetic.to_u8(img)
work = torch.zeros(1025, dtype=torch.float64, device="cuda")
for _ in range(3):
    lop.global_reduce(img, "sum", work=work)
    lop.global_reduce(u8, "max", work=work)
torch.cuda.synchronize()
print("ok")

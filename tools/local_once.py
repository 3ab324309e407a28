"""Run the bench's two local-operator cases once each (ncu target)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import synthetic
import paper_conf_ipps_membarthhtke12_b200 as lop

img = synthetic.angio(4096, 4096, seed=3, device="cuda")
u8 = synthetic.to_u8(img)
o = torch.empty(4096, 4096, dtype=torch.int32, device="cuda")
f = torch.empty_like(img)
m5 = np.full((5, 5), 0.5 / 25, np.float32)
m3 = np.full((3, 3), 0.5 / 9, np.float32)
for _ in range(2):
    lop.local([u8, u8.clone()], [np.ones((3, 3), np.int32)] * 2, "max", "absdiff", "clamp", out=o)
    lop.local([img, img.clone()], [m5, m3], "sum", "product", "clamp", out=f)
torch.cuda.synchronize()

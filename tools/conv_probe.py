"""Launch the convolution hot kernels a few times on 4096^2 (for ncu captures)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import synthetic  # noqa: E402
import paper_conf_ipps_membarthhtke12_b200 as lop  # noqa: E402

img = synthetic.angio(4096, 4096, seed=synthetic.config_seed(3), device="cuda")
u8 = synthetic.to_u8(img)
res = torch.empty_like(img)
u8o = torch.empty_like(u8)
i32o = torch.empty(u8.shape, dtype=torch.int32, device="cuda")
for _ in range(3):
    lop.gaussian(img, 5, "clamp", out=res)
    lop.sobel(img, 0, "clamp", out=res)
    lop.gaussian(u8, 5, "clamp", out=u8o)
    lop.sobel(u8, 0, "clamp", out=i32o)
torch.cuda.synchronize()
print("ok")

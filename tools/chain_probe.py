"""Launch the fused chain and its two passes on 4096^2 (for ncu captures)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import synthetic  # noqa: E402
import paper_conf_ipps_membarthhtke12_b200 as lop  # noqa: E402

img = synthetic.angio(4096, 4096, seed=3, device="cuda")
u8 = synthetic.to_u8(img)
gf, _ = lop.gaussian_mask(5, np.float32)
sxf = lop.sobel_mask(0, np.float32)
gi, gk = lop.gaussian_mask(5, np.int32)
sxi = lop.sobel_mask(0, np.int32)
for _ in range(2):
    lop.convolve_chain(img, gf, sxf, "clamp", fused=True)
    lop.convolve_chain(u8, gi, sxi, "clamp", shift1=gk, out_dtype=torch.int32, fused=True)
torch.cuda.synchronize()
print("ok")

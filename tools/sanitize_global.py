"""Small launches of the global reductions for compute-sanitizer (memcheck /
racecheck / initcheck): f32 and u8, every op, ragged widths, single pixels,
unaligned regions and frames, one scratch buffer reused by every call."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synthetic  # noqa: E402
import paper_conf_ipps_membarthhtke12_b200 as lop  # noqa: E402

work = torch.zeros(1025, dtype=torch.float64, device="cuda")
n = 0
for H, W in [(1, 1), (3, 2), (13, 17), (70, 257), (131, 600), (600, 1031)]:
    img = synthetic.uniform(H, W, seed=H + W).cuda()
    u8 = synthetic.uniform_u8(H, W, seed=H * W).cuda()
    frames = torch.stack([img, img * 0.5]).contiguous()
    uframes = torch.stack([u8, 255 - u8]).contiguous()
    for op in ("sum", "min", "max"):
        for x in (img, u8, frames, uframes):
            lop.global_reduce(x, op, work=work)
            n += 1
            if H > 4 and W > 4:
                lop.global_reduce(x, op, roi=(1, 2, W - 3, H - 3), work=work)
                n += 1
torch.cuda.synchronize()
assert work[-1].item() == 0.0
print("launches", n)

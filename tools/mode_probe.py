"""One bilateral launch per boundary mode on 4096^2 13x13 (for an ncu capture
comparing modes).  usage: python tools/mode_probe.py [mode ...]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synthetic  # noqa: E402
import paper_conf_ipps_membarthhtke12_b200 as lop  # noqa: E402

img = synthetic.angio(4096, 4096, seed=synthetic.config_seed(2), device="cuda")
out = torch.empty_like(img)
for m in (sys.argv[1:] or ["clamp", "constant"]):
    for _ in range(2):
        lop.bilateral(img, 3.0, 5.0, m, out=out)
torch.cuda.synchronize()

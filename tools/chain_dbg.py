import os, sys, numpy as np, torch
sys.path.insert(0, os.getcwd())
import synthetic, oracle
import paper_conf_ipps_membarthhtke12_b200 as lop
sys.path.insert(0, "tests")
from test_parity_gpu import _chain_pairs
mode = sys.argv[1] if len(sys.argv) > 1 else "clamp"
which = sys.argv[2] if len(sys.argv) > 2 else "f32"
if which == "f32":
    x = torch.stack([synthetic.uniform(67, 1032, seed=s + 70) for s in range(2)]).cuda(); pairs = _chain_pairs("f32"); cval = 0.25
else:
    x = torch.stack([synthetic.uniform_u8(67, 1040, seed=s + 80) for s in range(2)]).cuda(); pairs = _chain_pairs("u8"); cval = 99
for m1, k1, m2, k2 in pairs:
    os.environ["LOP_CHAIN_STREAM"] = "1"
    a = lop.convolve_chain(x, m1, m2, mode, constant=cval, shift1=k1, shift2=k2, fused=True)
    torch.cuda.synchronize()
    os.environ["LOP_CHAIN_STREAM"] = "0"
    b = lop.convolve_chain(x, m1, m2, mode, constant=cval, shift1=k1, shift2=k2, fused=True)
    print(mode, which, m1.shape, m2.shape, torch.equal(a, b), flush=True)

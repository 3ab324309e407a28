import os, sys
sys.path.insert(0, os.getcwd())
import torch, synthetic
import paper_conf_ipps_membarthhtke12_b200 as lop
x = synthetic.angio(4096, 4096, seed=1, device="cuda")
c = torch.empty(2048, 2048, device="cuda")
for _ in range(3):
    lop.pyramid_reduce(x, "mirror", out=c)
torch.cuda.synchronize()

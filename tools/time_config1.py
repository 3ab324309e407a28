import os, sys, json
sys.path.insert(0, os.getcwd())
import torch, synthetic
import paper_conf_ipps_membarthhtke12_b200 as lop
small = synthetic.angio(256, 256, seed=synthetic.config_seed(1), device="cuda")
so = torch.empty_like(small)
g = torch.cuda.CUDAGraph(); s2 = torch.cuda.Stream()
with torch.cuda.stream(s2):
    lop.bilateral(small, 1.0, 5.0, "clamp", size=3, out=so, stream=s2)
    with torch.cuda.graph(g, stream=s2):
        for _ in range(100):
            lop.bilateral(small, 1.0, 5.0, "clamp", size=3, out=so, stream=s2)
torch.cuda.synchronize()
a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
g.replay(); a.record()
for _ in range(10): g.replay()
b.record(); torch.cuda.synchronize()
print("config1 Gpx/s", 256*256*100*10/ a.elapsed_time(b) / 1e6)

mkdir -p gpurun_out/pt1
LOP_PIPELINE_TRACE=1 python - > gpurun_out/pt1/trace.txt 2>&1 <<'PY'
import torch, time, synthetic
import paper_conf_ipps_membarthhtke12_b200 as lop
H=W=4096
img = synthetic.angio(H, W, seed=2012002).pin_memory()
out = torch.empty_like(img).pin_memory()
for chunk in (512, 1024):
    p = lop.Pipeline(W, H, chunk_rows=chunk)
    for _ in range(3):
        t=time.perf_counter(); p.bilateral(img, out, 3.0, 5.0); print(chunk, (time.perf_counter()-t)*1e3, flush=True)
    p.close()
PY

# A/B: default build vs alternative .so on the 4096^2 and 1024^2 x 64 frames bilateral
mkdir -p gpurun_out/ab
python -c "import __graft_entry__ as g; g.build()"
for lib in "" "$@"; do
  LOP_LIBRARY=$lib python - <<'PY' >> gpurun_out/ab/ab.txt 2>&1
import os, torch, synthetic
import paper_conf_ipps_membarthhtke12_b200 as lop
lib = os.environ.get("LOP_LIBRARY") or "default"
def t(x, out, n=30):
    for _ in range(3): lop.bilateral(x, 3.0, 5.0, "clamp", out=out)
    a=torch.cuda.Event(enable_timing=True); b=torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(n): lop.bilateral(x, 3.0, 5.0, "clamp", out=out)
    b.record(); torch.cuda.synchronize(); return a.elapsed_time(b)/n
x = synthetic.angio(4096, 4096, seed=1, device="cuda"); o = torch.empty_like(x)
ms = t(x, o); print(lib, "4096^2", round(ms,4), "frac", round(168*4096*4096/(ms*1e-3)/4.6531e12,4))
f = torch.stack([synthetic.angio(1024,1024,seed=i,device="cuda") for i in range(64)]); of = torch.empty_like(f)
ms = t(f, of, 10); print(lib, "64x1024^2", round(ms,4), "frac", round(168*64*1024*1024/(ms*1e-3)/4.6531e12,4))
PY
done

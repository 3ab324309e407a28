import os, sys, numpy as np, torch
sys.path.insert(0, os.getcwd())
import synthetic
import paper_conf_ipps_membarthhtke12_b200 as lop
H, W = 129, 1031
rng = np.random.default_rng(H * 7 + W)
img = synthetic.uniform(H, W, seed=H + 11 * W).cuda()
ra = np.outer(rng.integers(-3, 4, 5), rng.integers(-3, 4, 5)).astype(np.int32)
rb = np.outer(rng.integers(-3, 4, 5), rng.integers(-3, 4, 5)).astype(np.int32)
ma, mb = ra.astype(np.float32) / 8, rb.astype(np.float32) / 4
z = np.zeros_like(mb)
for mode in ("clamp",):
    a = lop.convolve(img, ma, mode).cpu().numpy()
    b = lop.convolve(img, mb, mode).cpu().numpy()
    fa = lop.convolve2(img, ma, z, "l1", mode).cpu().numpy()
    fb = lop.convolve2(img, z, mb, "l1", mode).cpu().numpy()
    print("A |a| equal:", np.array_equal(fa, np.abs(a)), "B equal:", np.array_equal(fb, np.abs(b)))
    for comb in ("sumsq", "l1", "l2"):
        f = lop.convolve2(img, ma, mb, comb, mode).cpu().numpy()
        if comb == "l1": e = np.abs(a) + np.abs(b)
        else:
            e = a * a + b * b
            if comb == "l2": e = np.sqrt(e)
        d = np.argwhere(f != e)
        print(comb, np.array_equal(f, e), len(d), d[:3].tolist(), [(float(f[tuple(i)]), float(e[tuple(i)])) for i in d[:2]])
    s = a * a + b * b
    t = torch.from_numpy(s).cuda()
    print("torch sqrt == np sqrt:", np.array_equal(torch.sqrt(t).cpu().numpy(), np.sqrt(s)))

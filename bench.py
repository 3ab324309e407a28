#!/usr/bin/env python
"""bench.py -- throughput of the local-operator hot path on B200.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl lop|reference]
                    [--mode clamp] [--no-partitioned] [--no-extras]

One JSON line on rank 0 (driver contract):
  metric / unit   BASELINE.json's metric, in Mpixel/s
  value           whole-job Mpixel/s of the headline workload, inputs resident
                  in HBM, CUDA events on the launching stream, K steps between
                  barrier+synchronize, max over ranks
  partitioned     BASELINE configs 4 and 5 -- the paths that shard -- at this
                  N, each with the SAME total work at every N (strong
                  scaling): c4 = 1024 frames of 1024^2 split over the ranks
                  (no data-path collective), c5 = one 32768^2 image in row
                  bands with the NCCL halo exchange; per-rank ms, halo ms,
                  SFU fraction, NCCL communicator size
  e2e             the headline metric through the host pipeline API
                  (lop.Pipeline: pinned host in -> device -> pinned host out,
                  copies inside the timed region), with the pinned copy
                  ceiling measured in the same run and the fraction of it
  roofline        the dominant kernel against its bound (SFU for the
                  bilateral filter: 84 distinct ex2 per pixel = (13*13 - 1) / 2 with
                  symmetric pair-sharing; frac_vs_168_ex2_per_px against the
                  unshared count, which the pair kernel exceeds)
  cpu_baseline    the C oracle (double, OpenMP) on a bounded sample, rank 0, N=1
  clocks          nvidia-smi samples taken during the timed region
  gpu_launches    lop kernel launches inside the headline's timed region
                  (liblop counter, reset right before it)

Headline workload (identical at every N, so the scaling run's N=1 line is
this bench line): BASELINE config 2 with clamp -- every rank filters its own
4096x4096 f32 image per step (13x13, sigma_d=3, sigma_r=5), i.e. weak scaling
with no data-path collective.  The partitioned configs carry the strong
scaling of the frame and band splits.

Launch: under torchrun (WORLD_SIZE set) every rank runs; `--gpus N` with
N > 1 and no WORLD_SIZE re-executes itself under torch.distributed.run with
N ranks (127.0.0.1); --gpus disagreeing with WORLD_SIZE is an error.
--dry-run: plumbing only (gloo, CPU): every rank reports its partition of
configs 4 and 5; rank 0 prints them (tests/test_bench_launch.py).
"""
from __future__ import annotations

import argparse
import json
import math
import os
import socket
import statistics
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

BASELINE_METRIC = "Mpixel/s per filter at 1/2/4/8 B200; % of HBM GB/s or FP32/SFU roofline"
SM_COUNT = 148
MUFU_PER_CLK_PER_SM = 16          # MUFU.EX2 lanes per clock per SM on sm_100
C4_FRAMES, C4_SIZE = 1024, 1024   # BASELINE config 4
C5_SIZE = 32768                   # BASELINE config 5
SIGMA_D, SIGMA_R, WINDOW = 3.0, 5.0, 13


def parse(argv=None):
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=None,
                    help="ranks (default: WORLD_SIZE, else 1); N > 1 without torchrun self-launches")
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", choices=["lop", "reference"], default="lop")
    ap.add_argument("--workload", choices=["bilateral4096", "frames", "bands"],
                    default="bilateral4096", help="headline workload (default: config 2)")
    ap.add_argument("--mode", default="clamp")
    ap.add_argument("--no-extras", action="store_true", help="skip per-filter side measurements")
    ap.add_argument("--no-partitioned", action="store_true", help="skip the c4 / c5 records")
    ap.add_argument("--part-steps", type=int, default=5, help="timed steps of c4 / c5")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=10)
    ap.add_argument("--cpu-seconds", type=float, default=12.0)
    ap.add_argument("--dry-run", action="store_true", help="launch plumbing only (gloo, no GPU)")
    ap.add_argument("--backend", choices=["nccl", "gloo"], default="nccl",
                    help="process-group backend (gloo: ranks may share one GPU -- a test of "
                         "the N > 1 code path on a single-GPU box; halos are host-staged)")
    return ap.parse_args(argv)


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        d["_source"] = "measured (MEASURED_PEAKS.json)"
        return d
    return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "sm_max_mhz": 1965.0,
            "_source": "fallback (B200_PROFILING.md)"}


def sfu_peak_tex2(peaks) -> float:
    """148 SM x 16 MUFU.EX2 / clk x max SM clock, in T ex2 / s."""
    return SM_COUNT * MUFU_PER_CLK_PER_SM * float(peaks.get("sm_max_mhz", 1965.0)) * 1e6 / 1e12


# ------------------------------------------------------------- launching ----

def _free_port() -> int:
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def relaunch_if_needed(args, argv):
    """Returns an exit code if this process only launched the ranks, else None."""
    env_world = os.environ.get("WORLD_SIZE")
    if env_world is None:
        n = args.gpus or 1
        if n <= 1:
            return None
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1",
               "--nproc-per-node=%d" % n, "--master-addr=127.0.0.1",
               "--master-port=%d" % _free_port(), os.path.abspath(__file__)] + list(argv)
        print("[bench] --gpus %d without torchrun: launching %d ranks: %s" % (n, n, " ".join(cmd)),
              file=sys.stderr, flush=True)
        return subprocess.call(cmd)
    if args.gpus is not None and args.gpus != int(env_world):
        print(json.dumps({"error": "--gpus %d disagrees with WORLD_SIZE=%s" % (args.gpus, env_world)}),
              flush=True)
        return 2
    return None


# ------------------------------------------------------------ distributed ----

class Dist:
    def __init__(self):
        self.world = int(os.environ.get("WORLD_SIZE", "1"))
        self.rank = int(os.environ.get("RANK", "0"))
        self.local = int(os.environ.get("LOCAL_RANK", "0"))
        self.backend = None

    def device_index(self) -> int:
        """This rank's GPU: LOCAL_RANK (nccl); modulo the visible GPUs for gloo,
        whose ranks may share one GPU."""
        import torch
        n = torch.cuda.device_count()
        return self.local if self.backend != "gloo" or n == 0 else self.local % n

    def init(self, backend="nccl"):
        import torch
        import torch.distributed as dist
        if self.world > 1 and not dist.is_initialized():
            self.backend = backend
            if backend == "nccl":
                torch.cuda.set_device(self.local)
            dist.init_process_group(backend, device_id=(torch.device("cuda", self.local)
                                                        if backend == "nccl" else None))
            self.backend = backend
            # communicator evidence: the process group's size as NCCL sees it
            print("[bench] rank %d/%d: %s process group initialised, group size %d" %
                  (self.rank, self.world, backend, dist.get_world_size()), file=sys.stderr,
                  flush=True)

    def comm_info(self):
        if self.world == 1:
            return {"backend": None, "world_size": 1}
        import torch
        import torch.distributed as dist
        info = {"backend": dist.get_backend(), "world_size": dist.get_world_size()}
        if info["backend"] == "nccl":
            v = torch.cuda.nccl.version()
            info["nccl_version"] = ".".join(str(x) for x in v) if isinstance(v, tuple) else str(v)
        return info

    def barrier(self):
        if self.world > 1:
            import torch.distributed as dist
            dist.barrier()

    def _reduce(self, v, op):
        if self.world == 1:
            return v
        import torch
        import torch.distributed as dist
        dev = "cuda" if self.backend == "nccl" else "cpu"
        t = torch.tensor([v], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=op)
        return float(t.item())

    def max(self, v: float) -> float:
        if self.world == 1:
            return v
        import torch.distributed as dist
        return self._reduce(v, dist.ReduceOp.MAX)

    def gather(self, v: float) -> list:
        """v of every rank, in rank order."""
        if self.world == 1:
            return [v]
        import torch
        import torch.distributed as dist
        dev = "cuda" if self.backend == "nccl" else "cpu"
        t = torch.tensor([v], dtype=torch.float64, device=dev)
        out = [torch.zeros_like(t) for _ in range(self.world)]
        dist.all_gather(out, t)
        return [float(x.item()) for x in out]

    def gather_obj(self, obj):
        if self.world == 1:
            return [obj]
        import torch.distributed as dist
        out = [None] * self.world
        dist.all_gather_object(out, obj)
        return out

    def close(self):
        if self.world > 1:
            import torch.distributed as dist
            if dist.is_initialized():
                dist.destroy_process_group()


# ----------------------------------------------------------------- clocks ----

class ClockSampler:
    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index: int):
        self.gpu = gpu_index
        self.proc = None
        self.path = None

    def start(self):
        try:
            fd, self.path = tempfile.mkstemp(suffix=".csv")
            os.close(fd)
            self.fh = open(self.path, "w")
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.gpu), "--query-gpu=" + self.FIELDS,
                 "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=self.fh, stderr=subprocess.DEVNULL)
        except (OSError, FileNotFoundError):
            self.proc = None

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        self.fh.close()
        sm, smax, power, reasons = [], [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        with open(self.path) as f:
            for line in f:
                parts = [p.strip() for p in line.split(",")]
                if len(parts) < 9:
                    continue
                try:
                    sm.append(float(parts[1]))
                    smax.append(float(parts[2]))
                    power.append(float(parts[3]))
                except ValueError:
                    continue
                for n, v in zip(names, parts[5:9]):
                    if v.lower().startswith("active"):
                        reasons.add(n)
        os.unlink(self.path)
        return {"sm_mhz": statistics.median(sm) if sm else None,
                "sm_max_mhz": max(smax) if smax else None,
                "power_w_max": max(power) if power else None,
                "samples": len(sm), "reasons": sorted(reasons)}


# ------------------------------------------------------------------ timing ----

def time_steps(step, K, W, dist, stream, lop=None):
    """W warm-up steps, then K timed steps bracketed by barrier + synchronize;
    returns (total_ms max over ranks, per-step ms list on this rank, lop
    launches inside the timed region or None)."""
    import torch
    for i in range(W):
        step(i)
    torch.cuda.synchronize()
    dist.barrier()
    torch.cuda.synchronize()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
          for _ in range(K)]
    t0 = torch.cuda.Event(enable_timing=True)
    t1 = torch.cuda.Event(enable_timing=True)
    if lop is not None:
        lop.reset_launch_count()
    t0.record(stream)
    for i in range(K):
        ev[i][0].record(stream)
        step(i)
        ev[i][1].record(stream)
    t1.record(stream)
    launches = lop.launch_count() if lop is not None else None
    torch.cuda.synchronize()
    dist.barrier()
    torch.cuda.synchronize()
    total = t0.elapsed_time(t1)
    per = [a.elapsed_time(b) for a, b in ev]
    return dist.max(total), per, launches


def flush_l2(buf):
    buf.add_(1)          # write 512 MiB: evicts the 126 MB L2


# --------------------------------------------------------------- workloads ----

# --------------------------------------------------------------- workloads ----

def workload_c2(args, dist, lop, synthetic, dev, stream):
    """BASELINE config 2: one 4096^2 image per rank per step (weak scaling)."""
    import torch
    H = Wd = 4096
    n_sets = 3                             # rotating sets: 3 x 128 MiB > 126 MB L2
    seed = synthetic.config_seed(2) + 7919 * dist.rank
    base = synthetic.angio(H, Wd, seed=seed, device=dev)
    ins = [base.clone() for _ in range(n_sets)]
    outs = [torch.empty_like(base) for _ in range(n_sets)]

    def step(i):
        lop.bilateral(ins[i % n_sets], SIGMA_D, SIGMA_R, args.mode, size=WINDOW,
                      out=outs[i % n_sets], stream=stream)
    config = {"workload": "bilateral 4096x4096 f32, 13x13 (sigma_d=3), sigma_r=5, %s; "
                          "one image per rank per step (BASELINE config 2)" % args.mode,
              "height": H, "width": Wd, "window": WINDOW, "sigma_d": SIGMA_D,
              "sigma_r": SIGMA_R, "boundary": args.mode,
              "l2": "rotating %d input/output sets (%d MiB) > 126 MB L2" % (n_sets, n_sets * 128),
              "parallelism": "frame-parallel x%d (independent images)" % dist.world}
    return dict(step=step, px_rank=H * Wd, px_total=H * Wd * dist.world, config=config,
                scaling="weak", launches_per_step=1, base=base)


def workload_c4(args, dist, lop, synthetic, dev, stream):
    """BASELINE config 4: 1024 frames of 1024^2, contiguous frame ranges per
    rank (dist.frame_range), one batched launch per rank, no collective."""
    import torch
    from paper_conf_ipps_membarthhtke12_b200 import dist as ldist
    F, S = C4_FRAMES, C4_SIZE
    lo, hi = ldist.frame_range(F, dist.world, dist.rank)
    frames = synthetic.angio_frames(F, S, S, seed=synthetic.config_seed(4), first=lo,
                                    count=hi - lo, device=dev)
    out = torch.empty_like(frames)

    def step(i):
        lop.bilateral(frames, SIGMA_D, SIGMA_R, args.mode, size=WINDOW, out=out, stream=stream)
    config = {"workload": "%d frames x %d^2 f32 bilateral 13x13 %s, frame-parallel "
                          "(BASELINE config 4)" % (F, S, args.mode),
              "frames": F, "frame_size": S, "window": WINDOW, "boundary": args.mode,
              "frames_this_rank": [lo, hi],
              "l2": "inputs (4 GiB / N) larger than L2",
              "parallelism": "frame-parallel x%d, contiguous frame ranges" % dist.world}
    return dict(step=step, px_rank=(hi - lo) * S * S, px_total=F * S * S, config=config,
                scaling="strong", launches_per_step=1)


def workload_c5(args, dist, lop, synthetic, dev, stream):
    """BASELINE config 5: one 32768^2 image in row bands, NCCL halo exchange
    (dist.bilateral_bands: interior rows overlap the exchange)."""
    import torch
    from paper_conf_ipps_membarthhtke12_b200 import dist as ldist
    GH = GW = C5_SIZE
    band = ldist.Bands(GH, GW, dist.world, dist.rank, halo=WINDOW // 2, device=dev,
                       mode=args.mode)
    band.fill(lambda y0, y1: synthetic.angio(GH, GW, seed=synthetic.config_seed(5),
                                             device=dev, row_range=(y0, y1)))
    out = torch.empty_like(band.owned)

    def step(i):
        ldist.bilateral_bands(lop, band, SIGMA_D, SIGMA_R, args.mode, size=WINDOW, out=out,
                              stream=stream)

    def exchange_only(i):
        band.exchange(stream)
    config = {"workload": "%d^2 f32 bilateral 13x13 %s, row bands + NCCL halo exchange "
                          "(BASELINE config 5)" % (GH, args.mode),
              "height": GH, "width": GW, "window": WINDOW, "boundary": args.mode,
              "rows_this_rank": [band.y0, band.y1], "halo_rows": band.halo,
              "l2": "inputs (4 GiB / N) larger than L2",
              "parallelism": "row-bands x%d" % dist.world}
    return dict(step=step, px_rank=band.rows * GW, px_total=GH * GW, config=config,
                scaling="strong", launches_per_step=ldist.launches_per_band_step(band, WINDOW),
                exchange=exchange_only, halo_bytes=band.halo_bytes)


WORKLOADS = {"bilateral4096": workload_c2, "frames": workload_c4, "bands": workload_c5}


def sfu_roofline(peaks, px_per_launch, launch_ms):
    """SFU roofline of the bilateral pair kernel for `px_per_launch` pixels
    per launch of mean duration `launch_ms` (one GPU)."""
    taps = WINDOW * WINDOW - 1                 # algorithmic ex2 per pixel
    pair = os.environ.get("LOP_BILATERAL_PAIR", "1") != "0"
    ex2_px = taps // 2 if pair else taps
    ex2_per_launch = ex2_px * px_per_launch
    achieved = ex2_per_launch / (launch_ms / 1000.0) / 1e12
    achieved_168 = taps * px_per_launch / (launch_ms / 1000.0) / 1e12
    peak = sfu_peak_tex2(peaks)
    return {"bound": "alu",
            "kernel": ("lop::bilateral_pair_tm_kernel<6>" if os.environ.get("LOP_PAIR_TMEM", "1") != "0"
                       else "lop::bilateral_pair_kernel<6>") if pair else "lop::bilateral_sep_kernel<6>",
            "achieved": round(achieved, 4), "peak": round(peak, 4), "unit": "Tex2/s",
            "frac": round(achieved / peak, 4),
            "work_per_launch": "%d ex2 (= %d distinct per px x %d px)" % (ex2_per_launch, ex2_px,
                                                                         px_per_launch),
            "frac_vs_168_ex2_per_px": round(achieved_168 / peak, 4),
            "peak_basis": "148 SM x 16 MUFU.EX2/clk x %.0f MHz (sm_max_mhz, %s)" %
                          (float(peaks.get("sm_max_mhz", 1965.0)), peaks["_source"]),
            "avg_launch_ms": round(launch_ms, 5)}


def run_partitioned(args, dist, lop, synthetic, dev, stream, peaks):
    """Configs 4 and 5 at this N (same total work at every N): one record each."""
    import torch
    out = {}
    K, W = max(1, args.part_steps), 3
    peak = sfu_peak_tex2(peaks)
    ex2_px = (WINDOW * WINDOW - 1) // 2
    for name, make in (("c4", workload_c4), ("c5", workload_c5)):
        t_setup = time.perf_counter()
        wl = make(args, dist, lop, synthetic, dev, stream)
        torch.cuda.synchronize()
        setup_s = time.perf_counter() - t_setup
        total_ms, per, launches = time_steps(wl["step"], K, W, dist, stream, lop)
        rank_ms = statistics.mean(per)
        per_rank = dist.gather(rank_ms)
        value = wl["px_total"] * K / (total_ms / 1000.0) / 1e6
        rec = {"value": round(value, 2), "unit": "Mpixel/s", "scaling": "strong",
               "n_gpus": dist.world, "steps": K, "warmup": W,
               "ms_per_step": round(total_ms / K, 4),
               "per_rank_ms": [round(v, 4) for v in per_rank],
               "px_per_step": wl["px_total"],
               # SFU fraction of all N GPUs at the 84 distinct ex2 / px of the pair kernel
               "sfu_frac": round(ex2_px * wl["px_total"] / (total_ms / K / 1000.0) / 1e12 /
                                 (peak * dist.world), 4),
               "gpu_launches": launches,
               "launches_per_step_per_rank": wl["launches_per_step"],
               "setup_s": round(setup_s, 1),
               "config": wl["config"], "comm": dist.comm_info()}
        if "exchange" in wl:
            ex_ms, ex_per, _ = time_steps(wl["exchange"], K, W, dist, stream)
            rec["halo_exchange_ms"] = round(ex_ms / K, 4)
            rec["halo_exchange_per_rank_ms"] = [round(v, 4) for v in dist.gather(statistics.mean(ex_per))]
            rec["halo_bytes_per_rank"] = wl["halo_bytes"]
            rec["halo_note"] = ("exchange alone, timed like the steps; inside a step it overlaps "
                                "the interior rows (dist.bilateral_bands)")
        out[name] = rec
        del wl
        torch.cuda.empty_cache()
    return out


def measure_copy_ceiling(dev, nbytes, reps=10, trials=3):
    """Pinned host<->device copy rate with both directions busy at once (the
    pipeline's situation), GB/s per direction: best of `trials` timings of
    `reps` back-to-back pairs, after warm-up passes over the freshly pinned
    pages (the first DMA touching a pinned page is slower)."""
    import torch
    n = nbytes // 4
    h_src = torch.empty(n, dtype=torch.float32).pin_memory()
    h_dst = torch.empty(n, dtype=torch.float32).pin_memory()
    d_a = torch.empty(n, dtype=torch.float32, device=dev)
    d_b = torch.empty(n, dtype=torch.float32, device=dev)
    s1, s2 = torch.cuda.Stream(dev), torch.cuda.Stream(dev)

    def both():
        with torch.cuda.stream(s1):
            d_a.copy_(h_src, non_blocking=True)
        with torch.cuda.stream(s2):
            h_dst.copy_(d_b, non_blocking=True)
    for _ in range(3):
        both()
    torch.cuda.synchronize()
    best = 0.0
    for _ in range(trials):
        t = time.perf_counter()
        for _ in range(reps):
            both()
        torch.cuda.synchronize()
        best = max(best, reps * n * 4 / (time.perf_counter() - t) / 1e9)
    return best


def run_lop(args, dist, peaks):
    import torch
    import synthetic
    import paper_conf_ipps_membarthhtke12_b200 as lop

    dev = torch.device("cuda", dist.device_index())
    torch.cuda.set_device(dev)
    stream = torch.cuda.current_stream(dev)
    K, W = args.steps, max(3, args.warmup)
    wl = WORKLOADS[args.workload](args, dist, lop, synthetic, dev, stream)
    clocks = ClockSampler(dist.device_index())
    clocks.start()
    total_ms, per, launches = time_steps(wl["step"], K, W, dist, stream, lop)
    # keep the GPU busy a little longer so the sampler sees the clocks under load
    t_end = time.time() + max(0.0, 1.0 - total_ms / 1000.0)
    i = 0
    while time.time() < t_end:
        wl["step"](i)
        i += 1
        if i % 20 == 0:
            torch.cuda.synchronize()
    torch.cuda.synchronize()
    clk = clocks.stop()

    value = wl["px_total"] * K / (total_ms / 1000.0) / 1e6
    avg_launch_ms = sum(per) / len(per)
    # The symmetric pair-sharing kernel (default) needs (W^2-1)/2 = 84 distinct
    # ex2 per pixel (SURVEY §8(d)'s tighter bound): that is `achieved`/`frac`.
    # Against the W^2-1 = 168 of the unshared method (Listing 5) the ratio can
    # exceed 1 -- reported beside it as frac_vs_168_ex2_per_px.
    roofline = sfu_roofline(peaks, wl["px_rank"], avg_launch_ms)
    # DRAM traffic is not measurable inside this process (no profiler); the ncu
    # capture of the same kernel is committed under profiles/ 
    roofline["traffic"] = None
    roofline["traffic_note"] = ("dram bytes per launch (ncu --set full of the same kernel and "
                                "config): profiles/r02/ncu_full_bilateral_pair_tm_s10.md")
    result = dict(metric=BASELINE_METRIC, value=round(value, 2), unit="Mpixel/s",
                  n_gpus=dist.world, steps=K, warmup=W, ms_per_step=round(total_ms / K, 5),
                  higher_is_better=True, scaling=wl["scaling"], vs_baseline=None, dtype="f32",
                  data="synthetic", config=wl["config"], roofline=roofline, clocks=clk,
                  gpu_launches=int(launches), comm=dist.comm_info())

    # ---- e2e through the host pipeline API (rank-local, max over ranks)
    if args.workload == "bilateral4096" and args.e2e_steps > 0:
        result["e2e"] = run_e2e(args, dist, lop, wl["base"], dev)
    if not args.no_extras and dist.world == 1 and args.workload == "bilateral4096":
        result["filters"] = extras(lop, synthetic, dev, stream, peaks)
    del wl
    torch.cuda.empty_cache()
    if not args.no_partitioned:
        result["partitioned"] = run_partitioned(args, dist, lop, synthetic, dev, stream, peaks)
    return result


def run_e2e(args, dist, lop, base, dev):
    H = Wd = 4096
    K = args.e2e_steps
    # one host frame per step (distinct pinned buffers), streamed back to back
    host_in = base.cpu().unsqueeze(0).repeat(K, 1, 1).pin_memory()
    host_out = host_in.clone().pin_memory()
    # single synchronous image: 1024-row chunks (ramped); a frame stream: 2048-row
    # chunks (the fill / drain is paid once per stream; tools/pipe_frames_sweep.py)
    one = host_in[0]
    pipe1 = lop.Pipeline(Wd, H, device=dist.device_index(), chunk_rows=1024)
    pipe1.bilateral(one, host_out[0], SIGMA_D, SIGMA_R, args.mode, size=WINDOW)
    dist.barrier()
    t0 = time.perf_counter()
    pipe1.bilateral(one, host_out[0], SIGMA_D, SIGMA_R, args.mode, size=WINDOW)
    t_single = dist.max(time.perf_counter() - t0)
    pipe1.close()
    pipe = lop.Pipeline(Wd, H, device=dist.device_index(), chunk_rows=2048)
    # warm-up over every frame: the first DMA touching each pinned page is slower
    pipe.bilateral_frames(host_in, host_out, SIGMA_D, SIGMA_R, args.mode, size=WINDOW)
    dist.barrier()
    t0 = time.perf_counter()
    pipe.bilateral_frames(host_in, host_out, SIGMA_D, SIGMA_R, args.mode, size=WINDOW)
    t = dist.max(time.perf_counter() - t0)
    h2d, d2h = pipe.bytes_moved()
    pipe.close()
    # the copy ceiling in the same run: both directions busy at once, 64 MiB each
    ceil_gbs = measure_copy_ceiling(dev, H * Wd * 4)
    t_floor = max(h2d, d2h) / (ceil_gbs * 1e9)
    return {"value": round(H * Wd * dist.world * K / t / 1e6, 2),
            "unit": "Mpixel/s", "h2d_bytes_per_step": int(h2d // K),
            "d2h_bytes_per_step": int(d2h // K),
            "pcie_ceiling_gbs": round(ceil_gbs, 2),
            "frac": round(t_floor / t, 4),
            "single_image_call_Mpx_s": round(H * Wd * dist.world / t_single / 1e6, 2),
            "api": "lop.Pipeline.bilateral_frames (lop_pipeline_bilateral_frames): "
                   "%d steps = %d pinned host frames (the config-2 image) streamed "
                   "back to back in 2048-row chunks on 3 streams (H2D / kernel / "
                   "D2H), every frame's upload and download inside the timed "
                   "region; wall clock; single_image_call = one synchronous "
                   "lop_pipeline_bilateral call" % (K, K),
            "ceiling_method": "pinned H2D and D2H of 64 MiB at once on two streams, best of 3 x 10 "
                              "reps after 3 warm-ups, GB/s per direction; frac = max(h2d, d2h "
                              "bytes) / ceiling / time"}


def extras(lop, synthetic, dev, stream, peaks):
    """Per-filter side measurements (L2 flushed between iterations for the
    memory-bound ones): mode sweep of the bilateral (E5), Gaussian 5x5 and
    Sobel 3x3 on 4096^2 f32 / u8 (config 3), config 1 (256^2) via CUDA graph."""
    import torch
    out = {}
    H = Wd = 4096
    img = synthetic.angio(H, Wd, seed=synthetic.config_seed(2), device=dev)
    res = torch.empty_like(img)
    flush = torch.empty(128 * 1024 * 1024, dtype=torch.float32, device=dev)

    def timed(fn, n, do_flush):
        for _ in range(3):
            fn()
        ts = []
        for _ in range(n):
            if do_flush:
                flush_l2(flush)
            a = torch.cuda.Event(enable_timing=True)
            b = torch.cuda.Event(enable_timing=True)
            a.record(stream)
            fn()
            b.record(stream)
            torch.cuda.synchronize()
            ts.append(a.elapsed_time(b))
        return statistics.median(ts)

    modes = {}
    # two passes over the modes, the better median per mode (one slow sample of a mode -- a
    # clock dip, another process -- must not read as a mode effect)
    for _ in range(2):
        for mode in ("undefined", "clamp", "repeat", "mirror", "constant"):
            ms = timed(lambda: lop.bilateral(img, 3.0, 5.0, mode, size=13, out=res, stream=stream),
                       10, False)
            modes[mode] = max(modes.get(mode, 0.0), round(H * Wd / ms / 1e3, 1))
    out["bilateral_13x13_4096_f32_Mpx_s"] = modes
    v = list(modes.values())
    out["bilateral_mode_spread"] = round(max(v) / min(v) - 1.0, 4)
    hbm = float(peaks.get("hbm_gbs", 6650.0))
    out["conv_4096"] = conv_extras(lop, synthetic, dev, stream, hbm, img, timed)
    out["conv_4096"]["method"] = (
        "CUDA graph of 8 launches over 8 rotating input/output sets (footprint > L2, so every "
        "launch reads and writes DRAM), replayed; per-launch time = replay time / 8; also the "
        "median single launch after an L2 flush")
    # config 1: 256^2, 3x3, sigma_d = 1, sigma_r = 5, clamp -- launch-latency bound:
    # report CUDA-graph replays of 100 launches
    small = synthetic.angio(256, 256, seed=synthetic.config_seed(1), device=dev)
    so = torch.empty_like(small)
    g = torch.cuda.CUDAGraph()
    s2 = torch.cuda.Stream(dev)
    s2.wait_stream(stream)
    with torch.cuda.stream(s2):
        lop.bilateral(small, 1.0, 5.0, "clamp", size=3, out=so, stream=s2)
        with torch.cuda.graph(g, stream=s2):
            for _ in range(100):
                lop.bilateral(small, 1.0, 5.0, "clamp", size=3, out=so, stream=s2)
    stream.wait_stream(s2)
    ms = timed(lambda: g.replay(), 10, False)
    out["config1_bilateral_256_3x3_graph_Mpx_s"] = round(256 * 256 * 100 / ms / 1e3, 1)
    # multiresolution filter (N4, reading c28): 4 levels, 13 x 13 window, Mirror; the
    # bilateral levels dominate (SFU-bound), so report the time and the share of the
    # level-0 bilateral alone
    levels, srs = 4, [0.05, 0.08, 0.12, 0.0]
    ws = torch.empty(lop.multires_workspace_bytes(tuple(img.shape), levels), dtype=torch.uint8,
                     device=dev)
    ms_mr = timed(lambda: lop.multires_bilateral(img, levels, 3.0, srs, "mirror", out=res,
                                                 workspace=ws, stream=stream), 10, False)
    ms_b0 = timed(lambda: lop.bilateral(img, 3.0, 0.05, "mirror", size=13, out=res,
                                        stream=stream), 10, False)
    out["multires_bilateral_4096_4levels_13x13"] = {
        "ms": round(ms_mr, 4), "Mpx_s": round(H * Wd / ms_mr / 1e3, 1),
        "level0_bilateral_ms": round(ms_b0, 4),
        "level0_share": round(ms_b0 / ms_mr, 3),
        "launches": 3 * (levels - 1) + sum(1 for v in srs if v > 0)}
    return out


def conv_extras(lop, synthetic, dev, stream, hbm, img, timed):
    """Gaussian 5x5 / Sobel 3x3 on 4096^2 f32 and u8 (BASELINE config 3), the fused chain and
    the local MIN / MAX operators: HBM roofline."""
    import numpy as np
    import torch
    sets = 8
    u8 = synthetic.to_u8(img)
    f_in = [img.clone() for _ in range(sets)]
    f_out = [torch.empty_like(img) for _ in range(sets)]
    u_in = [u8.clone() for _ in range(sets)]
    u_out = [torch.empty_like(u8) for _ in range(sets)]
    i_out = [torch.empty(u8.shape, dtype=torch.int32, device=dev) for _ in range(sets)]
    cases = [("gaussian5x5_f32", lambda k, s: lop.gaussian(f_in[k], 5, "clamp", out=f_out[k],
                                                          stream=s), 8),
             ("sobel3x3_f32", lambda k, s: lop.sobel(f_in[k], 0, "clamp", out=f_out[k],
                                                     stream=s), 8),
             ("gaussian5x5_u8", lambda k, s: lop.gaussian(u_in[k], 5, "clamp", out=u_out[k],
                                                         stream=s), 2),
             ("sobel3x3_u8_i32", lambda k, s: lop.sobel(u_in[k], 0, "clamp", out=i_out[k],
                                                        stream=s), 5)]
    # fused Gaussian 5x5 -> Sobel 3x3 (one pass) vs the two passes
    gf, _ = lop.gaussian_mask(5, np.float32)
    sxf = lop.sobel_mask(0, np.float32)
    gi, gk = lop.gaussian_mask(5, np.int32)
    sxi = lop.sobel_mask(0, np.int32)
    mid_f = torch.empty_like(img)
    mid_u = torch.empty_like(u8)
    cases += [
        ("chain_gauss5_sobel3_f32",
         lambda k, s: lop.convolve_chain(f_in[k], gf, sxf, "clamp", out=f_out[k], stream=s), 8),
        ("chain_gauss5_sobel3_f32_fused_kernel",
         lambda k, s: lop.convolve_chain(f_in[k], gf, sxf, "clamp", out=f_out[k], stream=s,
                                         fused=True), 8),
        ("chain_gauss5_sobel3_f32_two_pass",
         lambda k, s: lop.convolve(lop.convolve(f_in[k], gf, "clamp", out=mid_f, stream=s), sxf,
                                   "clamp", out=f_out[k], stream=s), 8),
        ("chain_gauss5_sobel3_u8_i32",
         lambda k, s: lop.convolve_chain(u_in[k], gi, sxi, "clamp", shift1=gk, out=i_out[k],
                                         stream=s), 5),
        ("chain_gauss5_sobel3_u8_i32_fused_kernel",
         lambda k, s: lop.convolve_chain(u_in[k], gi, sxi, "clamp", shift1=gk, out=i_out[k],
                                         stream=s, fused=True), 5),
        ("chain_gauss5_sobel3_u8_i32_two_pass",
         lambda k, s: lop.convolve(lop.convolve(u_in[k], gi, "clamp", shift=gk, out=mid_u,
                                                stream=s), sxi, "clamp", out=i_out[k], stream=s),
         5)]
    # local MIN / MAX (Listing 9 convolve(mask, MIN/MAX, ...)): erosion / dilation
    cases += [
        ("erode5x5_u8", lambda k, s: lop.erode(u_in[k], 5, "clamp", out=u_out[k], stream=s), 2),
        ("dilate3x3_f32", lambda k, s: lop.dilate(f_in[k], 3, "clamp", out=f_out[k], stream=s), 8)]
    # two local operators + point-operator epilogue in one pass (N3): Sobel magnitude,
    # against the two Sobel passes alone (whose outputs a third pass would still combine)
    cases += [
        ("sobel_magnitude_l2_f32_fused",
         lambda k, s: lop.sobel_magnitude(f_in[k], "clamp", out=f_out[k], stream=s), 8),
        ("sobel_x_and_y_f32_two_passes",
         lambda k, s: (lop.sobel(f_in[k], 0, "clamp", out=f_out[k], stream=s),
                       lop.sobel(f_in[k], 1, "clamp", out=mid_f, stream=s)), 8),
        ("sobel_magnitude_l1_u8_i32_fused",
         lambda k, s: lop.sobel_magnitude(u_in[k], "clamp", out=i_out[k], stream=s), 5)]
    # local operator over two accessors (N2; Listing 9): two
    # consecutive frames, SUM of PRODUCT with a 5x5 and a 3x3 mask (a spatio-temporal
    # average), and MAX of ABSDIFF on u8 -> i32 (local contrast of two frames)
    f_in_b = [img.clone() for _ in range(sets)]
    u_in_b = [u8.clone() for _ in range(sets)]
    m5 = np.full((5, 5), 0.5 / 25, np.float32)
    m3 = np.full((3, 3), 0.5 / 9, np.float32)
    cases += [
        ("local_2acc_sum_product_f32",
         lambda k, s: lop.local([f_in[k], f_in_b[k]], [m5, m3], "sum", "product", "clamp",
                                out=f_out[k], stream=s), 12),
        ("local_2acc_max_absdiff_u8_i32",
         lambda k, s: lop.local([u_in[k], u_in_b[k]], [np.ones((3, 3), np.int32)] * 2, "max",
                                "absdiff", "clamp", out=i_out[k], stream=s), 6),
        # the same f32 operator with a point-operator prologue on both accessors (N3,
        # reading c27: window/level a I + b applied once per staged element)
        ("local_2acc_sum_product_f32_point_prologue",
         lambda k, s: lop.local([f_in[k], f_in_b[k]], [m5, m3], "sum", "product", "clamp",
                                out=f_out[k], stream=s, point=[(1.5, -0.25), (-1.0, 1.0)]), 12)]
    # global operator (sum of all pixels, deterministic two-level reduction)
    gres = torch.empty(1, dtype=torch.float64, device=dev)
    gwork = torch.zeros(1025, dtype=torch.float64, device=dev)     # LOP_GLOBAL_WORK_DOUBLES
    cases += [
        ("global_sum_f32", lambda k, s: lop.global_reduce(f_in[k], "sum", out=gres, work=gwork,
                                                          stream=s), 4),
        ("global_max_u8", lambda k, s: lop.global_reduce(u_in[k], "max", out=gres, work=gwork,
                                                         stream=s), 1),
        ("global_sumsq_f32", lambda k, s: lop.global_reduce(f_in[k], "sumsq", out=gres, work=gwork,
                                                            stream=s), 4),
        ("global_sumsq_u8", lambda k, s: lop.global_reduce(u_in[k], "sumsq", out=gres, work=gwork,
                                                           stream=s), 1)]
    # Laplacian-pyramid steps of the multiresolution filter (N4, reading c28):
    # REDUCE 4096^2 -> 2048^2 (4 B read per fine pixel + 4 B per coarse = 5 B / fine px),
    # band-pass EXPAND with the fine addend (coarse 1 B + addend 4 B + out 4 B = 9 B / fine px)
    red = [torch.empty(2048, 2048, device=dev) for _ in range(sets)]
    cases += [
        ("pyramid_reduce_f32", lambda k, s: lop.pyramid_reduce(f_in[k], "mirror", out=red[k],
                                                               stream=s), 5),
        ("pyramid_expand_bandpass_f32",
         lambda k, s: lop.pyramid_expand(red[k], img.shape, "mirror", addend=f_in[k], sign=-1.0,
                                         out=f_out[k], stream=s), 9)]
    res = {}
    H, W = img.shape
    for name, fn, bpp in cases:
        g = torch.cuda.CUDAGraph()
        s2 = torch.cuda.Stream(dev)
        s2.wait_stream(stream)
        with torch.cuda.stream(s2):
            for k in range(sets):
                fn(k, s2)
            with torch.cuda.graph(g, stream=s2):
                for k in range(sets):
                    fn(k, s2)
        stream.wait_stream(s2)
        ms = timed(lambda: g.replay(), 10, False) / sets
        ms_flush = timed(lambda: fn(0, stream), 10, True)
        gbs = H * W * bpp / ms / 1e6
        res[name] = {"Mpx_s": round(H * W / ms / 1e3, 1), "ms": round(ms, 5),
                     "GB_s": round(gbs, 1), "hbm_frac": round(gbs / hbm, 3), "bytes_per_px": bpp,
                     "single_launch_after_l2_flush_ms": round(ms_flush, 5)}
    return res


# ------------------------------------------------------------ CPU oracle ----

def cpu_oracle_rate(H, Wd, seconds, rows_per_chunk=None, mode="clamp"):
    """Time the C oracle (as it stands) on rows of the config-2 image until
    `seconds` elapse; returns (Mpixel/s, rows, cores)."""
    import oracle
    import synthetic
    img = synthetic.angio(H, Wd, seed=synthetic.config_seed(2)).numpy()
    cores = oracle.num_threads()
    rows_per_chunk = rows_per_chunk or max(1, cores)
    done, t_used = 0, 0.0
    while done < H and t_used < seconds:
        r1 = min(H, done + rows_per_chunk)
        t0 = time.perf_counter()
        oracle.bilateral_f32(img, 3.0, 5.0, mode, size=13, rows=(done, r1))
        t_used += time.perf_counter() - t0
        done = r1
    return done * Wd / t_used / 1e6, done, cores, t_used


def run_reference(args, dist):
    """--impl reference: the oracle timed on the host cores (rank 0 only)."""
    if dist.rank != 0:
        return None
    if dist.world > 1 and os.environ.get("OMP_NUM_THREADS") == "1":
        # torchrun sets OMP_NUM_THREADS=1 per rank; the one rank that runs the
        # oracle uses all host cores, as at N = 1 (libgomp reads it at load)
        os.environ["OMP_NUM_THREADS"] = str(os.cpu_count() or 1)
    import oracle
    oracle.build()
    H = Wd = 4096
    K, W = args.steps, max(3, args.warmup)
    per_step = max(0.5, min(5.0, 150.0 / (K + W)))
    import synthetic
    img = synthetic.angio(H, Wd, seed=synthetic.config_seed(2)).numpy()
    cores = oracle.num_threads()
    t0 = time.perf_counter()
    oracle.bilateral_f32(img, 3.0, 5.0, args.mode, size=13, rows=(0, 1))
    t_row = time.perf_counter() - t0
    rows = max(1, min(H, int(per_step / max(t_row, 1e-6))))
    y = 0

    def step():
        nonlocal y
        y0 = y % (H - rows + 1) if rows < H else 0
        oracle.bilateral_f32(img, 3.0, 5.0, args.mode, size=13, rows=(y0, y0 + rows))
        y += rows
    for _ in range(W):
        step()
    t0 = time.perf_counter()
    for _ in range(K):
        step()
    t = time.perf_counter() - t0
    value = rows * Wd * K / t / 1e6
    sample = ("%d rows x 4096 px of the config-2 image per step (of 4096 rows), "
              "13x13, sigma_d=3, sigma_r=5, %s" % (rows, args.mode))
    return dict(metric=BASELINE_METRIC, value=round(value, 4), unit="Mpixel/s", n_gpus=dist.world,
                steps=K, warmup=W, ms_per_step=round(t / K * 1000, 3), higher_is_better=True,
                scaling="weak", vs_baseline=None, dtype="f64", data="synthetic", impl="reference",
                config={"workload": "bilateral 4096x4096 f32 input, 13x13 (sigma_d=3), "
                                    "sigma_r=5, %s (BASELINE config 2), C oracle" % args.mode,
                        "parallelism": "OpenMP over rows, %d threads" % cores},
                cpu_baseline={"value": round(value, 4), "unit": "Mpixel/s", "cores": cores,
                              "kind": "oracle", "sample": sample},
                e2e={"value": round(value, 4), "unit": "Mpixel/s", "h2d_bytes_per_step": 0,
                     "d2h_bytes_per_step": 0})


def run_dry(args, dist):
    """--dry-run: the launch and partition plumbing without a GPU (gloo)."""
    from paper_conf_ipps_membarthhtke12_b200 import dist as ldist
    dist.init("gloo")
    lo, hi = ldist.frame_range(C4_FRAMES, dist.world, dist.rank)
    y0, y1 = ldist.band_range(C5_SIZE, dist.world, dist.rank)
    mine = {"rank": dist.rank, "c4_frames": [lo, hi], "c5_rows": [y0, y1],
            "pid": os.getpid()}
    plans = dist.gather_obj(mine)
    total = dist.gather(float(hi - lo))
    if dist.rank == 0:
        print(json.dumps({"dry_run": True, "n_gpus": dist.world, "comm": dist.comm_info(),
                          "ranks": plans, "c4_frames_total": int(sum(total))}), flush=True)
    dist.close()
    return 0


def main(argv=None):
    argv = sys.argv[1:] if argv is None else argv
    args = parse(argv)
    rc = relaunch_if_needed(args, argv)
    if rc is not None:
        return rc
    dist = Dist()
    if args.dry_run:
        return run_dry(args, dist)
    if args.impl == "reference":
        if dist.rank == 0:
            line = run_reference(args, dist)
            print(json.dumps(line), flush=True)
        return 0
    import torch
    if not torch.cuda.is_available():
        print(json.dumps({"error": "bench.py needs a CUDA device (no CPU fallback)"}))
        return 1
    dist.init(args.backend)
    peaks = load_peaks()
    res = run_lop(args, dist, peaks)
    if dist.rank == 0:
        if dist.world == 1 and not args.no_cpu_baseline:
            v, rows, cores, t = cpu_oracle_rate(4096, 4096, args.cpu_seconds, mode=args.mode)
            res["cpu_baseline"] = {"value": round(v, 4), "unit": "Mpixel/s", "cores": cores,
                                   "kind": "oracle",
                                   "sample": "first %d rows of the 4096x4096 config-2 image "
                                             "(%.1f s of CPU time), same filter" % (rows, t)}
        print(json.dumps(res), flush=True)
    dist.close()
    return 0


if __name__ == "__main__":
    sys.exit(main())

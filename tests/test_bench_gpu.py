"""bench.py end to end on the GPU: N = 1 (the driver's line: headline,
partitioned c4 / c5, e2e, roofline) and N = 2 ranks sharing the one GPU over a
gloo process group (--backend gloo: the N > 1 code path -- rank partition,
max-over-ranks timing, gather, host-staged band halos -- on a single-GPU
box; NCCL refuses two ranks on one device).  Short runs: the numbers are not
the point, the contract fields are."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _bench(args, timeout=900):
    env = dict(os.environ)
    for k in ("WORLD_SIZE", "RANK", "LOCAL_RANK", "MASTER_ADDR", "MASTER_PORT"):
        env.pop(k, None)
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py")] + args, cwd=ROOT, env=env,
                       capture_output=True, text=True, timeout=timeout)
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert r.returncode == 0, r.stderr[-3000:]
    return json.loads(lines[-1])


def _check_partitioned(line, n):
    for name in ("c4", "c5"):
        rec = line["partitioned"][name]
        assert rec["n_gpus"] == n and rec["scaling"] == "strong" and len(rec["per_rank_ms"]) == n
        assert rec["value"] > 0 and rec["px_per_step"] == 1024 ** 3
        assert rec["gpu_launches"] == rec["steps"] * rec["launches_per_step_per_rank"]
    # rank 0 (the printing rank) receives one 6-row halo from below for n > 1 (clamp)
    assert line["partitioned"]["c5"]["halo_bytes_per_rank"] == (0 if n == 1 else 6 * 32768 * 4)


def test_bench_single_gpu_contract():
    line = _bench(["--steps", "10", "--warmup", "3", "--no-extras", "--no-cpu-baseline",
                   "--e2e-steps", "2", "--part-steps", "2"])
    assert line["n_gpus"] == 1 and line["unit"] == "Mpixel/s" and line["steps"] == 10
    assert line["gpu_launches"] == 10
    assert line["roofline"]["bound"] == "alu" and 0 < line["roofline"]["frac"] < 1.2
    e2e = line["e2e"]
    assert e2e["h2d_bytes_per_step"] >= 4096 * 4096 * 4 and e2e["d2h_bytes_per_step"] == 4096 * 4096 * 4
    assert 0 < e2e["frac"] <= 1.05
    _check_partitioned(line, 1)


def test_bench_two_ranks_on_one_gpu_gloo():
    line = _bench(["--gpus", "2", "--backend", "gloo", "--steps", "4", "--warmup", "3",
                   "--no-extras", "--e2e-steps", "0", "--part-steps", "2"])
    assert line["n_gpus"] == 2 and line["comm"]["world_size"] == 2
    assert line["comm"]["backend"] == "gloo"
    _check_partitioned(line, 2)
    assert line["partitioned"]["c4"]["config"]["frames_this_rank"] == [0, 512]

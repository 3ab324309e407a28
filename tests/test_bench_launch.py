"""bench.py launch plumbing without a GPU: `--gpus N` self-launches N ranks
under torch.distributed.run (127.0.0.1) and every rank takes its share of the
partitioned configs 4 (frames) and 5 (row bands); `--gpus` disagreeing with
WORLD_SIZE is an error ("Next round" item 1)."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(args, env=None, timeout=300):
    e = dict(os.environ)
    for k in ("WORLD_SIZE", "RANK", "LOCAL_RANK", "MASTER_ADDR", "MASTER_PORT"):
        e.pop(k, None)
    e.update(env or {})
    res = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py")] + args, cwd=ROOT,
                         env=e, capture_output=True, text=True, timeout=timeout)
    lines = [ln for ln in res.stdout.splitlines() if ln.startswith("{")]
    return res, (json.loads(lines[-1]) if lines else None)


@pytest.mark.parametrize("n", [2, 3])
def test_gpus_n_spawns_n_ranks(n):
    res, line = _run(["--gpus", str(n), "--dry-run"])
    assert res.returncode == 0, res.stderr[-2000:]
    assert line["dry_run"] and line["n_gpus"] == n
    assert line["comm"] == {"backend": "gloo", "world_size": n}
    ranks = line["ranks"]
    assert [r["rank"] for r in ranks] == list(range(n))
    assert len({r["pid"] for r in ranks}) == n                    # n distinct processes
    # frames (config 4) and bands (config 5) tile their index ranges exactly
    assert ranks[0]["c4_frames"][0] == 0 and ranks[-1]["c4_frames"][1] == 1024
    assert ranks[0]["c5_rows"][0] == 0 and ranks[-1]["c5_rows"][1] == 32768
    for a, b in zip(ranks, ranks[1:]):
        assert a["c4_frames"][1] == b["c4_frames"][0] and a["c5_rows"][1] == b["c5_rows"][0]
    assert line["c4_frames_total"] == 1024
    assert "%d ranks" % n in res.stderr


def test_single_rank_default():
    res, line = _run(["--dry-run"])
    assert res.returncode == 0 and line["n_gpus"] == 1 and len(line["ranks"]) == 1


def test_gpus_disagreeing_with_world_size_fails():
    res, line = _run(["--gpus", "3", "--dry-run"], env={"WORLD_SIZE": "2", "RANK": "0"})
    assert res.returncode == 2 and "disagrees" in line["error"]

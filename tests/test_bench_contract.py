"""bench.py's JSON contract on the CPU-only arm (--impl reference: the oracle, timed on the
host cores): one JSON line with the keys the driver reads. The GPU arm's line is produced by
the same code path after the timed region (checked on the GPU box by running bench.py)."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.parametrize("wl", ["sdh_uniform_4k"])
def test_reference_arm_json_line(wl):
    r = subprocess.run([sys.executable, "bench.py", "--impl", "reference", "--workload", wl, "--steps", "1",
                        "--warmup", "0", "--cpu-seconds", "0.5"], cwd=ROOT, capture_output=True, text=True,
                       timeout=600)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    for k in ("impl", "metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
              "scaling", "vs_baseline", "dtype", "data", "config", "cpu_baseline", "e2e"):
        assert k in d, k
    assert d["impl"] == "reference" and d["value"] > 0 and d["config"]["workload"] == wl
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["value"] == d["value"]


@pytest.mark.parametrize("gpus", [2, 3])
def test_self_launch_reaches_n_ranks(gpus):
    """`python bench.py --gpus N` with no torchrun around it re-launches itself with N ranks
    (torch.distributed.run, 127.0.0.1 rendezvous); --dry-run joins a gloo group instead of
    NCCL, so the launch path is testable on CPU. The ranks' strips are the pair-balanced
    partition of the workload (disjoint, covering [0, n))."""
    r = subprocess.run([sys.executable, "bench.py", "--gpus", str(gpus), "--dry-run", "--workload", "sdh_uniform_4m"],
                       cwd=ROOT, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout
    d = json.loads(lines[0])
    assert d["dry_run"] and d["n_gpus"] == gpus and d["gpus_requested"] == gpus and d["combine"] == "nccl"
    assert sorted(x["rank"] for x in d["ranks"]) == list(range(gpus))
    assert len({x["pid"] for x in d["ranks"]}) == gpus            # one process per rank
    rows = sorted(tuple(x["rows"]) for x in d["ranks"])
    assert rows[0][0] == 0 and rows[-1][1] == d["n"]
    assert all(a[1] == b[0] for a, b in zip(rows, rows[1:]))


def test_world_size_must_match_gpus():
    """Under torchrun, --gpus must equal WORLD_SIZE (no silent single-GPU run)."""
    env = dict(os.environ, WORLD_SIZE="1", RANK="0", LOCAL_RANK="0")
    r = subprocess.run([sys.executable, "bench.py", "--gpus", "2", "--dry-run"], cwd=ROOT, capture_output=True,
                       text=True, timeout=300, env=env)
    assert r.returncode != 0 and "WORLD_SIZE = 1 but --gpus 2" in r.stderr

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

"""The kept round-2 evidence (profiles/r02_bench_*.json) is self-consistent: every bench line
carries the contract's keys, a clock record taken inside the timed region with no throttle
reason, and a roofline fraction that recomputes from its own achieved / peak; the value
recomputes from the workload's units and the step time. (CPU only: reads the files.)"""
import glob
import json
import os

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LINES = sorted(glob.glob(os.path.join(ROOT, "profiles", "r02_bench_*.json")))
BAD_REASONS = {"hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown"}


def load(path):
    with open(path) as f:
        return json.loads(f.read().strip().splitlines()[-1])


@pytest.mark.parametrize("path", LINES, ids=[os.path.basename(p) for p in LINES])
def test_bench_line_contract(path):
    d = load(path)
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
              "scaling", "dtype", "data", "config"):
        assert k in d, k
    assert d["value"] > 0 and d["warmup"] >= 3 or d.get("impl") == "reference"
    if d.get("impl") == "reference":
        assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
        return
    assert d["gpu_launches"] >= d["steps"]
    ck = d["clocks"]
    assert ck and ck["samples_inside"] >= 1
    assert not (set(ck["reasons"]) & BAD_REASONS)
    assert ck["sm_mhz"] >= 0.95 * ck["sm_max_mhz"]
    r = d["roofline"]
    assert r["bound"] in ("alu", "hbm", "tensor")
    assert abs(r["frac"] - r["achieved"] / r["peak"]) <= 1e-9 * max(1.0, r["frac"])
    e = d["e2e"]
    if e is not None:
        assert e["value"] > 0 and e["h2d_bytes_per_step"] > 0 and e["d2h_bytes_per_step"] > 0


def test_default_line_is_the_north_star_metric():
    d = load(os.path.join(ROOT, "profiles", "r02_bench_sdh_uniform_1m.json"))
    base = json.load(open(os.path.join(ROOT, "BASELINE.json")))
    assert d["metric"] == base["metric"]
    assert d["config"]["workload"] == "sdh_uniform_1m" and d["config"]["n"] == 1 << 20 and d["config"]["nb"] == 256
    assert d["cpu_baseline"]["kind"] == "oracle"
    # value = n(n-1)/2 pairs per step / step time
    n = d["config"]["n"]
    assert abs(d["value"] - n * (n - 1) / 2 / (d["ms_per_step"] * 1e-3) / 1e9) <= 1e-6 * d["value"]
    assert d["roofline"]["frac"] >= 0.6   # the north star's per-GPU bar

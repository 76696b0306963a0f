"""Write large-n golden results with the CPU oracle ONLY (never the CUDA path).

Usage: python tools/make_goldens.py <name> [<name> ...]   (names: see GOLDENS)
Each golden is tests/golden/<name>.json holding the inputs' recipe (generator,
seed, n), the parameters, the oracle's output (hist + edge-ambiguity counts, or
count + ambiguity) and how long the oracle took on how many threads.
"""
import json
import math
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
import tbs_inputs as g  # noqa: E402

GOLDENS = {
    # BASELINE.json configs[1]: SDH N=1M uniform 3D, 256 buckets (seed 2)
    "sdh_uniform_n1048576_nb256_seed2": dict(op="sdh", kind="uniform", n=1 << 20, seed=2, nb=256),
    # 2PCF on the clustered generator at N=1M (r = 0.03), a C3-recipe case small enough for the oracle
    "pcf_clustered_n1048576_r0.03_seed3": dict(op="pcf", kind="clustered", n=1 << 20, seed=3, r=0.03),
    # BASELINE.json configs[3] recipe at full size: SDH N=2M uniform, 16384 buckets (seed 4)
    "sdh_uniform_n2097152_nb16384_seed4": dict(op="sdh", kind="uniform", n=1 << 21, seed=4, nb=16384),
    # the north-star line at full size: SDH N=4M uniform, 256 buckets (seed 6)
    "sdh_uniform_n4194304_nb256_seed6": dict(op="sdh", kind="uniform", n=1 << 22, seed=6, nb=256),
    # BASELINE.json configs[2] at full size: 2PCF N=4M clustered, r = 0.03 (C3, seed 3)
    "pcf_clustered_n4194304_r0.03_seed3": dict(op="pcf", kind="clustered", n=1 << 22, seed=3, r=0.03),
    # BASELINE.json configs[0]: SDH N=4096 uniform, 64 buckets (seed 1)
    "sdh_uniform_n4096_nb64_seed1": dict(op="sdh", kind="uniform", n=4096, seed=1, nb=64),
}


def make(name):
    spec = GOLDENS[name]
    p = g.make(spec["kind"], spec["n"], spec["seed"])
    t0 = time.time()
    out = dict(name=name, spec=spec, generator="tbs_inputs." + spec["kind"], script="tools/make_goldens.py",
               threads=oracle.num_threads())
    if spec["op"] == "sdh":
        w = float(np.float32(math.sqrt(3) / spec["nb"]))
        h, a = oracle.sdh(p, w, spec["nb"])
        out.update(w=w, hist=[int(x) for x in h], amb=[int(x) for x in a])
    else:
        c, a = oracle.pcf(p, spec["r"])
        out.update(r=float(np.float32(spec["r"])), count=c, amb=a)
    out["oracle_seconds"] = round(time.time() - t0, 2)
    with open(os.path.join(ROOT, "tests", "golden", name + ".json"), "w") as f:
        json.dump(out, f, indent=0)
    print(name, out["oracle_seconds"], "s")


if __name__ == "__main__":
    for nm in sys.argv[1:]:
        make(nm)

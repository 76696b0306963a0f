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


def part_rows(n, parts, k):
    """Anchor rows of part k of `parts` with equal pair counts (sum over rows i of n-1-i):
    boundary R solves R (2n - R - 1) / 2 = k/parts * n (n - 1) / 2. Parts are disjoint and
    cover [0, n); the oracle's outputs over them add up to the full result."""
    def bound(j):
        if j == 0:
            return 0
        if j == parts:
            return n
        a = 2 * n - 1
        return int(round((a - math.sqrt(a * a - 4.0 * j / parts * n * (n - 1))) / 2))
    return bound(k), bound(k + 1)


def make(name, part=None, parts=None, outdir=None):
    """The golden `name`, or (part, parts) its k-th pair-balanced anchor-row part (for
    oracle runs longer than one job; merged by merge())."""
    spec = GOLDENS[name]
    p = g.make(spec["kind"], spec["n"], spec["seed"])
    rows = None if part is None else part_rows(spec["n"], parts, part)
    t0 = time.time()
    out = dict(name=name, spec=spec, generator="tbs_inputs." + spec["kind"], script="tools/make_goldens.py",
               threads=oracle.num_threads())
    if rows is not None:
        out.update(rows=list(rows), part=part, parts=parts)
    if spec["op"] == "sdh":
        w = float(np.float32(math.sqrt(3) / spec["nb"]))
        h, a = oracle.sdh(p, w, spec["nb"], rows=rows)
        out.update(w=w, hist=[int(x) for x in h], amb=[int(x) for x in a])
    else:
        c, a = oracle.pcf(p, spec["r"], rows=rows)
        out.update(r=float(np.float32(spec["r"])), count=c, amb=a)
    out["oracle_seconds"] = round(time.time() - t0, 2)
    fn = name + ("" if rows is None else f".part{part}of{parts}") + ".json"
    with open(os.path.join(outdir or os.path.join(ROOT, "tests", "golden"), fn), "w") as f:
        json.dump(out, f, indent=0)
    print(fn, out["oracle_seconds"], "s")


def make_split(name, part, parts, outdir, split):
    """Part `part` of `parts` computed as `split` pair-balanced anchor-row sub-ranges, one
    oracle call each (every call uses all OpenMP threads on rows of similar cost: a single call
    over a long triangular range leaves the threads holding its first, heaviest guided chunks
    running long after the others). The sub-range outputs are integer counts and add up to
    the part's; the file is the same as make(name, part, parts) writes."""
    spec = GOLDENS[name]
    n = spec["n"]
    p = g.make(spec["kind"], n, spec["seed"])
    b, e = part_rows(n, parts, part)
    # sub-range boundaries with equal pair counts inside [b, e)
    S = lambda x: x * (2 * n - x - 1) // 2
    tot = S(e) - S(b)
    bounds = [b]
    for k in range(1, split):
        target = S(b) + tot * k // split
        lo, hi = bounds[-1], e
        while lo < hi:
            mid = (lo + hi) // 2
            if S(mid) < target:
                lo = mid + 1
            else:
                hi = mid
        bounds.append(lo)
    bounds.append(e)
    t0 = time.time()
    w = float(np.float32(math.sqrt(3) / spec["nb"]))
    hist = np.zeros(spec["nb"], np.uint64)
    amb = np.zeros(spec["nb"] + 1, np.uint64)
    for k in range(split):
        h, a = oracle.sdh(p, w, spec["nb"], rows=(bounds[k], bounds[k + 1]))
        hist += h
        amb += a
        print(f"sub-range {k + 1}/{split} rows [{bounds[k]}, {bounds[k + 1]}) {time.time() - t0:.0f} s", flush=True)
    out = dict(name=name, spec=spec, generator="tbs_inputs." + spec["kind"], script="tools/make_goldens.py",
               threads=oracle.num_threads(), rows=[b, e], part=part, parts=parts, split=split,
               w=w, hist=[int(x) for x in hist], amb=[int(x) for x in amb], oracle_seconds=round(time.time() - t0, 2))
    fn = f"{name}.part{part}of{parts}.json"
    with open(os.path.join(outdir, fn), "w") as f:
        json.dump(out, f, indent=0)
    print(fn, out["oracle_seconds"], "s")


def merge(name, files):
    """Sum the parts' oracle outputs (integer counts: order-independent) into the golden."""
    ds = [json.load(open(f)) for f in files]
    parts = ds[0]["parts"]
    assert sorted(d["part"] for d in ds) == list(range(parts)) and all(d["name"] == name for d in ds)
    out = dict(name=name, spec=ds[0]["spec"], generator=ds[0]["generator"], script="tools/make_goldens.py",
               threads=ds[0]["threads"], merged_parts=[d["rows"] for d in sorted(ds, key=lambda d: d["part"])],
               oracle_seconds=round(sum(d["oracle_seconds"] for d in ds), 2))
    if "hist" in ds[0]:
        out.update(w=ds[0]["w"], hist=[int(sum(v)) for v in zip(*(d["hist"] for d in ds))],
                   amb=[int(sum(v)) for v in zip(*(d["amb"] for d in ds))])
    else:
        out.update(r=ds[0]["r"], count=sum(d["count"] for d in ds), amb=sum(d["amb"] for d in ds))
    with open(os.path.join(ROOT, "tests", "golden", name + ".json"), "w") as f:
        json.dump(out, f, indent=0)
    print(name, "merged from", len(ds), "parts")


if __name__ == "__main__":
    # python tools/make_goldens.py NAME...                    full goldens
    # python tools/make_goldens.py --part K PARTS OUTDIR NAME  one pair-balanced row part
    # python tools/make_goldens.py --part-split K PARTS OUTDIR NAME SPLIT   the part as SPLIT sub-ranges
    # python tools/make_goldens.py --merge NAME PART_FILE...   sum the parts
    a = sys.argv[1:]
    if a and a[0] == "--part":
        make(a[4], int(a[1]), int(a[2]), a[3])
    elif a and a[0] == "--part-split":      # --part-split K PARTS OUTDIR NAME SPLIT (SDH goldens)
        make_split(a[4], int(a[1]), int(a[2]), a[3], int(a[5]))
    elif a and a[0] == "--merge":
        merge(a[1], a[2:])
    else:
        for nm in a:
            make(nm)

"""B200 ablations of the paper's experiments, one JSON line each.

  nb sweep            (Fig. 5, L946-996 / L1020-1035): SDH N=1M uniform, default output stage
  output stage        (Fig. 4): lane-private (R=32) vs one copy per CTA vs global atomics
  clamp elision       (this design): bounding-box-proved no-clamp vs forced clamp
  clustered vs uniform(L1031-1035 contention remark): lane-private copies have no same-address traffic
Timing: CUDA events around each call after 2 warm-ups, best of 3.
"""
import json
import math
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_pitaksirianannt16_b200 as tbs  # noqa: E402
import tbs_inputs as g  # noqa: E402


def timed(f, reps=3):
    for _ in range(2):
        f()
    best = 1e30
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        f()
        b.record()
        torch.cuda.synchronize()
        best = min(best, a.elapsed_time(b))
    return best


def emit(**kw):
    print(json.dumps(kw), flush=True)


n = int(os.environ.get("ABL_N", 1 << 20))
pairs = n * (n - 1) // 2
pu = torch.from_numpy(g.uniform(n, 2)).cuda()
pc = torch.from_numpy(g.clustered(n, 3)).cuda()
for nb in (16, 64, 256, 512, 768, 1024, 2048, 4096, 6144, 8192, 16384, 32768, 49152, 65536, 98304, 131072):
    w = float(np.float32(math.sqrt(3) / nb))
    ms = timed(lambda: tbs.sdh(pu, w, nb))
    emit(ablation="nb_sweep", n=n, nb=nb, ms=ms, gpairs_s=pairs / ms / 1e6)
for mode in ("lane", "cta", "global"):
    w = float(np.float32(math.sqrt(3) / 256))
    ms = timed(lambda: tbs.sdh(pu, w, 256, hist_mode=mode), reps=1 if mode == "global" else 3)
    emit(ablation="output_stage", n=n, nb=256, mode=mode, ms=ms, gpairs_s=pairs / ms / 1e6)
for fc in (False, True):
    w = float(np.float32(math.sqrt(3) / 256))
    ms = timed(lambda: tbs.sdh(pu, w, 256, force_clamp=fc))
    emit(ablation="clamp", n=n, nb=256, force_clamp=fc, ms=ms, gpairs_s=pairs / ms / 1e6)
for name, p in (("uniform", pu), ("clustered", pc)):
    for nb in (64, 256, 16384):
        w = float(np.float32(math.sqrt(3) / nb))
        ms = timed(lambda: tbs.sdh(p, w, nb))
        emit(ablation="distribution", n=n, nb=nb, data=name, ms=ms, gpairs_s=pairs / ms / 1e6)
for m in (4096, 16384, 65536, 262144):
    q = torch.from_numpy(g.uniform(m, 1)).cuda()
    w = float(np.float32(math.sqrt(3) / 64))
    ms = timed(lambda: tbs.sdh(q, w, 64), reps=10)
    emit(ablation="size_sweep", n=m, nb=64, ms=ms, gpairs_s=m * (m - 1) / 2 / ms / 1e6)

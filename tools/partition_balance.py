"""Multi-GPU proxy on one B200 ("Multi-GPU without a cluster"): run each rank's
pair-balanced anchor strip (tbs_rank_rows) of the N=4M SDH / 2PCF on the single GPU, time
it with CUDA events, and report the strong-scaling efficiency the partition implies,
t_1 / (W * max_r t_r). The all-reduce (<= 2 KB here) is not included (NVLink latency ~10-30 us).
Also checks that the strips' partial results sum to the single-GPU result bit-exactly."""
import json
import math
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_pitaksirianannt16_b200 as tbs  # noqa: E402
import tbs_inputs as g  # noqa: E402


def timed(f):
    f()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    r = f()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b), r


n = int(os.environ.get("PB_N", 1 << 22))
for name, p, call in (
        ("sdh_uniform_4m", torch.from_numpy(g.uniform(n, 6)).cuda(),
         lambda p, rows: tbs.sdh(p, float(np.float32(math.sqrt(3) / 256)), 256, rows=rows)),
        ("pcf_clustered_4m", torch.from_numpy(g.clustered(n, 3)).cuda(),
         lambda p, rows: tbs.pcf(p, 0.03, rows=rows))):
    t1, full = timed(lambda: call(p, None))
    for W in (2, 4, 8):
        times, acc = [], None
        for r in range(W):
            rows = tbs.rank_rows(n, W, r)
            t, part = timed(lambda: call(p, rows))
            times.append(t)
            acc = part.clone() if acc is None else acc + part
        exact = bool(torch.equal(acc, full))
        print(json.dumps(dict(workload=name, n=n, world=W, t1_ms=t1, rank_ms=times,
                              efficiency=t1 / (W * max(times)), imbalance=max(times) / min(times),
                              sum_bit_exact=exact)), flush=True)

"""C1 (N = 4096, 64 buckets) kernel probe: per-call kernel time (CUDA events around the pair
kernel) for output-stage replications R and occupancy caps, printed as JSON lines. Env knobs
are the library's experiment hooks (TBS_LOG2R, TBS_OCC) and must be set before import."""
import json
import math
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_pitaksirianannt16_b200 as tbs  # noqa: E402
import tbs_inputs as g  # noqa: E402

n, nb = 4096, 64
w = float(np.float32(math.sqrt(3) / nb))
p = torch.from_numpy(g.uniform(n, 1)).cuda()
out = torch.empty(nb, dtype=torch.int64, device="cuda")
ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(200)]
for a, b in ev:            # materialise the cudaEvent_t handles passed through the C ABI
    a.record()
    b.record()
for _ in range(20):
    tbs.sdh(p, w, nb, out=out)
torch.cuda.synchronize()
for e in ev:
    tbs.sdh(p, w, nb, out=out, events=e)
torch.cuda.synchronize()
t = sorted(a.elapsed_time(b) * 1e3 for a, b in ev)
print(json.dumps(dict(log2r=os.environ.get("TBS_LOG2R"), occ=os.environ.get("TBS_OCC"), small=os.environ.get("TBS_SMALL_ITEMS"),
                      us_median=t[len(t) // 2], us_min=t[0], sum=int(out.sum().item()))))

"""Minimal driver for ncu captures: one warm-up call + one profiled call of a workload."""
import math
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_pitaksirianannt16_b200 as tbs  # noqa: E402
import tbs_inputs as g  # noqa: E402

wl = sys.argv[1] if len(sys.argv) > 1 else "sdh1m"
if wl == "sdh1m":
    p = torch.from_numpy(g.uniform(1 << 20, 2)).cuda()
    f = lambda: tbs.sdh(p, float(np.float32(math.sqrt(3) / 256)), 256)
elif wl == "pcf4m":
    p = torch.from_numpy(g.clustered(1 << 22, 3)).cuda()
    f = lambda: tbs.pcf(p, 0.03)
elif wl == "pcf1m":
    p = torch.from_numpy(g.clustered(1 << 20, 3)).cuda()
    f = lambda: tbs.pcf(p, 0.03)
elif wl == "sdh16k":
    p = torch.from_numpy(g.uniform(1 << 21, 4)).cuda()
    f = lambda: tbs.sdh(p, float(np.float32(math.sqrt(3) / 16384)), 16384)
elif wl == "hd64k":
    p = torch.from_numpy(g.uniform(1 << 16, 7, 64)).cuda().to(torch.bfloat16)
    f = lambda: tbs.pairmatrix_hd(p, 1.0 / 64)
elif wl == "pm64k":
    p = torch.from_numpy(g.uniform(1 << 16, 5)).cuda()
    f = lambda: tbs.pairmatrix(p, 1.0)
for _ in range(2):
    f()
torch.cuda.synchronize()
print("ok", wl)

"""A/B helper: SDH N=1M uniform at the given bucket counts (and forced output stages), best of
3 after 2 warm-ups; the library is the in-tree one or TBS_LIB_VARIANT. One JSON line each."""
import json
import math
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_pitaksirianannt16_b200 as tbs  # noqa: E402
import tbs_inputs as g  # noqa: E402

n = int(os.environ.get("ABL_N", 1 << 20))
pairs = n * (n - 1) // 2
pu = torch.from_numpy(g.uniform(n, 2)).cuda()
lib = os.path.basename(os.environ.get("TBS_LIB_VARIANT", "") or "main")
for spec in sys.argv[1:]:          # nb or nb:mode
    nb, _, mode = spec.partition(":")
    nb = int(nb)
    w = float(np.float32(math.sqrt(3) / nb))
    f = lambda: tbs.sdh(pu, w, nb, hist_mode=mode or None)
    for _ in range(2):
        f()
    best = 1e30
    for _ in range(3):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        f()
        b.record()
        torch.cuda.synchronize()
        best = min(best, a.elapsed_time(b))
    print(json.dumps(dict(lib=lib, n=n, nb=nb, mode=mode or "default", ms=round(best, 3), gpairs_s=round(pairs / best / 1e6, 1))), flush=True)

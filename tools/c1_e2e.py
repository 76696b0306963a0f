"""Host-side cost of the small-problem (BASELINE configs[0], N = 4096) call paths, per call:
the C-ABI host-pointer entry point (pinned / pageable input), the device path with explicit
copies, and the bare ctypes round trip. Prints one JSON line."""
import ctypes
import json
import math
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_pitaksirianannt16_b200 as tbs  # noqa: E402
import tbs_inputs as g  # noqa: E402

n, nb = 4096, 64
w = float(np.float32(math.sqrt(3) / nb))
p = g.uniform(n, 1)
pin = torch.from_numpy(p).pin_memory()
hh = np.zeros(nb, np.uint64)
dev = torch.device("cuda")
res = torch.empty(nb, dtype=torch.int64).pin_memory()


def per_call(f, k=2000):
    for _ in range(50):
        f()
    torch.cuda.synchronize()
    t = time.perf_counter()
    for _ in range(k):
        f()
    torch.cuda.synchronize()
    return (time.perf_counter() - t) / k * 1e6


def dev_path():
    d = pin.to(dev, non_blocking=True)
    res.copy_(tbs.sdh(d, w, nb))
    torch.cuda.current_stream().synchronize()


dp = pin.to(dev)
dout = torch.empty(nb, dtype=torch.int64, device=dev)
tiny = torch.zeros(1, device=dev)


def dev_only():
    tbs.sdh(dp, w, nb, out=dout)
    torch.cuda.current_stream().synchronize()


def floor_sync():
    tiny.add_(1.0)
    torch.cuda.current_stream().synchronize()


out = dict(n=n, nb=nb,
           us_one_torch_kernel_plus_sync=per_call(floor_sync),
           us_device_call_plus_sync=per_call(dev_only),
           us_ctypes_roundtrip=per_call(lambda: tbs.lib().tbs_version(), 20000),
           us_host_entry_pinned_in=per_call(lambda: tbs.sdh_host(pin.numpy(), w, nb, out=hh)),
           us_host_entry_pageable_in=per_call(lambda: tbs.sdh_host(p, w, nb, out=hh)),
           us_device_path_with_copies=per_call(dev_path))
pairs = n * (n - 1) / 2
out["gpairs_s_host_entry_pinned"] = pairs / out["us_host_entry_pinned_in"] / 1e3
print(json.dumps(out))

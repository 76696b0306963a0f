"""GPU tests of the windowed large-nb SDH stage (tbs_win.cuh, BASELINE
configs[3]). The points are reordered in space and every work item counts into a window of
buckets; the histogram is a function of the point set, and every pair's fp32 distance is computed
from the same two coordinates either way (p - a vs a - p: the same magnitude), so the windowed
histogram must equal the plain GPU histogram bit for bit — and meet the oracle's A_e rule."""
import json
import math
import os

import numpy as np
import pytest

import oracle
import tbs_inputs as g
from parity import check_sdh_float

pytestmark = pytest.mark.gpu
GOLD = os.path.join(os.path.dirname(__file__), "golden")


def hist(tbs, p, w, nb, mode):
    import torch
    h = tbs.sdh(torch.from_numpy(np.ascontiguousarray(p)).cuda(), w, nb, hist_mode=mode)
    torch.cuda.synchronize()
    return h.cpu().numpy().astype(np.uint64)


def w_of(nb, dim=3):
    return float(np.float32(math.sqrt(dim) / nb))


@pytest.mark.parametrize("nb", [1024, 16384, 70000])
@pytest.mark.parametrize("gen", ["uniform", "clustered"])
def test_window_equals_plain(tbs, nb, gen):
    """Single-segment items (nb 1024), multi-segment items (16384: ~4700-bucket intervals against
    a ~3400-row window at 70K points), and a plan that would otherwise take bucket passes."""
    n = 70001
    p = g.uniform(n, 41) if gen == "uniform" else g.clustered(n, 42)
    w = w_of(min(nb, 16384))
    hw = hist(tbs, p, w, nb, "window")
    hp = hist(tbs, p, w, nb, "nowindow")
    assert int(hw.sum()) == n * (n - 1) // 2
    assert hw.tolist() == hp.tolist()


def test_window_vs_oracle(tbs):
    n, nb = 66000, 16384
    p = g.clustered(n, 43)
    w = w_of(nb)
    ho, amb = oracle.sdh(p, w, nb)
    check_sdh_float(hist(tbs, p, w, nb, "window"), ho, amb)


@pytest.mark.parametrize("dim", [1, 2])
def test_window_low_dims_and_offset(tbs, dim):
    """dims 1 / 2 (padded coordinates are 0) and coordinates offset by 1000 (the ordering and the
    boxes work in absolute coordinates; the distances stay subtract-then-square)."""
    n, nb = 80000, 8192
    p = g.uniform(n, 44, dim) + (1000.0 if dim == 2 else 0.0)
    p = p.astype(np.float32)
    w = w_of(nb, dim)
    assert hist(tbs, p, w, nb, "window").tolist() == hist(tbs, p, w, nb, "nowindow").tolist()


def test_window_row_range_falls_back(tbs):
    """A row range names anchors by the caller's order: the windowed stage does not apply and
    the call equals the plain one."""
    import torch
    n, nb = 70000, 16384
    p = torch.from_numpy(g.uniform(n, 45)).cuda()
    a = tbs.sdh(p, w_of(nb), nb, rows=(1000, 30000), hist_mode="window").cpu().tolist()
    b = tbs.sdh(p, w_of(nb), nb, rows=(1000, 30000), hist_mode="nowindow").cpu().tolist()
    assert a == b


def test_window_2m_16k_golden(tbs):
    """BASELINE configs[3] at full size: the windowed histogram against the oracle golden and
    bit-equal to the plain two-replica stage."""
    n, nb = 1 << 21, 16384
    p = g.uniform(n, 4)
    hw = hist(tbs, p, w_of(nb), nb, "window")
    assert int(hw.sum()) == n * (n - 1) // 2
    gp = os.path.join(GOLD, "sdh_uniform_n2097152_nb16384_seed4.json")
    gold = json.load(open(gp))
    check_sdh_float(hw, gold["hist"], gold["amb"])
    assert hw.tolist() == hist(tbs, p, w_of(nb), nb, "nowindow").tolist()

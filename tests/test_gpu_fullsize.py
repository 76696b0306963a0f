"""GPU parity at BASELINE.json's full sizes, in the launch configuration bench.py times
(the default tbs.sdh / tbs.pcf / tbs.pairmatrix paths).

Where the O(N^2) oracle is too slow, the check is either (a) against a committed
golden written by tools/make_goldens.py (oracle only), (b) against the oracle on
sampled anchor strips (the row-range API computes exactly those pairs), or (c)
against the O(L^3) exact lattice closed form (oracle.lattice_closed), plus the
histogram-mass invariant.
"""
import json
import math
import os

import numpy as np
import pytest

import oracle
import tbs_inputs as g
from parity import check_knn_float, check_matrix, check_pcf_float, check_sdh_float

pytestmark = pytest.mark.gpu
GOLD = os.path.join(os.path.dirname(__file__), "golden")


def dev(p):
    import torch
    return torch.from_numpy(np.ascontiguousarray(p)).cuda()


def host(t):
    import torch
    torch.cuda.synchronize()
    return t.cpu().numpy()


def strips(n, width=48):
    return [(0, width), (n // 2, n // 2 + width), (n - width, n)]


def w_of(nb):
    return float(np.float32(math.sqrt(3) / nb))


# ---------------------------------------------------------------- configs[1]: SDH N=1M, 256 buckets
def test_sdh_1m_uniform_vs_golden(tbs):
    gold = json.load(open(os.path.join(GOLD, "sdh_uniform_n1048576_nb256_seed2.json")))
    p = g.uniform(1 << 20, 2)
    h = host(tbs.sdh(dev(p), gold["w"], 256)).astype(np.uint64)
    d = check_sdh_float(h, gold["hist"], gold["amb"])
    assert int(h.sum()) == (1 << 20) * ((1 << 20) - 1) // 2
    print("1M golden:", d)


def test_sdh_1m_lattice_exact(tbs):
    """L=100 lattice (N=10^6), w=1, 256 buckets (172 populated): exact vs closed form."""
    p = g.lattice(100, 2)
    h = host(tbs.sdh(dev(p), 1.0, 256, lattice=True))
    assert h.tolist() == oracle.lattice_closed(100, 1, 0, 256)[0].tolist()


# ---------------------------------------------------------------- 2PCF (configs[2])
def test_pcf_1m_clustered_vs_golden(tbs):
    gold = json.load(open(os.path.join(GOLD, "pcf_clustered_n1048576_r0.03_seed3.json")))
    p = g.clustered(1 << 20, 3)
    c = int(host(tbs.pcf(dev(p), 0.03))[0])
    check_pcf_float(c, gold["count"], gold["amb"])


def test_pcf_4m_clustered_vs_golden(tbs):
    """BASELINE.json configs[2] at full size: N=4M clustered, r=0.03 against the full oracle
    count (tools/make_goldens.py, 8.8e12 pairs on the CPU)."""
    gold = json.load(open(os.path.join(GOLD, "pcf_clustered_n4194304_r0.03_seed3.json")))
    p = g.clustered(1 << 22, 3)
    c = int(host(tbs.pcf(dev(p), 0.03))[0])
    check_pcf_float(c, gold["count"], gold["amb"])
    assert c > 2 ** 32


def test_pcf_4m_clustered_strips(tbs):
    n = 1 << 22
    p = g.clustered(n, 3)
    d = dev(p)
    for rows in strips(n):
        c = int(host(tbs.pcf(d, 0.03, rows=rows))[0])
        co, amb = oracle.pcf(p, 0.03, rows=rows)
        check_pcf_float(c, co, amb)
    total = int(host(tbs.pcf(d, 0.03))[0])
    assert total > 2 ** 32            # the count needs the u64 path
    acc = 0
    for r in range(8):                 # the 8-rank partition sums to the single-GPU count exactly
        acc += int(host(tbs.pcf(d, 0.03, rows=tbs.rank_rows(n, 8, r)))[0])
    assert acc == total


def test_pcf_4m_lattice_exact(tbs):
    """L=160 lattice (N=4,096,000), r=10 (r^2 = 100 exact): exact vs closed form."""
    p = g.lattice(160, 6)
    c = int(host(tbs.pcf(dev(p), 10.0))[0])
    assert c == oracle.lattice_closed(160, 1, 0, 1, r2=100)[1]


# ---------------------------------------------------------------- configs[3]: N=2M, 16384 buckets
@pytest.mark.parametrize("mode", [None, "global"])
def test_sdh_2m_16k_lattice_exact(tbs, mode):
    """L=128 lattice (N=2^21), w=2^-6, 16384 buckets (highest bucket 14078): exact vs closed form,
    default (smem) output stage and the partially privatised global histogram."""
    p = g.lattice(128, 4)
    h = host(tbs.sdh(dev(p), 2.0 ** -6, 16384, lattice=True, hist_mode=mode))
    ref = oracle.lattice_closed(128, 1, 6, 16384)[0]
    assert h.tolist() == ref.tolist()
    assert int(np.nonzero(ref)[0].max()) == 14078      # floor(64 * sqrt(3) * 127)


@pytest.mark.parametrize("mode", [None, "global"])
def test_sdh_2m_16k_uniform(tbs, mode):
    n, nb = 1 << 21, 16384
    p = g.uniform(n, 4)
    d = dev(p)
    h = host(tbs.sdh(d, w_of(nb), nb, hist_mode=mode)).astype(np.uint64)
    assert int(h.sum()) == n * (n - 1) // 2
    gp = os.path.join(GOLD, "sdh_uniform_n2097152_nb16384_seed4.json")
    if os.path.exists(gp):
        gold = json.load(open(gp))
        check_sdh_float(h, gold["hist"], gold["amb"])
    for rows in strips(n, 32):
        hs = host(tbs.sdh(d, w_of(nb), nb, rows=rows, hist_mode=mode))
        ho, amb = oracle.sdh(p, w_of(nb), nb, rows=rows)
        check_sdh_float(hs, ho, amb)


# ---------------------------------------------------------------- north-star line: SDH N=4M, 256 buckets
def test_sdh_4m_uniform_strips_and_mass(tbs):
    n = 1 << 22
    p = g.uniform(n, 6)
    d = dev(p)
    h = host(tbs.sdh(d, w_of(256), 256))
    assert int(h.sum()) == n * (n - 1) // 2
    for rows in strips(n):
        hs = host(tbs.sdh(d, w_of(256), 256, rows=rows))
        ho, amb = oracle.sdh(p, w_of(256), 256, rows=rows)
        check_sdh_float(hs, ho, amb)


@pytest.mark.parametrize("part", [0, 1])
def test_sdh_4m_uniform_vs_golden_part(tbs, part):
    """North-star workload at full size on each pair-balanced anchor-row part (rows [0, 1228483)
    and [1228483, 4194304): half of the 8.8e12 pairs each) through the row-range API, against the
    CPU oracle's histogram of exactly those pairs (tools/make_goldens.py --part 0 2: 43 min;
    --part-split 1 2 ... 48: 43 min, both on a GPU box's 16 host threads)."""
    gold = json.load(open(os.path.join(GOLD, "parts", f"sdh_uniform_n4194304_nb256_seed6.part{part}of2.json")))
    n = gold["spec"]["n"]
    rb, re = gold["rows"]
    p = g.uniform(n, gold["spec"]["seed"])
    h = host(tbs.sdh(dev(p), gold["w"], 256, rows=(rb, re))).astype(np.uint64)
    d = check_sdh_float(h, gold["hist"], gold["amb"])
    # pairs (i, j), rb <= i < re, i < j < n
    assert int(h.sum()) == sum(gold["hist"]) == (re - rb) * (2 * n - rb - re - 1) // 2
    print(f"4M golden part {part}:", d)


def test_sdh_4m_uniform_vs_golden(tbs):
    """North-star workload at full size, whole histogram (bench.py's default launch, all
    8.8e12 pairs) against the merged oracle golden (both pair-balanced parts)."""
    gold = json.load(open(os.path.join(GOLD, "sdh_uniform_n4194304_nb256_seed6.json")))
    assert gold["merged_parts"] == [[0, 1228483], [1228483, 4194304]]
    n = gold["spec"]["n"]
    p = g.uniform(n, gold["spec"]["seed"])
    h = host(tbs.sdh(dev(p), gold["w"], 256)).astype(np.uint64)
    d = check_sdh_float(h, gold["hist"], gold["amb"])
    assert int(h.sum()) == sum(gold["hist"]) == n * (n - 1) // 2
    print("4M golden:", d)


def test_sdh_4m_lattice_exact(tbs):
    """L=160 lattice (N=4,096,000), w=1, 256 buckets: d_max = 275.4 so buckets >= 256 clamp
    into 255 (the clamp path); exact vs closed form."""
    p = g.lattice(160, 6)
    h = host(tbs.sdh(dev(p), 1.0, 256, lattice=True))
    assert h.tolist() == oracle.lattice_closed(160, 1, 0, 256)[0].tolist()


def test_sdh_4m_clustered_float_mass_strips(tbs):
    n = 1 << 22
    p = g.clustered(n, 3)
    d = dev(p)
    h = host(tbs.sdh(d, w_of(256), 256))
    assert int(h.sum()) == n * (n - 1) // 2
    rows = (n // 3, n // 3 + 48)
    hs = host(tbs.sdh(d, w_of(256), 256, rows=rows))
    ho, amb = oracle.sdh(p, w_of(256), 256, rows=rows)
    check_sdh_float(hs, ho, amb)


# ---------------------------------------------------------------- configs[4]: Type-III N=64K
def test_pairmatrix_64k_sampled_rows(tbs):
    """configs[4] per run: 1024 sampled rows of the full 64K x 64K matrix
    computed in the bench's launch configuration, each against the oracle row by row."""
    import torch
    n = 1 << 16
    p = g.uniform(n, 5)
    out = tbs.pairmatrix(dev(p), 1.0)                      # 17.2 GB fp32 on the device
    rng = np.random.default_rng(0)
    rows = sorted(set([0, 1, n - 1] + rng.choice(n, 1021, replace=False).tolist()))
    idx = torch.tensor(rows, device=out.device)
    got = host(out.index_select(0, idx))
    del out
    torch.cuda.empty_cache()
    worst = 0.0
    for k, r in enumerate(rows):
        ref = oracle.pairmatrix(p, 1.0, rows=(r, r + 1))[0]
        worst = max(worst, check_matrix(got[k], ref))
    assert len(rows) >= 1024 and worst <= 1e-5


@pytest.mark.slow
def test_pairmatrix_64k_full_matrix(tbs):
    """configs[4] full check (SURVEY §8(d) C5 "full check once"): all 4.29e9 entries of the
    64K x 64K Gaussian matrix, computed in one call, against the oracle in 1024-row blocks
    (max relative error <= 1e-5; the worst block's value is written to gpurun_out/ if present)."""
    import json
    import os
    import torch
    n, blk = 1 << 16, 1024
    p = g.uniform(n, 5)
    out = tbs.pairmatrix(dev(p), 1.0)
    torch.cuda.synchronize()
    worst, where = 0.0, -1
    for b in range(0, n, blk):
        got = host(out[b:b + blk])
        ref = oracle.pairmatrix(p, 1.0, rows=(b, b + blk))
        e = check_matrix(got, ref)
        if e > worst:
            worst, where = e, b
    del out
    torch.cuda.empty_cache()
    if os.path.isdir("gpurun_out"):
        with open(os.path.join("gpurun_out", "pairmatrix_64k_full.json"), "w") as f:
            json.dump(dict(n=n, entries=n * n, blocks=n // blk, max_rel_err=worst, worst_block_row=where), f)
    assert worst <= 1e-5


# ---------------------------------------------------------------- NEXT-3 at full size: N=64K, d=64 (17.2 GB fp32)
def test_pairmatrix_hd_64k_sampled_rows(tbs):
    import torch
    n, d = 1 << 16, 64
    x = torch.from_numpy(g.uniform(n, 7, d)).cuda().to(torch.bfloat16)
    xb = x.view(torch.int16).cpu().numpy().view(np.uint16)
    out = tbs.pairmatrix_hd(x, 1.0 / d)
    rng = np.random.default_rng(1)
    rows = sorted(set([0, n - 1] + rng.integers(0, n, 62).tolist()))
    got = host(out.index_select(0, torch.tensor(rows, device=out.device))).astype(np.float64)
    del out
    torch.cuda.empty_cache()
    xf = (xb.astype(np.uint32) << 16).view(np.float32).astype(np.float64)
    nrm = (xf * xf).sum(1)
    g32 = np.float64(np.float32(1.0 / d))
    for k, r in enumerate(rows):
        ref = oracle.pairmatrix_hd(xb, 1.0 / d, rows=(r, r + 1))[0]
        B = 2.0 ** -23 * (d / 16 + 8) * (nrm[r] + nrm + 2 * np.abs(xf) @ np.abs(xf[r]))
        assert np.all(np.abs(got[k] - ref) <= ref * (g32 * B + 2e-6)), r


# ---------------------------------------------------------------- NEXT-3 at the d = 512 bench size (CTA pairs, banded raster)
def test_pairmatrix_hd_64k_d512_sampled_rows(tbs):
    import torch
    n, d = 1 << 16, 512
    x = torch.from_numpy(g.uniform(n, 7, d)).cuda().to(torch.bfloat16)
    xb = x.view(torch.int16).cpu().numpy().view(np.uint16)
    out = tbs.pairmatrix_hd(x, 1.0 / d)
    rng = np.random.default_rng(2)
    rows = sorted(set([0, 127, 128, 255, 256, n - 1] + rng.integers(0, n, 26).tolist()))
    got = host(out.index_select(0, torch.tensor(rows, device=out.device))).astype(np.float64)
    del out
    torch.cuda.empty_cache()
    xf = (xb.astype(np.uint32) << 16).view(np.float32).astype(np.float64)
    nrm = (xf * xf).sum(1)
    g32 = np.float64(np.float32(1.0 / d))
    for k, r in enumerate(rows):
        ref = oracle.pairmatrix_hd(xb, 1.0 / d, rows=(r, r + 1))[0]
        B = 2.0 ** -23 * (d / 16 + 8) * (nrm[r] + nrm + 2 * np.abs(xf) @ np.abs(xf[r]))
        assert np.all(np.abs(got[k] - ref) <= ref * (g32 * B + 2e-6)), r


# ---------------------------------------------------------------- NEXT-2: kernel-density sum at the bench size
def test_kde_1m_strips(tbs):
    """bench.py kde_uniform_1m (N = 1M, gamma = 1): anchor strips computed through the row-range
    API in the bench's launch configuration, each within 1e-5 relative of the oracle's strip."""
    n = 1 << 20
    p = g.uniform(n, 2)
    pt = dev(p)
    for rb, re in [(0, 300), (n // 3, n // 3 + 300), (n - 300, n)]:
        got = float(host(tbs.kde(pt, 1.0, rows=(rb, re)))[0])
        ref = oracle.kde(p, 1.0, rows=(rb, re))
        assert abs(got - ref) <= 1e-5 * ref, (rb, got, ref)


# ---------------------------------------------------------------- NEXT-2: kNN at the bench size
def test_knn_1m_sampled_strips(tbs):
    """bench.py knn_uniform_1m_k8: 1M uniform points, k = 8 (3 partner segments + merge)."""
    n, k = 1 << 20, 8
    p = g.uniform(n, 2)
    i, d = tbs.knn(dev(p), k)
    gi, gd = host(i).astype(np.int64), host(d)
    for rb, re in strips(n, 16):
        check_knn_float(p, k, gi[rb:re], gd[rb:re], rows=(rb, re))


def test_knn_lattice_2_5m_exact_strips(tbs):
    """137^3 = 2.57M lattice points: enough anchor tiles for the single-segment path
    (direct output, no merge); bit-exact against the oracle on strips."""
    L, k = 137, 16
    p = g.lattice(L, 5)
    n = len(p)
    i, d = tbs.knn(dev(p), k)
    gi, gd = host(i).astype(np.int64), host(d)
    for rb, re in strips(n, 8):
        oi, od = oracle.knn(p, k, rows=(rb, re))
        assert np.array_equal(gi[rb:re], oi) and np.array_equal(gd[rb:re], od.astype(np.float32))


# ---------------------------------------------------------------- maximum size (TBS_MAX_N = 2^30)
def test_max_n_strips(tbs):
    """n = TBS_MAX_N = 2^30 (12 GiB of points, 12 GiB of SoA scratch): every index the kernels
    form (tiles, chunks, SoA offsets, row bounds) stays in range. Points are coincident except
    the last, at distance 5 (w = 1, exact), so each strip's histogram is known in closed form:
    anchor i pairs with n-1-i partners, all at distance 0 except the pair with the last point."""
    import torch
    n = 1 << 30
    p = torch.zeros((n, 3), dtype=torch.float32, device="cuda")
    p[n - 1, 0] = 3.0
    p[n - 1, 1] = 4.0
    try:
        for rows in ((0, 1), (n - 5000, n - 2000), (n - 2, n)):
            b, e = rows
            h = tbs.sdh(p, 1.0, 8, rows=rows, lattice=True).cpu().numpy()
            pairs = (e - b) * (2 * n - b - e - 1) // 2
            far = e - b if e < n else e - b - 1          # pairs (i, n-1) with i in the strip, i < n-1
            assert int(h.sum()) == pairs and int(h[5]) == far and int(h[0]) == pairs - far, (rows, h)
            c = int(tbs.pcf(p, 4.5, rows=rows).item())
            assert c == pairs - far
    finally:
        del p
        torch.cuda.empty_cache()

"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

Acceptance (BASELINE.json north star):
  * lattice SDH / 2PCF: bit-exact;
  * float SDH: mass exact, cumulative counts within the edge-ambiguity counts A_e;
  * float 2PCF: within A_r;
  * Type-III: max relative error <= 1e-5.
Small cases span several tiles (anchor tile 2048, partner chunk 1024) and ragged
tails; full BASELINE.json sizes are checked in the bench's launch configuration on
sampled anchor strips (the oracle computes them row by row) and on exact lattice
closed forms.
"""
import math

import numpy as np
import pytest

import oracle
import tbs_inputs as g
from parity import check_knn_float, check_matrix, check_pcf_float, check_sdh_float

pytestmark = pytest.mark.gpu


def dev(p):
    import torch
    return torch.from_numpy(np.ascontiguousarray(p)).cuda()


def sdh_gpu(tbs, p, w, nb, **kw):
    import torch
    h = tbs.sdh(dev(p), w, nb, **kw)
    torch.cuda.synchronize()
    return h.cpu().numpy().astype(np.uint64)


def w_of(nb, dim=3):
    return float(np.float32(math.sqrt(dim) / nb))


# ------------------------------------------------------------------ SDH float
@pytest.mark.parametrize("n", [2, 3, 5, 100, 1023, 1024, 1025, 2047, 2048, 2049, 3071, 4096, 5000, 10007])
def test_sdh_uniform_ragged(tbs, n):
    p = g.uniform(n, 100 + n)
    nb = 64
    h = sdh_gpu(tbs, p, w_of(nb), nb)
    ho, amb = oracle.sdh(p, w_of(nb), nb)
    check_sdh_float(h, ho, amb)


@pytest.mark.parametrize("kind,nb,offset", [("uniform", 64, 0.0), ("uniform", 256, 0.0), ("uniform", 16384, 0.0),
                                             ("clustered", 256, 0.0), ("uniform", 256, 1000.0)])
def test_sdh_diag_band(tbs, kind, nb, offset):
    """SURVEY §8(c) diagnostic beside the 1e-6 acceptance rule: with the oracle's 5e-7 band
    counts, no edge may see more pairs moved than lie within 5e-7 of it (the fp32 error budget,
    DESIGN §10, is <= ~4e-7 relative, whatever the coordinates' offset). The numbers are also
    appended to gpurun_out/diag_band.jsonl when that directory exists."""
    import json
    import os
    n = 30000
    p = g.make(kind, n, 90 + nb) + np.float32(offset)
    w = w_of(nb)
    h = sdh_gpu(tbs, p, w, nb)
    ho, amb, amb2 = oracle.sdh_bands(p, w, nb)
    d = check_sdh_float(h, ho, amb, amb2)
    if os.path.isdir("gpurun_out"):
        with open(os.path.join("gpurun_out", "diag_band.jsonl"), "a") as f:
            f.write(json.dumps(dict(kind=kind, n=n, nb=nb, offset=offset, **d)) + "\n")
    assert d["edges_over_diag_band"] == 0, d


@pytest.mark.parametrize("n", [20001, 30000])
def test_sdh_main_config_ragged(tbs, n):
    """Sizes above the small-problem switch: the main tile configuration, ragged tail."""
    p = g.clustered(n, 31)
    h = sdh_gpu(tbs, p, w_of(256), 256)
    ho, amb = oracle.sdh(p, w_of(256), 256)
    check_sdh_float(h, ho, amb)
    c = int(tbs.pcf(dev(p), 0.02).item())
    co, ca = oracle.pcf(p, 0.02)
    check_pcf_float(c, co, ca)


def test_sdh_config1(tbs):
    """BASELINE.json configs[0]: N=4096 uniform, 64 buckets (golden from tools/make_goldens.py)."""
    import json, os
    gold = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "sdh_uniform_n4096_nb64_seed1.json")))
    p = g.uniform(4096, 1)
    h = sdh_gpu(tbs, p, gold["w"], 64)
    d = check_sdh_float(h, gold["hist"], gold["amb"])
    assert int(h.sum()) == 8386560
    print(d)


@pytest.mark.parametrize("kind,nb", [("clustered", 256), ("uniform", 1000), ("uniform", 16384), ("clustered", 3)])
def test_sdh_float_nb(tbs, kind, nb):
    p = g.make(kind, 6000, 7)
    h = sdh_gpu(tbs, p, w_of(nb), nb)
    ho, amb = oracle.sdh(p, w_of(nb), nb)
    check_sdh_float(h, ho, amb)


@pytest.mark.parametrize("mode", ["lane", "cta", "global"])
def test_sdh_hist_modes_float(tbs, mode):
    p = g.clustered(5000, 9)
    h = sdh_gpu(tbs, p, w_of(256), 256, hist_mode=mode)
    ho, amb = oracle.sdh(p, w_of(256), 256)
    check_sdh_float(h, ho, amb)


@pytest.mark.parametrize("dim", [1, 2, 4])
def test_sdh_dims(tbs, dim):
    p = g.uniform(3000, 50 + dim, dim)
    w = w_of(128, dim)
    h = sdh_gpu(tbs, p, w, 128)
    ho, amb = oracle.sdh(p, w, 128)
    check_sdh_float(h, ho, amb)


def test_sdh_offset_coordinates(tbs):
    """Coordinates far from the origin: the kernel subtracts before it squares, so the
    fp32 error stays relative to the distance (DESIGN.md §Error budget)."""
    p = g.uniform(4000, 3) + np.float32(1000.0)
    h = sdh_gpu(tbs, p, w_of(256), 256)
    ho, amb = oracle.sdh(p, w_of(256), 256)
    check_sdh_float(h, ho, amb)


def test_sdh_all_coincident(tbs):
    p = np.full((3000, 3), 0.3, np.float32)
    h = sdh_gpu(tbs, p, 0.01, 16)
    assert h[0] == 3000 * 2999 // 2 and h[1:].sum() == 0


@pytest.mark.parametrize("n", [0, 1])
def test_sdh_degenerate(tbs, n):
    import torch
    p = torch.zeros((n, 3), dtype=torch.float32, device="cuda")
    h = tbs.sdh(p, 0.1, 8)
    assert h.cpu().tolist() == [0] * 8


# ------------------------------------------------------------------ SDH lattice (bit-exact)
@pytest.mark.parametrize("n", [2, 17, 1500, 2048, 2049, 4096, 6001, 13824])
def test_sdh_lattice_exact(tbs, n):
    p = g.lattice(24, 5)[:n]
    # (w, nb) chosen so the bounding box selects each exact variant (d_max = 23 sqrt(3)):
    # bias only, X = (k_max + 1) m < 362 (w = 1, 1/2, 3/4 @ 80, 5/4, 1/8 with X = 319), the
    # one-sided fp32 fix-up without clamp (1/16: X = 638; 3/32: X = 1275), the clamped
    # two-sided fp32 fix-up (3/4 @ 7 buckets)
    for (w, nb, m, j) in [(1.0, 64, 1, 0), (0.5, 80, 1, 1), (0.75, 7, 3, 2), (0.75, 80, 3, 2), (1.25, 40, 5, 2),
                          (0.125, 320, 1, 3), (0.0625, 640, 1, 4), (0.09375, 400, 3, 5)]:
        h = sdh_gpu(tbs, p, w, nb, lattice=True)
        assert h.tolist() == oracle.sdh_lattice(p, m, j, nb).tolist(), (n, w, nb)


def test_sdh_lattice_bias_only_boundary(tbs):
    """Bias-only exact variant at its limit: lattice {0..208}^3, w = 1, so the largest
    X = (k_max + 1) m = 361 (361^2 = 130321 < 2^17); every s = k^2 + 2k (one below the next
    edge) and every exact square k^2 up to 360^2 that the subset reaches must bucket exactly."""
    p = g.lattice(209, 21)[:15000]
    p = np.concatenate([p, np.array([[0, 0, 0], [208, 208, 208], [208, 0, 0], [0, 208, 208]], np.float32)])
    h = sdh_gpu(tbs, p, 1.0, 400, lattice=True)
    assert h.tolist() == oracle.sdh_lattice(p, 1, 0, 400).tolist()


@pytest.mark.parametrize("L,j", [(20, 9), (17, 10)])
def test_sdh_lattice_one_sided_large_x(tbs, L, j):
    """One-sided fp32 exact variant where 4^j s exceeds 2^24 (the r02 relaxation): w = 2^-j on
    {0..L-1}^3, x = sqrt(4^j s) reaches ~16900 (L 20, j 9) and ~28400 (L 17, j 10) — up to
    0.87 of its 2^15 admission limit; corners added so the extreme distances occur."""
    p = g.lattice(L, 22 + j)[:6000]
    c = float(L - 1)
    p = np.concatenate([p, np.array([[0, 0, 0], [c, c, c], [c, 0, 0], [0, c, c]], np.float32)])
    nb = int(math.ceil(math.sqrt(3.0) * c * 2 ** j)) + 40
    h = sdh_gpu(tbs, p, 2.0 ** -j, nb, lattice=True)
    assert h.tolist() == oracle.sdh_lattice(p, 1, j, nb).tolist()


def test_sqrt_approx_bound():
    """The bias-only lattice variant assumes |sqrt.approx(s) / sqrt(s) - 1| <= 2^-22 for every
    integer s < 2^24 (exhaustive on this GPU; tools/sqrt_bound.cu), with its 2^-19 bias
    leaving a 4x margin."""
    import json
    import os
    import subprocess
    import tempfile
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    exe = os.path.join(tempfile.mkdtemp(), "sqrt_bound")
    subprocess.run([os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc"), "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-o", exe,
                    os.path.join(root, "tools", "sqrt_bound.cu")], check=True)
    r = json.loads(subprocess.run([exe], check=True, capture_output=True, text=True).stdout)
    assert r["log2_int"] <= -22.0 and r["log2_1_4"] <= -22.0, r
    # the FMA-pipe square root (sqrt_sw2, TBS_SW_SQRT slots) is at least as tight as MUFU
    assert r["sw_log2_int"] <= -23.0 and r["sw_log2_1_4"] <= -23.0, r


@pytest.mark.parametrize("mode", [None, "lane", "cta", "global"])
def test_sdh_lattice_modes_config1(tbs, mode):
    """L=16 lattice (N=4096, the configs[0] size), w=2^-1, 64 buckets: closed form."""
    p = g.lattice(16, 1)
    h = sdh_gpu(tbs, p, 0.5, 64, lattice=True, hist_mode=mode)
    assert h.tolist() == oracle.lattice_closed(16, 1, 1, 64)[0].tolist()
    assert h.tolist() == oracle.sdh_lattice(p, 1, 1, 64).tolist()


def test_sdh_lattice_float_mode_agrees(tbs):
    """Float mode on a lattice with a dyadic width: exact except for pairs whose
    distance is (numerically) on an edge — still inside the A_e rule."""
    p = g.lattice(20, 2)
    h = sdh_gpu(tbs, p, 0.5, 64)
    ho, amb = oracle.sdh(p, 0.5, 64)
    check_sdh_float(h, ho, amb)


# ------------------------------------------------------------------ row ranges / multi-GPU partition
@pytest.mark.parametrize("rows", [(0, 1), (1, 2), (5, 3000), (2047, 2049), (2048, 4096), (4000, 6000), (5999, 6000)])
def test_sdh_row_ranges(tbs, rows):
    p = g.lattice(20, 11)[:6000]
    h = sdh_gpu(tbs, p, 1.0, 40, lattice=True, rows=rows)
    assert h.tolist() == oracle.sdh_lattice(p, 1, 0, 40, rows=rows).tolist()


@pytest.mark.parametrize("world", [2, 3, 4, 8])
def test_partition_sums_bit_exact(tbs, world):
    """Sum over the W rank strips (what all_reduce computes) == the W=1 result, bit-exact."""
    import torch
    p = dev(g.clustered(9000, 4))
    full = tbs.sdh(p, w_of(256), 256).cpu()
    acc = torch.zeros(256, dtype=torch.int64)
    cacc = 0
    for r in range(world):
        rows = tbs.rank_rows(9000, world, r)
        acc += tbs.sdh(p, w_of(256), 256, rows=rows).cpu()
        cacc += int(tbs.pcf(p, 0.03, rows=rows).item())
    assert torch.equal(acc, full)
    assert cacc == int(tbs.pcf(p, 0.03).item())


# ------------------------------------------------------------------ 2PCF
@pytest.mark.parametrize("n", [2, 999, 2048, 4097, 13824])
def test_pcf_lattice_exact(tbs, n):
    p = g.lattice(24, 3)[:n]
    for r in (1.0, 3.0, 10.0, 40.0):
        c = int(tbs.pcf(dev(p), r).item())
        assert c == oracle.pcf(p, r)[0], (n, r)


def test_pcf_clustered_float(tbs):
    p = g.clustered(20000, 3)
    for r in (0.0, 0.01, 0.03, 0.2):
        c = int(tbs.pcf(dev(p), r).item())
        co, amb = oracle.pcf(p, r)
        check_pcf_float(c, co, amb)


def test_pcf_equals_cumulative_sdh_lattice(tbs):
    p = dev(g.lattice(18, 6))
    h = tbs.sdh(p, 1.0, 30, lattice=True).cpu().numpy()
    for e in (1, 5, 17):
        assert int(tbs.pcf(p, float(e)).item()) == int(h[:e].sum())


@pytest.mark.parametrize("dim", [1, 2, 4])
def test_pcf_dims(tbs, dim):
    p = g.uniform(3000, 60 + dim, dim)
    c = int(tbs.pcf(dev(p), 0.1).item())
    co, amb = oracle.pcf(p, 0.1)
    check_pcf_float(c, co, amb)


# ------------------------------------------------------------------ Type-III
@pytest.mark.parametrize("n", [1, 5, 1000, 1027, 2048, 3001])
@pytest.mark.parametrize("kernel", ["gaussian", "dist2", "dist"])
def test_pairmatrix(tbs, n, kernel):
    p = g.uniform(n, 200 + n)
    out = tbs.pairmatrix(dev(p), 1.0, kernel=kernel).cpu().numpy()
    ref = oracle.pairmatrix(p, 1.0, ktype=tbs.KERNELS[kernel])
    check_matrix(out, ref)
    if kernel == "gaussian":
        assert np.all(np.diag(out) == 1.0)


def test_pairmatrix_rows_gamma(tbs):
    p = g.uniform(2500, 8)
    out = tbs.pairmatrix(dev(p), 3.5, rows=(700, 1333)).cpu().numpy()
    check_matrix(out, oracle.pairmatrix(p, 3.5, rows=(700, 1333)))


# ------------------------------------------------------------------ host-pointer ABI
def test_host_pointer_entry_points(tbs):
    p = g.clustered(7000, 5)
    h = tbs.sdh_host(p, w_of(256), 256)
    assert h.tolist() == sdh_gpu(tbs, p, w_of(256), 256).tolist()
    assert tbs.pcf_host(p, 0.02) == int(tbs.pcf(dev(p), 0.02).item())
    q = p[:700]
    np.testing.assert_array_equal(tbs.pairmatrix_host(q, 2.0), tbs.pairmatrix(dev(q), 2.0).cpu().numpy())


def test_launch_counter_moves(tbs):
    before = tbs.launch_count()
    sdh_gpu(tbs, g.uniform(3000, 1), 0.05, 32)
    assert tbs.launch_count() >= before + 1           # small problem: one fused launch
    before = tbs.launch_count()
    sdh_gpu(tbs, g.uniform(40000, 1), 0.05, 32)
    assert tbs.launch_count() >= before + 2           # loader + pair kernel


# ------------------------------------------------------------------ NEXT-2: kernel-density pair sum, NEXT-1: RDF
def kde_gpu(tbs, p, gamma, **kw):
    import torch
    v = tbs.kde(dev(p), gamma, **kw)
    torch.cuda.synchronize()
    return float(v.item())


@pytest.mark.parametrize("n", [2, 3, 1000, 2049, 5000, 30011])
@pytest.mark.parametrize("gamma", [1.0, 100.0])
def test_kde(tbs, n, gamma):
    """Tolerance 1e-5 relative: ex2.approx (2 ulp) of an argument with ~3u relative error,
    fp32 group partials of <= 32 terms, Kahan fp32 per thread, fp64 across threads."""
    p = g.clustered(n, 40 + n)
    ref = oracle.kde(p, gamma)
    got = kde_gpu(tbs, p, gamma)
    assert abs(got - ref) <= 1e-5 * abs(ref) + 1e-30, (got, ref)


def test_kde_rows_partition_and_dims(tbs):
    p = g.uniform(6000, 77)
    ref = oracle.kde(p, 3.0)
    acc = sum(kde_gpu(tbs, p, 3.0, rows=tbs.rank_rows(6000, 4, r)) for r in range(4))
    assert abs(acc - ref) <= 1e-5 * ref
    for dim in (1, 2, 4):
        q = g.uniform(2500, 80 + dim, dim)
        r = oracle.kde(q, 2.0)
        assert abs(kde_gpu(tbs, q, 2.0) - r) <= 1e-5 * r
    assert kde_gpu(tbs, np.zeros((0, 3), np.float32), 1.0) == 0.0
    assert kde_gpu(tbs, np.zeros((40, 3), np.float32), 5.0) == 780.0      # C(40,2) coincident pairs


def test_kde_host_entry_point(tbs):
    import ctypes
    p = g.clustered(3000, 5)
    out = np.zeros(1, np.float64)
    assert tbs.lib().tbs_kde(p.ctypes.data, 3000, ctypes.c_float(1.5), out.ctypes.data) == 0
    assert abs(out[0] - oracle.kde(p, 1.5)) <= 1e-5 * out[0]


def _ideal(w, nb, dim, pairs, volume):
    """Ideal-gas shell counts with the ball volume from scipy's Gamma function (test side)."""
    from scipy.special import gamma as G
    c = math.pi ** (dim / 2) / G(dim / 2 + 1)
    k = np.arange(nb, dtype=np.float64)
    return pairs * c * (((k + 1) * w) ** dim - (k * w) ** dim) / volume


@pytest.mark.parametrize("dim", [1, 2, 3, 4])
def test_rdf_lattice_exact_dims(tbs, dim):
    """RDF (NEXT-1, reading R6) on integer-valued points: the histograms are exact on both
    sides, so g agrees to the rounding of two independently written normalisations."""
    import torch
    n, nb, w = 6000, 48, 0.5
    p = np.floor(g.uniform(n, 60 + dim, dim) * 40.0).astype(np.float32)
    gr = tbs.rdf(dev(p), w, nb, 40.0 ** dim, lattice=True)
    torch.cuda.synchronize()
    go, ho, _ = oracle.rdf_points(p, w, nb, 40.0 ** dim, lattice=(1, 1))
    assert ho[:nb].sum() > 0
    np.testing.assert_allclose(gr.cpu().numpy(), go, rtol=1e-12, atol=0)


@pytest.mark.parametrize("dim,rows", [(1, None), (2, None), (3, None), (4, None), (3, (1000, 7777))])
def test_rdf_float_dims(tbs, dim, rows):
    """Float inputs: the GPU's g may differ from the oracle's only through pairs within the
    1e-6 band of an edge, so |g_gpu[k] - g_or[k]| <= (A_k + A_{k+1}) / ideal_k (A from the
    ORACLE's band counts, ideal_k from the test's own ball volume) + rounding; the whole
    vector is also within that bound of the oracle pipeline on a row strip."""
    import torch
    n, nb = 9000, 64
    w = float(np.float32(math.sqrt(dim) / nb))
    p = g.uniform(n, 70 + dim, dim)
    gr = tbs.rdf(dev(p), w, nb, 1.0, rows=rows).cpu().numpy()
    torch.cuda.synchronize()
    go, ho, amb = oracle.rdf_points(p, w, nb, 1.0, rows=rows)
    ideal = _ideal(np.float64(np.float32(w)), nb, dim, oracle.pairs_of_rows(n, rows), 1.0)
    a = amb.astype(np.float64)
    bound = (a[:nb] + a[1:nb + 1]) / ideal + 1e-12 * np.abs(go)
    assert np.all(np.abs(gr - go) <= bound), np.max(np.abs(gr - go) - bound)
    np.testing.assert_allclose(go, ho[:nb] / ideal, rtol=1e-9)   # the test's ideal = the oracle's


def test_rdf_host_entry_and_degenerate(tbs):
    """tbs_rdf with host buffers equals the device path; n < 2 gives g = 0; a pair beyond
    nb w (clamp bucket) never enters g."""
    import ctypes
    p = g.uniform(3000, 77)
    nb, w = 32, 0.05
    out = np.zeros(nb, np.float64)
    assert tbs.lib().tbs_rdf(p.ctypes.data, 3000, 3, ctypes.c_float(w), nb, ctypes.c_double(1.0),
                             out.ctypes.data) == 0, tbs.last_error()
    np.testing.assert_array_equal(out, tbs.rdf(dev(p), w, nb, 1.0).cpu().numpy())
    assert not tbs.rdf(dev(p[:1]), w, nb, 1.0).cpu().numpy().any()
    q = np.array([[0, 0, 0], [5, 0, 0]], np.float32)
    assert not tbs.rdf(dev(q), w, nb, 1.0).cpu().numpy().any()


# ------------------------------------------------------------------ output-stage replication R and bucket-range passes
@pytest.mark.parametrize("nb,m,j", [(700, 1, 3), (2048, 1, 5), (4096, 1, 6), (8192, 1, 7), (60000, 1, 10),
                                    (100000, 1, 11)])
def test_sdh_lattice_replication_and_passes(tbs, nb, m, j):
    """nb spans R = 16, 8, 4 (one CTA copy each) and 2-3 bucket-range passes: exact."""
    p = g.lattice(24, 9)[:9000]
    w = m * 2.0 ** -j
    h = sdh_gpu(tbs, p, w, nb, lattice=True)
    assert h.tolist() == oracle.sdh_lattice(p, m, j, nb).tolist()


@pytest.mark.parametrize("nb", [64, 1000, 70000])
def test_sdh_forced_passes_float(tbs, nb):
    p = g.clustered(7000, 12)
    w = float(np.float32(math.sqrt(3) / min(nb, 4000)))
    h = sdh_gpu(tbs, p, w, nb, hist_mode="passes" if nb < 50000 else None)
    ho, amb = oracle.sdh(p, w, nb)
    check_sdh_float(h, ho, amb)


# ------------------------------------------------------------------ CUDA-graph capture of the stream-ordered API
def test_cuda_graph_capture_replay(tbs):
    """tbs_*_ex enqueue only stream-ordered work (cudaMallocAsync scratch, memset, kernels,
    cudaFreeAsync), so a call can be captured once and replayed; replays recompute from the
    (possibly updated) input buffer."""
    import torch
    p = dev(g.clustered(9000, 8))
    w = float(np.float32(math.sqrt(3) / 256))
    h = torch.empty(256, dtype=torch.int64, device="cuda")
    c = torch.empty(1, dtype=torch.int64, device="cuda")
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        tbs.sdh(p, w, 256, out=h)              # warm-up outside capture (occupancy cache, attributes)
        tbs.pcf(p, 0.03, out=c)
    torch.cuda.synchronize()
    graph = torch.cuda.CUDAGraph()
    with torch.cuda.graph(graph, stream=s):
        tbs.sdh(p, w, 256, out=h)
        tbs.pcf(p, 0.03, out=c)
    for seed in (8, 9):
        p.copy_(torch.from_numpy(g.clustered(9000, seed)))
        graph.replay()
        torch.cuda.synchronize()
        ho, amb = oracle.sdh(p.cpu().numpy(), w, 256)
        check_sdh_float(h.cpu().numpy(), ho, amb)
        co, ca = oracle.pcf(p.cpu().numpy(), 0.03)
        check_pcf_float(int(c.item()), co, ca)


# ------------------------------------------------------------------ NEXT-3: high-dimensional Type-III on tcgen05
def _bf16_bits(a):
    u = np.ascontiguousarray(a, dtype=np.float32).view(np.uint32).astype(np.uint64)
    return ((u + ((u >> 16) & 1) + 0x7FFF) >> 16).astype(np.uint16)


def _hd_bound(xbits):
    """Per-entry bound on |s_gpu - s|: exact bf16 products, fp32 accumulation in
    the tensor core (K-chunks of 16 summed in sequence) and in the norms:
    2^-23 (d/16 + 8) (|x_i|^2 + |x_j|^2 + 2 sum_k |x_ik x_jk|)."""
    x = (xbits.astype(np.uint32) << 16).view(np.float32).astype(np.float64)
    nrm = (x * x).sum(1)
    ax = np.abs(x)
    return 2.0 ** -23 * (x.shape[1] / 16 + 8) * (nrm[:, None] + nrm[None, :] + 2 * ax @ ax.T)


@pytest.mark.parametrize("n,d", [(1, 8), (5, 3), (128, 64), (300, 40), (1000, 128), (1029, 100), (2048, 64),
                                 (777, 192), (520, 256), (300, 512), (257, 1000)])
@pytest.mark.parametrize("kernel", ["gaussian", "dist2", "dist"])
def test_pairmatrix_hd(tbs, n, d, kernel):
    import torch
    rng = np.random.default_rng(n * 131 + d)
    xb = _bf16_bits(rng.random((n, d), dtype=np.float32))
    xt = torch.from_numpy(xb.view(np.int16)).cuda().view(torch.bfloat16)
    gamma = 1.0 / d
    got = tbs.pairmatrix_hd(xt, gamma, kernel=kernel).cpu().numpy().astype(np.float64)
    ref = oracle.pairmatrix_hd(xb, gamma, ktype=tbs.KERNELS[kernel])
    B = _hd_bound(xb)
    if kernel == "gaussian":
        g32 = np.float64(np.float32(gamma))
        tol = ref * (g32 * B + 2e-6) + 1e-30
    elif kernel == "dist2":
        tol = B + 1e-30
    else:
        tol = np.sqrt(B) + 1e-6 * ref
    err = np.abs(got - ref)
    assert np.all(err <= tol), (float(err.max()), float((err / tol).max()))


def test_pairmatrix_hd_rows_and_host(tbs):
    import torch
    rng = np.random.default_rng(5)
    xb = _bf16_bits(rng.standard_normal((700, 96)).astype(np.float32))
    xt = torch.from_numpy(xb.view(np.int16)).cuda().view(torch.bfloat16)
    full = tbs.pairmatrix_hd(xt, 0.01).cpu().numpy()
    part = tbs.pairmatrix_hd(xt, 0.01, rows=(130, 419)).cpu().numpy()
    assert np.array_equal(part, full[130:419])
    host = np.empty((700, 700), np.float32)
    assert tbs.lib().tbs_pairmatrix_hd(xb.ctypes.data, 700, 96, tbs._Kernel(0, 0.01), host.ctypes.data) == 0
    assert np.array_equal(host, full)
    ref = oracle.pairmatrix_hd(xb, 0.01)
    assert np.all(np.abs(full - ref) <= ref * (0.01 * _hd_bound(xb) + 2e-6))


@pytest.mark.parametrize("rows", [(0, 256), (128, 384), (300, 700), (511, 513), (255, 257), (699, 700), (5, 5)])
@pytest.mark.parametrize("n", [700, 702])
def test_pairmatrix_hd_pair_tile_rows(tbs, rows, n):
    """Row ranges that cut the CTA-pair tiles (256 rows: CTA 0 rows 0-127, CTA 1 rows 128-255)
    anywhere, with n % 4 == 0 (TMA-store path) and != 0 (masked path): equal to the full matrix."""
    import torch
    rng = np.random.default_rng(n + rows[0])
    xb = _bf16_bits(rng.standard_normal((n, 136)).astype(np.float32))
    xt = torch.from_numpy(xb.view(np.int16)).cuda().view(torch.bfloat16)
    full = tbs.pairmatrix_hd(xt, 0.01).cpu().numpy()
    part = tbs.pairmatrix_hd(xt, 0.01, rows=rows).cpu().numpy()
    assert part.shape == (rows[1] - rows[0], n)
    assert np.array_equal(part, full[rows[0]:rows[1]])


@pytest.mark.parametrize("n,d", [(9000, 64), (6000, 520), (6000, 448), (3000, 200)])
def test_pairmatrix_hd_many_tiles_sampled(tbs, n, d):
    """More pair tiles than clusters (persistent round-robin / banded raster at d > 128):
    sampled row strips against the oracle with the derived bound."""
    import torch
    rng = np.random.default_rng(n + d)
    xb = _bf16_bits(rng.random((n, d), dtype=np.float32))
    xt = torch.from_numpy(xb.view(np.int16)).cuda().view(torch.bfloat16)
    gamma = 1.0 / d
    full = tbs.pairmatrix_hd(xt, gamma).cpu().numpy().astype(np.float64)
    g32 = np.float64(np.float32(gamma))
    for r0 in (0, 2000, n - 300):
        rr = (r0, r0 + 300)
        ref = oracle.pairmatrix_hd(xb, gamma, rows=rr)
        x = (xb.astype(np.uint32) << 16).view(np.float32).astype(np.float64)
        nrm = (x * x).sum(1)
        ax = np.abs(x)
        B = 2.0 ** -23 * (d / 16 + 8) * (nrm[rr[0]:rr[1], None] + nrm[None, :] + 2 * ax[rr[0]:rr[1]] @ ax.T)
        assert np.all(np.abs(full[rr[0]:rr[1]] - ref) <= ref * (g32 * B + 2e-6) + 1e-30)


# ------------------------------------------------------------------ NEXT-2: all-point kNN (reading R5)
def knn_gpu(tbs, p, k, rows=None):
    import torch
    i, d = tbs.knn(dev(p), k, rows=rows)
    torch.cuda.synchronize()
    return i.cpu().numpy().astype(np.int64), d.cpu().numpy()


@pytest.mark.parametrize("L,cut,k", [(12, None, 1), (12, None, 6), (12, None, 8), (12, None, 13), (12, None, 26),
                                     (16, 3001, 4), (16, 4095, 16), (20, 7777, 32), (10, 1000, 18)])
def test_knn_lattice_exact(tbs, L, cut, k):
    """Integer lattice: squared distances exact in fp32, so idx and dist are bit-exact,
    including the smaller-index-first rule on the many lattice ties."""
    p = g.lattice(L, 30 + L)[:cut]
    oi, od = oracle.knn(p, k)
    gi, gd = knn_gpu(tbs, p, k)
    assert np.array_equal(gi, oi)
    assert np.array_equal(gd, od.astype(np.float32))


@pytest.mark.parametrize("kind,n,k", [("uniform", 3000, 1), ("uniform", 5000, 5), ("clustered", 9000, 8),
                                      ("clustered", 4097, 16), ("uniform", 12345, 32), ("uniform", 20000, 3)])
def test_knn_float(tbs, kind, n, k):
    p = g.make(kind, n, 50 + n)
    gi, gd = knn_gpu(tbs, p, k)
    check_knn_float(p, k, gi, gd)


def test_knn_rows_dims_and_edges(tbs):
    p = g.lattice(14, 3)[:2700]
    oi, od = oracle.knn(p, 7)
    parts = [knn_gpu(tbs, p, 7, rows=(2700 * r // 4, 2700 * (r + 1) // 4)) for r in range(4)]
    assert np.array_equal(np.concatenate([x[0] for x in parts]), oi)
    assert np.array_equal(np.concatenate([x[1] for x in parts]), od.astype(np.float32))
    gi, gd = knn_gpu(tbs, p, 7, rows=(1000, 1013))
    assert np.array_equal(gi, oi[1000:1013])
    for dim in (1, 2, 4):
        q = g.uniform(3000, 90 + dim, dim)
        gi, gd = knn_gpu(tbs, q, 6)
        check_knn_float(q, 6, gi, gd)
    # coincident points: every distance 0, ties by index
    z = np.zeros((300, 3), np.float32)
    gi, gd = knn_gpu(tbs, z, 5)
    assert np.array_equal(gi, oracle.knn(z, 5)[0]) and np.all(gd == 0)
    # k > n - 1, n = 1, n = 0
    q = g.uniform(5, 4)
    gi, gd = knn_gpu(tbs, q, 9)
    oi, od = oracle.knn(q, 9)
    assert np.array_equal(gi, oi) and np.all(np.isinf(gd[:, 4:]))
    gi, gd = knn_gpu(tbs, q[:1], 3)
    assert gi.tolist() == [[-1, -1, -1]] and np.all(np.isinf(gd))
    assert knn_gpu(tbs, q[:0], 3)[0].shape == (0, 3)


def test_knn_host_entry_point_and_einval(tbs):
    p = g.lattice(9, 5)
    gi, gd = tbs.knn_host(p, 10)
    oi, od = oracle.knn(p, 10)
    assert np.array_equal(gi.astype(np.int64), oi) and np.array_equal(gd, od.astype(np.float32))
    with pytest.raises(tbs.TbsError):
        tbs.knn(dev(p), 33)
    with pytest.raises(tbs.TbsError):
        tbs.knn(dev(p), 0)


# ------------------------------------------------------------------ TBS_VALIDATE (SURVEY §8(b) debug flag)
def test_validate_flag(tbs):
    """The debug flag checks what the loader recorded before any pair kernel runs: non-finite
    coordinates (SDH, 2PCF, RDF) and, under TBS_EXACT_LATTICE, non-integer coordinates or a
    bounding box whose squared pair distances could reach 2^24. Valid inputs give the same
    result as without the flag."""
    import torch
    lat = g.lattice(12, 3)
    ok = tbs.sdh(dev(lat), 0.5, 40, lattice=True, validate=True)
    assert ok.cpu().tolist() == tbs.sdh(dev(lat), 0.5, 40, lattice=True).cpu().tolist()
    bad = lat.copy()
    bad[7, 1] = 3.5                                   # not integer-valued
    with pytest.raises(tbs.TbsError, match="integer-valued"):
        tbs.sdh(dev(bad), 0.5, 40, lattice=True, validate=True)
    wide = lat.copy()
    wide[0] = (0, 0, 0)
    wide[1] = (5000, 0, 0)                            # 5000^2 >= 2^24
    with pytest.raises(tbs.TbsError, match="2\\^24"):
        tbs.sdh(dev(wide), 1.0, 40, lattice=True, validate=True)
    p = g.uniform(3000, 5)
    p[100, 2] = np.nan
    for call in (lambda x: tbs.sdh(x, 0.01, 64, validate=True), lambda x: tbs.pcf(x, 0.1, validate=True),
                 lambda x: tbs.rdf(x, 0.01, 64, 1.0, validate=True)):
        with pytest.raises(tbs.TbsError, match="non-finite"):
            call(dev(p))
    p[100, 2] = np.inf
    with pytest.raises(tbs.TbsError, match="non-finite"):
        tbs.sdh(dev(p), 0.01, 64, validate=True)
    q = g.uniform(3000, 5)                            # float data passes (non-integer is fine)
    assert int(tbs.sdh(dev(q), 0.01, 64, validate=True).sum().item()) == 3000 * 2999 // 2
    torch.cuda.synchronize()


# ------------------------------------------------------------------ small-problem host-buffer path
def test_host_small_path(tbs):
    """Host-buffer calls with n <= 16K move points and result with copy kernels over mapped
    pinned memory (the caller's pinned buffers, or the staging area for pageable ones) around
    the fused small-problem kernel: repeated and interleaved calls, pageable and pinned buffers,
    many radii, and the sizes around the switch all give the oracle's result."""
    import torch
    nb = 64
    pts = {n: g.uniform(n, 300 + n) for n in (2, 3000, 4096, 16384, 65536)}
    want = {n: oracle.sdh(p, w_of(nb), nb) for n, p in pts.items() if n <= 16384}
    for rep in range(3):
        for n in (2, 3000, 4096, 16384):
            h = tbs.sdh_host(pts[n], w_of(nb), nb)
            check_sdh_float(h, *want[n])
    pin = torch.from_numpy(pts[4096]).pin_memory()
    for _ in range(3):
        check_sdh_float(tbs.sdh_host(pin.numpy(), w_of(nb), nb), *want[4096])
    for k in list(range(10)) + [0, 1]:
        r = 0.02 + 0.01 * k
        c = tbs.pcf_host(pts[3000], r)
        co, ca = oracle.pcf(pts[3000], r)
        check_pcf_float(c, co, ca)
    tbs.release()
    check_sdh_float(tbs.sdh_host(pts[3000], w_of(nb), nb), *want[3000])
    h = tbs.sdh_host(pts[65536], w_of(nb), nb)                     # above the small-problem switch
    assert int(h.sum()) == 65536 * 65535 // 2
    assert h.tolist() == tbs.sdh(dev(pts[65536]), w_of(nb), nb).cpu().tolist()


def test_host_small_path_mixed_sequence(tbs):
    """The small host-buffer path keeps a per-thread device scratch zero between calls (the
    fused kernel's last CTA re-zeroes what it used): interleave operations, point counts and
    output sizes so every call's output region is one an earlier call dirtied differently."""
    import ctypes
    seq = [("sdh", 4096, 64), ("kde", 3000, 0), ("sdh", 2, 300), ("pcf", 16384, 0), ("sdh", 3000, 1000),
           ("kde", 4096, 0), ("sdh", 16384, 8192), ("pcf", 5, 0), ("sdh", 4096, 64), ("kde", 2, 0)]
    for rep in range(2):
        for op, n, nb in seq:
            p = g.uniform(n, 500 + n)
            if op == "sdh":
                ho, amb = oracle.sdh(p, w_of(nb), nb)
                check_sdh_float(tbs.sdh_host(p, w_of(nb), nb), ho, amb)
            elif op == "pcf":
                co, ca = oracle.pcf(p, 0.05)
                check_pcf_float(tbs.pcf_host(p, 0.05), co, ca)
            else:
                out = np.zeros(1, np.float64)
                assert tbs.lib().tbs_kde(p.ctypes.data, n, ctypes.c_float(1.5), out.ctypes.data) == 0
                ko = oracle.kde(p, 1.5)
                assert abs(out[0] - ko) <= 1e-5 * max(ko, 1e-30)

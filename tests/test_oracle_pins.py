"""Pins for the CPU oracle (oracle/), independent of the oracle's own code.

PAPER.md prints no worked example with values, so every pin is a
mathematical one: hand cases, brute force with independent numpy/scipy/torch
routines, mass, exact lattice closed forms, the uniform-cube distance law, and
cross-API identities. Each test names the passage it follows.
"""
import json
import math
import os

import numpy as np
import pytest
from scipy.spatial.distance import pdist

import oracle
import tbs_inputs as g
import cube_cdf  # tests/cube_cdf.py (sibling helper)

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def brute_sdh(p, w, nb):
    """Independent SDH: scipy pdist (i<j pairs, L290-296) -> floor(d/w) clamped (Q1, Q2)."""
    d = pdist(p.astype(np.float64))
    q = d / np.float64(np.float32(w))
    b = np.minimum(np.floor(q), nb - 1).astype(np.int64)
    return np.bincount(b, minlength=nb).astype(np.uint64), d


def brute_lattice(p, m, j, nb):
    """Independent exact lattice bucketing with python integers (math.isqrt)."""
    pi = p.astype(np.int64)
    n = len(pi)
    h = np.zeros(nb, np.uint64)
    for i in range(n):
        s = ((pi[i + 1:] - pi[i]) ** 2).sum(axis=1)
        for sv in s.tolist():
            k = min(math.isqrt(sv << (2 * j)) // m, nb - 1)
            h[k] += 1
    return h


# ---------------------------------------------------------------- hand cases (golden)
def test_hand_cases_golden():
    """tests/golden/hand_cases.json: values derived by hand (see its 'why' fields)."""
    with open(os.path.join(GOLDEN, "hand_cases.json")) as f:
        cases = json.load(f)["cases"]
    for c in cases:
        p = np.array(c["points"], np.float32).reshape(-1, 3)
        if c["op"] == "sdh":
            h, _ = oracle.sdh(p, c["w"], c["nb"])
            assert h.tolist() == c["hist"], c["why"]
        elif c["op"] == "sdh_lattice":
            h = oracle.sdh_lattice(p, c["m"], c["j"], c["nb"])
            assert h.tolist() == c["hist"], c["why"]
        elif c["op"] == "pcf":
            cnt, _ = oracle.pcf(p, c["r"])
            assert cnt == c["count"], c["why"]
        elif c["op"] == "pairmatrix":
            out = oracle.pairmatrix(p, c["gamma"])
            np.testing.assert_allclose(out, np.array(c["out"]), rtol=1e-15, err_msg=c["why"])


@pytest.mark.parametrize("n", [0, 1])
def test_degenerate_sizes(n):
    p = g.uniform(n, 1)
    h, a = oracle.sdh(p, 0.1, 16)
    assert h.sum() == 0 and a.sum() == 0
    assert oracle.pcf(p, 0.5)[0] == 0


def test_all_coincident():
    p = np.full((300, 3), 0.25, np.float32)
    h, a = oracle.sdh(p, 0.01, 10)
    assert h[0] == 300 * 299 // 2 and h[1:].sum() == 0
    assert oracle.pcf(p, 1e-3)[0] == 300 * 299 // 2
    assert oracle.pcf(p, 0.0)[0] == 0          # d < 0 never (reading Q4: strict)


# ---------------------------------------------------------------- brute force
@pytest.mark.parametrize("kind,n,nb,seed", [("uniform", 1500, 64, 11), ("uniform", 777, 7, 12),
                                            ("clustered", 1800, 256, 13)])
def test_sdh_bruteforce(kind, n, nb, seed):
    p = g.make(kind, n, seed)
    w = float(np.float32(math.sqrt(3) / nb))
    h, amb = oracle.sdh(p, w, nb)
    hb, d = brute_sdh(p, w, nb)
    assert h.tolist() == hb.tolist()
    # ambiguity counts: |d - e w| <= 1e-6 e w for e = 1..nb-1
    wd = np.float64(np.float32(w))
    e = np.rint(d / wd)
    ok = (e >= 1) & (e <= nb - 1) & (np.abs(d - e * wd) <= 1e-6 * e * wd)
    ab = np.bincount(e[ok].astype(np.int64), minlength=nb + 1)
    assert amb.tolist() == ab.tolist()


def test_sdh_dims_1_2_4():
    for dim in (1, 2, 4):
        p = g.uniform(600, 21 + dim, dim)
        w = float(np.float32(math.sqrt(dim) / 32))
        h, _ = oracle.sdh(p, w, 32)
        hb, _ = brute_sdh(p, w, 32)
        assert h.tolist() == hb.tolist()


def test_mass_invariant_4096():
    """Sum of the histogram = n(n-1)/2 exactly (each unordered pair once, L290-296)."""
    p = g.uniform(4096, 1)
    h, _ = oracle.sdh(p, float(np.float32(math.sqrt(3) / 64)), 64)
    assert int(h.sum()) == 4096 * 4095 // 2 == 8386560


def test_pcf_bruteforce():
    p = g.clustered(2000, 3)
    for r in (0.0, 0.005, 0.03, 0.3, 2.0):
        c, a = oracle.pcf(p, r)
        d = pdist(p.astype(np.float64))
        rr = np.float64(np.float32(r))
        assert c == int((d < rr).sum())
        assert a == int((np.abs(d - rr) <= 1e-6 * rr).sum())


def test_pcf_equals_cumulative_sdh_on_lattice():
    """2PCF(r = e w) == sum_{b<e} SDH[b] (reading Q4), exact on lattices."""
    p = g.lattice(9, 5)
    h = oracle.sdh_lattice(p, 1, 0, 20)
    for e in range(1, 20):
        c, _ = oracle.pcf(p, float(e))
        assert c == int(h[:e].sum())


# ---------------------------------------------------------------- rows
def test_row_ranges_partition():
    p = g.uniform(1000, 7)
    w = float(np.float32(0.02))
    full, famb = oracle.sdh(p, w, 100)
    cuts = [0, 1, 170, 171, 500, 999, 1000]
    acc = np.zeros(100, np.uint64)
    accc = 0
    for a, b in zip(cuts[:-1], cuts[1:]):
        acc += oracle.sdh(p, w, 100, rows=(a, b))[0]
        accc += oracle.pcf(p, 0.1, rows=(a, b))[0]
    assert acc.tolist() == full.tolist()
    assert accc == oracle.pcf(p, 0.1)[0]


def test_row_range_is_anchor_subset():
    """rows [a,b): anchors i in [a,b) with all partners j>i."""
    p = g.uniform(400, 8)
    d = np.sqrt(((p[:, None, :].astype(np.float64) - p[None, :, :]) ** 2).sum(-1))
    i, j = np.triu_indices(400, 1)
    sel = (i >= 100) & (i < 250)
    w = np.float64(np.float32(0.05))
    b = np.minimum(np.floor(d[i[sel], j[sel]] / w), 39).astype(np.int64)
    h, _ = oracle.sdh(p, 0.05, 40, rows=(100, 250))
    assert h.tolist() == np.bincount(b, minlength=40).tolist()


# ---------------------------------------------------------------- lattice exact mode
@pytest.mark.parametrize("L,m,j,nb", [(6, 2, 0, 6), (7, 1, 1, 8), (7, 3, 1, 12), (5, 1, 0, 3), (6, 5, 3, 40)])
def test_lattice_oracle_vs_bruteforce(L, m, j, nb):
    p = g.lattice(L, 100 + L)
    h = oracle.sdh_lattice(p, m, j, nb)
    assert h.tolist() == brute_lattice(p, m, j, nb).tolist()
    assert int(h.sum()) == len(p) * (len(p) - 1) // 2


@pytest.mark.parametrize("L,m,j,nb", [(6, 2, 0, 6), (7, 1, 1, 8), (7, 3, 1, 12), (5, 1, 0, 3), (8, 1, 2, 50)])
def test_lattice_closed_form_vs_bruteforce(L, m, j, nb):
    """O(L^3) closed form == brute force on a permuted lattice (any point order)."""
    p = g.lattice(L, 7)
    hc, _ = oracle.lattice_closed(L, m, j, nb)
    assert hc.tolist() == brute_lattice(p, m, j, nb).tolist()


def test_lattice_closed_known_values():
    """Values recomputed independently in SURVEY Appendix A item 4."""
    assert oracle.lattice_closed(6, 2, 0, 6)[0].tolist() == [1940, 9472, 10068, 1712, 28, 0]
    assert oracle.lattice_closed(7, 1, 1, 8)[0].tolist() == [0, 0, 2394, 864, 5415, 1050, 6632, 42298]


def test_lattice_closed_pcf():
    """Closed-form lattice 2PCF (s < r^2) == brute force == oracle.pcf at r = 4 (r^2 = 16)."""
    p = g.lattice(8, 3)
    _, c = oracle.lattice_closed(8, 1, 0, 4, r2=16)
    d2 = pdist(p.astype(np.float64), "sqeuclidean")
    assert c == int((d2 < 16).sum()) == oracle.pcf(p, 4.0)[0]


def test_float_mode_equals_lattice_mode_on_dyadic_width():
    """On integer points with a dyadic width, floor(d/w) in double is exact."""
    p = g.lattice(9, 2)
    for (m, j) in [(1, 0), (3, 2), (1, 3)]:
        w = m * 2.0 ** -j
        hf, _ = oracle.sdh(p, w, 64)
        hl = oracle.sdh_lattice(p, m, j, 64)
        assert hf.tolist() == hl.tolist()


def test_lattice_rejects_non_integer():
    with pytest.raises(ValueError):
        oracle.sdh_lattice(np.array([[0.5, 0, 0], [1, 1, 1]], np.float32), 1, 0, 4)


# ---------------------------------------------------------------- uniform cube law
def test_cube_cdf_quadrature_pins():
    for r in (0.1, 0.5, 0.9, 1.0):
        assert abs(cube_cdf.F(r) - cube_cdf.F_closed_le1(r)) < 1e-9
    assert cube_cdf.F(math.sqrt(3)) == 1.0
    # mean distance = int_0^sqrt3 (1 - F) dr = Robbins' constant
    from scipy import integrate
    mean, _ = integrate.quad(lambda r: 1 - cube_cdf.F(r), 0, math.sqrt(3), points=[1, math.sqrt(2)], limit=200)
    assert abs(mean - cube_cdf.ROBBINS) < 1e-7


def test_sdh_uniform_matches_cube_law():
    """E[h_k] = C(n,2) (F(r_{k+1}) - F(r_k)); tolerance 6 sigma with the U-statistic
    variance C(n,2) p(1-p) + n(n-1)(n-2) zeta_1 (pairs sharing a point correlate)."""
    n, nb = 4096, 64
    w = float(np.float32(math.sqrt(3) / nb))
    p = g.uniform(n, 1)
    h, _ = oracle.sdh(p, w, nb)
    edges = [cube_cdf.F(k * np.float64(np.float32(w))) for k in range(nb)] + [1.0]
    pk = np.diff(np.array(edges))
    npairs = n * (n - 1) // 2
    # zeta_1 estimated from per-point row histograms (independent numpy computation)
    x = p.astype(np.float64)
    zeta = np.zeros(nb)
    cnt = np.zeros((n, nb))
    for i in range(0, n, 512):
        d = np.sqrt(((x[i:i + 512, None, :] - x[None, :, :]) ** 2).sum(-1))
        b = np.minimum(np.floor(d / np.float64(np.float32(w))), nb - 1).astype(np.int64)
        for r in range(b.shape[0]):
            row = np.bincount(b[r], minlength=nb).astype(np.float64)
            row[0] -= 1                      # self pair
            cnt[i + r] = row
    zeta = (cnt / (n - 1)).var(axis=0)
    var = npairs * pk * (1 - pk) + n * (n - 1) * (n - 2) * zeta
    dev = np.abs(h.astype(np.float64) - npairs * pk)
    assert np.all(dev <= 6 * np.sqrt(var) + 1), (dev / np.sqrt(var + 1e-12)).max()


# ---------------------------------------------------------------- Type-III
def test_pairmatrix_vs_cdist():
    import torch
    p = g.uniform(700, 4)
    gamma = 1.0
    out = oracle.pairmatrix(p, gamma)
    t = torch.from_numpy(p.astype(np.float64))
    d = torch.cdist(t, t, compute_mode="donot_use_mm_for_euclid_dist")
    ref = torch.exp(-gamma * d * d).numpy()
    np.testing.assert_allclose(out, ref, rtol=1e-13, atol=0)
    assert np.array_equal(out, out.T)
    assert np.all(np.diag(out) == 1.0)
    rows = oracle.pairmatrix(p, gamma, rows=(100, 140))
    assert np.array_equal(rows, out[100:140])
    d2 = oracle.pairmatrix(p, 0.0, ktype=1)
    np.testing.assert_allclose(d2, (d * d).numpy(), rtol=1e-13, atol=1e-300)
    d1 = oracle.pairmatrix(p, 0.0, ktype=2)
    np.testing.assert_allclose(d1, d.numpy(), rtol=1e-13, atol=1e-300)


def test_pairmatrix_lattice_values():
    p = g.lattice(4, 1)
    out = oracle.pairmatrix(p, 0.5)
    s = ((p[:, None, :].astype(np.int64) - p[None, :, :]) ** 2).sum(-1)
    np.testing.assert_allclose(out, np.exp(-0.5 * s.astype(np.float64)), rtol=1e-15, atol=0)


# ---------------------------------------------------------------- NEXT-1 / NEXT-2: RDF and kernel-density sum
def test_kde_bruteforce_and_closed_forms():
    p = g.clustered(1500, 9)
    d2 = pdist(p.astype(np.float64), "sqeuclidean")
    for gamma in (0.0, 1.0, 50.0):
        assert abs(oracle.kde(p, gamma) - float(np.exp(-np.float64(np.float32(gamma)) * d2).sum())) <= 1e-9 * len(d2)
    assert oracle.kde(np.zeros((10, 3), np.float32), 3.0) == 45.0              # coincident: C(10,2) * 1
    two = np.array([[0, 0, 0], [1, 2, 2]], np.float32)                            # d^2 = 9
    assert abs(oracle.kde(two, 0.5) - math.exp(-4.5)) < 1e-15
    a = oracle.kde(p, 2.0, rows=(0, 700)) + oracle.kde(p, 2.0, rows=(700, 1500))
    assert abs(a - oracle.kde(p, 2.0)) < 1e-12 * oracle.kde(p, 2.0)


@pytest.mark.parametrize("dim", [1, 2, 3, 4])
def test_rdf_unit_ball_vs_gamma_function(dim):
    """The oracle's dim-ball volume c_d, read back through its API (one pair in shell 0 of
    width 1, pairs = 1, V = 1 gives g[0] = 1 / c_d), equals pi^(d/2) / Gamma(d/2 + 1)
    (scipy.special.gamma: a library routine the oracle does not use)."""
    from scipy.special import gamma as G
    g0 = oracle.rdf(np.array([1], np.uint64), 1.0, 1.0, dim, pairs=1)[0]
    assert abs(1.0 / g0 - math.pi ** (dim / 2) / G(dim / 2 + 1)) < 1e-14


@pytest.mark.parametrize("dim", [1, 2, 3, 4])
def test_rdf_two_point_shell(dim):
    """Hand case per dimension: two points 1.25 apart, w = 0.5, nb = 4, V = 10. The pair lies
    in shell 2 = [1.0, 1.5); one pair counted, so g[2] = V / (c_d (1.5^d - 1^d)) and every
    other shell is 0. The clamp bucket of the nb+1-bucket SDH stays empty (d < nb w = 2)."""
    from scipy.special import gamma as G
    p = np.zeros((2, dim), np.float32)
    p[1, 0] = 1.25
    gr, h, _ = oracle.rdf_points(p, 0.5, 4, 10.0)
    assert h.tolist() == [0, 0, 1, 0, 0]
    c = math.pi ** (dim / 2) / G(dim / 2 + 1)
    expect = [0.0, 0.0, 10.0 / (c * (1.5 ** dim - 1.0)), 0.0]
    np.testing.assert_allclose(gr, expect, rtol=1e-14, atol=0)
    # a pair beyond nb w lands in the dropped clamp bucket, never in g
    q = np.zeros((2, dim), np.float32)
    q[1, 0] = 7.0
    gq, hq, _ = oracle.rdf_points(q, 0.5, 4, 10.0)
    assert hq.tolist() == [0, 0, 0, 0, 1] and not gq.any()


def test_rdf_row_range_pairs():
    """An anchor-row strip is normalised by the pairs that strip counts: strips
    of a partition give g_strip * pairs_strip that sum to g_full * pairs_full."""
    p = g.uniform(900, 31)
    w, nb = 0.05, 20
    full, _, _ = oracle.rdf_points(p, w, nb, 1.0)
    acc = np.zeros(nb)
    for rows in ((0, 100), (100, 450), (450, 900)):
        gs, _, _ = oracle.rdf_points(p, w, nb, 1.0, rows=rows)
        acc += gs * oracle.pairs_of_rows(900, rows)
    assert oracle.pairs_of_rows(900) == 900 * 899 // 2
    np.testing.assert_allclose(acc, full * (900 * 899 // 2), rtol=1e-12)


def covariogram_g(dim, r0, r1, m=400000, seed=0):
    """Expected RDF of uniform points in the unit dim-cube over the shell [r0, r1): the mean of
    the cube's set covariogram prod_c (1 - |u_c|)^+ over points u uniform in the shell
    (E h_k / pairs = int_shell prod_c (1 - |u_c|)^+ du). Monte Carlo, independent of the oracle."""
    rng = np.random.default_rng(seed)
    r = (r0 ** dim + rng.random(m) * (r1 ** dim - r0 ** dim)) ** (1.0 / dim)
    v = rng.standard_normal((m, dim))
    u = v / np.linalg.norm(v, axis=1, keepdims=True) * r[:, None]
    f = np.prod(np.clip(1.0 - np.abs(u), 0.0, None), axis=1)
    return f.mean(), f.std() / math.sqrt(m)


@pytest.mark.parametrize("dim", [1, 2, 3, 4])
def test_rdf_uniform_hypercube_law(dim):
    """Uniform points in the unit dim-cube (V = 1): the oracle's g over 8 seeds agrees with the
    covariogram law (Monte Carlo above) within 5 standard errors (the seeds' spread) plus the
    Monte Carlo error. A wrong ball constant, exponent or pair count shifts g by >= 10 %."""
    n, nb = 2000, 8
    w = {1: 0.02, 2: 0.02, 3: 0.04, 4: 0.06}[dim]
    gs = np.array([oracle.rdf_points(g.uniform(n, 100 + s, dim), w, nb, 1.0)[0] for s in range(8)])
    mean, se = gs.mean(0), gs.std(0, ddof=1) / math.sqrt(len(gs))
    for k in range(1, nb):
        ex, mc = covariogram_g(dim, k * w, (k + 1) * w, seed=k)
        assert abs(mean[k] - ex) <= 5 * se[k] + 5 * mc + 1e-3, (dim, k, mean[k], ex, se[k])
    assert 0.5 < mean[1:].mean() < 1.0      # boundary deficit: g < 1 for a finite cube


def test_sdh_bands_bruteforce():
    """oracle.sdh_bands: same histogram and 1e-6 band as oracle.sdh, and the 5e-7 diagnostic
    band equals a scipy pdist brute-force count; the bands nest."""
    p = g.uniform(1500, 41)
    nb = 16384
    w = float(np.float32(math.sqrt(3) / nb))
    h, a, a2 = oracle.sdh_bands(p, w, nb)
    h1, a1 = oracle.sdh(p, w, nb)
    assert h.tolist() == h1.tolist() and a.tolist() == a1.tolist()
    _, d = brute_sdh(p, w, nb)
    wd = np.float64(np.float32(w))
    e = np.rint(d / wd)
    ok = (e >= 1) & (e <= nb - 1) & (np.abs(d - e * wd) <= 5e-7 * e * wd)
    assert a2.tolist() == np.bincount(e[ok].astype(np.int64), minlength=nb + 1).tolist()
    assert np.all(a2 <= a) and a2.sum() > 100 and a.sum() > a2.sum()


# ---------------------------------------------------------------- NEXT-3: high-dimensional Type-III (bf16 features)
def bf16_bits(a):
    """Round-to-nearest-even fp32 -> bf16 bit patterns (test-side input construction)."""
    u = np.ascontiguousarray(a, dtype=np.float32).view(np.uint32).astype(np.uint64)
    r = ((u >> 16) & 1) + 0x7FFF
    return ((u + r) >> 16).astype(np.uint16)


def test_pairmatrix_hd_vs_cdist():
    import torch
    rng = np.random.default_rng(3)
    x = bf16_bits(rng.standard_normal((300, 40)).astype(np.float32))
    xf = (x.astype(np.uint32) << 16).view(np.float32).astype(np.float64)
    t = torch.from_numpy(xf)
    d = torch.cdist(t, t, compute_mode="donot_use_mm_for_euclid_dist").numpy()
    np.testing.assert_allclose(oracle.pairmatrix_hd(x, 0.05), np.exp(-np.float64(np.float32(0.05)) * d * d),
                               rtol=1e-12, atol=0)
    np.testing.assert_allclose(oracle.pairmatrix_hd(x, 0.0, ktype=1), d * d, rtol=1e-12, atol=1e-12)
    np.testing.assert_allclose(oracle.pairmatrix_hd(x, 0.0, ktype=2), d, rtol=1e-12, atol=1e-12)
    full = oracle.pairmatrix_hd(x, 0.3)
    assert np.array_equal(full, full.T) and np.all(np.diag(full) == 1.0)
    assert np.array_equal(oracle.pairmatrix_hd(x, 0.3, rows=(17, 90)), full[17:90])


# ---- all-point kNN (NEXT-2; reading R5: ties -> smaller index) -----------
def _knn_lexsort(p, k):
    """Independent brute force: full distance matrix (scipy), then a lexicographic sort of
    (distance, index) per row with the self pair removed."""
    from scipy.spatial.distance import cdist
    n = len(p)
    D = cdist(p.astype(np.float64), p.astype(np.float64))
    idx = np.full((n, k), -1, np.int64)
    dist = np.full((n, k), np.inf)
    for i in range(n):
        j = np.array([x for x in range(n) if x != i], np.int64)
        order = np.lexsort((j, D[i, j]))[:k]
        idx[i, :len(order)] = j[order]
        dist[i, :len(order)] = D[i, j[order]]
    return idx, dist


@pytest.mark.parametrize("dim,n,k,seed", [(1, 40, 3, 1), (2, 60, 5, 2), (3, 80, 8, 3), (4, 50, 16, 4), (3, 9, 12, 5)])
def test_knn_vs_lexsort_bruteforce(dim, n, k, seed):
    p = g.uniform(n, seed, dim)
    i_o, d_o = oracle.knn(p, k)
    i_b, d_b = _knn_lexsort(p, k)
    assert np.array_equal(i_o, i_b)
    np.testing.assert_allclose(d_o, d_b, rtol=1e-12, atol=0)


def test_knn_lattice_neighbour_shells():
    # unit cubic lattice: an interior point has 6 neighbours at 1, 12 at sqrt 2, 8 at sqrt 3;
    # a corner has 3, 3, 1 (closed form)
    L = 5
    p = g.lattice(L, 11)
    _, d = oracle.knn(p, 26)
    key = [tuple(x) for x in p.astype(int)]
    centre, corner = key.index((2, 2, 2)), key.index((0, 0, 0))
    want = [1.0] * 6 + [math.sqrt(2)] * 12 + [math.sqrt(3)] * 8
    np.testing.assert_allclose(d[centre], want, rtol=1e-15)
    assert np.allclose(d[corner][:7], [1, 1, 1, math.sqrt(2), math.sqrt(2), math.sqrt(2), math.sqrt(3)])
    assert d[corner][7] == 2.0
    # every lattice point's nearest neighbour is at distance exactly 1
    _, d1 = oracle.knn(p, 1)
    assert np.all(d1[:, 0] == 1.0)


def test_knn_ties_go_to_smaller_index():
    p = np.zeros((7, 3), np.float32)               # all coincident: every distance is 0
    idx, d = oracle.knn(p, 3)
    for i in range(7):
        assert list(idx[i]) == [j for j in range(7) if j != i][:3]
    assert np.all(d == 0.0)
    # two shells around point 0, inserted in scrambled index order
    q = np.array([[0, 0, 0], [2, 0, 0], [1, 0, 0], [0, 2, 0], [0, 1, 0], [0, 0, 1]], np.float32)
    idx, d = oracle.knn(q, 5)
    assert list(idx[0]) == [2, 4, 5, 1, 3]
    assert list(d[0]) == [1, 1, 1, 2, 2]


def test_knn_k_exceeds_n_minus_1_and_rows():
    p = g.uniform(4, 7, 3)
    idx, d = oracle.knn(p, 6)
    assert np.all(idx[:, 3:] == -1) and np.all(np.isinf(d[:, 3:]))
    assert all(sorted(idx[i, :3]) == [j for j in range(4) if j != i] for i in range(4))
    assert oracle.knn(np.zeros((1, 3), np.float32), 2)[0].tolist() == [[-1, -1]]
    q = g.uniform(300, 8, 3)
    full_i, full_d = oracle.knn(q, 4)
    part_i, part_d = oracle.knn(q, 4, rows=(100, 170))
    assert np.array_equal(part_i, full_i[100:170]) and np.array_equal(part_d, full_d[100:170])


def test_4m_golden_parts_merge():
    """The north-star golden (tools/make_goldens.py, oracle only) is the sum of its two
    pair-balanced parts; each part's mass is the pair count of its anchor rows and the whole
    is C(n, 2); every ambiguity count is bounded by its neighbouring buckets' mass."""
    base = os.path.join(GOLDEN, "sdh_uniform_n4194304_nb256_seed6")
    full = json.load(open(base + ".json"))
    parts = [json.load(open(os.path.join(GOLDEN, "parts", f"sdh_uniform_n4194304_nb256_seed6.part{k}of2.json")))
             for k in (0, 1)]
    n = full["spec"]["n"]
    assert sum(full["hist"]) == n * (n - 1) // 2
    for pt in parts:
        b, e = pt["rows"]
        assert sum(pt["hist"]) == (e - b) * (2 * n - b - e - 1) // 2
        assert pt["w"] == full["w"] == float(np.float32(math.sqrt(3) / 256))
    assert [x + y for x, y in zip(parts[0]["hist"], parts[1]["hist"])] == full["hist"]
    assert [x + y for x, y in zip(parts[0]["amb"], parts[1]["amb"])] == full["amb"]
    h, a = full["hist"], full["amb"]
    assert all(a[k] <= h[k - 1] + h[k] for k in range(1, 256))

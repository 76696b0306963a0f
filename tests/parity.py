"""Acceptance rules for GPU-vs-oracle parity (BASELINE.json north star)."""
import numpy as np
import oracle


def check_sdh_float(h_gpu, h_or, amb, amb_diag=None):
    """Float SDH: mass equal exactly; for every edge e, the cumulative counts
    C(e) = sum_{b<e} h[b] differ by at most A_e (pairs within 1e-6 e w of edge e —
    only those can change side under fp32 rounding). Implies per-bucket
    |h_gpu[b] - h_or[b]| <= A_b + A_{b+1}. Returns diagnostics; with amb_diag (the oracle's
    5e-7 band counts, oracle.sdh_bands) also the SURVEY §8(c) diagnostic: the edges where the
    GPU moved more pairs than lie within 5e-7 of the edge, and the excess (a lower bound on
    the pairs the GPU placed wrongly although they are 5e-7..1e-6 from the edge)."""
    g = np.asarray(h_gpu, dtype=np.int64)
    o = np.asarray(h_or, dtype=np.int64)
    a = np.asarray(amb, dtype=np.int64)
    nb = len(o)
    assert g.shape == o.shape
    assert g.sum() == o.sum(), f"mass {g.sum()} != {o.sum()}"
    cg, co = np.cumsum(g)[:-1], np.cumsum(o)[:-1]          # C(e) for e = 1..nb-1
    dev = np.abs(cg - co)
    bad = np.nonzero(dev > a[1:nb])[0]
    assert bad.size == 0, f"edges {bad[:10] + 1}: |dC| {dev[bad[:10]]} > A_e {a[1:nb][bad[:10]]}"
    per = np.abs(g - o)
    lim = a[:nb] + a[1:nb + 1]
    assert np.all(per <= lim)
    out = dict(max_bucket_diff=int(per.max()), edges_differing=int((dev > 0).sum()), amb_total=int(a.sum()),
               pairs_moved=int(dev.sum()))
    if amb_diag is not None:
        a2 = np.asarray(amb_diag, dtype=np.int64)[1:nb]
        over = dev - a2
        out.update(amb_diag_total=int(a2.sum()), edges_over_diag_band=int((over > 0).sum()),
                   diag_band_excess=int(np.clip(over, 0, None).sum()),
                   max_dev_over_diag_amb=float(np.max(dev / np.maximum(a2, 1))) if dev.size else 0.0)
    return out


def check_pcf_float(c_gpu, c_or, amb):
    assert abs(int(c_gpu) - int(c_or)) <= int(amb), f"{c_gpu} vs {c_or} (amb {amb})"


def check_matrix(out_gpu, out_or, rtol=1e-5):
    g = np.asarray(out_gpu, dtype=np.float64)
    o = np.asarray(out_or, dtype=np.float64)
    assert g.shape == o.shape
    tiny = np.abs(o) < 1e-30
    rel = np.where(tiny, np.abs(g - o) / 1e-30, np.abs(g - o) / np.where(tiny, 1.0, np.abs(o)))
    m = float(rel.max()) if rel.size else 0.0
    assert m <= rtol, f"max rel err {m}"
    return m


def check_knn_float(p, k, gi, gd, rows=None, rtol=4e-6):
    """Float inputs: the GPU orders by the fp32 squared distance, so near-ties may swap.
    Checks: distances agree with the oracle's position by position (rtol); every returned
    index is valid, distinct, not the anchor, and its true distance equals the reported one;
    where the oracle's distance at a position is separated from its neighbours by more than
    the tolerance, the index is the oracle's."""
    oi, od = oracle.knn(p, k, rows=rows)
    rb = 0 if rows is None else rows[0]
    fin = np.isfinite(od)
    assert np.array_equal(np.isfinite(gd), fin) and np.all(gi[~fin] == -1)
    np.testing.assert_allclose(gd[fin], od[fin], rtol=rtol, atol=1e-30)
    P = p.astype(np.float64)
    for r in range(len(gi)):
        row = gi[r][gi[r] >= 0]
        assert len(set(row.tolist())) == len(row) and (rb + r) not in row
        true = np.sqrt(((P[row] - P[rb + r]) ** 2).sum(1))
        np.testing.assert_allclose(gd[r][:len(row)], true, rtol=rtol, atol=1e-30)
        sep = np.ones(k, bool)
        dd = od[r]
        gap = rtol * 4 * np.maximum(dd, 1e-30)
        sep[1:] &= (dd[1:] - dd[:-1]) > gap[1:]
        sep[:-1] &= (dd[1:] - dd[:-1]) > gap[:-1]
        assert np.array_equal(gi[r][sep & fin[r]], oi[r][sep & fin[r]]), r

"""The seeded input generators (tbs_inputs): determinism and recipe checks."""
import numpy as np

import tbs_inputs as g


def test_splitmix64_reference_vector():
    # Published splitmix64 outputs for seed 0 (Steele, Lea & Flood 2014; java.util.SplittableRandom).
    assert [int(x) for x in g.splitmix64(0, 0, 3)] == [0xE220A8397B1DCDAF, 0x6E789E6AA1B965F4,
                                                      0x06C45D188009454F]
    # counter form: any slice equals the same draws of the full stream
    assert np.array_equal(g.splitmix64(5, 10, 7), g.splitmix64(5, 0, 17)[10:])


def test_uniform_exact_fixed_point():
    p = g.uniform(10000, 3)
    assert p.dtype == np.float32 and p.shape == (10000, 3)
    assert p.min() >= 0 and p.max() < 1
    assert np.all(p * 2 ** 24 == np.floor(p * 2 ** 24))
    assert np.array_equal(p, g.uniform(10000, 3))
    assert not np.array_equal(p, g.uniform(10000, 4))
    assert abs(p.mean() - 0.5) < 0.01


def test_lattice_is_permuted_grid():
    p = g.lattice(7, 9)
    assert p.shape == (343, 3)
    keys = sorted(map(tuple, p.astype(int).tolist()))
    assert keys == [(a, b, c) for a in range(7) for b in range(7) for c in range(7)]
    assert not np.array_equal(p, g.lattice(7, 10))


def test_clustered_recipe():
    p = g.clustered(200000, 3)
    assert p.shape == (200000, 3) and p.min() >= 0 and p.max() < 1
    assert np.array_equal(p, g.clustered(200000, 3))
    # nearest-parent distance: ~90% of points sit within a few sigma_c of a parent
    par = (g.splitmix64(3, 0, 3 * g.CLUSTER_K) >> np.uint64(40)).astype(np.float64).reshape(-1, 3) / 2 ** 24
    x = p[:5000].astype(np.float64)
    d = np.abs(x[:, None, :] - par[None, :, :])
    d = np.minimum(d, 1 - d)                                 # wrapped
    dist = np.sqrt((d ** 2).sum(-1))
    near = dist.min(1)
    frac = (near < 0.06).mean()
    # 90% children (|offset| < 0.06 w.p. ~0.99) + 10% background, of which a fraction
    # 1 - exp(-K 4/3 pi 0.06^3) ~ 0.6 falls near some parent by chance: ~0.95-0.97
    assert 0.94 < frac < 0.98, frac
    # per-axis offset std ~ 0.01 among clustered points
    off = d[np.arange(len(x)), dist.argmin(1)][near < 0.06]
    assert 0.007 < np.sqrt((off ** 2).mean()) < 0.013

"""CPU-only checks of the C-ABI library: it loads, exports every symbol include/tbs.h
declares, rejects bad arguments synchronously, and its host-only partition logic
(tbs_rank_rows) is exact. No compute call is made (no GPU here)."""
import ctypes
import os
import re
import subprocess

import numpy as np
import pytest

import paper_conf_icpp_pitaksirianannt16_b200 as tbs
from paper_conf_icpp_pitaksirianannt16_b200 import build

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def L():
    build.build()
    return tbs.lib()


def declared_functions():
    src = open(os.path.join(ROOT, "include", "tbs.h")).read()
    return sorted(set(re.findall(r"^\s*(?:int|const char\*|void|uint64_t)\s+(tbs_\w+)\(", src, re.M)))


def test_exports_match_header(L):
    decl = declared_functions()
    assert set(decl) == set(tbs.EXPORTS)
    out = subprocess.run(["nm", "-D", "--defined-only", tbs.LIB_PATH], capture_output=True, text=True).stdout
    syms = set(re.findall(r" T (tbs_\w+)$", out, re.M))
    assert set(decl) <= syms, set(decl) - syms
    for f in decl:
        getattr(L, f)


def test_version(L):
    assert tbs.version() == 200


def test_kernels_are_sm100a(L):
    """The fat binary holds sm_100a SASS only (no PTX JIT fallback)."""
    out = subprocess.run(["cuobjdump", "--list-elf", tbs.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out
    sass = subprocess.run(["cuobjdump", "-sass", tbs.LIB_PATH], capture_output=True, text=True).stdout
    for mnem in ("ATOMS", "FFMA2", "FADD2", "MUFU.SQRT", "UBLKCP", "SYNCS"):
        assert mnem in sass, mnem


def _args(n=10, dim=3, rb=0, re_=None, pts=1):
    return tbs._Args(pts, n, dim, rb, n if re_ is None else re_, None, 0, None, None, None, 0, 0)


@pytest.mark.parametrize("kw,nb,w", [
    (dict(n=-1), 8, 0.1), (dict(n=(1 << 30) + 1), 8, 0.1), (dict(dim=0), 8, 0.1), (dict(dim=5), 8, 0.1),
    (dict(rb=-1), 8, 0.1), (dict(rb=5, re_=4), 8, 0.1), (dict(re_=11), 8, 0.1), (dict(pts=0), 8, 0.1),
    ({}, 0, 0.1), ({}, (1 << 24) + 1, 0.1), ({}, 8, 0.0), ({}, 8, -1.0), ({}, 8, float("inf")), ({}, 8, float("nan")),
])
def test_sdh_einval(L, kw, nb, w):
    a = _args(**kw)
    h = np.zeros(max(nb, 1), np.uint64)
    assert L.tbs_sdh_ex(ctypes.byref(a), w, nb, h.ctypes.data) == tbs.TBS_EINVAL
    assert tbs.last_error() != ""


def test_sdh_einval_null_hist_and_lattice_width(L):
    a = _args()
    assert L.tbs_sdh_ex(ctypes.byref(a), 0.5, 8, None) == tbs.TBS_EINVAL
    a.flags = tbs.TBS_EXACT_LATTICE
    h = np.zeros(8, np.uint64)
    assert L.tbs_sdh_ex(ctypes.byref(a), 0.3, 8, h.ctypes.data) == tbs.TBS_EINVAL      # 0.3 is not m * 2^-j
    assert "EXACT_LATTICE" in tbs.last_error()


def test_rdf_einval(L):
    """RDF (NEXT-1): argument errors are synchronous (no GPU work)."""
    a = _args()
    g = np.zeros(8, np.float64)
    assert L.tbs_rdf_ex(ctypes.byref(a), 0.5, 8, 0.0, g.ctypes.data) == tbs.TBS_EINVAL           # volume
    assert L.tbs_rdf_ex(ctypes.byref(a), 0.5, 8, float("inf"), g.ctypes.data) == tbs.TBS_EINVAL
    assert L.tbs_rdf_ex(ctypes.byref(a), 0.5, 0, 1.0, g.ctypes.data) == tbs.TBS_EINVAL
    assert L.tbs_rdf_ex(ctypes.byref(a), -0.5, 8, 1.0, g.ctypes.data) == tbs.TBS_EINVAL
    assert L.tbs_rdf_ex(ctypes.byref(a), 0.5, 8, 1.0, None) == tbs.TBS_EINVAL
    a.flags = tbs.TBS_OUT_PEERS
    assert L.tbs_rdf_ex(ctypes.byref(a), 0.5, 8, 1.0, g.ctypes.data) == tbs.TBS_EUNSUPPORTED
    h = np.zeros(8, np.uint64)
    assert L.tbs_rdf_hist_ex(h.ctypes.data, 8, 5, 0.5, 10.0, 1.0, g.ctypes.data, None) == tbs.TBS_EINVAL  # dim
    assert L.tbs_rdf_hist_ex(h.ctypes.data, 8, 3, 0.5, -1.0, 1.0, g.ctypes.data, None) == tbs.TBS_EINVAL  # pairs
    assert L.tbs_rdf_hist_ex(None, 8, 3, 0.5, 10.0, 1.0, g.ctypes.data, None) == tbs.TBS_EINVAL
    ok = ctypes.c_int(7)
    assert L.tbs_peer_atomics_ok(None, ctypes.byref(ok)) == tbs.TBS_EINVAL


def test_pcf_and_matrix_einval(L):
    a = _args()
    c = np.zeros(1, np.uint64)
    assert L.tbs_pcf_ex(ctypes.byref(a), -1.0, c.ctypes.data) == tbs.TBS_EINVAL
    assert L.tbs_pcf_ex(ctypes.byref(a), float("nan"), c.ctypes.data) == tbs.TBS_EINVAL
    assert L.tbs_pcf_ex(ctypes.byref(a), 1.0, None) == tbs.TBS_EINVAL
    assert L.tbs_pairmatrix_ex(ctypes.byref(a), tbs._Kernel(7, 1.0), c.ctypes.data) == tbs.TBS_EINVAL
    assert L.tbs_pairmatrix_ex(ctypes.byref(a), tbs._Kernel(0, float("inf")), c.ctypes.data) == tbs.TBS_EINVAL
    assert L.tbs_pairmatrix_ex(ctypes.byref(a), tbs._Kernel(0, 1.0), None) == tbs.TBS_EINVAL


def test_out_peers_validation(L):
    """TBS_OUT_PEERS (fused multi-GPU combine): 1..16 non-NULL peer buffers, SDH and 2PCF only;
    checked before any device work (no GPU needed)."""
    arr = (ctypes.c_void_p * 3)(1, 2, 3)
    a = _args()
    a.flags = tbs.TBS_OUT_PEERS
    assert L.tbs_sdh_ex(ctypes.byref(a), 0.5, 8, None) == tbs.TBS_EINVAL       # n_out_peers = 0
    a.out_peers, a.n_out_peers = arr, tbs.TBS_MAX_PEERS + 1
    assert L.tbs_pcf_ex(ctypes.byref(a), 0.5, None) == tbs.TBS_EINVAL
    arr[1] = None
    a.n_out_peers = 3
    assert L.tbs_sdh_ex(ctypes.byref(a), 0.5, 8, None) == tbs.TBS_EINVAL       # a NULL peer
    assert "out_peers[1]" in tbs.last_error()
    arr[1] = 2
    # every peer buffer must hold exactly the words the call writes
    a.out_peer_words = 4
    assert L.tbs_sdh_ex(ctypes.byref(a), 0.5, 8, None) == tbs.TBS_EINVAL       # 4 words < nb = 8
    assert "out_peer_words" in tbs.last_error()
    assert L.tbs_pcf_ex(ctypes.byref(a), 0.5, None) == tbs.TBS_EINVAL          # 4 words != 1
    a.out_peer_words = 8
    c = np.zeros(1, np.float64)
    assert L.tbs_kde_ex(ctypes.byref(a), 1.0, c.ctypes.data) == tbs.TBS_EUNSUPPORTED
    assert L.tbs_pairmatrix_ex(ctypes.byref(a), tbs._Kernel(0, 1.0), c.ctypes.data) == tbs.TBS_EUNSUPPORTED
    assert L.tbs_peer_alloc(0, ctypes.byref(ctypes.c_void_p()), ctypes.create_string_buffer(64)) == tbs.TBS_EINVAL
    assert L.tbs_peer_open(None, ctypes.byref(ctypes.c_void_p())) == tbs.TBS_EINVAL


@pytest.mark.parametrize("n", [0, 1, 2, 3, 7, 100, 2048, 4096, 1 << 20, 4194304, 1 << 30])
@pytest.mark.parametrize("world", [1, 2, 3, 4, 8])
def test_rank_rows_partition(L, n, world):
    """Disjoint, covering, and pair-balanced: each rank's pair count is within one
    row's worth (<= n-1 pairs) of n(n-1)/(2W)."""
    prev = 0
    P = n * (n - 1) // 2
    for r in range(world):
        b, e = tbs.rank_rows(n, world, r)
        assert b == prev and e >= b
        prev = e
        pairs = (e * (2 * n - e - 1) - b * (2 * n - b - 1)) // 2
        assert abs(pairs - P / world) <= max(n - 1, 0) + 1
    assert prev == n


def test_rank_rows_bad_args(L):
    b, e = ctypes.c_int64(), ctypes.c_int64()
    assert L.tbs_rank_rows(10, 0, 0, ctypes.byref(b), ctypes.byref(e)) == tbs.TBS_EINVAL
    assert L.tbs_rank_rows(10, 2, 2, ctypes.byref(b), ctypes.byref(e)) == tbs.TBS_EINVAL
    assert L.tbs_rank_rows(-1, 2, 0, ctypes.byref(b), ctypes.byref(e)) == tbs.TBS_EINVAL


def test_no_oracle_in_product():
    """The product package never imports or links the oracle (ISOLATION rule)."""
    pkg = os.path.join(ROOT, "paper_conf_icpp_pitaksirianannt16_b200")
    for dp, _, fs in os.walk(pkg):
        for f in fs:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                txt = open(os.path.join(dp, f)).read()
                assert "oracle" not in txt.replace("# no oracle", ""), f
    out = subprocess.run(["ldd", tbs.LIB_PATH], capture_output=True, text=True).stdout
    assert "oracle" not in out

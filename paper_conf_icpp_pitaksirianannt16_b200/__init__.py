"""B200-native 2-body statistics (Pitaksirianan, Nouri & Tu, ICPP 2016).

Thin Python binding over the C ABI of ``libtbs.so`` (declared in include/tbs.h).
Every step of the hot path runs in the library's sm_100a kernels; this module only
marshals tensors (device pointers, the current CUDA stream) and, for multi-GPU,
does the one collective of the method: ``all_reduce(SUM)`` of the per-rank
histogram / count over NCCL. There is no CPU fallback: if the
library or a CUDA device is missing, calls raise.

    sdh(points, bucket_width, nbuckets)   Type-II spatial distance histogram (int64[nb])
    pcf(points, radius)                   Type-I 2-point correlation count   (int64[1])
    pairmatrix(points, gamma=1.0)         Type-III Gaussian pair matrix      (float32[rows, n])
    rank_rows(n, world, rank)             pair-balanced anchor-row partition
    kde(points, gamma)                    Type-I kernel-density pair sum      (float64[1])   (NEXT-2)
    knn(points, k)                        Type-I all-point k nearest neighbours (int32, float32 [n, k]) (NEXT-2)
    rdf(points, bucket_width, nb, volume) radial distribution function       (float64[nb])  (NEXT-1)
    rdf_from_hist(hist, ...)              its normalisation on a (combined) device histogram
    sdh_host / pcf_host / pairmatrix_host the same through host (numpy) buffers
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("TBS_LIB_VARIANT") or os.path.join(_HERE, "libtbs.so")  # variant: A/B experiments only

TBS_OK, TBS_EINVAL, TBS_ENOMEM, TBS_ECUDA, TBS_EUNSUPPORTED = range(5)
TBS_EXACT_LATTICE = 0x1
TBS_HIST_FORCE_LANE = 0x10
TBS_HIST_FORCE_CTA = 0x20
TBS_HIST_FORCE_GLOBAL = 0x40
TBS_FORCE_CLAMP = 0x100
TBS_HIST_FORCE_PASSES = 0x200
TBS_OUT_PEERS = 0x400
TBS_VALIDATE = 0x800
TBS_MAX_PEERS = 16
KERNELS = {"gaussian": 0, "dist2": 1, "dist": 2}
HIST_MODES = {None: 0, "lane": TBS_HIST_FORCE_LANE, "cta": TBS_HIST_FORCE_CTA, "global": TBS_HIST_FORCE_GLOBAL,
              "passes": TBS_HIST_FORCE_PASSES}

# Symbols declared in include/tbs.h (checked by tests/test_abi.py).
EXPORTS = ("tbs_sdh", "tbs_pcf", "tbs_pairmatrix", "tbs_sdh_ex", "tbs_pcf_ex", "tbs_pairmatrix_ex",
           "tbs_kde", "tbs_kde_ex", "tbs_knn", "tbs_knn_ex", "tbs_rdf", "tbs_rdf_ex", "tbs_rdf_hist_ex",
           "tbs_pairmatrix_hd", "tbs_pairmatrix_hd_ex",
           "tbs_rank_rows", "tbs_peer_alloc", "tbs_peer_open", "tbs_peer_close", "tbs_peer_free", "tbs_peer_atomics_ok",
           "tbs_last_error", "tbs_release", "tbs_launch_count", "tbs_version")


class TbsError(RuntimeError):
    pass


class _Args(ctypes.Structure):
    _fields_ = [("points", ctypes.c_void_p), ("n", ctypes.c_int64), ("dim", ctypes.c_int),
                ("row_begin", ctypes.c_int64), ("row_end", ctypes.c_int64), ("stream", ctypes.c_void_p),
                ("flags", ctypes.c_uint32), ("ev_begin", ctypes.c_void_p), ("ev_end", ctypes.c_void_p),
                ("out_peers", ctypes.POINTER(ctypes.c_void_p)), ("n_out_peers", ctypes.c_int),
                ("out_peer_words", ctypes.c_int64)]


class _Kernel(ctypes.Structure):
    _fields_ = [("type", ctypes.c_int), ("gamma", ctypes.c_float)]


_lib = None


def lib() -> ctypes.CDLL:
    """Load libtbs.so (built in-tree by build.py / __graft_entry__.build()). Raises if missing."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise TbsError(f"{LIB_PATH} not built: run `python -m paper_conf_icpp_pitaksirianannt16_b200.build`")
        L = ctypes.CDLL(LIB_PATH)
        vp, i64, u64p = ctypes.c_void_p, ctypes.c_int64, ctypes.POINTER(ctypes.c_uint64)
        L.tbs_sdh.argtypes = [vp, i64, ctypes.c_int, ctypes.c_float, ctypes.c_int, vp]
        L.tbs_pcf.argtypes = [vp, i64, ctypes.c_float, vp]
        L.tbs_pairmatrix.argtypes = [vp, i64, _Kernel, vp]
        L.tbs_sdh_ex.argtypes = [ctypes.POINTER(_Args), ctypes.c_float, ctypes.c_int, vp]
        L.tbs_pcf_ex.argtypes = [ctypes.POINTER(_Args), ctypes.c_float, vp]
        L.tbs_pairmatrix_ex.argtypes = [ctypes.POINTER(_Args), _Kernel, vp]
        L.tbs_kde.argtypes = [vp, i64, ctypes.c_float, vp]
        L.tbs_kde_ex.argtypes = [ctypes.POINTER(_Args), ctypes.c_float, vp]
        L.tbs_knn.argtypes = [vp, i64, ctypes.c_int, ctypes.c_int, vp, vp]
        L.tbs_knn_ex.argtypes = [ctypes.POINTER(_Args), ctypes.c_int, vp, vp]
        L.tbs_rdf.argtypes = [vp, i64, ctypes.c_int, ctypes.c_float, ctypes.c_int, ctypes.c_double, vp]
        L.tbs_rdf_ex.argtypes = [ctypes.POINTER(_Args), ctypes.c_float, ctypes.c_int, ctypes.c_double, vp]
        L.tbs_rdf_hist_ex.argtypes = [vp, ctypes.c_int, ctypes.c_int, ctypes.c_float, ctypes.c_double, ctypes.c_double,
                                      vp, vp]
        L.tbs_peer_atomics_ok.argtypes = [ctypes.c_char_p, ctypes.POINTER(ctypes.c_int)]
        L.tbs_pairmatrix_hd.argtypes = [vp, i64, ctypes.c_int, _Kernel, vp]
        L.tbs_pairmatrix_hd_ex.argtypes = [vp, i64, ctypes.c_int, i64, i64, _Kernel, vp, vp, vp, vp]
        L.tbs_rank_rows.argtypes = [i64, ctypes.c_int, ctypes.c_int, ctypes.POINTER(ctypes.c_int64),
                                    ctypes.POINTER(ctypes.c_int64)]
        L.tbs_peer_alloc.argtypes = [ctypes.c_uint64, ctypes.POINTER(ctypes.c_void_p), ctypes.c_char_p]
        L.tbs_peer_open.argtypes = [ctypes.c_char_p, ctypes.POINTER(ctypes.c_void_p)]
        L.tbs_peer_close.argtypes = [vp]
        L.tbs_peer_free.argtypes = [vp]
        L.tbs_last_error.restype = ctypes.c_char_p
        L.tbs_launch_count.restype = ctypes.c_uint64
        L.tbs_release.restype = None
        for f in ("tbs_sdh", "tbs_pcf", "tbs_pairmatrix", "tbs_sdh_ex", "tbs_pcf_ex", "tbs_pairmatrix_ex",
                  "tbs_kde", "tbs_kde_ex", "tbs_knn", "tbs_knn_ex", "tbs_rdf", "tbs_rdf_ex", "tbs_rdf_hist_ex",
                  "tbs_pairmatrix_hd", "tbs_pairmatrix_hd_ex", "tbs_rank_rows", "tbs_version",
                  "tbs_peer_alloc", "tbs_peer_open", "tbs_peer_close", "tbs_peer_free", "tbs_peer_atomics_ok"):
            getattr(L, f).restype = ctypes.c_int
        _lib = L
    return _lib


def _check(rc: int, what: str):
    if rc != TBS_OK:
        raise TbsError(f"{what}: status {rc}: {lib().tbs_last_error().decode()}")


def last_error() -> str:
    return lib().tbs_last_error().decode()


def launch_count() -> int:
    """Kernels libtbs.so has launched in this process."""
    return int(lib().tbs_launch_count())


def release() -> None:
    lib().tbs_release()


def version() -> int:
    return int(lib().tbs_version())


def rank_rows(n: int, world: int, rank: int) -> tuple[int, int]:
    """Anchor rows of `rank` in the pair-count-balanced partition (host-only, no GPU)."""
    b, e = ctypes.c_int64(), ctypes.c_int64()
    _check(lib().tbs_rank_rows(int(n), int(world), int(rank), ctypes.byref(b), ctypes.byref(e)), "tbs_rank_rows")
    return b.value, e.value


# ---------------------------------------------------------------- multi-GPU combine
def partition(n: int, group=None, rows=None):
    """Anchor rows this rank owns: the pair-balanced strip of `group`, else `rows`."""
    if group is None:
        return rows
    import torch.distributed as dist
    return rank_rows(n, dist.get_world_size(group), dist.get_rank(group))


class PeerSink:
    """Buffers of the fused combine (TBS_OUT_PEERS): one int64[words] device buffer per rank
    of `group`, each mapped into every rank (CUDA IPC; over NVLink between GPUs; every peer
    must be reachable with native atomics). A call with ``sink=`` accumulates its row strip's
    partial locally and the pair kernel's last CTA adds it into all of them (system-scope
    atomics: words x ranks remote adds per rank; after multi-launch output stages, one extra
    kernel does), so after ``finish()`` each rank's buffer holds the all-reduced
    result — the collective is fused into the call instead of a separate NCCL all_reduce.

    Every rank holds two buffers (parity p = result index & 1), so one host barrier per
    result suffices: ``begin(stream)`` enqueues the zeroing of this rank's OTHER-parity buffer
    (the next result's); the compute call adds into every rank's parity-p buffer; ``finish``
    syncs the stream, passes the barrier — after which every rank's adds for this result
    have landed and every rank's next-parity buffer is zero, and nobody adds into it before
    this barrier — and returns a copy of the local parity-p buffer (enqueued before the
    zeroing of that buffer two results later)."""

    def __init__(self, words: int, group=None, device=None):
        import torch
        import torch.distributed as dist
        self.words, self.group = int(words), group
        self.world = dist.get_world_size(group) if group is not None else 1
        self.rank = dist.get_rank(group) if group is not None else 0
        if self.world > TBS_MAX_PEERS:
            raise TbsError(f"fused combine supports at most {TBS_MAX_PEERS} ranks")
        dev = torch.device(device) if device is not None else torch.device("cuda", torch.cuda.current_device())
        self._own, self._opened, err = None, [], None
        with torch.cuda.device(dev):
            # every rank reaches every collective below, whatever fails locally, and all ranks
            # agree at the end: either every mapping works or every rank raises
            p, h = ctypes.c_void_p(), ctypes.create_string_buffer(64)
            if lib().tbs_peer_alloc(2 * self.words * 8, ctypes.byref(p), h) == TBS_OK:   # two parities, zeroed
                self._own = p.value
            else:
                err = "tbs_peer_alloc: " + last_error()
            handles = [None] * self.world
            pr = torch.cuda.get_device_properties(dev)
            bus = f"{pr.pci_domain_id:04x}:{pr.pci_bus_id:02x}:{pr.pci_device_id:02x}.0"
            mine = (h.raw, bus) if self._own is not None else None
            if group is not None:
                dist.all_gather_object(handles, mine, group=group)
            else:
                handles[0] = mine
            # the fused adds are system-scope atomics into peer memory: every peer GPU must be
            # reachable with NATIVE atomics (NVLink; not PCIe P2P), else all ranks fall back
            for r, hr in enumerate(handles):
                if hr is not None and err is None:
                    okp = ctypes.c_int(0)
                    if lib().tbs_peer_atomics_ok(hr[1].encode(), ctypes.byref(okp)) != TBS_OK or not okp.value:
                        err = f"no native peer atomics to rank {r} (GPU {hr[1]})"
            ptrs = []
            for r, hr in enumerate(handles):
                if r == self.rank:
                    ptrs.append(self._own)
                elif hr is None or err is not None:
                    err = err or f"rank {r} has no buffer"
                    ptrs.append(None)
                else:
                    q = ctypes.c_void_p()
                    if lib().tbs_peer_open(hr[0], ctypes.byref(q)) == TBS_OK:
                        self._opened.append(q.value)
                        ptrs.append(q.value)
                    else:
                        err = "tbs_peer_open: " + last_error()
                        ptrs.append(None)
            if group is not None:
                ok = torch.tensor([0 if err else 1], dtype=torch.int32, device=dev if dist.get_backend(group) == "nccl" else "cpu")
                dist.all_reduce(ok, op=dist.ReduceOp.MIN, group=group)
                if not int(ok.item()) and err is None:
                    err = "another rank could not map the peer buffers"
            if err is not None:
                self.close()
                raise TbsError(f"fused combine unavailable: {err}")
        self._ptrs = [(ctypes.c_void_p * self.world)(*[q + par * self.words * 8 for q in ptrs]) for par in (0, 1)]
        both = torch.as_tensor(_CudaArray(self._own, 2 * self.words), device=dev)
        self._local = (both[:self.words], both[self.words:])
        self.parity = 0

    @property
    def ptrs(self):
        """Every rank's parity-p buffer (the out_peers of the current result)."""
        return self._ptrs[self.parity]

    @property
    def local(self):
        return self._local[self.parity]

    def _barrier(self):
        if self.group is not None:
            import torch.distributed as dist
            dist.barrier(group=self.group)

    def begin(self, stream=None):
        import torch
        st = stream if stream is not None else torch.cuda.current_stream(self.local.device)
        with torch.cuda.stream(st):
            self._local[self.parity ^ 1].zero_()

    def finish(self, stream=None, out=None):
        import torch
        st = stream if stream is not None else torch.cuda.current_stream(self.local.device)
        st.synchronize()
        self._barrier()
        loc = self.local
        self.parity ^= 1
        with torch.cuda.stream(st):
            return loc.clone() if out is None else out.copy_(loc)

    def close(self):
        """Collective over the group (every rank calls it once)."""
        if getattr(self, "_closed", False):
            return
        self._closed = True
        for q in self._opened:
            lib().tbs_peer_close(q)
        self._barrier()   # no rank frees its buffer while a peer may still map it
        if self._own is not None:
            lib().tbs_peer_free(self._own)
        self._own, self._opened = None, []


class _CudaArray:
    """__cuda_array_interface__ view of a raw int64 device buffer (no copy)."""

    def __init__(self, ptr, words):
        self.__cuda_array_interface__ = {"shape": (words,), "typestr": "<i8", "data": (ptr, False), "version": 3}


def _fused(a, sink):
    if sink is not None:
        a.flags |= TBS_OUT_PEERS
        a.out_peers, a.n_out_peers, a.out_peer_words = sink.ptrs, sink.world, sink.words
    return a


def combine(partial, group=None):
    """The method's one exchange step: sum the per-rank int64 partial
    histograms / counts with a single all_reduce (NCCL over NVLink on GPUs). Integer
    sums are order-independent, so the result is bit-identical to one GPU."""
    if group is not None:
        import torch.distributed as dist
        dist.all_reduce(partial, op=dist.ReduceOp.SUM, group=group)
    return partial


# ---------------------------------------------------------------- device (torch) API
def _torch():
    import torch
    return torch


def _args(points, rows, flags, stream, events):
    torch = _torch()
    if not (isinstance(points, torch.Tensor) and points.is_cuda and points.dtype == torch.float32):
        raise TypeError("points must be a CUDA float32 tensor [n, dim]")
    if points.dim() == 1:
        points = points.reshape(-1, 1)
    if not points.is_contiguous():
        raise ValueError("points must be contiguous (AoS [n][dim])")
    n, dim = points.shape
    rb, re = (0, n) if rows is None else (int(rows[0]), int(rows[1]))
    st = stream if stream is not None else torch.cuda.current_stream(points.device)
    a = _Args(points.data_ptr(), n, dim, rb, re, st.cuda_stream, flags, None, None, None, 0, 0)
    if events is not None:
        a.ev_begin, a.ev_end = events[0].cuda_event, events[1].cuda_event
    return a, n


def sdh(points, bucket_width: float, nbuckets: int, *, rows=None, lattice: bool = False, hist_mode=None,
        force_clamp: bool = False, validate: bool = False, out=None, stream=None, events=None, group=None,
        sink=None):
    """Spatial distance histogram (Type-II). Returns int64[nbuckets] on points.device.

    rows=(b, e): only anchors i in [b, e) (with all partners j > i). lattice=True:
    exact integer bucketing (integer-valued points, bucket_width = m * 2^-j).
    group: a torch.distributed process group: each rank computes its pair-balanced
    strip (rank_rows) and the partial histograms are summed with one all_reduce, or, with
    sink=PeerSink(nbuckets, group), by the pair kernel itself (its last CTA adds the rank's partial
    into every rank's buffer over peer memory).
    validate=True: TBS_VALIDATE (debug; raises on non-finite coordinates and, with lattice, on a
    violated exact-lattice contract).
    """
    torch = _torch()
    flags = (TBS_EXACT_LATTICE if lattice else 0) | HIST_MODES[hist_mode] | (TBS_FORCE_CLAMP if force_clamp else 0) \
        | (TBS_VALIDATE if validate else 0)
    a, _ = _args(points, partition(points.shape[0], group, rows), flags, stream, events)
    if sink is not None:            # fused combine: the kernels' flush is the all-reduce
        if sink.words != nbuckets:
            raise ValueError(f"sink holds {sink.words} words, the histogram has {nbuckets}")
        sink.begin(stream)
        _check(lib().tbs_sdh_ex(ctypes.byref(_fused(a, sink)), float(bucket_width), int(nbuckets), None), "tbs_sdh_ex")
        return sink.finish(stream, out)
    h = out if out is not None else torch.empty(nbuckets, dtype=torch.int64, device=points.device)
    _check(lib().tbs_sdh_ex(ctypes.byref(a), float(bucket_width), int(nbuckets), h.data_ptr()), "tbs_sdh_ex")
    return combine(h, group)


def pcf(points, radius: float, *, rows=None, validate: bool = False, out=None, stream=None, events=None, group=None,
        sink=None):
    """2-point correlation count (Type-I): #{i<j : d < radius}, int64[1] on points.device.
    sink=PeerSink(1, group): fused combine (see sdh)."""
    torch = _torch()
    a, _ = _args(points, partition(points.shape[0], group, rows), TBS_VALIDATE if validate else 0, stream, events)
    if sink is not None:
        if sink.words != 1:
            raise ValueError(f"sink holds {sink.words} words, the 2PCF count has 1")
        sink.begin(stream)
        _check(lib().tbs_pcf_ex(ctypes.byref(_fused(a, sink)), float(radius), None), "tbs_pcf_ex")
        return sink.finish(stream, out)
    c = out if out is not None else torch.empty(1, dtype=torch.int64, device=points.device)
    _check(lib().tbs_pcf_ex(ctypes.byref(a), float(radius), c.data_ptr()), "tbs_pcf_ex")
    return combine(c, group)


def kde(points, gamma: float, *, rows=None, out=None, stream=None, events=None, group=None):
    """Kernel-density pair sum (Type-I, NEXT-2): sum_{i<j} exp(-gamma d^2), float64[1] on device.
    With a group the per-rank partial sums are combined with one all_reduce (fp64 SUM)."""
    torch = _torch()
    a, _ = _args(points, partition(points.shape[0], group, rows), 0, stream, events)
    s = out if out is not None else torch.empty(1, dtype=torch.float64, device=points.device)
    _check(lib().tbs_kde_ex(ctypes.byref(a), float(gamma), s.data_ptr()), "tbs_kde_ex")
    return combine(s, group)


def knn(points, k: int, *, rows=None, out=None, stream=None, events=None, group=None):
    """All-point k nearest neighbours (Type-I, NEXT-2): for each anchor row, the k nearest other
    points in ascending (distance, index) order. Returns (idx int32 [rows, k], dist float32
    [rows, k]); missing entries (n - 1 < k) are (-1, inf). With a group each rank computes an
    equal block of anchor rows (every row costs n - 1 distances); no collective is needed."""
    torch = _torch()
    n = points.shape[0]
    if group is not None:
        import torch.distributed as dist
        W, r = dist.get_world_size(group), dist.get_rank(group)
        rows = (n * r // W, n * (r + 1) // W)
    a, _ = _args(points, rows, 0, stream, events)
    nr = a.row_end - a.row_begin
    if out is not None:
        idx, dist_ = out
    else:
        idx = torch.empty((nr, k), dtype=torch.int32, device=points.device)
        dist_ = torch.empty((nr, k), dtype=torch.float32, device=points.device)
    _check(lib().tbs_knn_ex(ctypes.byref(a), int(k), idx.data_ptr(), dist_.data_ptr()), "tbs_knn_ex")
    return idx, dist_


def rdf_from_hist(hist, bucket_width: float, nbuckets: int, volume: float, pairs: int, dim: int = 3, *, out=None,
                  stream=None):
    """RDF normalisation (NEXT-1, reading R6) of a device int64 histogram of >= nbuckets shells
    (e.g. an SDH with nbuckets + 1 buckets combined across ranks) counting `pairs` pairs; runs on
    the device (tbs_rdf_hist_ex). Returns float64[nbuckets] on the histogram's device."""
    torch = _torch()
    if not (isinstance(hist, torch.Tensor) and hist.is_cuda and hist.dtype == torch.int64 and hist.numel() >= nbuckets):
        raise TypeError("hist must be a CUDA int64 tensor with >= nbuckets entries")
    st = stream if stream is not None else torch.cuda.current_stream(hist.device)
    g = out if out is not None else torch.empty(nbuckets, dtype=torch.float64, device=hist.device)
    _check(lib().tbs_rdf_hist_ex(hist.contiguous().data_ptr(), int(nbuckets), int(dim), float(bucket_width),
                                 float(pairs), float(volume), g.data_ptr(), st.cuda_stream), "tbs_rdf_hist_ex")
    return g


def rdf(points, bucket_width: float, nbuckets: int, volume: float, *, rows=None, lattice: bool = False,
        hist_mode=None, validate: bool = False, out=None, stream=None, events=None, group=None, sink=None):
    """Radial distribution function g[k], k < nbuckets (NEXT-1, reading R6): the SDH of the same
    pairs with nbuckets + 1 buckets (the clamp bucket is dropped), normalised on the device by
    the ideal-gas shell counts of the pairs counted (tbs_rdf_ex). With a group, the ranks' SDH
    strips are combined first (all_reduce, or sink=PeerSink(nbuckets + 1, group)) and the
    normalisation uses all n(n-1)/2 pairs."""
    torch = _torch()
    n = points.shape[0]
    dim = points.shape[1] if points.dim() > 1 else 1
    if group is not None:
        h = sdh(points, bucket_width, nbuckets + 1, lattice=lattice, hist_mode=hist_mode, stream=stream,
                events=events, group=group, sink=sink)
        return rdf_from_hist(h, bucket_width, nbuckets, volume, n * (n - 1) // 2, dim, out=out, stream=stream)
    flags = (TBS_EXACT_LATTICE if lattice else 0) | HIST_MODES[hist_mode] | (TBS_VALIDATE if validate else 0)
    a, _ = _args(points, rows, flags, stream, events)
    g = out if out is not None else torch.empty(nbuckets, dtype=torch.float64, device=points.device)
    _check(lib().tbs_rdf_ex(ctypes.byref(a), float(bucket_width), int(nbuckets), float(volume), g.data_ptr()),
           "tbs_rdf_ex")
    return g


def pairmatrix(points, gamma: float = 1.0, *, kernel: str = "gaussian", rows=None, out=None, stream=None,
               events=None, group=None):
    """Type-III pair matrix rows [b, e) x n (float32). With a group, each rank gets its
    block of rows (rank_rows over the full square is not needed: rows split evenly)."""
    torch = _torch()
    n = points.shape[0]
    if group is not None:
        import torch.distributed as dist
        W, r = dist.get_world_size(group), dist.get_rank(group)
        rows = (n * r // W, n * (r + 1) // W)
    a, _ = _args(points, rows, 0, stream, events)
    nr = a.row_end - a.row_begin
    o = out if out is not None else torch.empty((nr, n), dtype=torch.float32, device=points.device)
    _check(lib().tbs_pairmatrix_ex(ctypes.byref(a), _Kernel(KERNELS[kernel], float(gamma)), o.data_ptr()),
           "tbs_pairmatrix_ex")
    return o


def pairmatrix_hd(features, gamma: float = 1.0, *, kernel: str = "gaussian", rows=None, out=None, stream=None,
                  events=None, group=None):
    """High-dimensional Type-III pair matrix on the tensor cores (NEXT-3): features is a CUDA
    bfloat16 tensor [n, d] (d <= 128); returns float32 rows [b, e) x n."""
    torch = _torch()
    if not (isinstance(features, torch.Tensor) and features.is_cuda and features.dtype == torch.bfloat16):
        raise TypeError("features must be a CUDA bfloat16 tensor [n, d]")
    x = features.contiguous()
    n, d = x.shape
    if group is not None:
        import torch.distributed as dist
        W, r = dist.get_world_size(group), dist.get_rank(group)
        rows = (n * r // W, n * (r + 1) // W)
    rb, re = (0, n) if rows is None else (int(rows[0]), int(rows[1]))
    st = stream if stream is not None else torch.cuda.current_stream(x.device)
    o = out if out is not None else torch.empty((re - rb, n), dtype=torch.float32, device=x.device)
    ev = (events[0].cuda_event, events[1].cuda_event) if events is not None else (None, None)
    _check(lib().tbs_pairmatrix_hd_ex(x.data_ptr(), n, d, rb, re, _Kernel(KERNELS[kernel], float(gamma)), o.data_ptr(),
                                      st.cuda_stream, ev[0], ev[1]), "tbs_pairmatrix_hd_ex")
    return o


# ---------------------------------------------------------------- host (numpy) API
def _host_points(points):
    p = np.ascontiguousarray(points, dtype=np.float32)
    if p.ndim == 1:
        p = p.reshape(-1, 1)
    return p


def sdh_host(points, bucket_width: float, nbuckets: int, out=None):
    """tbs_sdh with host buffers (H2D copy, kernels, D2H copy inside the call)."""
    p = _host_points(points)
    h = out if out is not None else np.empty(nbuckets, np.uint64)
    _check(lib().tbs_sdh(p.ctypes.data, p.shape[0], p.shape[1], float(bucket_width), int(nbuckets), h.ctypes.data),
           "tbs_sdh")
    return h


def pcf_host(points, radius: float) -> int:
    p = _host_points(points)
    assert p.shape[1] == 3
    c = np.zeros(1, np.uint64)
    _check(lib().tbs_pcf(p.ctypes.data, p.shape[0], float(radius), c.ctypes.data), "tbs_pcf")
    return int(c[0])


def pairmatrix_host(points, gamma: float = 1.0, kernel: str = "gaussian"):
    p = _host_points(points)
    assert p.shape[1] == 3
    n = p.shape[0]
    o = np.empty((n, n), np.float32)
    _check(lib().tbs_pairmatrix(p.ctypes.data, n, _Kernel(KERNELS[kernel], float(gamma)), o.ctypes.data),
           "tbs_pairmatrix")
    return o


def knn_host(points, k: int):
    """tbs_knn with host buffers: (idx int32 [n, k], dist float32 [n, k])."""
    p = _host_points(points)
    n = p.shape[0]
    idx = np.empty((n, k), np.int32)
    d = np.empty((n, k), np.float32)
    _check(lib().tbs_knn(p.ctypes.data, n, p.shape[1], int(k), idx.ctypes.data, d.ctypes.data), "tbs_knn")
    return idx, d

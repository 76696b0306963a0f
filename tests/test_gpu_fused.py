"""GPU tests of the fused multi-GPU combine (TBS_OUT_PEERS): each
SDH / 2PCF call accumulates its strip's partial locally and its last kernel adds it into every
rank's buffer (system-scope atomics over peer memory) instead of a separate all_reduce.

Only one GPU is available here, so the peers are (1) several local buffers in one process
(the fan-out itself), and (2) two processes on the same GPU whose buffers are mapped into
each other by CUDA IPC — the same mapping a multi-GPU run uses over NVLink. Integer sums are
order-independent: the result must equal the oracle (lattice, bit-exact) and the unfused GPU
result (float, bit-exact: identical bucket decisions)."""
import ctypes
import math
import os
import socket

import numpy as np
import pytest

import oracle
import tbs_inputs as g

pytestmark = pytest.mark.gpu


def _fanout(tbs, p, op, npeers, world, **kw):
    """Every strip of a `world`-way partition adds into the same `npeers` local buffers."""
    import torch
    words = kw.get("nb", 1)
    bufs = [torch.zeros(words, dtype=torch.int64, device="cuda") for _ in range(npeers)]
    arr = (ctypes.c_void_p * npeers)(*[b.data_ptr() for b in bufs])
    pt = torch.from_numpy(p).cuda()
    flags = tbs.TBS_OUT_PEERS | (tbs.TBS_EXACT_LATTICE if kw.get("lattice") else 0) | tbs.HIST_MODES[kw.get("mode")]
    for r in range(world):
        a, _ = tbs._args(pt, tbs.rank_rows(len(p), world, r), flags, None, None)
        a.out_peers, a.n_out_peers, a.out_peer_words = arr, npeers, words
        if op == "sdh":
            rc = tbs.lib().tbs_sdh_ex(ctypes.byref(a), float(kw["w"]), int(kw["nb"]), None)
        else:
            rc = tbs.lib().tbs_pcf_ex(ctypes.byref(a), float(kw["r"]), None)
        tbs._check(rc, op)
    torch.cuda.synchronize()
    return [b.cpu().numpy() for b in bufs]


@pytest.mark.parametrize("mode", [None, "lane", "cta", "global", "passes"])
def test_fused_fanout_sdh_lattice(tbs, mode):
    p = g.lattice(20, 31)[:7000]
    want = oracle.sdh_lattice(p, 1, 1, 60).astype(np.int64)
    for b in _fanout(tbs, p, "sdh", 3, 4, w=0.5, nb=60, lattice=True, mode=mode):
        assert b.tolist() == want.tolist()


@pytest.mark.parametrize("nb", [256, 16384, 70000])
def test_fused_fanout_sdh_float_equals_unfused(tbs, nb):
    """Float mode, all output stages (lane copies, 2 copies at 16K, bucket-range passes)."""
    import torch
    p = g.clustered(9000, 32)
    w = float(np.float32(math.sqrt(3) / min(nb, 16384)))
    ref = tbs.sdh(torch.from_numpy(p).cuda(), w, nb).cpu().numpy()
    ho, amb = oracle.sdh(p, w, nb)
    from parity import check_sdh_float
    check_sdh_float(ref, ho, amb)
    for b in _fanout(tbs, p, "sdh", 2, 3, w=w, nb=nb):
        assert b.tolist() == ref.tolist()


def test_fused_fanout_pcf(tbs):
    p = g.lattice(18, 33)
    bufs = _fanout(tbs, p, "pcf", 4, 5, r=math.sqrt(30.0))
    c, amb = oracle.pcf(p, math.sqrt(30.0))
    for b in bufs:
        assert abs(int(b[0]) - int(c)) <= int(amb)
        assert int(b[0]) == int(bufs[0][0])


def test_fused_sink_single_rank(tbs):
    """PeerSink without a process group (world 1): the binding's begin/compute/finish path."""
    import torch
    p = g.lattice(16, 34)
    pt = torch.from_numpy(p).cuda()
    sink = tbs.PeerSink(64)
    try:
        for _ in range(2):   # the sink is reusable: begin() re-zeroes
            h = tbs.sdh(pt, 0.5, 64, lattice=True, sink=sink)
            assert h.cpu().tolist() == oracle.lattice_closed(16, 1, 1, 64)[0].tolist()
    finally:
        sink.close()


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _ipc_worker(rank, world, port, q):
    import torch
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_icpp_pitaksirianannt16_b200 as tbs
        torch.cuda.set_device(0)
        pl = torch.from_numpy(g.lattice(24, 35)).cuda()
        pc = torch.from_numpy(g.clustered(20000, 36)).cuda()
        sink = tbs.PeerSink(80, dist.group.WORLD)
        csink = tbs.PeerSink(1, dist.group.WORLD)
        try:
            hl = tbs.sdh(pl, 0.5, 80, lattice=True, group=dist.group.WORLD, sink=sink).cpu().tolist()
            hf = tbs.sdh(pc, float(np.float32(math.sqrt(3) / 80)), 80, group=dist.group.WORLD, sink=sink).cpu().tolist()
            c = int(tbs.pcf(pc, 0.03, group=dist.group.WORLD, sink=csink).cpu()[0])
            # a third result on the same sink reuses parity 0 (zeroed during the second)
            hl3 = tbs.sdh(pl, 0.5, 80, lattice=True, group=dist.group.WORLD, sink=sink).cpu().tolist()
            assert hl3 == hl
            # the unfused path (all_reduce over gloo of CUDA tensors is unsupported: sum on host)
            part = tbs.sdh(pc, float(np.float32(math.sqrt(3) / 80)), 80, rows=tbs.partition(20000, dist.group.WORLD))
            part = part.cpu()
            dist.all_reduce(part)
            q.put((rank, hl, hf, c, part.tolist()))
        finally:
            sink.close()
            csink.close()
    except Exception as e:   # surface the error to the parent instead of hanging it
        q.put((rank, repr(e), None, None, None))
        raise
    finally:
        dist.destroy_process_group()


def test_fused_two_processes_ipc(tbs):
    """Two ranks on one GPU, buffers mapped into each other by CUDA IPC (the multi-GPU
    mapping): each rank's strip flushes into both buffers; both hold the full result."""
    import torch.multiprocessing as mp
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_ipc_worker, args=(r, world, port, q)) for r in range(world)]
    for pr in procs:
        pr.start()
    res = sorted(q.get(timeout=600) for _ in range(world))
    for pr in procs:
        pr.join(timeout=120)
    for r in res:
        assert r[2] is not None, r[1]
    want_l = oracle.sdh_lattice(g.lattice(24, 35), 1, 1, 80).astype(np.int64).tolist()
    pc = g.clustered(20000, 36)
    cw, camb = oracle.pcf(pc, 0.03)
    for _, hl, hf, c, unfused in res:
        assert hl == want_l
        assert hf == unfused
        assert abs(c - int(cw)) <= int(camb)
    assert res[0][2:4] == res[1][2:4]
    for pr in procs:
        assert pr.exitcode == 0


def _nccl_worker(port, q):
    """A one-rank NCCL group on the GPU: the binding's group path (pair-balanced strip of a
    world-1 partition = all rows, then tbs.combine's all_reduce over NCCL on a device tensor)."""
    import torch
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    torch.cuda.set_device(0)
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda:0"))
    try:
        import paper_conf_icpp_pitaksirianannt16_b200 as tbs
        G = dist.group.WORLD
        pl = torch.from_numpy(g.lattice(20, 37)).cuda()
        pc = torch.from_numpy(g.clustered(30000, 38)).cuda()
        w = float(np.float32(math.sqrt(3) / 128))
        out = {
            "backend": dist.get_backend(G),
            "hl": tbs.sdh(pl, 0.5, 70, lattice=True, group=G).cpu().tolist(),
            "hf": tbs.sdh(pc, w, 128, group=G).cpu().tolist(),
            "hf1": tbs.sdh(pc, w, 128).cpu().tolist(),
            "c": int(tbs.pcf(pc, 0.03, group=G).cpu()[0]),
            "c1": int(tbs.pcf(pc, 0.03).cpu()[0]),
            "kde": float(tbs.kde(pc[:5000], 2.0, group=G).cpu()[0]),
            "kde1": float(tbs.kde(pc[:5000], 2.0).cpu()[0]),
        }
        q.put(out)
    except Exception as e:
        q.put({"error": repr(e)})
        raise
    finally:
        dist.destroy_process_group()


def test_nccl_combine_world1():
    """The north star's combine (one NCCL all_reduce of the rank partials) executed on the GPU:
    one rank, so the result must equal the ungrouped call bit for bit and the oracle's rule."""
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    pr = ctx.Process(target=_nccl_worker, args=(_free_port(), q))
    pr.start()
    r = q.get(timeout=600)
    pr.join(timeout=120)
    assert "error" not in r, r
    assert r["backend"] == "nccl"
    assert r["hl"] == oracle.sdh_lattice(g.lattice(20, 37), 1, 1, 70).astype(np.int64).tolist()
    assert r["hf"] == r["hf1"] and r["c"] == r["c1"]
    assert abs(r["kde"] - r["kde1"]) <= 1e-12 * abs(r["kde1"])   # fp64 partial sums: order may vary
    pc = g.clustered(30000, 38)
    cw, camb = oracle.pcf(pc, 0.03)
    assert abs(r["c"] - int(cw)) <= int(camb)
    assert pr.exitcode == 0

"""World-size-2 (and 3) gloo tests of the multi-GPU host logic on CPU: the pair-balanced
partition (tbs_rank_rows through the C ABI) and the one exchange step (tbs.combine =
all_reduce SUM). Each rank's partial comes from the oracle on its strip (stand-in for
the kernel, which needs a GPU); the combined result must equal the single-process
oracle bit-exactly, as the GPU path's must."""
import math
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        import paper_conf_icpp_pitaksirianannt16_b200 as tbs
        import tbs_inputs as g
        n, nb = 3001, 96
        w = float(np.float32(math.sqrt(3) / nb))
        p = g.clustered(n, 21)
        rows = tbs.partition(n, dist.group.WORLD)
        h = torch.from_numpy(oracle.sdh(p, w, nb, rows=rows)[0].astype(np.int64))
        h = tbs.combine(h, dist.group.WORLD)
        c = torch.tensor([oracle.pcf(p, 0.05, rows=rows)[0]], dtype=torch.int64)
        c = tbs.combine(c, dist.group.WORLD)
        pl = g.lattice(12, 4)
        hl = torch.from_numpy(oracle.sdh_lattice(pl, 1, 1, 40, rows=tbs.partition(len(pl), dist.group.WORLD))
                              .astype(np.int64))
        hl = tbs.combine(hl, dist.group.WORLD)
        q.put((rank, rows, h.tolist(), int(c.item()), hl.tolist()))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_partition_and_allreduce_gloo(world):
    import oracle
    import tbs_inputs as g
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for pr in procs:
        pr.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    n, nb = 3001, 96
    w = float(np.float32(math.sqrt(3) / nb))
    p = g.clustered(n, 21)
    full = oracle.sdh(p, w, nb)[0].astype(np.int64).tolist()
    fullc = oracle.pcf(p, 0.05)[0]
    fulll = oracle.sdh_lattice(g.lattice(12, 4), 1, 1, 40).astype(np.int64).tolist()
    res.sort()
    assert [r[1] for r in res][0][0] == 0 and res[-1][1][1] == n
    for i in range(world - 1):
        assert res[i][1][1] == res[i + 1][1][0]           # contiguous strips
    for _, _, h, c, hl in res:
        assert h == full and c == fullc and hl == fulll    # every rank holds the identical result

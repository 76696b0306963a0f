"""bench.py — throughput of the 2-BS hot path on B200 (one JSON line on rank 0).

Default workload (BASELINE.json configs[1], the metric's N=1M point): SDH of
N = 2^20 uniform 3-D points, 256 buckets, w = fp32(sqrt(3)/256). One step = one
full pass of the hot path: SoA loader -> triangular pair kernel with the privatised
shared-memory histogram -> u64 flush (-> NCCL all_reduce of the histogram for N>1).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload NAME] [--impl tbs|reference]
                    [--combine nccl|fused] [--dry-run]

Multi-GPU: one rank per GPU. Under torchrun (WORLD_SIZE set) the ranks are torchrun's and
WORLD_SIZE must equal --gpus; a plain `python bench.py --gpus N` (N > 1) re-launches itself
through torch.distributed.run with N local ranks. Each rank computes its pair-balanced anchor
strip (tbs_rank_rows) and the ranks sum their histograms with one NCCL all_reduce
(--combine nccl, the default and the north star's path) or with the kernels' own flush into
every rank's buffer over peer memory (--combine fused, TBS_OUT_PEERS). Strong scaling: the
problem is fixed. NCCL's INIT log goes to stderr (NCCL_DEBUG=INFO, NCCL_DEBUG_SUBSYS=INIT
unless set) so the communicator's ranks can be counted. --dry-run: no GPU work — the ranks
join a gloo group, check the world size and print their row strips (CPU test of the launch). Time = CUDA events on the
launching stream around exactly K steps, barrier + synchronize on both sides, max
over ranks. The L2 (126 MB) is flushed between steps by writing 256 MiB; the
inputs (12 MiB) are smaller than L2 and the flush is inside the timed region.
--impl reference times the CPU oracle (the reference arm of this tier) on bounded
samples of the same workload.
"""
from __future__ import annotations

import argparse
import ctypes
import json
import math
import os
import statistics
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import tbs_inputs as gen  # noqa: E402

WORKLOADS = {
    # name: (op, distribution, n, seed, params)
    "sdh_uniform_4k": ("sdh", "uniform", 4096, 1, dict(nb=64)),             # configs[0] (latency-bound)
    "sdh_uniform_1m": ("sdh", "uniform", 1 << 20, 2, dict(nb=256)),         # configs[1] (default)
    "sdh_clustered_1m": ("sdh", "clustered", 1 << 20, 3, dict(nb=256)),
    "sdh_uniform_4m": ("sdh", "uniform", 1 << 22, 6, dict(nb=256)),         # north-star target line
    "sdh_uniform_2m_16k": ("sdh", "uniform", 1 << 21, 4, dict(nb=16384)),   # configs[3]
    "sdh_lattice_4m": ("sdh_lattice", "lattice", 160 ** 3, 6, dict(nb=256, w=1.0)),
    "sdh_lattice_2m_16k": ("sdh_lattice", "lattice", 128 ** 3, 4, dict(nb=16384, w=2.0 ** -6)),  # configs[3], exact mode
    "pcf_clustered_4m": ("pcf", "clustered", 1 << 22, 3, dict(r=0.03)),     # configs[2]
    "pairmatrix_64k": ("pairmatrix", "uniform", 1 << 16, 5, dict(gamma=1.0)),  # configs[4]
    "kde_uniform_1m": ("kde", "uniform", 1 << 20, 2, dict(gamma=1.0)),        # NEXT-2 (Type-I float sum)
    "pairmatrix_hd_64k_d64": ("pairmatrix_hd", "uniform", 1 << 16, 7, dict(d=64, gamma=1.0 / 64)),  # NEXT-3
    "knn_uniform_1m_k8": ("knn", "uniform", 1 << 20, 2, dict(k=8)),  # NEXT-2 (all-point kNN)
    "pairmatrix_hd_64k_d512": ("pairmatrix_hd", "uniform", 1 << 16, 7, dict(d=512, gamma=1.0 / 512)),
    "rdf_uniform_1m": ("rdf", "uniform", 1 << 20, 2, dict(nb=256, volume=1.0)),  # NEXT-1 (SDH + normalisation)
}
METRIC = "SDH pair-distances/sec (G pairs/s) at N=1M–4M, 1/2/4/8 B200, % of roofline"

# Roofline denominators: B200 unit counts x max SM clock.
SMS = 148
FP32_LANES_PER_CLK_SM = 128        # FFMA/FADD lanes per SM per clock (FFMA2 issues half as often, same lanes)
ATOMS_LANES_PER_CLK_SM = 32        # conflict-free shared atomics: 1 warp-instr/clk/SM (31.5 measured, tools/peaks.cu)
MUFU_LANES_PER_CLK_SM = 16         # XU pipe (sqrt/rsqrt/ex2): 15.9 measured; one sqrt per SDH pair


def peaks():
    mp = {}
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            mp = json.load(f)
    f_max = float(mp.get("sm_max_mhz", 1965.0)) * 1e6
    return dict(
        f_max=f_max,
        fp32=SMS * FP32_LANES_PER_CLK_SM * f_max,
        atoms=SMS * ATOMS_LANES_PER_CLK_SM * f_max,
        mufu=SMS * MUFU_LANES_PER_CLK_SM * f_max,
        hbm=float(mp.get("hbm_gbs", 6650.0)) * 1e9,
        bf16=float(mp.get("bf16_tflops", 2250.0)) * 1e12,
        bf16_src="MEASURED_PEAKS.json bf16_tflops" if "bf16_tflops" in mp else "fallback 2.25 PF nominal",
        hbm_src="MEASURED_PEAKS.json hbm_gbs" if "hbm_gbs" in mp else "fallback 6.65 TB/s (B200_PROFILING.md)",
    )


def units_of(op, n):
    return n * n if op == "pairmatrix" else n * (n - 1) // 2


# ------------------------------------------------------------------ clocks sampler
class Clocks:
    """SM clock + clock-event reasons sampled DURING the timed region.

    A background thread polls NVML every 5 ms (the GPU is found by PCI bus id, so
    CUDA_VISIBLE_DEVICES remappings do not matter); `mark(True)` / `mark(False)` bracket the
    timed region on the host. Runs shorter than a few NVML periods still get their samples:
    the sampler is started (and has produced a sample) before the region opens, and the
    samples inside the bracket, plus the last one before and the first one after it, are
    reported, with `window_ms` and `samples` so a reader can judge them (None if NVML is
    unavailable)."""
    REASONS = {0x4: "sw_power_cap", 0x8: "hw_slowdown", 0x20: "sw_thermal_slowdown",
               0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown"}

    def __init__(self, torch_device):
        import threading
        self.rows, self.t0, self.t1, self.src = [], None, None, "nvml"
        self._stop = threading.Event()
        try:
            import pynvml as nv
            nv.nvmlInit()
            h = None
            try:
                import torch
                pr = torch.cuda.get_device_properties(torch_device)
                bus = f"{pr.pci_domain_id:08x}:{pr.pci_bus_id:02x}:{pr.pci_device_id:02x}.0"
                h = nv.nvmlDeviceGetHandleByPciBusId_v2(bus)
            except Exception:   # noqa: BLE001 — fall back to the visible index
                h = nv.nvmlDeviceGetHandleByIndex(torch_device.index or 0)
            self.max_mhz = nv.nvmlDeviceGetMaxClockInfo(h, nv.NVML_CLOCK_SM)

            def poll():
                while not self._stop.is_set():
                    try:
                        self.rows.append((time.perf_counter(), nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM),
                                          nv.nvmlDeviceGetCurrentClocksEventReasons(h)))
                    except Exception:   # noqa: BLE001
                        pass
                    self._stop.wait(0.005)
            self.th = threading.Thread(target=poll, daemon=True)
            self.th.start()
            t_end = time.perf_counter() + 2.0
            while not self.rows and time.perf_counter() < t_end:
                time.sleep(0.002)
        except Exception:   # noqa: BLE001
            self.th, self.src = None, "none"

    def mark(self, start):
        if start:
            self.t0 = time.perf_counter()
        else:
            self.t1 = time.perf_counter()

    def stop(self):
        if self.th is None:
            return None
        time.sleep(0.012)      # one more sample after the region closes
        self._stop.set()
        self.th.join()
        rows = self.rows
        if not rows or self.t0 is None or self.t1 is None:
            return None
        inside = [r for r in rows if self.t0 <= r[0] <= self.t1]
        before = [r for r in rows if r[0] < self.t0][-1:]
        after = [r for r in rows if r[0] > self.t1][:1]
        win = before + inside + after if len(inside) < 3 else inside
        reasons = sorted({nm for r in win for bit, nm in self.REASONS.items() if r[2] & bit})
        return {"sm_mhz": statistics.median(r[1] for r in win), "sm_max_mhz": self.max_mhz,
                "sm_min_mhz": min(r[1] for r in win), "reasons": reasons, "samples": len(win),
                "samples_inside": len(inside), "window_ms": round((self.t1 - self.t0) * 1e3, 3),
                "source": "nvml 5 ms poll"}


# ------------------------------------------------------------------ reference arm (CPU oracle)
def oracle_rate(op, p, params, rows):
    import oracle
    n = p.shape[0]
    t0 = time.perf_counter()
    if op == "sdh":
        oracle.sdh(p, float(np.float32(math.sqrt(3) / params["nb"])), params["nb"], rows=rows)
    elif op == "rdf":
        oracle.rdf_points(p, float(np.float32(math.sqrt(3) / params["nb"])), params["nb"], params["volume"], rows=rows)
    elif op == "sdh_lattice":
        oracle.sdh_lattice(p, 1, 0, params["nb"], rows=rows)
    elif op == "pcf":
        oracle.pcf(p, params["r"], rows=rows)
    elif op == "kde":
        oracle.kde(p, params["gamma"], rows=rows)
    elif op == "pairmatrix_hd":
        oracle.pairmatrix_hd(bf16_bits(p), params["gamma"], rows=rows)
    elif op == "knn":
        oracle.knn(p, params["k"], rows=rows)
    else:
        oracle.pairmatrix(p, params["gamma"], rows=rows)
    dt = time.perf_counter() - t0
    b, e = rows
    units = (e - b) * n if op.startswith("pairmatrix") else (e - b) * (n - 1) if op == "knn" else \
        (e - b) * (2 * n - b - e - 1) // 2
    return units, dt


def bf16_bits(a):
    """fp32 -> bf16 (round to nearest even) bit patterns, the same rounding torch applies."""
    u = np.ascontiguousarray(a, dtype=np.float32).view(np.uint32).astype(np.uint64)
    return ((u + ((u >> np.uint64(16)) & np.uint64(1)) + np.uint64(0x7FFF)) >> np.uint64(16)).astype(np.uint16)


def sample_rows(op, n, target_units):
    """Anchor rows [0, R) holding about target_units pairs (matrix: entries)."""
    per = n if op.startswith("pairmatrix") else max(n - 1, 1)
    return (0, int(min(n, max(1, target_units // per))))


def cpu_baseline(op, p, params, seconds):
    import oracle
    n = p.shape[0]
    u, dt = oracle_rate(op, p, params, sample_rows(op, n, 2e8 if not op.startswith("pairmatrix") else 2e7))
    rate = u / dt
    rows = sample_rows(op, n, rate * seconds)
    u, dt = oracle_rate(op, p, params, rows)
    return dict(value=u / dt / 1e9, unit="G pairs/s" if not op.startswith("pairmatrix") else "G entries/s",
                cores=oracle.num_threads(), kind="oracle",
                sample=f"anchor rows [{rows[0]},{rows[1]}) of the same N={n} input ({u:.3e} "
                       f"{'pairs' if not op.startswith('pairmatrix') else 'entries'}, {dt:.1f} s, fp64, OpenMP)")


def run_reference(args, wl):
    op, dist_, n, seed, params = WORKLOADS[wl]
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    p = gen.make(dist_, n, seed, params.get("d", 3))
    unit = "G pairs/s" if not op.startswith("pairmatrix") else "G entries/s"
    import oracle
    # each step: a bounded anchor-row sample, sized for ~120 s over the whole run
    per_step = max(2.0, 120.0 / max(1, args.steps + args.warmup))
    u0, dt0 = oracle_rate(op, p, params, sample_rows(op, n, 2e8 if not op.startswith("pairmatrix") else 2e7))
    rows = sample_rows(op, n, u0 / dt0 * per_step)
    for _ in range(args.warmup):
        oracle_rate(op, p, params, rows)
    tot_u, tot_t = 0, 0.0
    for _ in range(args.steps):
        u, dt = oracle_rate(op, p, params, rows)
        tot_u += u
        tot_t += dt
    v = tot_u / tot_t / 1e9
    metric = METRIC if op in ("sdh", "sdh_lattice") else f"{op} throughput ({unit})"   # as the tbs arm names it
    line = {"impl": "reference", "metric": metric, "value": v, "unit": unit, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": tot_t / args.steps * 1e3,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": wl, "n": n, "distribution": dist_, "seed": seed, **params},
            "cpu_baseline": {"value": v, "unit": unit, "cores": oracle.num_threads(), "kind": "oracle",
                             "sample": f"per step anchor rows [{rows[0]},{rows[1]}) of the N={n} input"},
            "e2e": {"value": v, "unit": unit, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------ GPU arm
def relaunch(args):
    """`--gpus N` without torchrun: run this script under torch.distributed.run with N local
    ranks (rendezvous on 127.0.0.1) and exit with its status."""
    import socket
    import subprocess
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    env = dict(os.environ)
    env.setdefault("NCCL_DEBUG", "INFO")
    env.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
    env.setdefault("NCCL_DEBUG_FILE", "/dev/stderr")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", f"--master-port={port}", os.path.abspath(__file__)] + sys.argv[1:]
    print(f"[bench] launching {args.gpus} ranks: {' '.join(cmd)}", file=sys.stderr, flush=True)
    sys.exit(subprocess.run(cmd, env=env).returncode)


def dry_run(args):
    """The launch path without GPU work: gloo group, world == --gpus, each rank's strip."""
    import torch
    import torch.distributed as dist

    import paper_conf_icpp_pitaksirianannt16_b200 as tbs
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    n = WORKLOADS[args.workload][2]
    if world > 1:
        dist.init_process_group("gloo")
    rows = list(tbs.rank_rows(n, world, rank))
    got = [None] * world
    if world > 1:
        dist.all_gather_object(got, (rank, os.getpid(), rows))
        dist.barrier()
        dist.destroy_process_group()
    else:
        got = [(rank, os.getpid(), rows)]
    if rank == 0:
        print(json.dumps({"dry_run": True, "n_gpus": world, "gpus_requested": args.gpus, "workload": args.workload,
                          "n": n, "combine": args.combine, "impl": args.impl,
                          "ranks": [{"rank": r, "pid": pid, "rows": rw} for r, pid, rw in got]}), flush=True)
    del torch


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--workload", default="sdh_uniform_1m", choices=sorted(WORKLOADS))
    ap.add_argument("--impl", default="tbs", choices=["tbs", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=12.0)
    ap.add_argument("--combine", default="nccl", choices=["nccl", "fused"],
                    help="N > 1, SDH / 2PCF: NCCL all_reduce (default) or the fused peer-memory flush")
    ap.add_argument("--dry-run", action="store_true", help="launch path only (gloo, no GPU work)")
    ap.add_argument("--graph", default="auto", choices=["auto", "on", "off"],
                    help="replay each step from a CUDA graph (auto: one GPU, n <= 64K, Type-I/II)")
    args = ap.parse_args()
    if "WORLD_SIZE" not in os.environ and args.gpus > 1:
        return relaunch(args)
    world_env = int(os.environ.get("WORLD_SIZE", "1"))
    assert world_env == args.gpus, f"WORLD_SIZE = {world_env} but --gpus {args.gpus}"
    if args.dry_run:
        return dry_run(args)
    assert args.warmup >= 3 or args.impl == "reference", "timing rules: >= 3 warm-up steps"
    wl = args.workload
    if args.impl == "reference":
        return run_reference(args, wl)

    import torch
    import torch.distributed as dist

    import paper_conf_icpp_pitaksirianannt16_b200 as tbs

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    pg = None
    if world > 1:
        for k, v in (("NCCL_DEBUG", "INFO"), ("NCCL_DEBUG_SUBSYS", "INIT"), ("NCCL_DEBUG_FILE", "/dev/stderr")):
            os.environ.setdefault(k, v)      # communicator ranks in the log, stdout kept for the JSON line
        dist.init_process_group("nccl", device_id=dev)
        pg = dist.group.WORLD

    op, dist_, n, seed, params = WORKLOADS[wl]
    p_host = gen.make(dist_, n, seed, params.get("d", 3))
    pts = torch.from_numpy(p_host).to(dev)
    if op == "pairmatrix_hd":
        pts = pts.to(torch.bfloat16)        # the API's feature type (input construction, untimed)
    st = torch.cuda.current_stream(dev)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    nb = params.get("nb", 1)
    w = float(np.float32(math.sqrt(3) / nb)) if op in ("sdh", "rdf") else params.get("w", 1.0)
    out = None
    if op in ("sdh", "sdh_lattice"):
        out = torch.empty(nb, dtype=torch.int64, device=dev)
    elif op == "rdf":
        out = torch.empty(nb, dtype=torch.float64, device=dev)
    elif op == "pcf":
        out = torch.empty(1, dtype=torch.int64, device=dev)
    elif op == "kde":
        out = torch.empty(1, dtype=torch.float64, device=dev)
    elif op == "knn":
        rows_pm = (n * rank // world, n * (rank + 1) // world)
        out = (torch.empty((rows_pm[1] - rows_pm[0], params["k"]), dtype=torch.int32, device=dev),
               torch.empty((rows_pm[1] - rows_pm[0], params["k"]), dtype=torch.float32, device=dev))
    else:
        rows_pm = (n * rank // world, n * (rank + 1) // world)
        out = torch.empty((rows_pm[1] - rows_pm[0], n), dtype=torch.float32, device=dev)

    # N > 1, Type-I/II: one NCCL all_reduce of the per-rank histogram / count (--combine nccl),
    # or the combine fused into the kernels' flush (every partial added into every rank's buffer
    # over NVLink peer memory, TBS_OUT_PEERS; --combine fused), falling back to NCCL if the peer
    # mapping cannot be set up (no native peer atomics, ...). config.combine records what ran.
    sink, combine = None, "none"
    if pg is not None and op in ("sdh", "sdh_lattice", "pcf"):
        combine = "nccl-allreduce"
        if args.combine == "fused":
            try:
                sink = tbs.PeerSink(nb if op != "pcf" else 1, pg, dev)
                combine = "fused-peer"
            except Exception as e:   # noqa: BLE001 — report and use the collective instead
                print(f"[bench] fused combine unavailable ({e}); using NCCL all_reduce", file=sys.stderr)
    elif pg is not None:
        combine = "nccl-allreduce" if op == "kde" else "none (row-sharded output)"

    def step(events=None):
        if op == "sdh":
            tbs.sdh(pts, w, nb, out=out, events=events, group=pg, sink=sink)
        elif op == "sdh_lattice":
            tbs.sdh(pts, w, nb, lattice=True, out=out, events=events, group=pg, sink=sink)
        elif op == "rdf":
            tbs.rdf(pts, w, nb, params["volume"], out=out, events=events, group=pg)
        elif op == "pcf":
            tbs.pcf(pts, params["r"], out=out, events=events, group=pg, sink=sink)
        elif op == "kde":
            tbs.kde(pts, params["gamma"], out=out, events=events, group=pg)
        elif op == "pairmatrix_hd":
            tbs.pairmatrix_hd(pts, params["gamma"], out=out, events=events, group=pg)
        elif op == "knn":
            tbs.knn(pts, params["k"], out=out, events=events, group=pg)
        else:
            tbs.pairmatrix(pts, params["gamma"], out=out, events=events, group=pg)

    kev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    for a, b in kev:            # materialise the cudaEvent_t handles passed through the C ABI
        a.record(st)
        b.record(st)
    for _ in range(args.warmup):
        flush.fill_(1)
        step()
    torch.cuda.synchronize(dev)
    # Launch-bound steps (small n, one GPU): capture one step (loader + pair kernel + flush) in a
    # CUDA graph and replay it, so the timed steps measure the device work, not the host's
    # per-launch latency. The kernels' own events are not captured: the step events time it.
    graph, graph_launches = None, 0
    if args.graph == "on" or (args.graph == "auto" and world == 1 and n <= 65536
                              and op in ("sdh", "sdh_lattice", "pcf", "kde")):
        try:
            side = torch.cuda.Stream(dev)
            side.wait_stream(st)
            with torch.cuda.stream(side):
                step()
            st.wait_stream(side)
            torch.cuda.synchronize(dev)
            graph = torch.cuda.CUDAGraph()
            lc = tbs.launch_count()
            with torch.cuda.graph(graph):
                step()
            graph_launches = tbs.launch_count() - lc
            graph.replay()
            torch.cuda.synchronize(dev)
        except Exception as e:   # noqa: BLE001 — report and time the plain launches
            print(f"[bench] CUDA graph capture failed ({e}); timing plain launches", file=sys.stderr)
            graph = None
    if pg is not None:
        dist.barrier()
    torch.cuda.synchronize(dev)
    clocks = Clocks(dev) if rank == 0 else None
    l0 = tbs.launch_count()
    t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    sev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    if clocks:
        clocks.mark(True)
    t0.record(st)
    for k in range(args.steps):
        flush.fill_(k & 0xFF)    # L2 flush between steps (256 MiB > 126 MB L2), outside the step events
        sev[k][0].record(st)
        if graph is not None:
            graph.replay()
        else:
            step(events=kev[k])
        sev[k][1].record(st)
    t1.record(st)
    torch.cuda.synchronize(dev)
    if clocks:
        clocks.mark(False)
    if pg is not None:
        dist.barrier()
    launches = tbs.launch_count() - l0 if graph is None else graph_launches * args.steps
    ck = clocks.stop() if clocks else None
    region_ms = t0.elapsed_time(t1)                          # whole bracket, L2 flushes included
    ms = sum(a.elapsed_time(b) for a, b in sev)               # the K steps themselves
    # the dominant kernel's time: its own events, or under a graph the whole step (conservative)
    kms = [a.elapsed_time(b) for a, b in (kev if graph is None else sev)]
    if pg is not None:
        tt = torch.tensor([ms, sum(kms) / len(kms), region_ms], dtype=torch.float64, device=dev)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        ms, kavg, region_ms = tt.tolist()
    else:
        kavg = sum(kms) / len(kms)

    is_matrix = op in ("pairmatrix", "pairmatrix_hd")
    units = units_of("pairmatrix" if is_matrix else "sdh", n) * (2 if op == "knn" else 1)  # kNN: ordered pairs
    value = units * args.steps / (ms * 1e-3) / 1e9
    unit = "G pairs/s" if not is_matrix else "G entries/s"
    pk = peaks()
    # dominant kernel (pair kernel / matrix kernel) on this rank: its share of the units
    if is_matrix:
        rows_pm = (n * rank // world, n * (rank + 1) // world)
        rank_units = (rows_pm[1] - rows_pm[0]) * n
        bytes_ = rank_units * 4.0
        achieved = bytes_ / (kavg * 1e-3)
        roof = {"bound": "hbm", "achieved": achieved / 1e9, "peak": pk["hbm"] / 1e9, "unit": "GB/s",
                "frac": achieved / pk["hbm"], "peak_source": pk["hbm_src"] + " (a read+write copy; this kernel only writes)",
                "frac_of_nominal": achieved / 7.7e12,   # HGX HBM3e 7.7 TB/s (B200_PROFILING.md), context
                "algorithmic_bytes_per_launch": bytes_}
        rp = os.path.join(ROOT, "profiles", "r02_peaks.json")
        if os.path.exists(rp):
            # this kernel only WRITES: the measured write-only ceiling (cudaMemset of 8 GiB,
            # tools/peaks.cu) is the tighter reference than the read+write copy bandwidth
            wpk = json.load(open(rp))["hbm_memset_GBps"] * 1e9
            roof["write_peak_GBps"] = wpk / 1e9
            roof["frac_of_write_peak"] = achieved / wpk
        if op == "pairmatrix_hd":
            # the Gram contraction: 2 d flops per entry on the bf16 tensor cores; the bound is
            # whichever of (output bytes / HBM, flops / tensor peak) takes longer
            flops = 2.0 * params["d"] * rank_units
            tfrac = flops / (kavg * 1e-3) / pk["bf16"]
            roof["tensor_view"] = {"achieved": flops / (kavg * 1e-3) / 1e12, "peak": pk["bf16"] / 1e12,
                                   "unit": "TFLOP/s", "frac": tfrac, "peak_source": pk["bf16_src"],
                                   "algorithmic_flops_per_launch": flops}
            if flops / pk["bf16"] > bytes_ / pk["hbm"]:
                roof = {"bound": "tensor", "achieved": flops / (kavg * 1e-3) / 1e12, "peak": pk["bf16"] / 1e12,
                        "unit": "TFLOP/s", "frac": tfrac, "peak_source": pk["bf16_src"],
                        "algorithmic_flops_per_launch": flops,
                        "hbm_view": {"achieved": achieved / 1e9, "peak": pk["hbm"] / 1e9, "unit": "GB/s",
                                     "frac": achieved / pk["hbm"]}}
    else:
        rb, re = tbs.rank_rows(n, world, rank)
        rank_units = (re - rb) * (2 * n - rb - re - 1) // 2
        if op == "knn":
            rb, re = n * rank // world, n * (rank + 1) // world
            rank_units = (re - rb) * (n - 1)
        pairs_s = rank_units / (kavg * 1e-3)
        if op == "knn":
            peak = pk["fp32"] / 6
            bound_note = "FP32 pipe: 6 lane-ops per ordered pair (3 sub + 3 mul/fma); compare + rare insert on ALU"
        elif op == "pcf":
            peak = pk["fp32"] / 6
            bound_note = "FP32 pipe: 6 lane-ops/pair (3 sub + 3 mul/fma)"
        elif op == "kde":
            peak = min(pk["fp32"] / 8, pk["mufu"])
            bound_note = "min(FP32 pipe / 8 lane-ops per pair (distance 6, scale, sum), MUFU / 1 ex2 per pair)"
        else:
            peak = min(pk["fp32"] / 6, pk["atoms"])
            bound_note = "min(FP32 pipe / 6 lane-ops per pair, shared-atomic lanes / 1 per pair)"
        roof = {"bound": "alu", "achieved": pairs_s / 1e9, "peak": peak / 1e9, "unit": "G pairs/s",
                "frac": pairs_s / peak, "peak_source": f"{bound_note}; 148 SMs x unit lanes/clk x "
                                                      f"{pk['f_max'] / 1e6:.0f} MHz (DESIGN.md §Roofline)",
                "frac_fp32": pairs_s * 6 / pk["fp32"]}
        if op in ("sdh", "sdh_lattice", "rdf"):
            roof["mufu_cap"] = pk["mufu"] / 1e9         # one MUFU.SQRT per pair: this design's ceiling
            roof["frac_of_mufu_cap"] = pairs_s / pk["mufu"]
            if nb + 32 > 768:
                # fewer than 32 lane-private replicas fit (DESIGN.md §7 a8): the increments hit
                # random banks of R shared copies; the measured ceiling of that access pattern
                # (tools/peaks.cu, profiles/r02_peaks.json) bounds this design: nb >= 8192 runs
                # R <= 2 copies in one 256-thread CTA per SM (atoms_random_16k_r2_1x256, C4's exact
                # layout), smaller nb more replicas (atoms_random_256, one copy: a lower bound)
                rp = os.path.join(ROOT, "profiles", "r02_peaks.json")
                if os.path.exists(rp):
                    key = "atoms_random_16k_r2_1x256" if nb >= 8192 else "atoms_random_256"
                    cap = json.load(open(rp))[key]["per_clk_per_sm"] * SMS * pk["f_max"]
                    roof["atoms_random_cap"] = cap / 1e9
                    roof["atoms_random_cap_source"] = f"profiles/r02_peaks.json {key}"
                    roof["frac_of_atoms_random_cap"] = pairs_s / cap
    roof["traffic"] = None
    prof = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(prof):
        try:
            roof["traffic"] = json.load(open(prof)).get(wl)
        except Exception:
            pass
    roof["kernel_ms_avg"] = kavg

    # e2e: host buffers through the public API, H2D of the points and D2H of the result each step
    e2e = None
    if op in ("sdh", "sdh_lattice", "pcf", "kde", "knn", "rdf"):
        ph = torch.from_numpy(p_host).pin_memory()
        if world == 1 and op != "sdh_lattice":     # the simple host-pointer entry points
            hh = np.zeros(nb if op == "sdh" else 1, np.uint64)
            kh = np.zeros(1, np.float64)
            gh = np.zeros(nb, np.float64)

            # the C-ABI host-buffer entry points (tbs_sdh / tbs_pcf / tbs_kde: the north star's
            # signatures) called directly, arguments marshalled once; status checked every call
            L, pptr = tbs.lib(), ph.numpy().ctypes.data
            ch = np.zeros(1, np.uint64)
            cw, cg, cr = ctypes.c_float(w), ctypes.c_float(params.get("gamma", 0.0)), ctypes.c_float(params.get("r", 0.0))

            def e2e_step():
                if op == "sdh":
                    rc = L.tbs_sdh(pptr, n, 3, cw, nb, hh.ctypes.data)
                elif op == "rdf":
                    rc = L.tbs_rdf(pptr, n, 3, cw, nb, ctypes.c_double(params["volume"]), gh.ctypes.data)
                elif op == "kde":
                    rc = L.tbs_kde(pptr, n, cg, kh.ctypes.data)
                elif op == "knn":
                    tbs.knn_host(ph.numpy(), params["k"])
                    rc = 0
                else:
                    rc = L.tbs_pcf(pptr, n, cr, ch.ctypes.data)
                if rc:
                    raise tbs.TbsError(f"e2e call: status {rc}: {tbs.last_error()}")
        else:
            res_h = torch.empty((out[1] if op == "knn" else out).shape, dtype=(out[1] if op == "knn" else out).dtype).pin_memory()

            def e2e_step():
                d = ph.to(dev, non_blocking=True)
                if op == "sdh":
                    r = tbs.sdh(d, w, nb, group=pg, sink=sink)
                elif op == "rdf":
                    r = tbs.rdf(d, w, nb, params["volume"], group=pg)
                elif op == "sdh_lattice":
                    r = tbs.sdh(d, w, nb, lattice=True, group=pg, sink=sink)
                elif op == "kde":
                    r = tbs.kde(d, params["gamma"], group=pg)
                elif op == "knn":
                    r = tbs.knn(d, params["k"], group=pg)[1]
                else:
                    r = tbs.pcf(d, params["r"], group=pg, sink=sink)
                res_h.copy_(r)
        for _ in range(2):
            e2e_step()
        torch.cuda.synchronize(dev)
        if pg is not None:
            dist.barrier()
        ke = max(2, args.steps // 2)
        tw = time.perf_counter()
        for _ in range(ke):
            e2e_step()
        torch.cuda.synchronize(dev)
        te = time.perf_counter() - tw
        if pg is not None:
            tt = torch.tensor([te], dtype=torch.float64, device=dev)
            dist.all_reduce(tt, op=dist.ReduceOp.MAX)
            te = tt.item()
        d2h = int(out[0].numel() * 8) if op == "knn" else int(out.numel() * 8)
        e2e = {"value": units * ke / te / 1e9, "unit": unit, "h2d_bytes_per_step": int(p_host.nbytes),
               "d2h_bytes_per_step": d2h}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline(op if op != "sdh_lattice" else "sdh_lattice", p_host, params, args.cpu_seconds)

    if rank == 0:
        cfg = {"workload": wl, "n": n, "distribution": dist_, "seed": seed, **params,
               "l2": "flushed between steps (256 MiB write between the per-step CUDA events; inputs 12 B/point < L2)",
               "timed_region_ms": region_ms,
               "parallelism": f"rows{world}" if world > 1 else "single",
               "step": "loader + pair kernel + flush" + (f" + combine ({combine})" if world > 1 else ""),
               "combine": combine, "cuda_graph": graph is not None}
        if op in ("sdh", "rdf"):
            cfg["bucket_width"] = w
        if op == "rdf":
            cfg["step"] += " + RDF normalisation kernel (an nb + 1-bucket SDH)"
        line = {"metric": METRIC if op in ("sdh", "sdh_lattice") else f"{op} throughput ({unit})",
                "value": value, "unit": unit, "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
                "ms_per_step": ms / args.steps, "higher_is_better": True, "scaling": "strong",
                "vs_baseline": None, "dtype": "f32", "data": "synthetic", "config": cfg,
                "roofline": roof, "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": int(launches),
                "clocks": ck}
        print(json.dumps(line), flush=True)
    if sink is not None:
        sink.close()
    if pg is not None:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()

#!/usr/bin/env python3
"""Benchmark: unordered DFS on B200 (BASELINE.json metric
"GTEPS & ms per full DFS (1 B200); batched-root DFS/sec at 1/2/4/8 GPUs").

One step = one full unordered DFS (reset + persistent traversal + finalize)
over the resident graph, from the step's root.  Roots follow the paper's methodology (64 sources,
average TEPS): the config's headline root followed by 63 seeded roots with degree > 0;
step s of rank r uses root (r + s*N) mod 64.  With N > 1 every rank holds a replica of the graph
and runs its own roots (weak scaling, no data-path collective).

The JSON line (rank 0) carries, besides the contract keys:
  roofline      dominant kernel (persistent traversal): algorithmic bytes per launch
                over its CUDA-event time, against MEASURED_PEAKS.json hbm_gbs; `step` adds
                SURVEY §8(d)'s B_min (with the 4n reset term) over the whole step
  cpu_baseline  the oracle (Alg 1) pinned to one host core, median over whole traversals
  e2e           the public C ABI with host buffers (dfs_run into pinned host memory)
  batch1024     C5 (configs[4]): 1,024 seeded roots on the road graph partitioned contiguously
                across the N ranks (strong scaling), DFS/s without and with the NCCL gather of
                the parent arrays to rank 0, roofline, all-core oracle baseline, I1-I6 checks
  rmat24        C3 (configs[2], N = 1): GTEPS, ms, roofline of the 128-wide kernel
--impl reference = the CPU oracle (Alg 1, oracle/) timed on the host cores, same workload.

`python bench.py --gpus N` without torchrun re-launches itself under torch.distributed.run
with N ranks (one per GPU, NCCL).

Usage: python bench.py [--gpus N] [--steps K] [--warmup W] [--config road24m] [--impl b200|reference]
"""
from __future__ import annotations

import argparse
import json
import os
import socket
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "GTEPS & ms per full DFS (1 B200); batched-root DFS/sec at 1/2/4/8 GPUs"
L2_BYTES = 126 * 1024 * 1024


def log(*a):
    print(*a, file=sys.stderr, flush=True)


def parse(argv=None):
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="road24m",
                    choices=["road24m", "grid256", "rmat24", "path100m", "caterpillar", "batch1024"])
    ap.add_argument("--batch-roots", type=int, default=1024)
    ap.add_argument("--concurrency", type=int, default=0,
                    help="batch: traversals in flight per GPU (0 = library auto)")
    ap.add_argument("--impl", default="b200", choices=["b200", "reference"])
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-validate", action="store_true")
    ap.add_argument("--no-batch", action="store_true", help="skip the batch1024 sub-record")
    ap.add_argument("--no-rmat", action="store_true", help="skip the rmat24 sub-record")
    ap.add_argument("--no-span", action="store_true", help="skip the span (eccentricity floor) record")
    ap.add_argument("--no-gather", action="store_true", help="batch: skip the with-gather pass")
    ap.add_argument("--cpu-seconds", type=float, default=12.0)
    ap.add_argument("--nroots", type=int, default=64)
    ap.add_argument("--set", action="append", default=[], metavar="KEY=VALUE",
                    help="dfs_options field for the timed runs (A/B experiments)")
    return ap.parse_args(argv)


def roots_for(g, root0, k):
    import graphgen
    rs = [int(root0)] + [int(x) for x in graphgen.random_roots(g, k - 1, seed=0x6A7)]
    return rs[:k]


def cpu_model():
    try:
        with open("/proc/cpuinfo") as f:
            for ln in f:
                if ln.startswith("model name"):
                    return ln.split(":", 1)[1].strip()
    except OSError:
        pass
    import platform
    return platform.processor() or "cpu"


def host_cores():
    try:
        return len(os.sched_getaffinity(0))
    except AttributeError:  # pragma: no cover
        return os.cpu_count() or 1


# ------------------------------------------------------------------------------ clocks
class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled every 200 ms during the timed region."""
    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception as e:  # pragma: no cover
            log("clock sampler unavailable:", e)
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unavailable"]}
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=2)
        except Exception:
            self.proc.kill()
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 7:
                continue
            try:
                sm.append(float(f[0])); mx.append(float(f[1]))
            except ValueError:
                continue
            for nm, v in zip(names, f[3:7]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "samples": len(sm), "reasons": sorted(reasons)}


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md)"


def traffic_from_profile(workload):
    """ncu dram__bytes_read.sum + dram__bytes_write.sum of one traversal-kernel launch
    (profiles/ncu_traffic.json, written from the committed `ncu --set full` captures)."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        v = d.get(workload)
        return v.get("bytes") if isinstance(v, dict) else v
    return None


def parse_sets(sets):
    opts = {}
    for kv in sets:
        k, _, v = kv.partition("=")
        opts[k] = int(v)
    return opts


# ------------------------------------------------------------------------------ oracle (CPU)
def cpu_oracle_pinned(g, roots, seconds, steps=None):
    """oracle.dfs (Alg 1) on ONE host core (sched_setaffinity), whole traversals, bounded by
    `seconds` (or exactly `steps` traversals); returns (GTEPS of the median traversal, median ms,
    count, core)."""
    import oracle
    deg = np.diff(g.row_ptr)
    old = os.sched_getaffinity(0)
    core = min(old)
    os.sched_setaffinity(0, {core})
    ms, gteps = [], []
    try:
        t_all = 0.0
        for q in range(10**9):
            r = roots[q % len(roots)]
            t0 = time.perf_counter()
            p = oracle.dfs(g.row_ptr, g.col_idx, r)
            dt = time.perf_counter() - t0
            t_all += dt
            ms.append(dt * 1e3)
            gteps.append(int(deg[p != -2].sum()) / dt / 1e9)
            if (steps is not None and len(ms) >= steps) or (steps is None and t_all >= seconds):
                break
    finally:
        os.sched_setaffinity(0, old)
    return float(np.median(gteps)), float(np.median(ms)), len(ms), core


def cpu_oracle_pool(g, roots, seconds):
    """C5 CPU baseline: a pool of threads over ALL host cores, one root per task (oracle.dfs
    releases the GIL in C); bounded by `seconds`.  Returns (DFS/s, completed, threads)."""
    import oracle
    nthreads = host_cores()
    lock = threading.Lock()
    state = {"next": 0, "done": 0}
    t0 = time.perf_counter()

    def worker():
        while True:
            with lock:
                if time.perf_counter() - t0 >= seconds:
                    return
                q = state["next"]
                state["next"] += 1
            oracle.dfs(g.row_ptr, g.col_idx, int(roots[q % len(roots)]))
            with lock:
                state["done"] += 1

    th = [threading.Thread(target=worker) for _ in range(nthreads)]
    for t in th:
        t.start()
    for t in th:
        t.join()
    el = time.perf_counter() - t0
    return state["done"] / el, state["done"], nthreads, el


# ------------------------------------------------------------------------------ launch
def free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def relaunch(a):
    """`--gpus N` without torchrun: re-execute this script under torch.distributed.run, one rank
    per GPU (the driver's own N > 1 launch goes straight to main())."""
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={a.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(free_port()),
           os.path.abspath(__file__), *sys.argv[1:]]
    log("relaunch:", " ".join(cmd))
    return subprocess.call(cmd)


def main():
    a = parse()
    if "WORLD_SIZE" not in os.environ and a.gpus > 1:
        sys.exit(relaunch(a))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if a.impl == "reference":
        return reference_arm(a, world, rank)

    import torch
    import torch.distributed as dist
    # one rank per GPU over NCCL.  DFS_BENCH_BACKEND=gloo (test aid only: exercises the N > 1 code
    # paths with several ranks sharing the GPUs of a smaller box; collectives on host tensors)
    backend = os.environ.get("DFS_BENCH_BACKEND", "nccl")
    gpu = local % max(1, torch.cuda.device_count()) if backend != "nccl" else local
    torch.cuda.set_device(gpu)
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", gpu))
        else:
            dist.init_process_group(backend)
    dev = torch.device("cuda", gpu)
    a.coll_dev = dev if backend == "nccl" else torch.device("cpu")
    a.gpu = gpu
    import graphgen

    if a.config == "batch1024":
        g = graphgen.road(4900, 4900)
        rec = {"metric": METRIC, "n_gpus": world}
        b = batch_leg(a, g, world, rank, local, dev)
        if rank == 0:
            rec.update({"value": b["dfs_per_s"], "unit": "DFS/s", "steps": b["roots"], "warmup": a.warmup,
                        "ms_per_step": b["ms_per_dfs"], "higher_is_better": True, "scaling": "strong",
                        "vs_baseline": None, "dtype": "int32", "data": "synthetic",
                        "config": {"workload": "batch1024", "n": g.n, "m": g.m},
                        "batch1024": b})
            print(json.dumps(rec), flush=True)
        if world > 1:
            dist.destroy_process_group()
        return

    t0 = time.time()
    g, root0, undirected, desc = graphgen.config_graph(a.config)
    log(f"[rank {rank}] graph {a.config}: n={g.n} m={g.m} built in {time.time() - t0:.1f}s")
    rec = single_root_leg(a, a.config, g, root0, undirected, desc, world, rank, local, headline=True)

    if not a.no_batch and a.config in ("road24m",):
        b = batch_leg(a, g, world, rank, local, dev)
        if rank == 0:
            rec["batch1024"] = b
    if rank == 0 and world == 1 and not a.no_rmat and a.config != "rmat24":
        del g
        t0 = time.time()
        gr, rr, und, desc_r = graphgen.config_graph("rmat24")
        log(f"[rank {rank}] graph rmat24: n={gr.n} m={gr.m} built in {time.time() - t0:.1f}s")
        sub = single_root_leg(a, "rmat24", gr, rr, und, desc_r, 1, 0, local, headline=False)
        rec["rmat24"] = sub
    if rank == 0:
        print(json.dumps(rec), flush=True)
    if world > 1:
        dist.destroy_process_group()


# ------------------------------------------------------------------------------ span
def bfs_eccentricity(row_ptr, col_idx, r):
    """Largest BFS distance from r (level-synchronous frontier BFS in numpy; not the oracle)."""
    rp = np.asarray(row_ptr, dtype=np.int64)
    col = np.asarray(col_idx)
    dist_ = np.full(len(rp) - 1, -1, np.int32)
    dist_[r] = 0
    f = np.array([r], dtype=np.int64)
    d = 0
    while True:
        s = rp[f]
        c = rp[f + 1] - s
        tot = int(c.sum())
        if tot == 0:
            break
        nb = col[np.repeat(s - (np.cumsum(c) - c), c) + np.arange(tot)]
        nb = np.unique(nb[dist_[nb] < 0])
        if nb.size == 0:
            break
        d += 1
        dist_[nb] = d
        f = nb.astype(np.int64)
    return d


def span_record(g, my_roots, step_ms, clk, k=2):
    """The latency floor of the first k timed roots ("span"): any traversal that
    builds a tree needs ecc(root) sequential claims, each at least one L2 hit (~250 cycles) plus
    one global atomic (~318 cycles) after its parent's claim (B300_MICROARCH L2/ATOMG latencies),
    at the SM clock sampled during the timed region."""
    mhz = (clk or {}).get("sm_mhz") or 1965.0
    per_level_us = 570.0 / mhz
    out = []
    for r in list(dict.fromkeys(my_roots))[:k]:
        ecc = bfs_eccentricity(g.row_ptr, g.col_idx, int(r))
        ms = [t for rr, t in zip(my_roots, step_ms) if rr == r]
        med = float(np.median(ms))
        floor = ecc * per_level_us / 1e3
        out.append({"root": int(r), "bfs_ecc": ecc, "ms_median": round(med, 4), "floor_ms": round(floor, 4),
                    "frac_of_floor": round(floor / med, 4)})
    return {"roots": out, "per_level_cycles": 570,
            "what": "latency floor = BFS eccentricity x (L2 hit + atomic) per level; no tree-building traversal "
                    "from that root can be faster; the DFS's own span is longer (scripts/span_sim.c)"}


# ------------------------------------------------------------------------------ single root
def single_root_leg(a, workload, g, root0, undirected, desc, world, rank, local, headline):
    """Single-root traversals on one GPU per rank (weak-scaled replicas for N > 1).  Returns the
    full JSON record (headline) or the sub-record (rmat24) on rank 0."""
    import torch
    import torch.distributed as dist

    import oracle
    from paper_conf_ppopp_niul0c26_b200 import Graph, Options
    from paper_conf_ppopp_niul0c26_b200 import dfs as dfsmod

    roots = roots_for(g, root0, a.nroots)
    deg = np.diff(g.row_ptr)
    G = Graph(g.row_ptr, g.col_idx)
    out = torch.empty(g.n, dtype=torch.int32, device="cuda")
    stream = torch.cuda.current_stream()
    ws_bytes = (g.n + 1) * 4 + g.m * 4 + g.n * 4
    flush_l2 = ws_bytes < 2 * L2_BYTES
    scratch = torch.empty(2 * L2_BYTES // 4, dtype=torch.int32, device="cuda") if flush_l2 else None
    opts = parse_sets(a.set)
    timed_opts = Options(**opts)

    steps = a.steps if headline else max(5, min(a.steps, 10))
    my_roots = [roots[(rank + s * world) % len(roots)] for s in range(steps)]
    # m_r / n_r per root are fixed (the reach set is unique): computed once, outside timing, from
    # a validated run; the first runs are also checked against the oracle (I1-I6 exact)
    m_r, n_r, valid = {}, {}, {}
    for q, r in enumerate(sorted(set(my_roots))):
        p = G.run(r, out=out, options=timed_opts)
        vis = (p != -2).cpu().numpy()
        m_r[r] = int(deg[vis].sum())
        n_r[r] = int(vis.sum())
        if not a.no_validate and q < 2:
            res = oracle.check_tree(g.row_ptr, g.col_idx, r, p.cpu().numpy(), i7=True, undirected=undirected)
            valid[r] = {k: getattr(res, k) for k in ("i1", "i2", "i3", "i4", "i5", "i6", "i7")}
            valid[r]["n_cross_I7"] = res.n_cross
            assert res.ok or res.failed() == ["i7"], (r, res)
    for s in range(max(3, a.warmup)):
        G.run(my_roots[s % len(my_roots)], out=out, options=timed_opts)
    torch.cuda.synchronize()

    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(steps)]
    trav_ms = []
    clocks = ClockSampler(getattr(a, "gpu", local)).start()
    launches0 = G.launch_count()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    for s in range(steps):
        if flush_l2:
            scratch.fill_(s)
        ev[s][0].record(stream)
        _, st = G.run(my_roots[s], out=out, options=timed_opts, stats=True)
        ev[s][1].record(stream)
        trav_ms.append(st.traversal_ms)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    launches = G.launch_count() - launches0
    clk = clocks.stop()
    step_ms = [e0.elapsed_time(e1) for e0, e1 in ev]
    my_time = sum(step_ms) / 1e3
    my_edges = sum(m_r[r] for r in my_roots)
    # roofline of the dominant kernel (persistent traversal, launched on `stream`; its duration
    # is the library's CUDA-event pair around the launch, dfs_stats.traversal_ms): algorithmic
    # bytes per launch = 12 B per reached vertex (uint32 row_ptr pair + parent write) + 8 B per
    # scanned edge (col_idx entry + one visited probe); the step-level figure adds
    # SURVEY §8(d)'s 4n reset term over the whole step time
    kbytes = sum(12.0 * n_r[r] + 8.0 * m_r[r] for r in my_roots)
    sbytes = kbytes + 4.0 * g.n * steps
    # SURVEY §8(d)'s B_sec: the same accesses at 32-byte sector granularity (random accesses)
    secbytes = sum(4.0 * g.n + 64.0 * n_r[r] + 32.0 * n_r[r] * (1.0 + 4.0 * (m_r[r] / max(1, n_r[r])) / 32.0)
                   + 32.0 * m_r[r] for r in my_roots)
    my_trav = sum(trav_ms) / 1e3

    from paper_conf_ppopp_niul0c26_b200 import batch
    (t_job, _), (edges,) = batch.reduce_max_sum([my_time, my_trav], [float(my_edges)], world,
                                                device=a.coll_dev)
    if rank != 0:
        G.close()
        return None

    peak, peak_src = measured_peaks()
    achieved = kbytes / my_trav / 1e9            # rank 0's own launches (per-GPU kernel figure)
    roof = {"bound": "hbm", "achieved": round(achieved, 3), "peak": peak, "unit": "GB/s",
            "frac": round(achieved / peak, 6), "traffic": traffic_from_profile(workload),
            "kernel": (f"b200dfs::dfs_walker_kernel<{st.walker_lanes}> (sub-warp walkers)" if st.walker_lanes != 32
                       else f"b200dfs::dfs_persistent_kernel ({st.window}-wide windows)"), "peak_source": peak_src,
            "bytes_per_launch_avg": round(kbytes / steps, 1),
            "launch_ms_avg": round(my_trav * 1e3 / steps, 4),
            "kernel_share_of_step": round(my_trav / my_time, 4),
            "step": {"bytes_B_min_avg": round(sbytes / steps, 1),
                     "achieved": round(sbytes / my_time / 1e9, 3),
                     "frac": round(sbytes / my_time / 1e9 / peak, 6),
                     "what": "SURVEY 8(d) B_min = 4n + 12 n_r + 8 m_r over the whole step (reset + traversal + finalize)"},
            "step_sector": {"bytes_B_sec_avg": round(secbytes / steps, 1),
                            "achieved": round(secbytes / my_time / 1e9, 3),
                            "frac": round(secbytes / my_time / 1e9 / peak, 6),
                            "what": "SURVEY 8(d) B_sec = 4n + 64 n_r + 32 n_r (1 + 4 d/32) + 32 m_r (32-byte sectors "
                                    "for random accesses) over the whole step"}}
    gteps = edges / t_job / 1e9
    ms_per_dfs = t_job * 1e3 / steps
    rec = {"metric": METRIC, "value": round(gteps, 6), "unit": "GTEPS", "n_gpus": world,
           "steps": steps, "warmup": a.warmup, "ms_per_step": round(ms_per_dfs, 4),
           "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "int32",
           "data": "synthetic",
           "config": {"workload": workload, "desc": desc, "n": g.n, "m": g.m, "roots": len(set(my_roots)),
                      "root_policy": "headline root + 63 seeded degree>0 roots, round robin (P:1523-1526)",
                      "l2": ("flushed between steps (2x L2 write)" if flush_l2 else
                             f"inputs larger than L2 ({ws_bytes / 1e6:.0f} MB CSR+parent)"),
                      "parallelism": f"replicas x{world}" if world > 1 else "single GPU",
                      "blocks": st.blocks, "warps_per_block": st.warps_per_block,
                      "options": opts or "library defaults"},
           "ms_per_dfs": round(ms_per_dfs, 4), "dfs_per_s": round(steps * world / t_job, 3),
           "ms_per_dfs_median": round(float(np.median(step_ms)), 4),
           "gpu_launches": int(launches), "clocks": clk, "roofline": roof, "validation": valid}
    if headline and not a.no_span and workload in ("road24m", "grid256", "rmat24"):   # (deep configs: 10^6+ BFS levels)
        rec["span"] = span_record(g, my_roots, step_ms, clk)
    if headline and not a.no_cpu_baseline and world == 1:
        v, ms, cnt, core = cpu_oracle_pinned(g, roots, a.cpu_seconds)
        rec["cpu_baseline"] = {"value": round(v, 6), "unit": "GTEPS", "cores": 1, "kind": "oracle",
                               "sample": f"{cnt} whole Alg-1 traversals of {workload} (round-robin roots), "
                                         f"median {ms:.1f} ms; pinned to host core {core} "
                                         f"(sched_setaffinity) of {host_cores()}; {cpu_model()}",
                               "statistic": "median GTEPS over traversals"}
    if headline and not a.no_e2e:
        rec["e2e"] = e2e_leg(a, g, my_roots, m_r, dfsmod, G)
    G.close()
    return rec


# ------------------------------------------------------------------------------ C5 batch
def batch_leg(a, g, world, rank, local, dev):
    """C5 (BASELINE.json configs[4]): `--batch-roots` seeded roots on the replicated road graph,
    partitioned contiguously across ranks (strong scaling).  Pass 1: traversals only
    (dfs_run_batch_ex, chunks of device-resident parent rows, K traversals in flight per GPU).
    Pass 2: the same with every chunk's parent rows gathered to rank 0 over NCCL (bounded
    sub-chunks into a reused rank-0 device buffer: the result sink).  Times are device events,
    max over ranks.  After timing, 4 rows of the last chunk per rank are checked against the
    oracle (I1-I6 exact); the all-core CPU baseline runs on rank 0 at N = 1."""
    import torch
    import torch.distributed as dist

    import graphgen
    import oracle
    from paper_conf_ppopp_niul0c26_b200 import Graph, Options
    from paper_conf_ppopp_niul0c26_b200 import batch

    roots = graphgen.random_roots(g, a.batch_roots, seed=0xC5)
    k = len(roots)
    lo, hi = batch.partition(k, world, rank)
    mine = [int(r) for r in roots[lo:hi]]
    G = Graph(g.row_ptr, g.col_idx)
    opts = parse_sets(a.set)
    if a.concurrency > 0:
        opts["concurrency"] = a.concurrency
    o = Options(**opts)
    cap = max(b - a_ for a_, b in (batch.partition(k, world, p) for p in range(world)))
    # rows per dfs_run_batch call: up to 512 (fewer call boundaries, each of which waits for the
    # slowest in-flight traversal), bounded by 40% of the free device memory; the same on every rank
    free_b, _ = torch.cuda.mem_get_info()
    rows_fit = max(8, int(0.4 * free_b // (g.n * 4)))
    if world > 1:
        (rows_fit_min,), _ = batch.reduce_max_sum([-float(rows_fit)], [], world, device=a.coll_dev)
        rows_fit = int(-rows_fit_min)
    rows = max(1, min(512, cap, rows_fit))
    out_rows = torch.empty((rows, g.n), dtype=torch.int32, device=dev)
    G.run_batch(mine[:min(rows, 8)], out=out_rows[:min(rows, 8)], options=o)      # warm-up
    torch.cuda.synchronize()
    sub = 8                                                   # rows per gather round
    sink = None
    if world > 1 and rank == 0 and not a.no_gather:
        sink = [torch.empty((sub, g.n), dtype=torch.int32, device=a.coll_dev) for _ in range(world)]

    lanes = []

    def one_pass(gather):
        counts = []
        launches0 = G.launch_count()
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        if gather and world > 1 and rows >= 2 * sub:
            # exchange overlapped with the traversals: chunks of `grows` rows alternate between
            # two halves of the row buffer; chunk c's rows go to rank 0 (async NCCL gathers on
            # the communicator's stream) while chunk c + 1 traverses into the other half, and a
            # half is reused only after its gathers completed
            grows = max(sub, (rows // 2) // sub * sub)
            halves = [out_rows[:grows], out_rows[grows:2 * grows]]
            pending = [[], []]
            for ci, c0 in enumerate(range(0, cap, grows)):
                buf = halves[ci % 2]
                for w, _ in pending[ci % 2]:
                    w.wait()
                pending[ci % 2] = []
                chunk = mine[c0:c0 + grows]
                if chunk:
                    _, st = G.run_batch(chunk, out=buf[:len(chunk)], options=o, stats=True)
                    counts.append(st.root_counts.copy())
                    lanes.append(st.walker_lanes)
                src_rows = buf if a.coll_dev.type == "cuda" else buf.cpu()
                pending[ci % 2] = batch.gather_chunk_to_rank0(src_rows, len(chunk), min(grows, cap - c0), sub,
                                                              sink, world, rank, async_op=True)
            for pw in pending:
                for w, _ in pw:
                    w.wait()
        else:
            for c0 in range(0, cap, rows):
                chunk = mine[c0:c0 + rows]
                if chunk:
                    _, st = G.run_batch(chunk, out=out_rows[:len(chunk)], options=o, stats=True)
                    counts.append(st.root_counts.copy())
                    lanes.append(st.walker_lanes)
                if gather and world > 1:
                    src_rows = out_rows if a.coll_dev.type == "cuda" else out_rows.cpu()
                    batch.gather_chunk_to_rank0(src_rows, len(chunk), min(rows, cap - c0), sub, sink, world, rank)
        e1.record()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1)
        launches = G.launch_count() - launches0
        (t_max,), _ = batch.reduce_max_sum([ms], [], world, device=a.coll_dev)
        return t_max, ms, np.concatenate(counts) if counts else np.zeros((0, 2)), launches

    clocks = ClockSampler(getattr(a, "gpu", local)).start()
    t_trav, my_ms, counts, launches = one_pass(False)
    t_gath = None
    if not a.no_gather and world > 1:
        t_gath, _, _, _ = one_pass(True)
    clk = clocks.stop()
    # algorithmic bytes of this rank's traversals (SURVEY 8(d) B_min per traversal)
    my_bytes = float(sum(4.0 * g.n + 12.0 * nv + 8.0 * mv for nv, mv in counts))
    my_edges = float(counts[:, 1].sum()) if len(counts) else 0.0
    # validation of rows produced by the timed run (the last chunk), outside timing
    vals = []
    if not a.no_validate and mine:
        last0 = ((len(mine) - 1) // rows) * rows
        for q in range(min(4, len(mine) - last0)):
            r = mine[last0 + q]
            res = oracle.check_tree(g.row_ptr, g.col_idx, r, out_rows[q].cpu().numpy(), i7=False, undirected=True)
            assert res.ok, (r, res)
            vals.append(int(res.ok))
    _, (tot_bytes, tot_edges, nval, nok) = batch.reduce_max_sum(
        [], [my_bytes, my_edges, float(len(vals)), float(sum(vals))], world, device=a.coll_dev)
    # e2e: the public C symbol dfs_run_batch with HOST buffers (roots in host memory, parent rows
    # into pinned host memory), wall clock with a device sync on both sides; a bounded sample of
    # E roots per rank (the full 1,024 x 96 MB of rows would not fit in host memory)
    e2e = None
    if not a.no_e2e:
        import ctypes
        from paper_conf_ppopp_niul0c26_b200 import dfs as dfsmod
        lib = dfsmod.load_library()
        E = min(64, len(mine))
        hroots = np.ascontiguousarray(np.array(mine[:E], dtype=np.int32))
        hout = torch.empty((max(E, 1), g.n), dtype=torch.int32).pin_memory()
        h = ctypes.c_void_p(G._h)
        assert lib.dfs_run_batch(h, hroots.ctypes.data, E, ctypes.c_void_p(hout.data_ptr())) == 0   # warm-up
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        rc = lib.dfs_run_batch(h, hroots.ctypes.data, E, ctypes.c_void_p(hout.data_ptr()))
        torch.cuda.synchronize()
        el = time.perf_counter() - t0
        assert rc == 0, rc
        del hout
        (el_max,), (roots_all,) = batch.reduce_max_sum([el], [float(E)], world, device=a.coll_dev)
        e2e = {"value": round(roots_all / el_max, 3), "unit": "DFS/s", "h2d_bytes_per_step": int(E * 4),
               "d2h_bytes_per_step": int(E * g.n * 4), "roots_per_rank": E,
               "what": f"dfs_run_batch(resident graph, {E} host roots, pinned host parents_out) per rank; "
                       "wall clock, max over ranks"}
    G.close()
    if rank != 0:
        return None
    peak, peak_src = measured_peaks()
    conc = opts.get("concurrency", 0) or "auto (8)"
    kl = lanes[0] if lanes else 32
    b = {"roots": k, "dfs_per_s": round(k / (t_trav * 1e-3), 3), "ms_per_dfs": round(t_trav / k, 4),
         "region_ms": round(t_trav, 3), "gteps": round(tot_edges / (t_trav * 1e-3) / 1e9, 4),
         "partition": f"contiguous slices of {k} seeded roots over {world} rank(s) (strong scaling)",
         "concurrency": conc, "rows_per_call": rows, "gpu_launches": int(launches), "clocks": clk,
         "roofline": {"bound": "hbm", "achieved": round(my_bytes / (my_ms * 1e-3) / 1e9, 3), "peak": peak,
                      "unit": "GB/s", "frac": round(my_bytes / (my_ms * 1e-3) / 1e9 / peak, 6),
                      "traffic": traffic_from_profile("batch"), "traffic_what": "ncu dram read+write of one "
                      "traversal-kernel launch of a K = 8 batch (profiles/r02/ncu/ncu_batch.md)",
                      "kernel": (f"b200dfs::dfs_walker_kernel<{kl}> (sub-warp walkers)" if kl != 32
                                 else "b200dfs::dfs_persistent_kernel"),
                      "peak_source": peak_src,
                      "what": "rank 0: SURVEY 8(d) B_min (4n + 12 n_r + 8 m_r) x its roots / its batch region time "
                              "(concurrent traversal kernels overlap, so the region is the kernel time)"},
         "validation": {"rows_checked": int(nval), "rows_ok_I1_I6": int(nok),
                        "what": "4 rows of the last timed chunk per rank, oracle.check_tree I1-I6 exact"}}
    if e2e is not None:
        b["e2e"] = e2e
    if world == 1:
        b["with_gather"] = {"dfs_per_s": b["dfs_per_s"], "region_ms": b["region_ms"], "bytes_to_rank0": 0,
                            "what": "N=1: the parent rows are already on rank 0 (no exchange step)"}
    elif t_gath is not None:
        b["with_gather"] = {"dfs_per_s": round(k / (t_gath * 1e-3), 3), "region_ms": round(t_gath, 3),
                            "bytes_to_rank0": int((k - (hi - lo)) * g.n * 4),
                            "what": f"each chunk's parent rows gathered to rank 0 (NCCL gather, {sub}-row rounds "
                                    "into a reused rank-0 device buffer), overlapped with the next chunk's "
                                    "traversals (double-buffered rows, async gathers)"}
    if world == 1 and not a.no_cpu_baseline:
        v, done, nth, el = cpu_oracle_pool(g, roots, a.cpu_seconds)
        b["cpu_baseline"] = {"value": round(v, 4), "unit": "DFS/s", "cores": nth, "kind": "oracle",
                             "sample": f"{done} whole Alg-1 traversals of the batch roots in {el:.1f} s, "
                                       f"a pool of {nth} threads (one root per task) on {cpu_model()}"}
    return b


def e2e_leg(a, g, my_roots, m_r, dfsmod, G):
    """Public C ABI with host buffers.

    e2e (headline): the graph is resident (like a model's weights); each step is one user call
    dfs_run(handle, root, parent_out) with parent_out in pinned host memory — the step's input
    (the root) goes host -> device and the result (n int32 parents) comes back device -> host
    inside the timed region.
    with_upload: additionally dfs_graph_create from the host CSR and dfs_graph_destroy per step.
    """
    import ctypes

    import torch
    lib = dfsmod.load_library()
    out = torch.empty(g.n, dtype=torch.int32).pin_memory()
    k = max(1, min(5, a.steps))
    h = ctypes.c_void_p(G._h)
    ts, edges = [], 0
    for s in range(k + 1):
        r = my_roots[s % len(my_roots)]
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        rc = lib.dfs_run(h, int(r), ctypes.c_void_p(out.data_ptr()))
        torch.cuda.synchronize()
        dt = time.perf_counter() - t0
        assert rc == 0, rc
        if s > 0:                      # first is warm-up
            ts.append(dt)
            edges += m_r[r]
    rec = {"value": round(edges / sum(ts) / 1e9, 6), "unit": "GTEPS", "h2d_bytes_per_step": 4,
           "d2h_bytes_per_step": int(g.n * 4), "steps": k, "ms_per_step": round(sum(ts) / k * 1e3, 3),
           "what": "dfs_run(resident graph, root, pinned host parent_out); wall clock, cuda sync both sides"}
    # with the CSR upload in every step
    rp = np.ascontiguousarray(g.row_ptr)
    ci = np.ascontiguousarray(g.col_idx)
    ku = max(1, min(2, a.steps))
    tu, eu = [], 0
    for s in range(ku + 1):
        r = my_roots[s % len(my_roots)]
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        hu = lib.dfs_graph_create(rp.ctypes.data, ci.ctypes.data, g.n, g.m)
        assert hu, lib.dfs_last_error()
        rc = lib.dfs_run(hu, int(r), ctypes.c_void_p(out.data_ptr()))
        lib.dfs_graph_destroy(hu)
        torch.cuda.synchronize()
        dt = time.perf_counter() - t0
        assert rc == 0, rc
        if s > 0:
            tu.append(dt)
            eu += m_r[r]
    rec["with_upload"] = {"value": round(eu / sum(tu) / 1e9, 6), "unit": "GTEPS",
                          "h2d_bytes_per_step": int((g.n + 1) * 8 + g.m * 4),
                          "d2h_bytes_per_step": int(g.n * 4), "steps": ku,
                          "ms_per_step": round(sum(tu) / ku * 1e3, 3),
                          "what": "dfs_graph_create(host CSR) + dfs_run(pinned host out) + dfs_graph_destroy"}
    return rec


def reference_arm(a, world, rank):
    """The CPU oracle (Alg 1, oracle/dfs_oracle.c) as the reference implementation: rank 0 only
    (the other ranks exit without work), one pinned host core, each step one whole traversal."""
    import graphgen
    if world > 1 and rank != 0:
        return
    g, root0, undirected, desc = graphgen.config_graph(a.config if a.config != "batch1024" else "road24m")
    roots = roots_for(g, root0, a.nroots)
    if a.warmup > 0:
        cpu_oracle_pinned(g, roots, 0, steps=min(a.warmup, 3))
    v, ms, cnt, core = cpu_oracle_pinned(g, roots, 0, steps=a.steps)
    rec = {"metric": METRIC, "value": round(v, 6), "unit": "GTEPS", "impl": "reference",
           "n_gpus": world, "steps": a.steps, "warmup": a.warmup, "ms_per_step": round(ms, 3),
           "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "int32",
           "data": "synthetic",
           "config": {"workload": a.config, "desc": desc, "n": g.n, "m": g.m},
           "cpu_baseline": {"value": round(v, 6), "unit": "GTEPS", "cores": 1, "kind": "oracle",
                            "sample": f"{cnt} whole Alg-1 traversals of {a.config}, median; pinned to host "
                                      f"core {core} of {host_cores()}; {cpu_model()}"},
           "e2e": {"value": round(v, 6), "unit": "GTEPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(rec), flush=True)


if __name__ == "__main__":
    main()

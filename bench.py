#!/usr/bin/env python3
"""Benchmark: unordered DFS on B200 (BASELINE.json metric
"GTEPS & ms per full DFS (1 B200); batched-root DFS/sec at 1/2/4/8 GPUs").

One step = one full unordered DFS (reset + persistent traversal + finalize)
over the resident graph, from the step's root.  Roots follow the paper's methodology (64 sources,
average TEPS): the config's headline root followed by 63 seeded roots with degree > 0;
step s of rank r uses root (r + s*N) mod 64.  With N > 1 every rank holds a replica of the graph
and runs its own roots (weak scaling, no data-path collective); the single exchange step is an
NCCL all_gather of the per-root summaries at the end.

value  = whole-job GTEPS = sum over ranks and steps of m_r (out-degree sum of the visited set,
         reading S6) / max over ranks of the sum of per-step device times (CUDA events).
e2e    = same metric through the public C ABI with HOST buffers: dfs_graph_create (host CSR ->
         device) + dfs_run (host parent_out) + dfs_graph_destroy per step.
--impl reference = the CPU oracle (Alg 1, oracle/) timed on the host cores, same workload.

Usage: python bench.py [--gpus N] [--steps K] [--warmup W] [--config road24m] [--impl b200|reference]
"""
from __future__ import annotations

import argparse
import json
import os
import platform
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


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="road24m",
                    choices=["road24m", "grid256", "rmat24", "path100m", "caterpillar", "batch1024"])
    ap.add_argument("--batch-roots", type=int, default=1024)
    ap.add_argument("--concurrency", type=int, default=0,
                    help="batch1024: traversals in flight per GPU (0 = auto)")
    ap.add_argument("--impl", default="b200", choices=["b200", "reference"])
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-validate", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=12.0)
    ap.add_argument("--nroots", type=int, default=64)
    return ap.parse_args()


def roots_for(g, root0, k):
    import graphgen
    rs = [int(root0)] + [int(x) for x in graphgen.random_roots(g, k - 1, seed=0x6A7)]
    return rs[:k]


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
        return float(d["hbm_gbs"]), "measured"
    return 6650.0, "fallback (B200_PROFILING.md)"


def traffic_from_profile(workload):
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return d.get(workload)
    return None


# ------------------------------------------------------------------------------ oracle (CPU)
def cpu_oracle(g, roots, seconds, steps=None):
    """Time oracle.dfs (Alg 1, one host core) over whole traversals; bounded by `seconds`."""
    import oracle
    tot_t, tot_e, done = 0.0, 0, 0
    for q in range(10**9):
        r = roots[q % len(roots)]
        t0 = time.perf_counter()
        p = oracle.dfs(g.row_ptr, g.col_idx, r)
        dt = time.perf_counter() - t0
        vis = p != -2
        tot_t += dt
        tot_e += int(np.diff(g.row_ptr)[vis].sum())
        done += 1
        if (steps is not None and done >= steps) or (steps is None and tot_t >= seconds):
            break
    return tot_e / tot_t / 1e9, tot_t / done * 1e3, done


# ------------------------------------------------------------------------------ main
def main():
    a = parse()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    import graphgen

    if a.impl == "reference":
        return reference_arm(a, world, rank)
    if a.config == "batch1024":
        return batch_arm(a, world, rank, local)

    import torch
    import torch.distributed as dist
    from paper_conf_ppopp_niul0c26_b200 import Graph, Options
    from paper_conf_ppopp_niul0c26_b200 import dfs as dfsmod

    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))

    t0 = time.time()
    g, root0, undirected, desc = graphgen.config_graph(a.config)
    log(f"[rank {rank}] graph {a.config}: n={g.n} m={g.m} built in {time.time() - t0:.1f}s")
    roots = roots_for(g, root0, a.nroots)
    deg = np.diff(g.row_ptr)

    G = Graph(g.row_ptr, g.col_idx)
    out = torch.empty(g.n, dtype=torch.int32, device="cuda")
    stream = torch.cuda.current_stream()
    ws_bytes = (g.n + 1) * 4 + g.m * 4 + g.n * 4
    flush_l2 = ws_bytes < 2 * L2_BYTES
    scratch = torch.empty(2 * L2_BYTES // 4, dtype=torch.int32, device="cuda") if flush_l2 else None

    my_roots = [roots[(rank + s * world) % len(roots)] for s in range(a.steps)]
    # m_r per root is fixed (the reach set is unique): computed once, outside timing, from a
    # validated run; the first run of each root is also checked against the oracle (I1-I6)
    m_r, valid = {}, {}
    import oracle
    for q, r in enumerate(sorted(set(my_roots))):
        p = G.run(r, out=out)
        vis = (p != -2).cpu().numpy()
        m_r[r] = int(deg[vis].sum())
        if not a.no_validate and q < 2:
            res = oracle.check_tree(g.row_ptr, g.col_idx, r, p.cpu().numpy(), i7=True, undirected=undirected)
            valid[r] = {k: getattr(res, k) for k in ("i1", "i2", "i3", "i4", "i5", "i6", "i7")}
            valid[r]["n_cross_I7"] = res.n_cross
            assert res.ok or res.failed() == ["i7"], (r, res)
    for s in range(a.warmup):
        G.run(my_roots[s % len(my_roots)], out=out)
    torch.cuda.synchronize()

    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(a.steps)]
    opt_stats = Options()
    trav_ms = []
    clocks = ClockSampler(local)
    clocks.start()
    launches0 = G.launch_count()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    for s in range(a.steps):
        if flush_l2:
            scratch.fill_(s)
        ev[s][0].record(stream)
        _, st = G.run(my_roots[s], out=out, options=opt_stats, stats=True)
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

    # exchange step: per-root summaries gathered over NCCL (roots, m_r, ms)
    summ = torch.tensor([[float(r), float(m_r[r]), float(t)] for r, t in zip(my_roots, step_ms)],
                        dtype=torch.float64, device="cuda")
    if world > 1:
        allsum = torch.empty((world * a.steps, 3), dtype=torch.float64, device="cuda")
        dist.all_gather_into_tensor(allsum, summ)
        tmax = torch.tensor([my_time], dtype=torch.float64, device="cuda")
        dist.all_reduce(tmax, op=dist.ReduceOp.MAX)
        t_job = float(tmax.item())
        edges = float(allsum[:, 1].sum().item())
    else:
        t_job = my_time
        edges = float(my_edges)
    if rank != 0:
        if world > 1:
            dist.destroy_process_group()
        return

    gteps = edges / t_job / 1e9
    ms_per_dfs = t_job * 1e3 / a.steps
    # roofline of the dominant kernel (persistent traversal): algorithmic bytes per launch =
    # 12 B per reached vertex (uint32 row_ptr pair + parent write) + 8 B per scanned edge
    # (col_idx + one visited probe)  (DESIGN.md §"Roofline")
    byte_sum, trav_sum = 0.0, 0.0
    peak, peak_src = measured_peaks()
    # n_r per root (visited count)
    n_r = {}
    for r in set(my_roots):
        p = G.run(r, out=out)
        n_r[r] = int((p != -2).sum().item())
    for r, tm in zip(my_roots, trav_ms):
        byte_sum += 12.0 * n_r[r] + 8.0 * m_r[r]
        trav_sum += tm / 1e3
    achieved = byte_sum / trav_sum / 1e9
    roof = {"bound": "hbm", "achieved": round(achieved, 3), "peak": peak, "unit": "GB/s",
            "frac": round(achieved / peak, 6), "traffic": traffic_from_profile(a.config),
            "kernel": "b200dfs::dfs_persistent_kernel<256>", "peak_source": peak_src,
            "kernel_share_of_step": round(trav_sum / t_job, 4),
            "bytes_per_launch_avg": round(byte_sum / len(my_roots), 1)}

    rec = {"metric": METRIC, "value": round(gteps, 6), "unit": "GTEPS", "n_gpus": world,
           "steps": a.steps, "warmup": a.warmup, "ms_per_step": round(ms_per_dfs, 4),
           "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "int32",
           "data": "synthetic",
           "config": {"workload": a.config, "desc": desc, "n": g.n, "m": g.m, "roots": len(set(my_roots)),
                      "root_policy": "headline root + 63 seeded degree>0 roots, round robin (P:1523-1526)",
                      "l2": ("flushed between steps (2x L2 write)" if flush_l2 else
                             f"inputs larger than L2 ({ws_bytes / 1e6:.0f} MB CSR+parent)"),
                      "parallelism": f"replicas x{world}" if world > 1 else "single GPU",
                      "blocks": st.blocks, "warps_per_block": st.warps_per_block},
           "ms_per_dfs": round(ms_per_dfs, 4), "dfs_per_s": round(a.steps * world / t_job, 3),
           "ms_per_dfs_median": round(float(np.median(step_ms)), 4),
           "gpu_launches": int(launches), "clocks": clk, "roofline": roof, "validation": valid}

    if not a.no_cpu_baseline and world == 1:
        v, ms, cnt = cpu_oracle(g, roots, a.cpu_seconds)
        rec["cpu_baseline"] = {"value": round(v, 6), "unit": "GTEPS", "cores": 1, "kind": "oracle",
                               "sample": f"{cnt} full Alg-1 traversals of {a.config} (round-robin roots), "
                                         f"{ms:.1f} ms each, 1 host thread ({platform.processor() or 'cpu'}, "
                                         f"{os.cpu_count()} host cores)"}
    if not a.no_e2e:
        rec["e2e"] = e2e_leg(a, g, my_roots, m_r, dfsmod, G)
    print(json.dumps(rec), flush=True)
    G.close()
    if world > 1:
        dist.destroy_process_group()


def batch_arm(a, world, rank, local):
    """C5 (BASELINE.json configs[4]): 1,024 seeded roots on the replicated road graph, partitioned
    contiguously across ranks (strong scaling); one NCCL all_gather of per-root summaries."""
    import torch
    import torch.distributed as dist

    import graphgen
    from paper_conf_ppopp_niul0c26_b200 import Graph
    from paper_conf_ppopp_niul0c26_b200 import batch

    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    dev = torch.device("cuda", local)
    t0 = time.time()
    g = graphgen.road(4900, 4900)
    roots = graphgen.random_roots(g, a.batch_roots, seed=0xC5)
    log(f"[rank {rank}] batch graph n={g.n} m={g.m} built in {time.time() - t0:.1f}s; {len(roots)} roots")
    G = Graph(g.row_ptr, g.col_idx)
    lo, hi = batch.partition(len(roots), world, rank)
    conc = a.concurrency if a.concurrency > 0 else 8          # library auto (DESIGN §8 sweep)
    # chunks of 4 waves of `conc` traversals (device-resident parent rows, 96 MB each)
    out_rows = torch.empty((max(1, min(4 * conc, hi - lo)), g.n), dtype=torch.int32, device=dev)
    for s_ in range(a.warmup):                       # warm-up traversals (untimed)
        G.run(int(roots[(lo + s_) % len(roots)]), out=out_rows[0])
    launches0 = G.launch_count()
    clocks = ClockSampler(local)
    clocks.start()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    res = batch.run_batch_chunked(G, out_rows, roots, world=world, rank=rank, device=dev, concurrency=conc)
    e1.record()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clk = clocks.stop()
    region_ms = e0.elapsed_time(e1)
    if world > 1:
        t = torch.tensor([region_ms], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        region_ms = float(t.item())
    launches = G.launch_count() - launches0
    if rank == 0:
        k = len(roots)
        rec = {"metric": METRIC, "value": round(res.gteps(), 6), "unit": "GTEPS", "n_gpus": world,
               "steps": k, "warmup": a.warmup, "ms_per_step": round(res.max_ms / max(1, hi - lo), 4),
               "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "int32",
               "data": "synthetic",
               "config": {"workload": "batch1024", "desc": "C5: road-maze 4900x4900, 1024 seeded roots "
                          "partitioned contiguously across ranks, NCCL all_gather of per-root summaries",
                          "n": g.n, "m": g.m, "roots": k, "parallelism": f"replicas x{world}",
                          "l2": f"inputs larger than L2 ({((g.n + 1) * 4 + g.m * 8 + g.n * 4) / 1e6:.0f} MB)"},
               "dfs_per_s": round(res.dfs_per_s(), 3),
               "dfs_per_s_region": round(k / (region_ms * 1e-3), 3),
               "region_ms": round(region_ms, 3), "gpu_launches": int(launches), "clocks": clk,
               "exchange": "all_gather_into_tensor of (k x 5) float64 summaries",
               "concurrency": conc}
        print(json.dumps(rec), flush=True)
    G.close()
    if world > 1:
        dist.destroy_process_group()


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
    """The CPU oracle (Alg 1, oracle/dfs_oracle.c) as the reference implementation."""
    import graphgen
    if world > 1 and rank != 0:
        return
    g, root0, undirected, desc = graphgen.config_graph(a.config)
    roots = roots_for(g, root0, a.nroots)
    cpu_oracle(g, roots, 0, steps=a.warmup) if a.warmup > 0 else None
    v, ms, cnt = cpu_oracle(g, roots, 0, steps=a.steps)
    rec = {"metric": METRIC, "value": round(v, 6), "unit": "GTEPS", "impl": "reference",
           "n_gpus": world, "steps": a.steps, "warmup": a.warmup, "ms_per_step": round(ms, 3),
           "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "int32",
           "data": "synthetic",
           "config": {"workload": a.config, "desc": desc, "n": g.n, "m": g.m},
           "cpu_baseline": {"value": round(v, 6), "unit": "GTEPS", "cores": 1, "kind": "oracle",
                            "sample": f"{cnt} full Alg-1 traversals of {a.config}, 1 host thread"},
           "e2e": {"value": round(v, 6), "unit": "GTEPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(rec), flush=True)


if __name__ == "__main__":
    main()

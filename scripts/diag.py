#!/usr/bin/env python3
"""Diagnostics sweep: traversal time, GTEPS and scheduler counters under option variants.

python scripts/diag.py --graph road:4900 --roots 3 --variants default,w16,nointer ...
Graphs: road:W  grid:W  rmat:S  path:N  cat:S  (see graphgen).  Prints one JSON line per run.
"""
import argparse
import json
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import graphgen  # noqa: E402

VARIANTS = {
    "default": {},
    "w16": dict(warps_per_block=16),
    "w8": dict(warps_per_block=8),
    "hot16": dict(hot_cutoff=16),
    "hot8": dict(hot_cutoff=8),
    "cold32": dict(cold_cutoff=32),
    "cold16": dict(cold_cutoff=16),
    "h8c16": dict(hot_cutoff=8, cold_cutoff=16),
    "random": dict(victim_policy=0),
    "nointer": dict(inter_steal=False),
    "nointra": dict(intra_steal=False),
    "b74": dict(blocks=74),
    "b1": dict(blocks=1),
    "det": dict(deterministic=True),
    "paper": dict(spill=False, inter_any=False),
    "paper_h8c16": dict(spill=False, inter_any=False, hot_cutoff=8, cold_cutoff=16),
    "nospill": dict(spill=False),
    "leader": dict(inter_any=False),
    "h8c8": dict(hot_cutoff=8, cold_cutoff=8),
    "h16c16": dict(hot_cutoff=16, cold_cutoff=16),
    "h16c32": dict(hot_cutoff=16, cold_cutoff=32),
    "h8c32": dict(hot_cutoff=8, cold_cutoff=32),
    "h4c8": dict(hot_cutoff=4, cold_cutoff=8),
    "h8c8i128": dict(hot_cutoff=8, cold_cutoff=8, spill_idle=128),
    "h8c8i8": dict(hot_cutoff=8, cold_cutoff=8, spill_idle=8),
    "h8c8w16": dict(hot_cutoff=8, cold_cutoff=8, warps_per_block=16),
    "h4c4": dict(hot_cutoff=4, cold_cutoff=4),
    "h4c4b256": dict(hot_cutoff=4, cold_cutoff=4, backoff_max_ns=256),
    "h4c4b8k": dict(hot_cutoff=4, cold_cutoff=4, backoff_max_ns=8192),
    "h4c8b256": dict(hot_cutoff=4, cold_cutoff=8, backoff_max_ns=256),
    "h4c4w16": dict(hot_cutoff=4, cold_cutoff=4, warps_per_block=16),
    "h4c4w24": dict(hot_cutoff=4, cold_cutoff=4, warps_per_block=24),
    "h4c4leader": dict(hot_cutoff=4, cold_cutoff=4, inter_any=False),
    "h4c4nospill": dict(hot_cutoff=4, cold_cutoff=4, spill=False),
    "h2c2": dict(hot_cutoff=2, cold_cutoff=2),
    "h2c4": dict(hot_cutoff=2, cold_cutoff=4),
    "h4c2": dict(hot_cutoff=4, cold_cutoff=2),
    "h2c2w16": dict(hot_cutoff=2, cold_cutoff=2, warps_per_block=16),
    "h2c2i1": dict(hot_cutoff=2, cold_cutoff=2, spill_idle=1),
    "h6c2": dict(hot_cutoff=6, cold_cutoff=2),
    "w32": dict(window=32),
    "w128": dict(window=128),
    "h2c2w32": dict(hot_cutoff=2, cold_cutoff=2, window=32),
    "h2c2w128": dict(hot_cutoff=2, cold_cutoff=2, window=128),
    "h4c4w32": dict(hot_cutoff=4, cold_cutoff=4, window=32),
    "h4c4w128": dict(hot_cutoff=4, cold_cutoff=4, window=128),
    "det32": dict(deterministic=True, window=32),
    "det128": dict(deterministic=True, window=128),
    "det_nospec": dict(deterministic=True, window=32, speculate=False),
    "det_pb1": dict(deterministic=True, window=32, pub_batch=1),
    "det_pb1_nospec": dict(deterministic=True, window=32, pub_batch=1, speculate=False),
    "h2c2pb1": dict(hot_cutoff=2, cold_cutoff=2, pub_batch=1),
    "h2c2pb2": dict(hot_cutoff=2, cold_cutoff=2, pub_batch=2),
    "h2c2pb4": dict(hot_cutoff=2, cold_cutoff=2, pub_batch=4),
    "h2c2pb16": dict(hot_cutoff=2, cold_cutoff=2, pub_batch=16),
    "h2c2nospec": dict(hot_cutoff=2, cold_cutoff=2, speculate=False),
    "h4c4pb4": dict(hot_cutoff=4, cold_cutoff=4, pub_batch=4),
    "A": dict(hot_cutoff=2, cold_cutoff=2, pub_batch=1),
    "A16": dict(hot_cutoff=2, cold_cutoff=2, pub_batch=1, warps_per_block=16),
    "A24": dict(hot_cutoff=2, cold_cutoff=2, pub_batch=1, warps_per_block=24),
    "A8": dict(hot_cutoff=2, cold_cutoff=2, pub_batch=1, warps_per_block=8),
    "B16": dict(hot_cutoff=4, cold_cutoff=4, pub_batch=1, warps_per_block=16),
    "A16nospec": dict(hot_cutoff=2, cold_cutoff=2, pub_batch=1, warps_per_block=16, speculate=False),
    "A16b8k": dict(hot_cutoff=2, cold_cutoff=2, pub_batch=1, warps_per_block=16, backoff_max_ns=8192),
    "det16": dict(deterministic=True),
    "paperdef": dict(hot_cutoff=32, cold_cutoff=64, spill=False, inter_any=False, pub_batch=1, speculate=False),
    "spec1": dict(speculate=1),
    "spec0": dict(speculate=0),
    "nohalf": dict(steal_half=False),
    "h1c1": dict(hot_cutoff=1, cold_cutoff=1),
    "h1c2": dict(hot_cutoff=1, cold_cutoff=2),
    "h4c4": dict(hot_cutoff=4, cold_cutoff=4),
    "h1c1nohalf": dict(hot_cutoff=1, cold_cutoff=1, steal_half=False),
    "nospill": dict(spill=False),
    "b37": dict(blocks=37),
    "b16": dict(blocks=16),
    "h4c4": dict(hot_cutoff=4, cold_cutoff=4),
    "pb8": dict(pub_batch=8),
    "w0": dict(collect_stats=2),
    "w0nospill": dict(collect_stats=2, spill=False),
    "w0det": dict(collect_stats=2, deterministic=True),
    "bmin256": dict(backoff_min_ns=256),
    "bmin1k": dict(backoff_min_ns=1024, backoff_max_ns=4096),
    "bmax512": dict(backoff_max_ns=512),
    "bmax8k": dict(backoff_max_ns=8192),
    "early": dict(speculate=6),
    "specpop": dict(speculate=10),
    "noleaf": dict(leaf_skip=False),
    "bulk": dict(leaf_skip=2),
    "bulkw16": dict(leaf_skip=2, warps_per_block=16),
    "pb4": dict(pub_batch=4),
    "pb16": dict(pub_batch=16),
    "spill128": dict(spill_idle=128),
    "spill1k": dict(spill_idle=1024),
    "nointra": dict(intra_steal=False),
    "detnoleaf": dict(deterministic=True, leaf_skip=False),
    "specboth": dict(speculate=14),
    "specpop128": dict(speculate=9, window=128),
    "pf2": dict(prefetch_lines=2),
    "pf4": dict(prefetch_lines=4),
    "pf8": dict(prefetch_lines=8),
    "detpf4": dict(deterministic=True, prefetch_lines=4),
    "early128": dict(speculate=5, window=128),
    "w0early": dict(collect_stats=2, speculate=6),
    "w0detearly": dict(collect_stats=2, deterministic=True, speculate=6),
    "cl2": dict(cluster=2),
    "cl4": dict(cluster=4),
    "cl8": dict(cluster=8),
    "cl2stats": dict(cluster=2, collect_stats=True),
    "cl4nospill": dict(cluster=4, spill=False),
    "cl1": dict(cluster=1),
    "noearly": dict(speculate=2 | 8),
    "st1": dict(steal_tries=1),
    "bulk_copy": dict(bulk_copy=True),
    "bulk_copy_v1": dict(bulk_copy=True, ring_cap=2),
    "v1": dict(ring_cap=2),
    "l2p32": dict(l2_persist_mb=32),
    "l2off": dict(l2_persist_mb=-1),
    "h2c1": dict(hot_cutoff=2, cold_cutoff=1),
    "w8": dict(warps_per_block=8),
    "b32": dict(blocks=32),
    "b74": dict(blocks=74),
    "h1c4": dict(hot_cutoff=1, cold_cutoff=4),
    "si64": dict(spill_idle=64),
    "si256": dict(spill_idle=256),
    "si8": dict(spill_idle=8),
    "pb2": dict(pub_batch=2),
    "bmin64": dict(backoff_min_ns=64),
    "bmax1k": dict(backoff_max_ns=1024),
    "bmax4k": dict(backoff_max_ns=4096),
    "l2p64": dict(l2_persist_mb=64),
    "spec128": dict(speculate=1 | 4 | 8),
    "l2p96": dict(l2_persist_mb=96),
    "w0nointra": dict(collect_stats=2, intra_steal=False),
    "sp8": dict(spill_period=8),
    "sp16": dict(spill_period=16),
    "sp64": dict(spill_period=64),
    "detbulk": dict(deterministic=True, bulk_copy=True),
    "early2st8": dict(speculate=2 | 4 | 8, steal_tries=8),
    "st2": dict(steal_tries=2),
    "st4": dict(steal_tries=4),
    "st8": dict(steal_tries=8),
    "st4stats": dict(steal_tries=4, collect_stats=True),
    "early2": dict(speculate=2 | 4 | 8),
    "detearly": dict(deterministic=True, speculate=2 | 4 | 8),
    "cl2late": dict(cluster=2, cluster_late=True),
    "cl2late_stats": dict(cluster=2, cluster_late=True, collect_stats=True),
}


def graph(spec):
    kind, _, arg = spec.partition(":")
    if kind == "road":
        w = int(arg)
        return graphgen.road(w, w)
    if kind == "grid":
        w = int(arg)
        return graphgen.grid(w, w)
    if kind == "rmat":
        return graphgen.rmat(int(arg), 16)
    if kind == "path":
        n = int(float(arg))
        return graphgen.path_chords(n, n // 100)
    if kind == "cat":
        k = int(arg)
        return graphgen.caterpillar(1 << k if k <= 30 else k, 94)     # cat:20 = spine 2^20 (C4b)
    raise ValueError(spec)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--graph", default="road:4900")
    ap.add_argument("--roots", type=int, default=3)
    ap.add_argument("--reps", type=int, default=2)
    ap.add_argument("--variants", default="default")
    ap.add_argument("--timeline", type=int, default=0, help="timeline sample period in us (0 = off)")
    ap.add_argument("--nostats", action="store_true", help="time the production (non-STATS) kernel")
    a = ap.parse_args()
    import torch
    from paper_conf_ppopp_niul0c26_b200 import Graph, Options
    t0 = time.time()
    g = graph(a.graph)
    print(f"# {a.graph}: n={g.n} m={g.m} gen {time.time() - t0:.1f}s", file=sys.stderr, flush=True)
    roots = [0] + list(graphgen.random_roots(g, a.roots - 1, seed=7))
    deg = np.diff(g.row_ptr)
    G = Graph(g.row_ptr, g.col_idx)
    out = torch.empty(g.n, dtype=torch.int32, device="cuda")
    G.run(0, out=out)
    TL = 8192
    if a.timeline:
        G.timeline(TL, a.timeline * 1000)
    for vn in a.variants.split(","):
        kw = dict(VARIANTS[vn])
        kw.setdefault("collect_stats", not a.nostats)
        o = Options(**kw)
        for r in roots:
            best = None
            for _ in range(a.reps):
                _, st = G.run(int(r), out=out, options=o, stats=True)
                if best is None or st.traversal_ms < best.traversal_ms:
                    best = st
            st = best
            warps = st.blocks * st.warps_per_block
            util = 1.0 - st.idle_ns / max(1.0, warps * st.traversal_ms * 1e6)
            rec = dict(graph=a.graph, variant=vn, root=int(r), ms=round(st.traversal_ms, 3),
                       cyc_total=[st.cyc_window, st.cyc_probe, st.cyc_claim, st.cyc_tail, st.cyc_outside],
                       total_ms=round(st.kernel_ms, 3), gteps=round(st.m_visited / st.traversal_ms / 1e6, 4),
                       n_visited=st.n_visited, util=round(util, 4), claims=st.claims,
                       failed=st.failed_claims, windows=st.windows, flushes=st.flushes,
                       refills=st.refills, intra=st.intra_steals, inter=st.inter_steals, cl=getattr(st, "cluster_steals", 0), blocks=st.blocks,
                       pops=getattr(st, "pops", 0), dead_pops=getattr(st, "dead_pops", 0),
                       attempts=st.steal_attempts, scans=st.inter_scans, spills=st.spills, chunks=st.chunks_allocated,
                       us_per_claim_per_warp=round(st.traversal_ms * 1e3 * warps * util / max(1, st.claims), 3),
                       windows_per_claim=round(st.windows / max(1, st.claims), 3),
                       cyc_per_window=[round(x / max(1, st.windows), 1) for x in
                                       (st.cyc_window, st.cyc_probe, st.cyc_claim, st.cyc_tail, st.cyc_outside)])
            if a.timeline:
                G.run(int(r), out=out, options=o)      # sampled run
                tl, prog, wprog = G.timeline(TL, a.timeline * 1000, fetch=True)
                k = int(np.nonzero(tl >= 0)[0].max()) + 1 if np.any(tl >= 0) else 0
                tl = tl[:k]
                prog = prog[:k]
                wprog = wprog[:k]
                if k >= 20:
                    rec["claims_by_5pct"] = [int(c[c > 0].max()) if np.any(c > 0) else 0 for c in np.array_split(prog, 20)]
                    if np.any(wprog > 0):      # collect_stats runs: windows scanned so far
                        rec["windows_by_5pct"] = [int(c[c > 0].max()) if np.any(c > 0) else 0
                                                  for c in np.array_split(wprog, 20)]
                valid = tl[tl >= 0]
                dec = [int(np.mean(c[c >= 0])) if np.any(c >= 0) else -1 for c in np.array_split(tl, 20)] if k >= 20 else []
                rec["timeline_us"] = a.timeline
                rec["busy_mean"] = round(float(valid.mean()), 1) if valid.size else None
                rec["busy_by_5pct"] = dec
            print(json.dumps(rec), flush=True)
    G.close()


if __name__ == "__main__":
    main()

"""Command-line driver: unordered DFS on a Matrix Market graph or a named synthetic config.

    python -m paper_conf_ppopp_niul0c26_b200.cli --mtx graph.mtx --roots 64 --csv perf.csv
    python -m paper_conf_ppopp_niul0c26_b200.cli --config road24m --roots 8
    python -m paper_conf_ppopp_niul0c26_b200.cli --config road24m --roots 256 --batch   # DFS/s

Mirrors the paper's measurement methodology: a set of source vertices (here: the
given ones, or `--roots` seeded vertices with out-degree > 0), one traversal per source, and the
average of traversed edges / runtime (MTEPS).  Writes one CSV row per source (the artifact's
per-graph perf CSV, is the model).  `--batch` runs all sources as one
`dfs_run_batch` (K traversals in flight, BASELINE configs[4]) and reports DFS/s.  Every traversal
runs in libdfs.so.
"""
from __future__ import annotations

import argparse
import csv
import json
import sys
import time


def main(argv=None) -> int:
    ap = argparse.ArgumentParser(prog="paper_conf_ppopp_niul0c26_b200.cli")
    src = ap.add_mutually_exclusive_group(required=True)
    src.add_argument("--mtx", help="Matrix Market coordinate file (SuiteSparse format)")
    src.add_argument("--config", help="named synthetic config (graphgen.CONFIGS)")
    ap.add_argument("--symmetric", action="store_true", help="store both directions of every entry")
    ap.add_argument("--roots", type=int, default=64, help="number of seeded source vertices")
    ap.add_argument("--root", type=int, action="append", help="explicit source vertex (repeatable)")
    ap.add_argument("--seed", type=int, default=0x6A7)
    ap.add_argument("--csv", help="write per-source results here")
    ap.add_argument("--save-parents", metavar="NPY",
                    help="also save the (sources x n) int32 parent arrays (numpy .npy) for checking")
    ap.add_argument("--batch", action="store_true",
                    help="one dfs_run_batch over all sources (concurrent traversals); reports DFS/s")
    ap.add_argument("--set", action="append", default=[], metavar="KEY=VALUE",
                    help="dfs_options field, e.g. --set hot_cutoff=32 --set cold_cutoff=64")
    a = ap.parse_args(argv)

    import graphgen
    import torch

    from . import Graph, Options
    t0 = time.time()
    if a.mtx:
        g = graphgen.read_mtx(a.mtx, symmetric=a.symmetric)
        name = a.mtx
    else:
        g, _, _, _ = graphgen.config_graph(a.config)
        name = a.config
    load_s = time.time() - t0
    roots = [int(r) for r in (a.root or graphgen.random_roots(g, a.roots, seed=a.seed))]
    opts = {}
    for kv in a.set:
        k, _, v = kv.partition("=")
        opts[k] = int(v)
    options = Options(**opts) if opts else None
    G = Graph(g.row_ptr, g.col_idx)
    out = torch.empty(g.n, dtype=torch.int32, device="cuda")
    G.run(roots[0], out=out, options=options)                 # warm-up
    rows = []
    saved = None
    if a.save_parents:
        import numpy as np
        saved = np.empty((len(roots), g.n), dtype=np.int32)
    if a.batch:
        bout = torch.empty((len(roots), g.n), dtype=torch.int32, device="cuda")
        G.run_batch(roots[:2], out=bout[:2], options=options)  # warm-up (scratch slots)
        bout, st = G.run_batch(roots, out=bout, options=options, stats=True)
        if saved is not None:
            saved[:] = bout.cpu().numpy()
        G.close()
        if saved is not None:
            np.save(a.save_parents, saved)
        per = [dict(root=r, n_visited=int(st.root_counts[q, 0]), m_visited=int(st.root_counts[q, 1]))
               for q, r in enumerate(roots)]
        if a.csv:
            with open(a.csv, "w", newline="") as f:
                w = csv.DictWriter(f, fieldnames=list(per[0]))
                w.writeheader()
                w.writerows(per)
        tot_e = sum(r["m_visited"] for r in per)
        print(json.dumps(dict(graph=name, n=g.n, m=g.m, sources=len(per), load_s=round(load_s, 2), batch=True,
                              kernel=("walkers x%d lanes" % st.walker_lanes) if st.walker_lanes != 32 else "warp",
                              ms=round(st.kernel_ms, 3), dfs_per_s=round(len(per) / st.kernel_ms * 1e3, 2),
                              aggregate_mteps=round(tot_e / st.kernel_ms / 1e3, 2))))
        return 0
    for q, r in enumerate(roots):
        _, st = G.run(r, out=out, options=options, stats=True)
        if saved is not None:
            saved[q] = out.cpu().numpy()
        rows.append(dict(root=r, n_visited=st.n_visited, m_visited=st.m_visited,
                         ms=round(st.kernel_ms, 4), mteps=round(st.m_visited / st.kernel_ms / 1e3, 2)))
    G.close()
    if saved is not None:
        np.save(a.save_parents, saved)
    if a.csv:
        with open(a.csv, "w", newline="") as f:
            w = csv.DictWriter(f, fieldnames=list(rows[0]))
            w.writeheader()
            w.writerows(rows)
    tot_e = sum(r["m_visited"] for r in rows)
    tot_ms = sum(r["ms"] for r in rows)
    summary = dict(graph=name, n=g.n, m=g.m, sources=len(rows), load_s=round(load_s, 2),
                   avg_mteps=round(sum(r["mteps"] for r in rows) / len(rows), 2),
                   aggregate_mteps=round(tot_e / tot_ms / 1e3, 2), avg_ms=round(tot_ms / len(rows), 4))
    print(json.dumps(summary))
    return 0


if __name__ == "__main__":
    sys.exit(main())

#!/usr/bin/env python3
"""A/B of two (or more) builds of libdfs.so inside one process on one GPU box.

Box-to-box variation between gpurun boxes is several percent, so kernel changes are decided by
alternating the builds on the same graph in the same process:

    python scripts/ab_libs.py --libs build_a/libdfs.so build_b/libdfs.so --config road24m \
        --reps 5 --steps 8 [--set key=value ...] [--out results.jsonl]

Each rep runs `steps` traversals per build (roots round robin over the bench's 64-root list) and
records the mean device time of the step (dfs_stats.kernel_ms) and of the traversal kernel
(traversal_ms); the builds alternate within every rep.  Prints one JSON line per build with the
median over reps.  Every build's first tree per root is checked with the oracle (I1-I6).
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--libs", nargs="+", required=True)
    ap.add_argument("--config", default="road24m")
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--steps", type=int, default=8)
    ap.add_argument("--nroots", type=int, default=16)
    ap.add_argument("--set", action="append", default=[], help="dfs_options KEY=VALUE (all builds)")
    ap.add_argument("--variant", action="append", default=[],
                    help="comma-separated dfs_options KEY=VALUE list; every build x variant is timed")
    ap.add_argument("--batch", type=int, default=0, help="time dfs_run_batch of this many roots instead")
    ap.add_argument("--validate", type=int, default=1)
    ap.add_argument("--out")
    a = ap.parse_args()

    import torch

    import graphgen
    import oracle
    from paper_conf_ppopp_niul0c26_b200 import Graph, Options
    from paper_conf_ppopp_niul0c26_b200 import dfs as dfsmod

    t0 = time.time()
    g, root0, undirected, _ = graphgen.config_graph(a.config)
    print(f"graph {a.config} n={g.n} m={g.m} in {time.time() - t0:.1f}s", file=sys.stderr, flush=True)
    roots = [int(root0)] + [int(x) for x in graphgen.random_roots(g, a.nroots - 1, seed=0x6A7)]
    opts = {}
    for kv in a.set:
        k, _, v = kv.partition("=")
        opts[k] = int(v)
    variants = []
    for v in (a.variant or [""]):
        d = dict(opts)
        for kv in filter(None, v.split(",")):
            k, _, x = kv.partition("=")
            d[k] = int(x)
        variants.append((v, Options(**d) if d else None))
    libs = [dfsmod.load_library(os.path.abspath(p)) for p in a.libs]
    Gs0 = [Graph(g.row_ptr, g.col_idx, lib=lib) for lib in libs]
    # one timed arm per (build, variant); arms of one build share its graph handle
    arms = [(Gs0[li], f"{p}" + (f" [{vn}]" if vn else ""), vo) for li, p in enumerate(a.libs) for vn, vo in variants]
    Gs = [x[0] for x in arms]
    names = [x[1] for x in arms]
    opts_of = [x[2] for x in arms]
    out = torch.empty(g.n, dtype=torch.int32, device="cuda")
    bout = torch.empty((a.batch, g.n), dtype=torch.int32, device="cuda") if a.batch else None
    broots = graphgen.random_roots(g, a.batch, seed=0xC5) if a.batch else None
    deg = np.diff(g.row_ptr)
    for G, p, o in zip(Gs, names, opts_of):
        for r in roots[:a.validate]:
            par = G.run(r, out=out, options=o).cpu().numpy()
            res = oracle.check_tree(g.row_ptr, g.col_idx, r, par, undirected=undirected)
            assert res.ok, (p, r, res)
        G.run(roots[0], out=out, options=o)
        if a.batch:                                  # scratch slots of the batch: allocated untimed
            G.run_batch(broots, out=bout, options=o)
    res = {p: {"step_ms": [], "trav_ms": [], "gteps": []} for p in names}
    s = 0
    for rep in range(a.reps):
        order = list(range(len(Gs))) if rep % 2 == 0 else list(reversed(range(len(Gs))))
        for i in order:
            G, p, o = Gs[i], names[i], opts_of[i]
            if a.batch:
                torch.cuda.synchronize()
                _, st = G.run_batch(broots, out=bout, options=o, stats=True)
                res[p]["step_ms"].append(st.kernel_ms / a.batch)
                res[p]["trav_ms"].append(st.kernel_ms / a.batch)
                res[p]["gteps"].append(st.m_visited / st.kernel_ms / 1e6)
                continue
            km, tm, ed = 0.0, 0.0, 0
            for q in range(a.steps):
                r = roots[(s + q) % len(roots)]
                _, st = G.run(r, out=out, options=o, stats=True)
                km += st.kernel_ms
                tm += st.traversal_ms
                ed += st.m_visited
            res[p]["step_ms"].append(km / a.steps)
            res[p]["trav_ms"].append(tm / a.steps)
            res[p]["gteps"].append(ed / km / 1e6)
        s += a.steps
    lines = []
    for p in names:
        d = res[p]
        rec = {"lib": p, "config": a.config, "set": opts, "batch": a.batch,
               "step_ms_median": round(float(np.median(d["step_ms"])), 4),
               "trav_ms_median": round(float(np.median(d["trav_ms"])), 4),
               "gteps_median": round(float(np.median(d["gteps"])), 4),
               "step_ms_reps": [round(x, 4) for x in d["step_ms"]]}
        lines.append(json.dumps(rec))
        print(lines[-1], flush=True)
    if a.out:
        with open(a.out, "a") as f:
            f.write("\n".join(lines) + "\n")
    for G in Gs0:
        G.close()


if __name__ == "__main__":
    main()

#!/usr/bin/env python3
"""Vertex-order experiment: the same graph under different vertex numberings (each adjacency
list keeps its entry order, so Alg 1's tree is the same up to renaming), timed on the GPU.

    python scripts/reorder_ab.py --config road24m --orders orig dfs0 rcm bfs0 --roots 8 --reps 3

A road traversal's step is a chain of dependent loads into fresh territory (row_ptr -> col_idx ->
probe -> claim); the numbering decides how often that territory shares cache lines with the last
vertex visited.  Prints one JSON line per order (median traversal ms over the roots).
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


def relabel(row_ptr, col_idx, order):
    """New vertex k = old vertex order[k]; lists keep their entry order."""
    rp = np.asarray(row_ptr, dtype=np.int64)
    col = np.asarray(col_idx, dtype=np.int64)
    n = len(rp) - 1
    perm = np.empty(n, dtype=np.int64)
    perm[order] = np.arange(n, dtype=np.int64)
    deg = np.diff(rp)[order]
    nrp = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(deg, out=nrp[1:])
    starts = rp[order]
    idx = np.repeat(starts - nrp[:-1], deg) + np.arange(int(nrp[-1]), dtype=np.int64)
    ncol = perm[col[idx]].astype(np.int32)
    return nrp, ncol, perm


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="road24m")
    ap.add_argument("--orders", nargs="+", default=["orig", "dfs0", "rcm", "bfs0"])
    ap.add_argument("--roots", type=int, default=8)
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--set", action="append", default=[])
    ap.add_argument("--lib")
    ap.add_argument("--validate", type=int, default=1)
    a = ap.parse_args()
    import scipy.sparse as sp
    import scipy.sparse.csgraph as cg
    import torch

    import graphgen
    import oracle
    from paper_conf_ppopp_niul0c26_b200 import Graph, Options
    from paper_conf_ppopp_niul0c26_b200 import dfs as dfsmod

    g, root0, undirected, _ = graphgen.config_graph(a.config)
    roots = [int(root0)] + [int(x) for x in graphgen.random_roots(g, 63, seed=0x6A7)][: a.roots - 1]
    n = g.n
    A = sp.csr_matrix((np.ones(g.m, dtype=np.int8), np.asarray(g.col_idx), np.asarray(g.row_ptr)), shape=(n, n))
    opts = {k: int(v) for k, _, v in (kv.partition("=") for kv in a.set)}
    o = Options(**opts) if opts else None
    lib = dfsmod.load_library(os.path.abspath(a.lib)) if a.lib else None
    for name in a.orders:
        t0 = time.time()
        if name == "orig":
            rp, col, perm = np.asarray(g.row_ptr), np.asarray(g.col_idx), np.arange(n)
        else:
            if name == "dfs0":
                order = cg.depth_first_order(A, 0, directed=True, return_predecessors=False)
            elif name == "bfs0":
                order = cg.breadth_first_order(A, 0, directed=True, return_predecessors=False)
            elif name == "rcm":
                order = cg.reverse_cuthill_mckee(A, symmetric_mode=True)
            else:
                raise SystemExit(f"unknown order {name}")
            if len(order) < n:                      # unreached vertices keep their relative order
                seen = np.zeros(n, dtype=bool)
                seen[order] = True
                order = np.concatenate([order, np.nonzero(~seen)[0]])
            rp, col, perm = relabel(g.row_ptr, g.col_idx, np.asarray(order, dtype=np.int64))
        t_ord = time.time() - t0
        kw = {"lib": lib} if lib is not None else {}
        G = Graph(rp, col, **kw)
        out = torch.empty(n, dtype=torch.int32, device="cuda")
        rr = [int(perm[r]) for r in roots]
        if a.validate:
            p = G.run(rr[0], out=out, options=o).cpu().numpy()
            res = oracle.check_tree(rp, col, rr[0], p, undirected=undirected)
            assert res.ok, (name, res)
        for r in rr[:2]:
            G.run(r, out=out, options=o)
        ms = {r: [] for r in rr}
        for _ in range(a.reps):
            for r in rr:
                _, st = G.run(r, out=out, options=o, stats=True)
                ms[r].append(st.traversal_ms)
        med = [float(np.median(v)) for v in ms.values()]
        print(json.dumps({"config": a.config, "order": name, "order_s": round(t_ord, 2), "set": opts,
                          "trav_ms_median": round(float(np.median(med)), 4), "trav_ms_mean": round(float(np.mean(med)), 4),
                          "per_root_ms": [round(x, 3) for x in med]}), flush=True)
        G.close()
        del G


if __name__ == "__main__":
    main()

#!/usr/bin/env python3
"""Run one configuration for ncu: warm-up traversal(s), then the traversal to capture.

    ncu --set full -k regex:<kernel> --launch-skip <warm-up launches> -c 1 -o out \
        python scripts/ncu_run.py --config road24m [--set walker_lanes=8 ...] [--batch K]
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="road24m")
    ap.add_argument("--set", action="append", default=[])
    ap.add_argument("--warmup", type=int, default=1)
    ap.add_argument("--runs", type=int, default=1)
    ap.add_argument("--batch", type=int, default=0)
    a = ap.parse_args()
    import torch

    import graphgen
    from paper_conf_ppopp_niul0c26_b200 import Graph, Options
    g, root, _, _ = graphgen.config_graph(a.config)
    opts = {}
    for kv in a.set:
        k, _, v = kv.partition("=")
        opts[k] = int(v)
    o = Options(**opts) if opts else None
    G = Graph(g.row_ptr, g.col_idx)
    if a.batch:
        roots = graphgen.random_roots(g, a.batch, seed=0xC5)
        out = torch.empty((a.batch, g.n), dtype=torch.int32, device="cuda")
        for _ in range(a.warmup + a.runs):
            G.run_batch(roots, out=out, options=o)
    else:
        out = torch.empty(g.n, dtype=torch.int32, device="cuda")
        for _ in range(a.warmup + a.runs):
            G.run(root, out=out, options=o)
    torch.cuda.synchronize()
    print("done", g.n, g.m, flush=True)


if __name__ == "__main__":
    main()

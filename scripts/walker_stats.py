#!/usr/bin/env python3
"""STATS counters of one traversal per walker width on a bench config (diagnostic):
    python scripts/walker_stats.py --config road24m --lanes 4 1 --blocks 18
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="road24m")
ap.add_argument("--lanes", type=int, nargs="+", default=[4, 1])
ap.add_argument("--blocks", type=int, default=18)
ap.add_argument("--roots", type=int, default=3)
ap.add_argument("--set", action="append", default=[])
a = ap.parse_args()
import torch  # noqa: E402

import graphgen  # noqa: E402
from paper_conf_ppopp_niul0c26_b200 import Graph, Options  # noqa: E402

g, root0, _, _ = graphgen.config_graph(a.config)
roots = [int(x) for x in graphgen.random_roots(g, a.roots, seed=0xC5)]
extra = {k: int(v) for k, _, v in (kv.partition("=") for kv in a.set)}
out = torch.empty(g.n, dtype=torch.int32, device="cuda")
with Graph(g.row_ptr, g.col_idx) as G:
    for lanes in a.lanes:
        for r in roots:
            o = Options(walker_lanes=lanes, blocks=a.blocks, collect_stats=True, **extra)
            G.run(r, out=out, options=o)
            _, st = G.run(r, out=out, options=o, stats=True)
            d = {k: getattr(st, k) for k in ("traversal_ms", "blocks", "warps_per_block", "claims", "failed_claims",
                                             "flushes", "refills", "intra_steals", "inter_steals", "steal_attempts",
                                             "windows", "pops", "donations", "spills", "chunks_allocated")}
            print(json.dumps({"lanes": lanes, "root": r, **d}), flush=True)

#!/usr/bin/env python3
"""Repeat small walker-kernel runs under option combinations and report which fail I1-I6
(debugging aid for dfs_walker.cuh; prints one line per combination)."""
import itertools
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import graphgen  # noqa: E402
import oracle  # noqa: E402
import torch  # noqa: E402
from paper_conf_ppopp_niul0c26_b200 import Graph, Options  # noqa: E402

g = graphgen.road(300, 200, seed=7)
reps = int(sys.argv[1]) if len(sys.argv) > 1 else 6
G = Graph(g.row_ptr, g.col_idx)
out = torch.empty(g.n, dtype=torch.int32, device="cuda")
for lanes, inter, donate, spill, sp in itertools.product([16, 8, 4], [0, 1], [0, 1], [0, 1], [1, 1024]):
    fails = []
    for rep in range(reps):
        r = [31337, 0, 777, 45000][rep % 4]
        out.fill_(-7)                        # poison: a claimed vertex without a parent write shows as -7
        o = Options(walker_lanes=lanes, inter_steal=inter, donate=donate, spill=spill, steal_period=sp,
                    collect_stats=True)
        p, st = G.run(r, out=out, options=o, stats=True)
        par = p.cpu().numpy()
        res = oracle.check_tree(g.row_ptr, g.col_idx, r, par, undirected=True)
        if not res.ok:
            fails.append(dict(root=r, failed=res.failed(), n_vis=res.n_visited, poison=int((par == -7).sum()),
                              claims=st.claims, donations=st.donations, intra=st.intra_steals,
                              flushes=st.flushes, refills=st.refills, spills=st.spills))
    print(f"lanes={lanes} inter={inter} donate={donate} spill={spill} steal_period={sp}: "
          f"{len(fails)}/{reps} fail {fails[:2]}", flush=True)

#!/usr/bin/env python3
"""Where dfs_graph_create's time goes (diagnostic): wall time of create from pageable and pinned
host CSR and from device CSR, the first run (scratch allocation) and a second run, destroy."""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import graphgen  # noqa: E402
from paper_conf_ppopp_niul0c26_b200 import Graph  # noqa: E402

g, root, _, _ = graphgen.config_graph(sys.argv[1] if len(sys.argv) > 1 else "road24m")
out = torch.empty(g.n, dtype=torch.int32, device="cuda")
srcs = {"pageable": (g.row_ptr, g.col_idx),
        "pinned": (torch.from_numpy(np.asarray(g.row_ptr)).pin_memory(), torch.from_numpy(np.asarray(g.col_idx)).pin_memory()),
        "device": (torch.from_numpy(np.asarray(g.row_ptr)).cuda(), torch.from_numpy(np.asarray(g.col_idx)).cuda())}
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 2
only = sys.argv[3].split(",") if len(sys.argv) > 3 else list(srcs)
for rep in range(reps):
    for name, (rp, ci) in srcs.items():
        if name not in only:
            continue
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        G = Graph(rp, ci)
        torch.cuda.synchronize()
        t1 = time.perf_counter()
        G.run(root, out=out)
        torch.cuda.synchronize()
        t2 = time.perf_counter()
        G.run(root, out=out)
        torch.cuda.synchronize()
        t3 = time.perf_counter()
        G.close()
        torch.cuda.synchronize()
        t4 = time.perf_counter()
        print(json.dumps({"lib": os.environ.get("DFS_LIB", "default"), "rep": rep, "src": name, "create_ms": round((t1 - t0) * 1e3, 2),
                          "first_run_ms": round((t2 - t1) * 1e3, 2), "second_run_ms": round((t3 - t2) * 1e3, 2),
                          "destroy_ms": round((t4 - t3) * 1e3, 2)}), flush=True)

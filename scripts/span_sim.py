#!/usr/bin/env python3
"""Run scripts/span_sim.c (the idealised parallel-DFS schedule model, DESIGN.md §8 "span") on a
bench config: BFS eccentricity of each root, ticks for a sweep of walker counts and steal delays.

    python scripts/span_sim.py --config road24m --roots 4 --walkers 2368 4736 20000 \
        --delays 0 2 --out profiles/r02/span/road24m.jsonl

CPU only (no GPU, no product code): graphgen builds the graph, gcc builds the model.
"""
from __future__ import annotations

import argparse
import os
import subprocess
import sys
import tempfile

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="road24m")
    ap.add_argument("--roots", type=int, default=4, help="the bench's first k roots")
    ap.add_argument("--walkers", type=int, nargs="+", default=[4736])
    ap.add_argument("--delays", type=int, nargs="+", default=[0])
    ap.add_argument("--out")
    a = ap.parse_args()
    import graphgen

    g, root0, _, _ = graphgen.config_graph(a.config)
    roots = ([int(root0)] + [int(x) for x in graphgen.random_roots(g, 63, seed=0x6A7)])[:a.roots]
    with tempfile.TemporaryDirectory() as d:
        exe = os.path.join(d, "span_sim")
        subprocess.run(["gcc", "-O2", "-o", exe, os.path.join(ROOT, "scripts", "span_sim.c")], check=True)
        np.asarray(g.row_ptr, dtype=np.int64).tofile(os.path.join(d, "rp.bin"))
        np.asarray(g.col_idx, dtype=np.int32).tofile(os.path.join(d, "col.bin"))
        lines = []
        for r in roots:
            for w in a.walkers:
                for dl in a.delays:
                    out = subprocess.run([exe, str(r), str(w), str(dl)], cwd=d, check=True,
                                         capture_output=True, text=True).stdout.strip()
                    out = out[:-1] + f', "config": "{a.config}"}}'
                    print(out, flush=True)
                    lines.append(out)
    if a.out:
        os.makedirs(os.path.dirname(a.out), exist_ok=True)
        with open(a.out, "w") as f:
            f.write("\n".join(lines) + "\n")


if __name__ == "__main__":
    main()

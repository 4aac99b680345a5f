"""bench.py's span record: the BFS eccentricity helper against closed forms (CPU)."""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402
import graphgen  # noqa: E402


def test_eccentricity_closed_forms():
    g = graphgen.grid(40, 25)
    assert bench.bfs_eccentricity(g.row_ptr, g.col_idx, 0) == 39 + 24          # corner: W + H - 2
    assert bench.bfs_eccentricity(g.row_ptr, g.col_idx, 12 * 40 + 20) == 20 + 12   # interior cell
    p = graphgen.path(1000)
    assert bench.bfs_eccentricity(p.row_ptr, p.col_idx, 0) == 999
    assert bench.bfs_eccentricity(p.row_ptr, p.col_idx, 500) == 500
    # isolated vertex and a star (hand-built CSR)
    rp = np.array([0, 0], dtype=np.int64)
    assert bench.bfs_eccentricity(rp, np.zeros(0, dtype=np.int32), 0) == 0
    n = 9
    rows = [list(range(1, n))] + [[0]] * (n - 1)
    rp = np.cumsum([0] + [len(r) for r in rows]).astype(np.int64)
    col = np.array([v for r in rows for v in r], dtype=np.int32)
    assert bench.bfs_eccentricity(rp, col, 0) == 1 and bench.bfs_eccentricity(rp, col, 3) == 2

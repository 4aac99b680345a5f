"""scripts/span_sim.c (the DFS schedule model DESIGN.md §8 quotes) on graphs whose answer is known
(CPU; builds the model with gcc)."""
import json
import os
import subprocess

import numpy as np
import pytest

import graphgen

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def exe(tmp_path_factory):
    d = tmp_path_factory.mktemp("span")
    out = str(d / "span_sim")
    subprocess.run(["gcc", "-O2", "-o", out, os.path.join(ROOT, "scripts", "span_sim.c")], check=True)
    return out


def _run(exe, g, root, walkers, tmp_path, delay=0):
    np.asarray(g.row_ptr, dtype=np.int64).tofile(tmp_path / "rp.bin")
    np.asarray(g.col_idx, dtype=np.int32).tofile(tmp_path / "col.bin")
    r = subprocess.run([exe, str(root), str(walkers), str(delay)], cwd=tmp_path, check=True,
                       capture_output=True, text=True)
    return json.loads(r.stdout)


def test_path_is_sequential(exe, tmp_path):
    """A path from one end: every claim depends on the previous one.  One walker: n - 1 claim
    steps and n pops on the way back; more walkers only share the pops of the exhausted entries
    (stolen from the stack bottom), never the claims."""
    g = graphgen.path(500)
    d1 = _run(exe, g, 0, 1, tmp_path)
    assert d1["bfs_ecc"] == 499 and d1["claims"] == 500 and d1["reach"] == 500
    assert d1["ticks"] == 499 + 500
    d64 = _run(exe, g, 0, 64, tmp_path)
    assert d64["claims"] == 500 and 499 <= d64["ticks"] < d1["ticks"]      # the span bounds it


def test_star_parallelises_only_through_stealing(exe, tmp_path):
    """A star from its centre: BFS eccentricity 1; one walker claims the leaves one per tick."""
    n = 200
    rows = [list(range(1, n))] + [[0]] * (n - 1)
    rp = np.cumsum([0] + [len(r) for r in rows]).astype(np.int64)
    col = np.array([v for r in rows for v in r], dtype=np.int32)
    g = graphgen.CSR(rp, col, "star")
    d1 = _run(exe, g, 0, 1, tmp_path)
    assert d1["bfs_ecc"] == 1 and d1["claims"] == n and d1["reach"] == n
    d8 = _run(exe, g, 0, 8, tmp_path)
    assert d8["ticks"] < d1["ticks"]                   # thieves take the centre's remaining scan


def test_more_walkers_never_slower_on_grid(exe, tmp_path):
    g = graphgen.grid(64, 64)
    t = [_run(exe, g, 0, w, tmp_path)["ticks"] for w in (1, 16, 256)]
    assert t[0] > t[1] >= t[2] * 0.9 and _run(exe, g, 0, 16, tmp_path)["bfs_ecc"] == 126

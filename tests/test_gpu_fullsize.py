"""Full-size parity: BASELINE.json configs C1-C4 at their full sizes, in the launch configuration
bench.py times (library defaults: 148 x 32 warps, cutoffs 1 / 1 with steal-half, two-choice;
C5: the batch defaults, 8 traversals in flight on 18-block shares).

Checks (exact, integer): I1-I6 via the oracle checker (O(n+m)); reach set / visited count equal
to the oracle's BFS; unique-tree inputs (caterpillar) bit-exact with Alg 1; C1 also bit-exact in
deterministic mode (the 65,535-deep snake).  Large configs can be skipped with
DFS_SKIP_FULLSIZE=1 (they take minutes to generate and check).
"""
import os

import numpy as np
import pytest

import graphgen
import oracle

torch = pytest.importorskip("torch")
pytestmark = [pytest.mark.gpu]

if torch.cuda.is_available():
    from paper_conf_ppopp_niul0c26_b200 import Graph, Options

SKIP_BIG = os.environ.get("DFS_SKIP_FULLSIZE", "0") == "1"


def _check(g, root, p, undirected=True):
    r = oracle.check_tree(g.row_ptr, g.col_idx, root, p, i7=False, undirected=undirected)
    assert all(getattr(r, k) == 1 for k in ("i1", "i2", "i3", "i4", "i5", "i6")), r
    return r


def test_c1_grid256_full():
    g, root, und, _ = graphgen.config_graph("grid256")
    with Graph(g.row_ptr, g.col_idx) as G:
        p = G.run(root).cpu().numpy()
        r = _check(g, root, p)
        assert r.n_visited == g.n and r.m_visited == g.m == 261_120
        d = G.run(root, options=Options(deterministic=True)).cpu().numpy()
        assert np.array_equal(d, oracle.dfs(g.row_ptr, g.col_idx, root))


@pytest.mark.skipif(SKIP_BIG, reason="DFS_SKIP_FULLSIZE=1")
@pytest.mark.parametrize("name", ["road24m", "rmat24", "path100m"])
def test_full_configs_valid(name):
    g, root, und, _ = graphgen.config_graph(name)
    roots = [root] + [int(x) for x in graphgen.random_roots(g, 1, seed=0x6A7)]
    with Graph(g.row_ptr, g.col_idx) as G:
        for r in roots:
            p = G.run(r).cpu().numpy()
            res = _check(g, r, p, und)
            reach = oracle.reach(g.row_ptr, g.col_idx, r)
            assert res.n_visited == int(reach.sum())
            if name != "rmat24":
                assert res.n_visited == g.n           # connected by construction


@pytest.mark.skipif(SKIP_BIG, reason="DFS_SKIP_FULLSIZE=1")
def test_caterpillar_full_bit_exact():
    g, root, und, _ = graphgen.config_graph("caterpillar")
    want = oracle.dfs(g.row_ptr, g.col_idx, root)
    with Graph(g.row_ptr, g.col_idx) as G:
        for r in (root, 2**19, g.n - 1):
            p = G.run(r).cpu().numpy()
            w = want if r == root else oracle.dfs(g.row_ptr, g.col_idx, r)
            assert np.array_equal(p, w)


@pytest.mark.skipif(SKIP_BIG, reason="DFS_SKIP_FULLSIZE=1")
def test_c5_batch1024_full():
    """configs[4] at full size in bench.py's launch configuration: 1,024 seeded roots on the
    4900^2 road graph through dfs_run_batch at the default concurrency (8 traversals in flight,
    18-block shares), 128 rows per call.  Every row reaches all n vertices (the graph is
    connected: I4 exact) with parent[root] = -1; 16 rows spread over the batch pass I1-I6 exact."""
    g, _, _, _ = graphgen.config_graph("road24m")
    roots = graphgen.random_roots(g, 1024, seed=0xC5)
    check = set(range(0, 1024, 64))
    rows = 128
    out = torch.empty((rows, g.n), dtype=torch.int32, device="cuda")
    with Graph(g.row_ptr, g.col_idx) as G:
        for c0 in range(0, 1024, rows):
            chunk = [int(r) for r in roots[c0:c0 + rows]]
            _, st = G.run_batch(chunk, out=out, stats=True)
            assert st.blocks == 148 // 8
            vis = (out != -2).sum(dim=1).cpu().numpy()
            assert (vis == g.n).all(), (c0, vis.min())
            assert (st.root_counts[:, 0] == g.n).all() and (st.root_counts[:, 1] == g.m).all()
            rt = torch.tensor(chunk, dtype=torch.int64, device="cuda")
            assert bool((out.gather(1, rt[:, None]) == -1).all())
            for q in range(len(chunk)):
                if c0 + q in check:
                    _check(g, chunk[q], out[q].cpu().numpy())

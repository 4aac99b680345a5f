"""Full-size parity: BASELINE.json configs C1-C4 at their full sizes, in the launch configuration
bench.py times (default options: 148 x 32 warps, hot 32 / cold 64, two-choice).

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

"""Pins of the oracle's Alg 1 to things other than itself.

* closed forms: path, star, complete binary tree, caterpillar, grid boustrophedon, path+chords;
* a library routine: scipy.sparse.csgraph.depth_first_order (lexicographic DFS over the stored
  CSR order) must give the same predecessor array on random graphs, directed and undirected,
  with adjacency lists in arbitrary (shuffled) order;
* reach set: scipy breadth_first_order / connected_components;
* invariants: n_visited, sum of out-degrees.
"""
import numpy as np
import pytest
import scipy.sparse as sp
from scipy.sparse.csgraph import breadth_first_order, connected_components, depth_first_order

import graphgen
import oracle


def _check_valid(g, root, parent, undirected=True):
    r = oracle.check_tree(g.row_ptr, g.col_idx, root, parent, i7=True, undirected=undirected)
    assert r.ok, r


def test_path_closed_form():
    n = 1000
    g = graphgen.path(n)
    p = oracle.dfs(g.row_ptr, g.col_idx, 0)
    assert p[0] == -1
    assert np.array_equal(p[1:], np.arange(n - 1))          # parent[i] = i-1, depth n-1
    k = 377                                                   # interior root: left arm first
    p = oracle.dfs(g.row_ptr, g.col_idx, k)
    assert p[k] == -1
    assert np.array_equal(p[:k], np.arange(1, k + 1))       # i < k: parent i+1
    assert np.array_equal(p[k + 1:], np.arange(k, n - 1))   # i > k: parent i-1
    _check_valid(g, k, p)


def test_star_closed_form():
    n = 50
    g = graphgen.star(n)
    p = oracle.dfs(g.row_ptr, g.col_idx, 0)
    assert p[0] == -1 and np.all(p[1:] == 0)
    leaf = 17
    p = oracle.dfs(g.row_ptr, g.col_idx, leaf)
    assert p[leaf] == -1 and p[0] == leaf
    others = np.setdiff1d(np.arange(1, n), [leaf])
    assert np.all(p[others] == 0)


def test_binary_tree_closed_form():
    n = 4095
    g = graphgen.binary_tree(n)
    p = oracle.dfs(g.row_ptr, g.col_idx, 0)
    i = np.arange(1, n)
    assert p[0] == -1 and np.array_equal(p[1:], (i - 1) // 2)


def test_caterpillar_closed_form():
    S, L = 300, 7
    g = graphgen.caterpillar(S, L)
    p = oracle.dfs(g.row_ptr, g.col_idx, 0)
    assert p[0] == -1
    assert np.array_equal(p[1:S], np.arange(S - 1))
    leaves = np.arange(S, S + S * L)
    assert np.array_equal(p[leaves], (leaves - S) // L)


def _snake_parent(W, H):
    """Boustrophedon Hamiltonian path of the W x H grid from vertex 0."""
    par = np.empty(W * H, dtype=np.int64)
    for r in range(H):
        for c in range(W):
            v = r * W + c
            if r % 2 == 0:
                par[v] = (v - W if r > 0 else -1) if c == 0 else v - 1
            else:
                par[v] = v - W if c == W - 1 else v + 1
    return par


@pytest.mark.parametrize("W,H", [(256, 256), (7, 5), (1, 9), (9, 1)])
def test_grid_boustrophedon(W, H):
    g = graphgen.grid(W, H)
    assert g.m == 2 * ((W - 1) * H + W * (H - 1))
    p = oracle.dfs(g.row_ptr, g.col_idx, 0)
    assert np.array_equal(p.astype(np.int64), _snake_parent(W, H))


def test_path_plus_chords_is_bare_path():
    n = 200_000
    g = graphgen.path_chords(n, 2_000, seed=7)
    assert g.m > 2 * (n - 1)
    p = oracle.dfs(g.row_ptr, g.col_idx, 0)
    assert np.array_equal(p[1:], np.arange(n - 1))


def _scipy_graph(g):
    data = np.ones(g.m, dtype=np.float64)
    return sp.csr_matrix((data, g.col_idx.astype(np.int32), g.row_ptr), shape=(g.n, g.n))


@pytest.mark.parametrize("seed", range(12))
def test_matches_scipy_dfs(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(5, 400))
    ne = int(rng.integers(n // 2, 4 * n))
    directed = bool(seed % 2)
    g = graphgen.random_graph(n, ne, seed=1000 + seed, symmetric=not directed)
    g = graphgen.shuffle_lists(g, seed)           # CSR order, not sorted order, decides
    root = int(rng.integers(0, n))
    p = oracle.dfs(g.row_ptr, g.col_idx, root)
    order, pred = depth_first_order(_scipy_graph(g), root, directed=True, return_predecessors=True)
    want = np.where(pred == -9999, -2, pred)
    want[root] = -1
    assert np.array_equal(p, want)
    assert set(order.tolist()) == set(np.nonzero(p != -2)[0].tolist())


@pytest.mark.parametrize("seed", range(6))
def test_reach_matches_scipy(seed):
    rng = np.random.default_rng(100 + seed)
    n = int(rng.integers(10, 3000))
    g = graphgen.random_graph(n, int(n * 0.7), seed=seed, symmetric=bool(seed % 2))
    root = int(rng.integers(0, n))
    vis = oracle.reach(g.row_ptr, g.col_idx, root)
    order = breadth_first_order(_scipy_graph(g), root, directed=True, return_predecessors=False)
    want = np.zeros(n, dtype=bool)
    want[order] = True
    assert np.array_equal(vis, want)
    p = oracle.dfs(g.row_ptr, g.col_idx, root)
    assert np.array_equal(p != -2, want)
    if seed % 2:   # undirected: the reach set is the root's connected component
        _, lab = connected_components(_scipy_graph(g), directed=False)
        assert np.array_equal(want, lab == lab[root])


def test_rmat_small_shape_and_validity():
    g = graphgen.rmat(14, 16)
    deg = g.degree()
    assert g.n == 1 << 14
    assert np.all(np.diff(g.row_ptr) >= 0)
    # symmetric, no self loops
    src = np.repeat(np.arange(g.n), deg)
    assert not np.any(src == g.col_idx)
    a = set(zip(src.tolist(), g.col_idx.tolist()))
    assert all((v, u) in a for (u, v) in list(a)[:5000])
    root = int(graphgen.random_roots(g, 1, seed=3)[0])
    p = oracle.dfs(g.row_ptr, g.col_idx, root)
    r = oracle.check_tree(g.row_ptr, g.col_idx, root, p, i7=True, undirected=True)
    assert r.ok
    assert r.m_visited == int(deg[p != -2].sum())


def test_road_generator_shape():
    g = graphgen.road(128, 96, seed=0x5EED)
    assert g.n == 128 * 96
    assert abs(g.m / g.n - 2.4) < 0.05                       # avg degree 2.4 (DESIGN recipe)
    _, lab = connected_components(_scipy_graph(g), directed=False)
    assert np.all(lab == lab[0])                             # spanning tree => connected
    p = oracle.dfs(g.row_ptr, g.col_idx, 0)
    _check_valid(g, 0, p)


def test_oracle_rejects_bad_args():
    g = graphgen.path(5)
    with pytest.raises(ValueError):
        oracle.dfs(g.row_ptr, g.col_idx, 5)
    with pytest.raises(ValueError):
        oracle.dfs(g.row_ptr, g.col_idx, -1)


def test_isolated_root_and_empty_graph():
    rp = np.zeros(4, dtype=np.int64)
    ci = np.zeros(0, dtype=np.int32)
    p = oracle.dfs(rp, ci, 2)
    assert p.tolist() == [-2, -2, -1]
    r = oracle.check_tree(rp, ci, 2, p, i7=True, undirected=True)
    assert r.ok and r.n_visited == 1 and r.m_visited == 0


def test_self_loops_and_duplicates():
    # 0 -> 0, 0 -> 1 (twice), 1 -> 2, 2 -> 0: duplicates and a self loop are non-tree entries
    rp = np.array([0, 4, 5, 6], dtype=np.int64)
    ci = np.array([0, 1, 1, 2, 2, 0], dtype=np.int32)
    p = oracle.dfs(rp, ci, 0)
    assert p.tolist() == [-1, 0, 1]
    assert oracle.check_tree(rp, ci, 0, p, i7=True).ok


def test_matrix_market_roundtrip_and_symmetric(tmp_path):
    """graphgen.read_mtx (input side, SuiteSparse format P:3294-3296): general files are read
    as directed edges; symmetric files store both directions; self loops / duplicates dropped."""
    g = graphgen.road(30, 20, seed=1)
    p = tmp_path / "g.mtx"
    graphgen.write_mtx(g, str(p))
    h = graphgen.read_mtx(str(p))
    assert np.array_equal(g.row_ptr, h.row_ptr) and np.array_equal(g.col_idx, h.col_idx)
    s = tmp_path / "s.mtx"
    s.write_text("%%MatrixMarket matrix coordinate real symmetric\n% c\n4 4 4\n2 1 1.5\n3 2 2\n4 4 7\n3 2 9\n")
    t = graphgen.read_mtx(str(s))
    assert t.row_ptr.tolist() == [0, 1, 3, 4, 4] and t.col_idx.tolist() == [1, 0, 2, 1]
    bad = tmp_path / "bad.mtx"
    bad.write_text("%%MatrixMarket matrix array real general\n2 2\n1\n2\n3\n4\n")
    with pytest.raises(ValueError):
        graphgen.read_mtx(str(bad))

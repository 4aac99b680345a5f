"""Pin the oracle's acceptance checker by set equality with brute force.

For tiny graphs (<= 8 vertices), over EVERY candidate parent array (tests/bruteforce.py):
  * {checker I1-I6 accepts} == async in-order-scan outcome set   (I6 is exactly that model)
  * {checker I1-I5 + I7 accepts} == classical DFS trees over all adjacency permutations
  * Alg 1 oracle tree ∈ both; k-agent work-stealing outcomes ⊆ I6 set.
A wrong sign, index or dropped constraint in the checker changes one of these sets.
"""
import numpy as np
import pytest

import oracle
from tests import bruteforce as bf


def _sets_for(row_ptr, col, root, undirected):
    adj = bf.lists(row_ptr, col)
    classical = bf.classical_trees(adj, root)
    scan = bf.async_scan_outcomes(adj, root)
    acc6, acc7 = set(), set()
    for cand in bf.arborescences(adj, root):
        r = oracle.check_tree(row_ptr, col, root, np.array(cand, dtype=np.int32),
                              i7=True, undirected=undirected)
        ok5 = all(getattr(r, k) == 1 for k in ("i1", "i2", "i3", "i4", "i5"))
        if ok5 and r.i6 == 1:
            acc6.add(cand)
        if ok5 and r.i7 == 1:          # I7 quantifies over all list orders; independent of I6
            acc7.add(cand)
    return adj, classical, scan, acc6, acc7


def _graphs(n_graphs, seed, nmin, nmax, directed_frac):
    rng = np.random.default_rng(seed)
    for k in range(n_graphs):
        n = int(rng.integers(nmin, nmax + 1))
        directed = rng.random() < directed_frac
        p = float(rng.uniform(0.3, 0.7))
        rp, col = bf.random_tiny_graph(rng, n, p, directed, self_loops=directed and k % 5 == 0)
        root = int(rng.integers(0, n))
        yield rp, col, root, not directed


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_checker_equals_bruteforce(seed):
    for rp, col, root, undirected in _graphs(25, seed, 3, 6, 0.34):
        adj, classical, scan, acc6, acc7 = _sets_for(rp, col, root, undirected)
        assert acc6 == scan, (adj, root)
        assert acc7 == classical, (adj, root)
        lex = tuple(oracle.dfs(rp, col, root).tolist())
        assert lex in classical and lex in scan


@pytest.mark.parametrize("seed", [11, 12])
def test_work_stealing_outcomes_are_scan_consistent(seed):
    for rp, col, root, undirected in _graphs(15, seed, 3, 5, 0.3):
        adj = bf.lists(rp, col)
        scan = bf.async_scan_outcomes(adj, root)
        for k in (2, 3):
            ws = bf.stealing_outcomes(adj, root, k)
            assert ws <= scan
            for cand in ws:
                assert oracle.check_tree(rp, col, root, np.array(cand, dtype=np.int32)).ok


def test_work_stealing_produces_non_classical_trees():
    """Why I7 cannot be enforced on parallel runs: stealing creates cross edges."""
    found = 0
    for rp, col, root, undirected in _graphs(20, 99, 5, 6, 0.0):
        adj = bf.lists(rp, col)
        ws = bf.stealing_outcomes(adj, root, 2)
        found += len(ws - bf.classical_trees(adj, root)) > 0
    assert found > 0


def test_seven_vertex_graphs():
    for rp, col, root, undirected in _graphs(4, 7, 7, 7, 0.25):
        adj, classical, scan, acc6, acc7 = _sets_for(rp, col, root, undirected)
        assert acc6 == scan and acc7 == classical


def test_checker_mutations_hit_named_invariant():
    import graphgen
    g = graphgen.grid(6, 5)
    p = oracle.dfs(g.row_ptr, g.col_idx, 0)
    assert oracle.check_tree(g.row_ptr, g.col_idx, 0, p, i7=True, undirected=True).ok

    q = p.copy(); q[3] = -1                              # second root
    assert oracle.check_tree(g.row_ptr, g.col_idx, 0, q).failed() == ["i1"]
    q = p.copy(); q[0] = 1                               # root not -1
    assert oracle.check_tree(g.row_ptr, g.col_idx, 0, q).failed() == ["i1"]
    q = p.copy(); q[7] = 20                              # parent edge does not exist
    assert oracle.check_tree(g.row_ptr, g.col_idx, 0, q).failed() == ["i2"]
    q = p.copy(); q[1], q[2] = 2, 1                      # 2-cycle between adjacent vertices
    assert oracle.check_tree(g.row_ptr, g.col_idx, 0, q).failed() == ["i3"]
    q = p.copy(); q[29] = -2                              # dropped reachable leaf
    r = oracle.check_tree(g.row_ptr, g.col_idx, 0, q)
    assert r.failed() == ["i4"]
    # a BFS tree is scan-consistent (all scanners in lock-step) but not a classical DFS tree
    import scipy.sparse as sp
    from scipy.sparse.csgraph import breadth_first_order
    A = sp.csr_matrix((np.ones(g.m), g.col_idx, g.row_ptr), shape=(g.n, g.n))
    _, pred = breadth_first_order(A, 0, directed=True, return_predecessors=True)
    q = np.where(pred == -9999, -1, pred).astype(np.int32)
    r = oracle.check_tree(g.row_ptr, g.col_idx, 0, q, i7=True, undirected=True)
    assert r.failed() == ["i7"] and r.n_cross > 0


def test_i5_closure_on_directed_graph():
    # 0 -> 1, 1 -> 2 ; claimed tree omits 2 but also the reach set contains 2 -> I4 fires first.
    rp = np.array([0, 1, 2, 2], dtype=np.int64)
    ci = np.array([1, 2], dtype=np.int32)
    r = oracle.check_tree(rp, ci, 0, np.array([-1, 0, -2], dtype=np.int32))
    assert r.failed() == ["i4"]


def test_i6_rejects_out_of_order_claim():
    # path a-b-c plus edge a-c (triangle), root a=0, lists sorted: a:[1,2] b:[0,2] c:[0,1].
    # Tree {b<-a, c<-a}: a scans pos 0 (claims b), b's scan of c at pos1 must wait for c's claim,
    # which happens at a's pos 1 -> consistent (a scans in order).  Tree {c<-a, b<-c}: a's position
    # 0 targets b, which is claimed only by c, whose claim happens at a's position 1 > 0 -> cycle.
    rp = np.array([0, 2, 4, 6], dtype=np.int64)
    ci = np.array([1, 2, 0, 2, 0, 1], dtype=np.int32)
    assert oracle.check_tree(rp, ci, 0, np.array([-1, 0, 0], dtype=np.int32)).ok
    r = oracle.check_tree(rp, ci, 0, np.array([-1, 2, 0], dtype=np.int32))
    assert r.failed() == ["i6"]


def _graphs_p(n_graphs, seed, n, p_lo, p_hi, directed_frac):
    rng = np.random.default_rng(seed)
    for k in range(n_graphs):
        directed = rng.random() < directed_frac
        p = float(rng.uniform(p_lo, p_hi))
        rp, col = bf.random_tiny_graph(rng, n, p, directed, self_loops=directed and k % 2 == 0)
        root = int(rng.integers(0, n))
        yield rp, col, root, not directed


def test_eight_vertex_graphs():
    """north_star / SURVEY T2: brute force on graphs of 8 vertices (the largest size named),
    undirected and directed (with self loops), sparse enough that the enumerations finish."""
    seen = 0
    for rp, col, root, undirected in _graphs_p(6, 8, 8, 0.25, 0.4, 0.5):
        adj, classical, scan, acc6, acc7 = _sets_for(rp, col, root, undirected)
        assert acc6 == scan and acc7 == classical, (adj, root)
        lex = tuple(oracle.dfs(rp, col, root).tolist())
        assert lex in classical and lex in scan
        seen += len(bf.reach_set(adj, root)) == 8
    assert seen >= 2          # at least two cases reach all 8 vertices

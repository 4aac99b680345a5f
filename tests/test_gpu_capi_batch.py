"""GPU parity through the four north-star C symbols and the batch path at its defaults.

* dfs_graph_create / dfs_run / dfs_run_batch / dfs_graph_destroy called directly through ctypes
  with HOST buffers (pageable numpy arrays: the library copies the CSR in, stages the parents
  out, and page-locks a pageable batch output for its concurrent path) — every tree checked
  against the oracle (I1-I6 exact; bit-exact where the spanning tree is unique);
* dfs_run_batch at the default concurrency (K = 8 traversals in flight, auto) with >= 8 roots:
  every row checked, per-root counts equal the oracle's;
* steal counters: Alg 3 and Alg 4 both move work on the stress configurations (a regression that
  silently disabled either would still produce valid trees, so the counters are asserted).
Reference: P:198-208 (problem), P:1067-1180 (Alg 3/4), north_star (C ABI, configs[4]).
"""
import ctypes

import numpy as np
import pytest

import graphgen
import oracle

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    from paper_conf_ppopp_niul0c26_b200 import Graph, Options
    from paper_conf_ppopp_niul0c26_b200 import dfs as dfsmod


def _valid(g, root, parent, undirected=True):
    r = oracle.check_tree(g.row_ptr, g.col_idx, root, np.asarray(parent), i7=True, undirected=undirected)
    assert all(getattr(r, k) == 1 for k in ("i1", "i2", "i3", "i4", "i5", "i6")), (g.name, root, r)
    assert r.n_visited == int(oracle.reach(g.row_ptr, g.col_idx, root).sum())
    return r


def test_north_star_symbols_with_host_buffers():
    lib = dfsmod.load_library()
    torch.cuda.set_device(0)
    for g, undirected, exact in ((graphgen.road(700, 500, seed=31), True, False),
                                 (graphgen.random_graph(50_000, 150_000, seed=5, symmetric=False), False, False),
                                 (graphgen.binary_tree((1 << 16) - 1), True, True)):
        rp = np.ascontiguousarray(g.row_ptr, dtype=np.int64)
        ci = np.ascontiguousarray(g.col_idx, dtype=np.int32)
        h = lib.dfs_graph_create(rp.ctypes.data, ci.ctypes.data, g.n, g.m)
        assert h, lib.dfs_last_error()
        try:
            roots = [int(x) for x in graphgen.random_roots(g, 10, seed=7)]
            parent = np.full(g.n, 12345, dtype=np.int32)                    # pageable host output
            assert lib.dfs_run(ctypes.c_void_p(h), roots[0], parent.ctypes.data) == 0
            _valid(g, roots[0], parent, undirected)
            if exact:
                assert np.array_equal(parent, oracle.dfs(g.row_ptr, g.col_idx, roots[0]))
            hroots = np.array(roots, dtype=np.int32)
            rows = np.full((len(roots), g.n), 777, dtype=np.int32)          # pageable host batch
            assert lib.dfs_run_batch(ctypes.c_void_p(h), hroots.ctypes.data, len(roots), rows.ctypes.data) == 0
            for q, r in enumerate(roots):
                _valid(g, r, rows[q], undirected)
                if exact:
                    assert np.array_equal(rows[q], oracle.dfs(g.row_ptr, g.col_idx, r))
            # errors through the plain symbols: bad root, NULL output
            assert lib.dfs_run(ctypes.c_void_p(h), g.n, parent.ctypes.data) == -1
            assert lib.dfs_run(ctypes.c_void_p(h), 0, None) == -1
        finally:
            lib.dfs_graph_destroy(ctypes.c_void_p(h))
    lib.dfs_graph_destroy(None)                                             # no-op


@pytest.mark.parametrize("graph", ["road", "rmat"])
def test_batch_default_concurrency_every_row(graph):
    """configs[4] at reduced size: >= 8 roots at the library default (K = 8 in flight, auto
    share of the SMs), device and pinned host outputs; every row equals the oracle's reach set
    and passes I1-I6; per-root counts match."""
    g = graphgen.road(1024, 1024, seed=0x5EED) if graph == "road" else graphgen.rmat(17, 16)
    roots = graphgen.random_roots(g, 12, seed=44)
    deg = np.diff(g.row_ptr)
    with Graph(g.row_ptr, g.col_idx) as G:
        out, st = G.run_batch(roots, stats=True)
        assert st.blocks == 148 // 8                                       # 8 in flight
        for q, r in enumerate(roots):
            res = _valid(g, int(r), out[q].cpu().numpy())
            assert tuple(st.root_counts[q]) == (res.n_visited, int(deg[out[q].cpu().numpy() != -2].sum()))
        hb = torch.empty((len(roots), g.n), dtype=torch.int32).pin_memory()
        G.run_batch(roots, out=hb)
        for q, r in enumerate(roots):
            _valid(g, int(r), hb[q].numpy())
        # explicit K = 16 (maximum), more roots than slots
        out16 = G.run_batch(roots, options=Options(concurrency=16))
        for q, r in enumerate(roots):
            _valid(g, int(r), out16[q].cpu().numpy())


def test_batch_empty_and_repeated_roots():
    """num_roots = 0 is a no-op (NULL arrays accepted); repeated roots give independent rows."""
    g = graphgen.road(128, 96, seed=3)
    lib = dfsmod.load_library()
    with Graph(g.row_ptr, g.col_idx) as G:
        assert lib.dfs_run_batch(ctypes.c_void_p(G._h), None, 0, None) == 0
        assert lib.dfs_run_batch(ctypes.c_void_p(G._h), None, -1, None) == -1
        assert G.run_batch([]).shape == (0, g.n)
        roots = [7, 7, 7, 7, 7, 7, 7, 7, 7, 0]
        out = G.run_batch(roots)
        for q, r in enumerate(roots):
            _valid(g, r, out[q].cpu().numpy())


def test_batch_host_rows_double_buffered():
    """Host (pinned) output rows of a concurrent batch: every slot runs many more traversals than
    its two device row buffers, so each buffer is reused while the previous row's copy to the host
    is in flight (copy stream + events); every row must still be the right traversal."""
    g = graphgen.road(256, 256, seed=0x5EED)
    roots = graphgen.random_roots(g, 40, seed=45)
    with Graph(g.row_ptr, g.col_idx) as G:
        for conc in (4, 8):
            hb = torch.full((len(roots), g.n), 31337, dtype=torch.int32).pin_memory()
            G.run_batch(roots, out=hb, options=Options(concurrency=conc))
            for q, r in enumerate(roots):
                row = hb[q].numpy()
                assert row[int(r)] == -1, (conc, q)                        # the row of root q
                _valid(g, int(r), row)


@pytest.mark.parametrize("opts", [dict(), dict(hot_cutoff=2, cold_cutoff=2, steal_half=False),
                                  dict(window=128), dict(warps_per_block=8, blocks=40)])
def test_both_steal_tiers_move_work(opts):
    g = graphgen.road(1024, 1024, seed=0x5EED)
    with Graph(g.row_ptr, g.col_idx) as G:
        p, st = G.run(0, options=Options(collect_stats=True, **opts), stats=True)
        _valid(g, 0, p.cpu().numpy())
        assert st.intra_steals > 0, st
        assert st.inter_steals > 0, st
        assert st.claims == st.n_visited - 1
        # with Alg 4 off no inter-block steal happens (the counter is live, not constant)
        p, st = G.run(0, options=Options(collect_stats=True, inter_steal=False, **opts), stats=True)
        _valid(g, 0, p.cpu().numpy())
        assert st.inter_steals == 0 and st.intra_steals > 0

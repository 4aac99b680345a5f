"""GPU parity of the sub-warp walker kernel (dfs_walker.cuh; dfs_options.walker_lanes = 16/8/4).

Same bars as the warp kernel: I1-I6 exact on every graph and option
set (I4 = reach set bit-exact), bit-exact with Alg 1 on tree inputs (unique spanning tree), steal
counters live, stress settings that force flush/refill/steal races on tiny rings.
"""
import numpy as np
import pytest

import graphgen
import oracle

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    from paper_conf_ppopp_niul0c26_b200 import DfsError, Graph, Options

LANES = [16, 8, 4, 2]


def _valid(g, root, parent, undirected=True):
    got = parent.cpu().numpy() if hasattr(parent, "cpu") else parent
    r = oracle.check_tree(g.row_ptr, g.col_idx, root, got, i7=True, undirected=undirected)
    assert all(getattr(r, k) == 1 for k in ("i1", "i2", "i3", "i4", "i5", "i6")), (g.name, root, r)
    assert r.n_visited == int(oracle.reach(g.row_ptr, g.col_idx, root).sum())
    return r


def _exact(g, root, parent):
    got = parent.cpu().numpy() if hasattr(parent, "cpu") else parent
    want = oracle.dfs(g.row_ptr, g.col_idx, root)
    assert np.array_equal(got, want), (g.name, root, int((got != want).sum()))


@pytest.mark.parametrize("lanes", LANES)
@pytest.mark.parametrize("name,build,nroots,undirected", [
    ("grid256", lambda: graphgen.grid(256, 256), 2, True),
    ("road1024", lambda: graphgen.road(1024, 1024, seed=0x5EED), 3, True),
    ("road_ragged", lambda: graphgen.road(999, 777, seed=11), 2, True),
    ("rmat16", lambda: graphgen.rmat(16, 16), 3, True),
    ("pathchords", lambda: graphgen.path_chords(400_000, 4_000, seed=2), 2, True),
    ("random_dir", lambda: graphgen.random_graph(30_000, 90_000, seed=3, symmetric=False,
                                                  allow_self=True, allow_dup=True), 3, False),
    ("shuffled", lambda: graphgen.shuffle_lists(graphgen.random_graph(20_000, 50_000, seed=4), 9), 2, True),
])
def test_walker_valid(lanes, name, build, nroots, undirected):
    g = build()
    roots = [int(r) for r in graphgen.random_roots(g, nroots, seed=lanes)]
    with Graph(g.row_ptr, g.col_idx) as G:
        for r in roots:
            p, st = G.run(r, options=Options(walker_lanes=lanes), stats=True)
            _valid(g, r, p, undirected)
            assert st.n_visited == int((p != -2).sum().item())


@pytest.mark.parametrize("lanes", LANES)
@pytest.mark.parametrize("name,build,roots", [
    ("path", lambda: graphgen.path(300_001), [0, 150_000]),
    ("star", lambda: graphgen.star(50_000), [0, 7]),
    ("bintree", lambda: graphgen.binary_tree((1 << 20) - 1), [0, 5]),
    ("caterpillar", lambda: graphgen.caterpillar(1 << 14, 94), [0, 5000]),
])
def test_walker_tree_inputs_bit_exact(lanes, name, build, roots):
    g = build()
    with Graph(g.row_ptr, g.col_idx) as G:
        for r in roots:
            _exact(g, r, G.run(r, options=Options(walker_lanes=lanes)))


@pytest.mark.parametrize("lanes", LANES)
@pytest.mark.parametrize("opts", [
    dict(ring_cap=2), dict(ring_cap=5, hot_cutoff=2, cold_cutoff=2), dict(hot_cutoff=8, cold_cutoff=16),
    dict(steal_half=False), dict(steal_period=8), dict(steal_tries=1), dict(spill=False),
    dict(inter_steal=False), dict(intra_steal=False), dict(blocks=3, warps_per_block=2),
    dict(blocks=1), dict(warps_per_block=1, blocks=5), dict(victim_policy=0), dict(speculate=0),
    dict(speculate=1), dict(leaf_skip=0), dict(leaf_skip=1), dict(pub_batch=4), dict(spill_period=1),
    dict(records=1), dict(records=1, ring_cap=3), dict(donate=0), dict(donate=0, steal_period=1024),
])
def test_walker_stress(lanes, opts):
    g = graphgen.road(300, 200, seed=7)
    gr = graphgen.rmat(13, 8, seed=5)
    with Graph(g.row_ptr, g.col_idx) as G, Graph(gr.row_ptr, gr.col_idx) as GR:
        for r in (0, 31337):
            _valid(g, r, G.run(r, options=Options(walker_lanes=lanes, **opts)))
        rr = int(graphgen.random_roots(gr, 1, seed=2)[0])
        _valid(gr, rr, GR.run(rr, options=Options(walker_lanes=lanes, **opts)))


@pytest.mark.parametrize("lanes", LANES)
def test_walker_counters_and_steals(lanes):
    g = graphgen.road(1024, 1024, seed=0x5EED)
    with Graph(g.row_ptr, g.col_idx) as G:
        p, st = G.run(0, options=Options(walker_lanes=lanes, collect_stats=True), stats=True, block_claims=True)
        r = _valid(g, 0, p)
        assert st.claims == r.n_visited - 1
        assert int(st.block_claims.sum()) == r.n_visited - 1
        assert st.intra_steals > 0 and st.inter_steals > 0, st
        p, st = G.run(0, options=Options(walker_lanes=lanes, collect_stats=True, inter_steal=False), stats=True)
        _valid(g, 0, p)
        assert st.inter_steals == 0 and st.intra_steals > 0


@pytest.mark.parametrize("lanes", LANES)
@pytest.mark.parametrize("records", [0, 1])
def test_walker_records_directed_long_lists(lanes, records):
    """Vertex records hold the first 6 neighbours: lists of 0..40 entries (directed, self loops,
    duplicates, unsorted) take both the record path and the col_idx path of the same list."""
    g = graphgen.shuffle_lists(graphgen.random_graph(20_000, 200_000, seed=12, symmetric=False,
                                                     allow_self=True, allow_dup=True), 4)
    with Graph(g.row_ptr, g.col_idx) as G:
        for r in (0, 999):
            _valid(g, r, G.run(r, options=Options(walker_lanes=lanes, records=records)), undirected=False)


@pytest.mark.parametrize("lanes", LANES)
def test_walker_deep_stack_flush_refill(lanes):
    """One walker holding ~n entries: grid snake / 10^6 path / caterpillar spine drive the
    per-walker ColdSeg through thousands of flushes and refills."""
    for g, root, exact in ((graphgen.grid(256, 256), 0, False), (graphgen.path(1_000_000), 0, True),
                           (graphgen.caterpillar(1 << 15, 30), 0, True)):
        with Graph(g.row_ptr, g.col_idx) as G:
            for opts in (dict(), dict(ring_cap=7), dict(blocks=1, warps_per_block=1)):
                p, st = G.run(root, options=Options(walker_lanes=lanes, collect_stats=True, **opts), stats=True)
                (_exact if exact else _valid)(g, root, p)


@pytest.mark.parametrize("lanes", LANES)
def test_walker_batch_errors_and_recovery(lanes):
    g = graphgen.road(600, 600, seed=2)
    roots = [int(r) for r in graphgen.random_roots(g, 10, seed=3)]
    with Graph(g.row_ptr, g.col_idx) as G:
        out = G.run_batch(roots, options=Options(walker_lanes=lanes))
        for q, r in enumerate(roots):
            _valid(g, r, out[q])
        with pytest.raises(DfsError) as e:
            G.run(0, options=Options(walker_lanes=lanes, max_pool_chunks=1, ring_cap=2))
        assert e.value.code == -2
        with pytest.raises(DfsError) as e:
            G.run(0, options=Options(walker_lanes=lanes, timeout_ms=1, blocks=1, warps_per_block=1))
        assert e.value.code == -5
        _valid(g, 5, G.run(5, options=Options(walker_lanes=lanes)))
        hb = torch.empty((len(roots), g.n), dtype=torch.int32)
        G.run_batch(roots, out=hb, options=Options(walker_lanes=lanes, concurrency=4))
        for q, r in enumerate(roots):
            _valid(g, r, hb[q].numpy())
    with pytest.raises(DfsError):
        with Graph(g.row_ptr, g.col_idx) as G:
            G.run(0, options=Options(walker_lanes=6))

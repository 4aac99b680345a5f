"""GPU parity: the CUDA path (through the C ABI) against the oracle, on the same seeded inputs.

Bars (DESIGN.md §"Parity"): integer work, tolerance 0.
  * deterministic single-warp mode: parent array bit-exact with Alg 1 (oracle.dfs);
  * tree-shaped inputs (unique spanning tree): bit-exact in every mode;
  * full parallel mode: checks I1-I6 exact (I4 = reach set bit-exact, visited count exact);
    I7 (classical DFS tree) reported, not required (stealing creates cross edges by design);
  * stress: tiny cutoffs, few warps/blocks, many roots — forces flush/refill/steal races.
"""
import numpy as np
import pytest

import graphgen
import oracle

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    from paper_conf_ppopp_niul0c26_b200 import DfsError, Graph, Options


def _exact(g, root, parent):
    want = oracle.dfs(g.row_ptr, g.col_idx, root)
    got = parent.cpu().numpy() if hasattr(parent, "cpu") else parent
    if not np.array_equal(got, want):
        bad = np.nonzero(got != want)[0]
        raise AssertionError(f"{g.name} root {root}: {bad.size} mismatches, first {bad[:5]} "
                             f"got {got[bad[:5]]} want {want[bad[:5]]}")


def _valid(g, root, parent, undirected=True):
    got = parent.cpu().numpy() if hasattr(parent, "cpu") else parent
    r = oracle.check_tree(g.row_ptr, g.col_idx, root, got, i7=True, undirected=undirected)
    assert all(getattr(r, k) == 1 for k in ("i1", "i2", "i3", "i4", "i5", "i6")), (g.name, root, r)
    reach = oracle.reach(g.row_ptr, g.col_idx, root)
    assert r.n_visited == int(reach.sum())
    return r


DET = None


def det():
    return Options(deterministic=True)


# ------------------------------------------------------------------ deterministic = Alg 1
@pytest.mark.parametrize("name,build,root", [
    ("grid256", lambda: graphgen.grid(256, 256), 0),                  # depth-65,535 snake
    ("grid_ragged", lambda: graphgen.grid(37, 53), 700),
    ("road512", lambda: graphgen.road(512, 300, seed=5), 0),
    ("path1e6", lambda: graphgen.path(1_000_000), 0),
    ("pathchords", lambda: graphgen.path_chords(300_000, 3_000, seed=2), 12345),
    ("caterpillar", lambda: graphgen.caterpillar(4096, 94), 0),
    ("rmat16", lambda: graphgen.rmat(16, 16), None),
    ("star", lambda: graphgen.star(100_000), 0),
    ("random_dir", lambda: graphgen.random_graph(20_000, 60_000, seed=3, symmetric=False,
                                                  allow_self=True, allow_dup=True), 17),
    ("shuffled", lambda: graphgen.shuffle_lists(graphgen.random_graph(5000, 30000, seed=4), 9), 1),
])
def test_deterministic_bit_exact(name, build, root):
    g = build()
    if root is None:
        root = int(graphgen.random_roots(g, 1, seed=1)[0])
    with Graph(g.row_ptr, g.col_idx) as G:
        for win, sp in ((32, 2), (128, 2), (32, 0), (128, 1), (32, 2 | 4 | 8)):
            p = G.run(root, options=Options(deterministic=True, window=win, speculate=sp))
            torch.cuda.synchronize()
            _exact(g, root, p)


def test_bulk_leaf_claims_respect_shared_in_lists():
    """Leaf map (bulk claims in 128-wide windows): a sink with two in-neighbours is not a leaf —
    Alg 1 reaches it through the first child, so claiming it early from the root would differ."""
    #   0 -> [1, 2];  1 -> [2];  2 -> []  (directed);  Alg 1 from 0: parent = [-1, 0, 1]
    rp = np.array([0, 2, 3, 3], dtype=np.int64)
    ci = np.array([1, 2, 2], dtype=np.int32)
    with Graph(rp, ci) as G:
        for win in (32, 128):
            assert G.run(0, options=Options(deterministic=True, window=win)).cpu().tolist() == [-1, 0, 1]
    # many sinks shared by two hubs, deterministic 128-wide windows: bit-exact with Alg 1
    rng = np.random.default_rng(5)
    n, k = 3000, 400
    rows = [[] for _ in range(n)]
    rows[0] = [1] + list(range(2 + 0, 2 + k))                 # root: hub 1, then sinks
    rows[1] = list(range(2, 2 + k)) + list(range(2 + k, n))   # hub 1 reaches the same sinks first
    for v in range(2 + k, n):
        rows[v] = sorted(rng.choice(n, 2, replace=False).tolist())
    rp = np.zeros(n + 1, dtype=np.int64)
    rp[1:] = np.cumsum([len(r) for r in rows])
    ci = np.array([x for r in rows for x in r], dtype=np.int32)
    g = graphgen.CSR(rp, ci, "shared_sinks")
    with Graph(rp, ci) as G:
        for win in (32, 128):
            _exact(g, 0, G.run(0, options=Options(deterministic=True, window=win)))
            _valid(g, 0, G.run(0, options=Options(window=win)), undirected=False)


# ------------------------------------------------------------------ unique trees: exact in parallel
@pytest.mark.parametrize("name,build,roots", [
    ("path", lambda: graphgen.path(200_001), [0, 100_000, 200_000]),
    ("star", lambda: graphgen.star(50_000), [0, 7]),
    ("bintree", lambda: graphgen.binary_tree((1 << 20) - 1), [0, 5, (1 << 19)]),
    ("caterpillar", lambda: graphgen.caterpillar(1 << 14, 94), [0, 5000]),
])
def test_tree_inputs_bit_exact_parallel(name, build, roots):
    g = build()
    with Graph(g.row_ptr, g.col_idx) as G:
        for r in roots:
            p = G.run(r)
            _exact(g, r, p)


# ------------------------------------------------------------------ parallel: I1-I6 exact
@pytest.mark.parametrize("name,build,nroots", [
    ("grid256", lambda: graphgen.grid(256, 256), 3),
    ("road1024", lambda: graphgen.road(1024, 1024, seed=0x5EED), 3),
    ("road_ragged", lambda: graphgen.road(999, 777, seed=11), 2),
    ("rmat18", lambda: graphgen.rmat(18, 16), 4),
    ("pathchords", lambda: graphgen.path_chords(1_000_000, 10_000, seed=1), 2),
    ("random_sparse", lambda: graphgen.random_graph(200_000, 150_000, seed=8), 4),  # many components
])
def test_parallel_valid(name, build, nroots):
    g = build()
    roots = [0] + list(graphgen.random_roots(g, nroots - 1, seed=42))
    with Graph(g.row_ptr, g.col_idx) as G:
        for r in roots:
            p = G.run(int(r))
            _valid(g, int(r), p)


def test_parallel_directed_with_self_loops_and_duplicates():
    g = graphgen.random_graph(100_000, 400_000, seed=77, symmetric=False, allow_self=True, allow_dup=True)
    with Graph(g.row_ptr, g.col_idx) as G:
        for r in graphgen.random_roots(g, 3, seed=5):
            p = G.run(int(r))
            _valid(g, int(r), p, undirected=False)


# ------------------------------------------------------------------ stress
@pytest.mark.parametrize("opts", [
    dict(hot_cutoff=4, cold_cutoff=4),
    dict(hot_cutoff=2, cold_cutoff=2),
    dict(hot_cutoff=6, cold_cutoff=2, spill_idle=1),
    dict(hot_cutoff=2, cold_cutoff=2, warps_per_block=3, blocks=5, spill=False),
    dict(hot_cutoff=8, cold_cutoff=8, warps_per_block=4, blocks=8),
    dict(inter_any=False, spill=False),
    dict(hot_cutoff=4, cold_cutoff=4, warps_per_block=2, blocks=64),
    dict(victim_policy=0),
    dict(intra_steal=False),
    dict(inter_steal=False),
    dict(blocks=1),
    dict(hot_cutoff=64, cold_cutoff=128),
    dict(hot_cutoff=2, cold_cutoff=2, window=128),
    dict(hot_cutoff=4, cold_cutoff=8, window=32),
    dict(hot_cutoff=1, cold_cutoff=1),
    dict(hot_cutoff=3, cold_cutoff=5, steal_half=False),
    dict(hot_cutoff=1, cold_cutoff=1, warps_per_block=2, blocks=3, spill_idle=1, pub_batch=3),
    dict(speculate=1, window=128, steal_half=False),
    dict(speculate=0),
    dict(speculate=1, window=128),
    dict(hot_cutoff=4, ring_cap=3, warps_per_block=4, blocks=6),
    dict(cluster=2),                                                  # §8(f)-3 DSMEM tier
    dict(cluster=4, hot_cutoff=2, window=128),
    dict(cluster=2, warps_per_block=4, blocks=8, spill=False, inter_steal=False),
    dict(cluster=8, warps_per_block=2, hot_cutoff=1, intra_steal=True, spill_idle=1),
    dict(cluster=2, cluster_late=True, steal_tries=3, hot_cutoff=2),
    dict(steal_tries=4),
    dict(steal_tries=8, warps_per_block=8, blocks=4, spill=False),
    dict(speculate=2 | 4 | 8),
    dict(bulk_copy=True),                                             # cp.async.bulk flush/refill
    dict(bulk_copy=False, l2_persist_mb=16),                          # warp copies; L2 policy window
    dict(bulk_copy=True, ring_cap=3, hot_cutoff=2, cold_cutoff=2, window=128),
])
def test_stress_options(opts):
    graphs = [graphgen.road(300, 300, seed=3), graphgen.rmat(14, 8, seed=9),
              graphgen.caterpillar(2000, 30), graphgen.path_chords(100_000, 2_000, seed=3)]
    o = Options(**opts)
    for g in graphs:
        with Graph(g.row_ptr, g.col_idx) as G:
            for r in list(graphgen.random_roots(g, 3, seed=len(opts))) + [0]:
                p = G.run(int(r), options=o)
                _valid(g, int(r), p)


def test_many_small_random_graphs():
    rng = np.random.default_rng(0)
    for k in range(40):
        n = int(rng.integers(2, 3000))
        g = graphgen.random_graph(n, int(rng.integers(0, 4 * n)), seed=k, symmetric=bool(k % 2),
                                  allow_self=bool(k % 3 == 0), allow_dup=bool(k % 5 == 0))
        o = Options(hot_cutoff=4, cold_cutoff=4) if k % 2 else None
        with Graph(g.row_ptr, g.col_idx) as G:
            r = int(rng.integers(0, n))
            p = G.run(r, options=o)
            _valid(g, r, p, undirected=bool(k % 2))
            if k % 4 == 0:
                _exact(g, r, G.run(r, options=det()))


# ------------------------------------------------------------------ API edge cases
def test_isolated_root_single_vertex_and_empty():
    rp = np.zeros(2, dtype=np.int64)
    with Graph(rp, np.zeros(0, dtype=np.int32)) as G:
        assert G.run(0).cpu().tolist() == [-1]
    rp = np.array([0, 1, 2, 2], dtype=np.int64)
    ci = np.array([1, 0], dtype=np.int32)
    with Graph(rp, ci) as G:
        assert G.run(2).cpu().tolist() == [-2, -2, -1]
        assert G.run(0).cpu().tolist() == [-1, 0, -2]


def test_host_and_device_buffers_and_batch():
    g = graphgen.road(200, 150, seed=1)
    roots = graphgen.random_roots(g, 6, seed=2)
    rp_d = torch.from_numpy(g.row_ptr).cuda()
    ci_d = torch.from_numpy(g.col_idx).cuda()
    with Graph(rp_d, ci_d) as G:                                # device inputs
        host_out = torch.empty(g.n, dtype=torch.int32).pin_memory()
        G.run(int(roots[0]), out=host_out)                       # host output
        _valid(g, int(roots[0]), host_out.numpy())
        out = G.run_batch(roots)                                 # device batch output
        for q, r in enumerate(roots):
            _valid(g, int(r), out[q])
        hb = torch.empty((len(roots), g.n), dtype=torch.int32)  # host batch output, device roots
        G.run_batch(torch.from_numpy(roots).cuda(), out=hb, options=det())
        for q, r in enumerate(roots):
            _exact(g, int(r), hb[q].numpy())
        assert G.launch_count() > 0


def test_errors():
    g = graphgen.grid(10, 10)
    with Graph(g.row_ptr, g.col_idx) as G:
        with pytest.raises(DfsError) as e:
            G.run(100)
        assert e.value.code == -1
        with pytest.raises(DfsError):
            G.run(0, options=Options(hot_cutoff=66))              # h_s > 32 lanes
        with pytest.raises(DfsError):
            G.run(0, options=Options(cold_cutoff=130))            # c_s > 64
        with pytest.raises(DfsError):
            G.run(0, options=Options(window=64))
        with pytest.raises(DfsError):
            G.run(0, options=Options(blocks=100000))
        with pytest.raises(DfsError):
            G.run(0, options=Options(cluster=3))                  # cluster sizes 2, 4, 8
    bad = g.row_ptr.copy(); bad[5] = bad[4] - 1                   # non-monotone row_ptr
    with pytest.raises(DfsError):
        Graph(bad, g.col_idx)
    badc = g.col_idx.copy(); badc[3] = g.n                        # neighbour out of range
    with pytest.raises(DfsError):
        Graph(g.row_ptr, badc)
    with pytest.raises(DfsError):
        Graph(torch.from_numpy(bad).cuda(), torch.from_numpy(g.col_idx).cuda())


def test_stats_counters():
    g = graphgen.road(512, 512, seed=3)
    with Graph(g.row_ptr, g.col_idx) as G:
        p, st = G.run(0, stats=True, options=Options(collect_stats=True))
        r = _valid(g, 0, p)
        assert st.n_visited == r.n_visited and st.m_visited == r.m_visited
        assert st.claims == r.n_visited - 1
        assert st.kernel_ms > 0 and 0 < st.traversal_ms <= st.kernel_ms
        p2, st2 = G.run(7, stats=True)                 # counts without the counter build
        r2 = _valid(g, 7, p2)
        assert st2.n_visited == r2.n_visited and st2.m_visited == r2.m_visited and st2.claims == 0


def test_stream_and_repeat_consistency():
    g = graphgen.rmat(15, 16, seed=3)
    r = int(graphgen.random_roots(g, 1, seed=3)[0])
    s = torch.cuda.Stream()
    with Graph(g.row_ptr, g.col_idx) as G:
        with torch.cuda.stream(s):
            ps = [G.run(r) for _ in range(5)]
        torch.cuda.synchronize()
        vis = [(p != -2).cpu().numpy() for p in ps]
        for p, v in zip(ps, vis):
            assert np.array_equal(v, vis[0])
            _valid(g, r, p)


@pytest.mark.parametrize("conc", [2, 3, 4])
def test_concurrent_batch(conc):
    """§8(f)-2: K traversals at once on K slots / streams / SM shares; every row valid."""
    g = graphgen.road(400, 300, seed=9)
    roots = graphgen.random_roots(g, 7, seed=conc)
    with Graph(g.row_ptr, g.col_idx) as G:
        out, st = G.run_batch(roots, options=Options(concurrency=conc), stats=True)
        tot_v = 0
        for q, r in enumerate(roots):
            res = _valid(g, int(r), out[q])
            tot_v += res.n_visited
            assert tuple(st.root_counts[q]) == (res.n_visited, res.m_visited)
        assert st.n_visited == tot_v
        hb = torch.empty((len(roots), g.n), dtype=torch.int32)
        G.run_batch(roots, out=hb, options=Options(concurrency=conc, hot_cutoff=4, window=128))
        for q, r in enumerate(roots):
            _valid(g, int(r), hb[q].numpy())
        # deterministic ignores concurrency and stays bit-exact
        d = G.run_batch(roots[:3], options=Options(concurrency=conc, deterministic=True))
        for q, r in enumerate(roots[:3]):
            _exact(g, int(r), d[q])
        with pytest.raises(DfsError):
            G.run_batch(roots, options=Options(concurrency=conc, blocks=148))   # blocks*conc > SMs


def test_one_level_stack_and_block_claims():
    """ring_cap=2 (v1 one-level stack: every push spills) stays valid; block claims sum to the
    claims (Fig 9 task counts)."""
    g = graphgen.road(300, 200, seed=12)
    with Graph(g.row_ptr, g.col_idx) as G:
        for opts in (dict(ring_cap=2), dict(ring_cap=3, blocks=1, inter_steal=False),
                     dict(ring_cap=2, deterministic=True)):
            p, st = G.run(0, options=Options(**opts), stats=True, block_claims=True)
            r = _valid(g, 0, p)
            assert int(st.block_claims.sum()) == r.n_visited - 1
            if opts.get("deterministic"):
                _exact(g, 0, p)


def test_fault_injection_timeout_enomem_and_recovery():
    """the watchdog and pool exhaustion end the kernel with DFS_ETIMEOUT / DFS_ENOMEM
    (no hang); the same handle then runs normally again (tables cleared after errors)."""
    g = graphgen.grid(256, 256)                     # det snake keeps ~65K entries on the stack
    with Graph(g.row_ptr, g.col_idx) as G:
        with pytest.raises(DfsError) as e:
            G.run(0, options=Options(deterministic=True, max_pool_chunks=2))
        assert e.value.code == -2                                    # DFS_ENOMEM
        _exact(g, 0, G.run(0, options=det()))                      # recovers
        with pytest.raises(DfsError) as e:
            G.run(0, options=Options(deterministic=True, timeout_ms=1))
        assert e.value.code == -5                                    # DFS_ETIMEOUT
        _valid(g, 0, G.run(0))
        with pytest.raises(DfsError) as e:                           # parallel + tiny pool
            G.run(0, options=Options(max_pool_chunks=1, ring_cap=2))
        assert e.value.code == -2
        _valid(g, 5, G.run(5))
        hb = graphgen.road(600, 600, seed=2)
    with Graph(hb.row_ptr, hb.col_idx) as G:                         # batch error propagates
        with pytest.raises(DfsError):
            G.run_batch([0, 1, 2, 3], options=Options(concurrency=2, ring_cap=2, max_pool_chunks=1))
        out = G.run_batch([0, 1, 2, 3], options=Options(concurrency=2))
        for q, r in enumerate([0, 1, 2, 3]):
            _valid(hb, r, out[q])


def test_cli_on_matrix_market(tmp_path, capsys):
    """The user-facing driver (f-4): .mtx in, per-source CSV + MTEPS summary out."""
    import json as _json
    from paper_conf_ppopp_niul0c26_b200 import cli
    g = graphgen.road(64, 48, seed=6)
    p = tmp_path / "road.mtx"
    graphgen.write_mtx(g, str(p))
    out_csv = tmp_path / "perf.csv"
    npy = tmp_path / "parents.npy"
    assert cli.main(["--mtx", str(p), "--roots", "4", "--csv", str(out_csv), "--set", "hot_cutoff=4",
                     "--save-parents", str(npy)]) == 0
    summary = _json.loads(capsys.readouterr().out.strip().splitlines()[-1])
    assert summary["sources"] == 4 and summary["n"] == g.n and summary["m"] == g.m
    rows = out_csv.read_text().strip().splitlines()
    assert len(rows) == 5 and rows[0].startswith("root,n_visited")
    assert all(int(r.split(",")[1]) == g.n for r in rows[1:])          # connected: all reached
    # every tree the CLI produced from the .mtx path is a valid DFS tree of the file's graph
    gm = graphgen.read_mtx(str(p))
    assert np.array_equal(gm.row_ptr, g.row_ptr) and np.array_equal(gm.col_idx, g.col_idx)
    parents = np.load(npy)
    assert parents.shape == (4, g.n)
    for q, line in enumerate(rows[1:]):
        _valid(gm, int(line.split(",")[0]), parents[q])
    # a directed file written from shuffled lists (not symmetrised; the reader sorts rows)
    gd = graphgen.shuffle_lists(graphgen.random_graph(3000, 9000, seed=8, symmetric=False), 3)
    pd = tmp_path / "dir.mtx"
    graphgen.write_mtx(gd, str(pd))
    gdm = graphgen.read_mtx(str(pd))
    assert cli.main(["--mtx", str(pd), "--root", "0", "--root", "17", "--save-parents", str(npy)]) == 0
    capsys.readouterr()
    parents = np.load(npy)
    for q, r in enumerate((0, 17)):
        _valid(gdm, r, parents[q], undirected=False)
    # --batch: one dfs_run_batch over all sources (concurrent traversals), DFS/s summary, rows valid
    assert cli.main(["--mtx", str(p), "--roots", "6", "--batch", "--csv", str(out_csv),
                     "--save-parents", str(npy)]) == 0
    summary = _json.loads(capsys.readouterr().out.strip().splitlines()[-1])
    assert summary["batch"] is True and summary["sources"] == 6 and summary["dfs_per_s"] > 0
    rows = out_csv.read_text().strip().splitlines()
    parents = np.load(npy)
    assert len(rows) == 7 and parents.shape == (6, g.n)
    for q, line in enumerate(rows[1:]):
        r = int(line.split(",")[0])
        assert int(line.split(",")[1]) == g.n
        _valid(gm, r, parents[q])


@pytest.mark.parametrize("cl", [2, 4])
def test_cluster_tier_moves_work_through_dsmem(cl):
    """§8(f)-3: with Alg 4 and the spill off, work leaves a CTA only through the cluster tier —
    every CTA of the root's cluster claims vertices, the steals are counted, the tree is valid
    (I1-I6), and the grid is whole clusters."""
    g = graphgen.road(512, 512, seed=21)
    with Graph(g.row_ptr, g.col_idx) as G:
        o = Options(cluster=cl, inter_steal=False, spill=False, collect_stats=True)
        p, st = G.run(0, options=o, stats=True, block_claims=True)
        _valid(g, 0, p)
        assert st.cluster_steals > 0
        assert st.blocks % cl == 0
        bc = st.block_claims
        assert int(bc.sum()) == st.n_visited - 1
        assert (bc[:cl] > 0).all() and (bc[cl:] == 0).all()       # work stayed in cluster 0
        # default-tier run on the same handle, then the cluster tier on a batch
        _valid(g, 5, G.run(5))
        roots = graphgen.random_roots(g, 4, seed=cl)
        out = G.run_batch(roots, options=Options(cluster=cl, concurrency=2))
        for q, r in enumerate(roots):
            _valid(g, int(r), out[q])


def test_bulk_copy_flush_refill_exact():
    """cp.async.bulk flush/refill (TMA ablation): deterministic mode stays bit-exact on
    deep stacks that flush and refill thousands of times (odd ring_cap makes every parity of ring
    slot vs ColdSeg position occur), and parallel runs stay valid."""
    for g, root in ((graphgen.grid(256, 256), 0), (graphgen.caterpillar(4096, 94), 0),
                    (graphgen.path_chords(200_000, 2_000, seed=4), 7)):
        with Graph(g.row_ptr, g.col_idx) as G:
            for rc in (0, 7, 64, 3):
                o = Options(deterministic=True, bulk_copy=True, ring_cap=rc)
                _exact(g, root, G.run(root, options=o))
                p, st = G.run(root, options=Options(bulk_copy=True, ring_cap=rc, collect_stats=True), stats=True)
                _valid(g, root, p)


def test_two_handles_from_two_host_threads():
    """Distinct handles are independent (dfs.h): two host threads, each with its own handle and
    its own stream, run single roots and batches at the same time; every result is valid, and a
    failing call in one thread sets that thread's dfs_last_error only."""
    import threading
    graphs = [graphgen.road(300, 200, seed=21), graphgen.rmat(14, 8, seed=22)]
    errors, results = [None, None], [None, None]

    def work(t):
        try:
            g = graphs[t]
            roots = [int(x) for x in graphgen.random_roots(g, 6, seed=30 + t)]
            s = torch.cuda.Stream()
            with torch.cuda.stream(s), Graph(g.row_ptr, g.col_idx) as G:
                singles = [G.run(r).cpu().numpy() for r in roots[:3]]
                rows = G.run_batch(roots).cpu().numpy()
                lib = G._lib
                bad = lib.dfs_run_ex(G._h, g.n + 5, None, None, None)
                results[t] = (roots, singles, rows, bad, lib.dfs_last_error())
        except Exception as e:  # noqa: BLE001 — reported by the main thread
            errors[t] = e

    ths = [threading.Thread(target=work, args=(t,)) for t in range(2)]
    for th in ths:
        th.start()
    for th in ths:
        th.join(timeout=600)
    assert errors == [None, None], errors
    for t in range(2):
        g = graphs[t]
        roots, singles, rows, bad, last = results[t]
        assert bad == -1 and last == -1                       # DFS_EINVAL, this thread's code
        for r, p in zip(roots[:3], singles):
            _valid(g, r, p, undirected=True)
        for q, r in enumerate(roots):
            _valid(g, r, rows[q], undirected=True)

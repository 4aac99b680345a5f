"""Multi-process host logic of the batched multi-GPU path on CPU with gloo.

NCCL cannot put two ranks on one GPU and this CI has none, so the partition / exchange / timing
logic of paper_conf_ppopp_niul0c26_b200.batch is exercised with world_size-2 gloo process
groups and an oracle-backed runner (a test fixture; the product runner is batch.gpu_runner).
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import graphgen
import oracle
from paper_conf_ppopp_niul0c26_b200 import batch


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def test_partition_covers_every_root_once():
    for k in (0, 1, 7, 1024, 1023):
        for P in (1, 2, 3, 4, 8):
            seen = []
            for p in range(P):
                lo, hi = batch.partition(k, P, p)
                assert 0 <= lo <= hi <= k
                assert (hi - lo) in (k // P, k // P + 1)
                seen.extend(range(lo, hi))
            assert seen == list(range(k))
    with pytest.raises(ValueError):
        batch.partition(4, 2, 2)


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        g = graphgen.road(40, 30, seed=3)
        roots = graphgen.random_roots(g, 11, seed=4)
        deg = np.diff(g.row_ptr)
        local = {}

        def runner(root, qi):
            p = oracle.dfs(g.row_ptr, g.col_idx, root)
            local[qi] = p
            vis = p != -2
            return int(vis.sum()), int(deg[vis].sum()), 1.0 + rank   # fake device ms

        res = batch.run_batch(runner, roots, world=world, rank=rank)
        lo, hi = res.my_range
        rows = torch.from_numpy(np.stack([local[i] for i in range(hi - lo)])) if hi > lo else \
            torch.empty((0, g.n), dtype=torch.int32)
        parents = batch.gather_parents(rows, g.n, len(roots), world, rank, chunk=2)
        q.put((rank, res.summaries, res.my_ms, res.max_ms, parents))
    finally:
        dist.destroy_process_group()


def test_run_batch_gloo_world2():
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = [q.get(timeout=240) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    out.sort(key=lambda t: t[0])
    g = graphgen.road(40, 30, seed=3)
    roots = graphgen.random_roots(g, 11, seed=4)
    deg = np.diff(g.row_ptr)
    want = []
    for r in roots:
        p = oracle.dfs(g.row_ptr, g.col_idx, int(r))
        want.append((int(r), int((p != -2).sum()), int(deg[p != -2].sum())))
    for rank, summ, my_ms, max_ms, parents in out:
        f = batch.SUMMARY_FIELDS
        assert summ.shape == (len(roots), len(f))
        assert [int(x) for x in summ[:, f.index("root")]] == [w[0] for w in want]
        assert [int(x) for x in summ[:, f.index("n_visited")]] == [w[1] for w in want]
        assert [int(x) for x in summ[:, f.index("m_visited")]] == [w[2] for w in want]
        # rank column says who ran each root: contiguous slices
        owners = summ[:, f.index("rank")].astype(int).tolist()
        assert owners == [0] * 5 + [1] * 6
        assert max_ms == max(o[2] for o in out)
        if rank == 0:
            assert parents.shape == (len(roots), g.n)
            for q_, r in enumerate(roots):
                assert np.array_equal(parents[q_], oracle.dfs(g.row_ptr, g.col_idx, int(r)))
        else:
            assert parents is None
    res0 = batch.BatchResult(out[0][1], (0, 5), out[0][2], out[0][3])
    assert res0.dfs_per_s() == pytest.approx(len(roots) / (out[0][3] * 1e-3))


def _worker_bench_exchange(rank, world, port, q):
    """bench.py's exchange helpers: reduce_max_sum (job time = max over ranks, totals = sums)
    and gather_chunk_to_rank0 (the C5 gather of parent rows into a reused rank-0 sink), with
    uneven slices (rank 1 holds one row fewer) so the padding path runs."""
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        mx, sm = batch.reduce_max_sum([1.0 + rank, 10.0 - rank], [2.0 * rank + 1, 5.0], world)
        n, nrows, sub = 17, 7, 3
        have = nrows - rank                                    # rank 0: 7 rows, rank 1: 6
        rows = torch.arange(nrows * n, dtype=torch.int32).reshape(nrows, n) + 1000 * rank
        sink = [torch.empty((sub, n), dtype=torch.int32) for _ in range(world)] if rank == 0 else None
        received = []
        rounds = 0
        for s0 in range(0, nrows, sub):
            # one round at a time so the test can copy out what the sink received
            rounds += batch.gather_chunk_to_rank0(rows[s0:], max(0, have - s0), min(sub, nrows - s0), sub,
                                                  sink, world, rank)
            if rank == 0:
                received.append([t.clone() for t in sink])
        # the async variant (bench pass 2 overlaps it with the next chunk's traversals) delivers
        # the same rows once its work handles are waited on
        received_async = []
        for s0 in range(0, nrows, sub):
            works = batch.gather_chunk_to_rank0(rows[s0:], max(0, have - s0), min(sub, nrows - s0), sub,
                                                sink, world, rank, async_op=True)
            assert len(works) == 1
            for w, _ in works:
                w.wait()
            if rank == 0:
                received_async.append([t.clone() for t in sink])
        if rank == 0:
            assert all(all(torch.equal(x, y) for x, y in zip(ra, rs)) for ra, rs in zip(received_async, received))
        q.put((rank, mx, sm, rounds, received))
    finally:
        dist.destroy_process_group()


def test_bench_exchange_gloo_world2():
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker_bench_exchange, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = sorted([q.get(timeout=240) for _ in range(world)], key=lambda t: t[0])
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    n, nrows, sub = 17, 7, 3
    for rank, mx, sm, rounds, received in out:
        assert mx == [2.0, 10.0] and sm == [4.0, 10.0]
        assert rounds == 3
    received = out[0][4]
    for r_i, s0 in enumerate(range(0, nrows, sub)):
        for src in range(world):
            have = nrows - src
            want = torch.arange(nrows * n, dtype=torch.int32).reshape(nrows, n) + 1000 * src
            got = received[r_i][src]
            for j in range(sub):
                row = s0 + j
                if row < have and row < nrows:
                    assert torch.equal(got[j], want[row]), (r_i, src, j)
                else:
                    assert bool((got[j] == -3).all()), (r_i, src, j)

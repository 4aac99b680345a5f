"""Batched independent traversals across GPUs (BASELINE.json configs[4]).

A single traversal does not shard (every claim is a fine-grained atomic on one visited set), so
multi-GPU use is limited to batches of independent roots: every rank holds a replica of the
graph (``Graph``), roots are partitioned contiguously — rank p gets ``[p*k/P, (p+1)*k/P)`` — and
the only cross-GPU traffic is one exchange step after the traversals: an
``all_gather_into_tensor`` of fixed-size per-root summaries (NCCL over NVLink on GPUs; gloo in
the CPU tests).  Optionally the parent arrays themselves are gathered to rank 0 in chunks.

The traversal itself is ``runner(root, row)`` — on GPUs a thin wrapper around
``Graph.run`` (``dfs_run_ex``) writing into row ``row`` of a device buffer; the host logic here
(partitioning, summaries, exchange, timing reduction) is independent of it so it can be tested
with world_size-2 gloo process groups on CPU (tests/test_dist_gloo.py).
"""
from __future__ import annotations

from dataclasses import dataclass
from typing import Callable, List, Optional, Sequence, Tuple

import numpy as np

#: per-root summary columns exchanged between ranks (float64: exact for ints < 2^53)
SUMMARY_FIELDS = ("root", "rank", "n_visited", "m_visited", "ms")


def partition(num_roots: int, world: int, rank: int) -> Tuple[int, int]:
    """Contiguous slice [lo, hi) of the root list owned by ``rank`` (sizes differ by <= 1)."""
    if world <= 0 or not (0 <= rank < world) or num_roots < 0:
        raise ValueError("bad partition arguments")
    return (rank * num_roots) // world, ((rank + 1) * num_roots) // world


@dataclass
class BatchResult:
    summaries: np.ndarray        # (num_roots, len(SUMMARY_FIELDS)), in global root order
    my_range: Tuple[int, int]
    my_ms: float                 # this rank's device time for its slice
    max_ms: float                # max over ranks (the job time)

    @property
    def total_edges(self) -> float:
        return float(self.summaries[:, SUMMARY_FIELDS.index("m_visited")].sum())

    def gteps(self) -> float:
        return self.total_edges / (self.max_ms * 1e-3) / 1e9

    def dfs_per_s(self) -> float:
        return self.summaries.shape[0] / (self.max_ms * 1e-3)


def run_batch(runner: Callable[[int, int], Tuple[int, int, float]], roots: Sequence[int],
              world: int = 1, rank: int = 0, group=None, device=None) -> BatchResult:
    """Run this rank's slice of ``roots`` and exchange summaries with every rank.

    ``runner(root, local_index) -> (n_visited, m_visited, ms)``.  With ``world > 1`` a
    ``torch.distributed`` process group must be initialised; ``device`` is where the exchange
    tensors live (a CUDA device for NCCL, CPU for gloo).
    """
    import torch
    k = len(roots)
    lo, hi = partition(k, world, rank)
    rows: List[List[float]] = []
    my_ms = 0.0
    for q, r in enumerate(roots[lo:hi]):
        nv, mv, ms = runner(int(r), q)
        my_ms += float(ms)
        rows.append([float(r), float(rank), float(nv), float(mv), float(ms)])
    nf = len(SUMMARY_FIELDS)
    dev = device if device is not None else torch.device("cpu")
    if world == 1:
        return BatchResult(np.asarray(rows, dtype=np.float64).reshape(-1, nf), (lo, hi), my_ms, my_ms)
    import torch.distributed as dist
    # fixed-size exchange: pad every rank's block to the largest slice
    cap = max(partition(k, world, p)[1] - partition(k, world, p)[0] for p in range(world))
    mine = torch.full((cap, nf), -1.0, dtype=torch.float64, device=dev)
    if rows:
        mine[:len(rows)] = torch.tensor(rows, dtype=torch.float64, device=dev)
    allb = torch.empty((world * cap, nf), dtype=torch.float64, device=dev)
    dist.all_gather_into_tensor(allb, mine, group=group)
    t = torch.tensor([my_ms], dtype=torch.float64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    allb = allb.cpu().numpy()
    out = np.empty((k, nf), dtype=np.float64)
    for p in range(world):
        plo, phi = partition(k, world, p)
        out[plo:phi] = allb[p * cap:p * cap + (phi - plo)]
    return BatchResult(out, (lo, hi), my_ms, float(t.item()))


def gather_parents(local_rows, n: int, num_roots: int, world: int, rank: int, group=None,
                   dst: int = 0, chunk: int = 8):
    """Optionally gather full parent arrays (num_roots x n int32) to rank ``dst`` in chunks of
    ``chunk`` rows per rank (bounded buffer), returning the array on ``dst`` and None elsewhere.
    ``local_rows`` is this rank's (hi-lo, n) int32 tensor."""
    import torch
    import torch.distributed as dist
    lo, hi = partition(num_roots, world, rank)
    if world == 1:
        return local_rows.cpu().numpy() if rank == dst else None
    out = np.empty((num_roots, n), dtype=np.int32) if rank == dst else None
    cap = max(partition(num_roots, world, p)[1] - partition(num_roots, world, p)[0] for p in range(world))
    for c0 in range(0, cap, chunk):
        rows = min(chunk, cap - c0)
        buf = torch.full((rows, n), -3, dtype=torch.int32, device=local_rows.device)
        have = max(0, min(rows, (hi - lo) - c0))
        if have > 0:
            buf[:have] = local_rows[c0:c0 + have]
        gl = [torch.empty_like(buf) for _ in range(world)] if rank == dst else None
        dist.gather(buf, gather_list=gl, dst=dst, group=group)
        if rank == dst:
            for p in range(world):
                plo, phi = partition(num_roots, world, p)
                take = max(0, min(rows, (phi - plo) - c0))
                if take:
                    out[plo + c0:plo + c0 + take] = gl[p][:take].cpu().numpy()
    return out


def gpu_runner(G, out_rows, collect: Optional[list] = None):
    """runner for ``run_batch`` backed by the library: Graph.run (dfs_run_ex) into row q of
    ``out_rows`` (a (rows, n) int32 CUDA tensor, reused modulo rows); stats give n_visited,
    m_visited and the device time of the call."""
    def run(root: int, q: int):
        row = out_rows[q % out_rows.shape[0]]
        _, st = G.run(root, out=row, stats=True)
        if collect is not None:
            collect.append(st)
        return st.n_visited, st.m_visited, st.kernel_ms
    return run


def run_batch_chunked(G, out_rows, roots, world: int = 1, rank: int = 0, group=None, device=None,
                      concurrency: int = 1) -> BatchResult:
    """GPU batch: this rank's slice goes to ``dfs_run_batch_ex`` in chunks of
    ``out_rows.shape[0]`` roots with ``concurrency`` traversals in flight (§8(f)-2).  Per-root
    (n_visited, m_visited) come from the library's per-root counts; a chunk's device time (CUDA
    events) is attributed evenly to its roots.  Then the summaries are exchanged (run_batch)."""
    from .dfs import Options
    k = len(roots)
    lo, hi = partition(k, world, rank)
    mine = [int(r) for r in roots[lo:hi]]
    rows = out_rows.shape[0]
    results = []
    for c0 in range(0, len(mine), rows):
        chunk = mine[c0:c0 + rows]
        _, st = G.run_batch(chunk, out=out_rows[:len(chunk)], options=Options(concurrency=concurrency),
                            stats=True)
        share = st.kernel_ms / len(chunk)
        for q in range(len(chunk)):
            results.append((int(st.root_counts[q, 0]), int(st.root_counts[q, 1]), share))
    it = iter(results)
    return run_batch(lambda root, q: next(it), roots, world=world, rank=rank, group=group, device=device)


def reduce_max_sum(maxvals: Sequence[float], sumvals: Sequence[float], world: int, device=None,
                   group=None) -> Tuple[List[float], List[float]]:
    """Job-level reduction of per-rank figures (bench.py): element-wise MAX over ranks of
    ``maxvals`` (device times: the job takes as long as its slowest rank) and SUM of ``sumvals``
    (edges, bytes, counts).  One all_reduce each; identity for world == 1."""
    if world == 1:
        return [float(x) for x in maxvals], [float(x) for x in sumvals]
    import torch
    import torch.distributed as dist
    dev = device if device is not None else torch.device("cpu")
    tm = torch.tensor([float(x) for x in maxvals], dtype=torch.float64, device=dev)
    ts = torch.tensor([float(x) for x in sumvals], dtype=torch.float64, device=dev)
    dist.all_reduce(tm, op=dist.ReduceOp.MAX, group=group)
    dist.all_reduce(ts, op=dist.ReduceOp.SUM, group=group)
    return tm.cpu().tolist(), ts.cpu().tolist()


def gather_chunk_to_rank0(rows, have: int, nrows: int, sub: int, sink, world: int, rank: int,
                          group=None, dst: int = 0, async_op: bool = False):
    """The C5 exchange step for one chunk of parent rows (bench.py batch pass 2): every rank
    sends rows [0, nrows) of ``rows`` (a (>= nrows, n) int32 tensor whose first ``have`` rows are
    valid; the rest are sent as -3 padding so every rank makes the same calls) to ``dst`` in
    rounds of ``sub`` rows; ``dst`` receives each round into ``sink`` (world tensors of
    (sub, n) — a reused buffer: the result sink).  Returns the number of rounds (the same on
    every rank).  Tensors live on the process group's device (CUDA for NCCL, CPU for gloo).

    ``async_op=True`` returns the list of the rounds' work handles instead: with NCCL the
    gathers then run on the communicator's stream while the caller launches the next chunk's
    traversals (``rows`` must stay untouched until the handles are waited on)."""
    import torch
    import torch.distributed as dist
    rounds = 0
    works = []
    n = rows.shape[1]
    for s0 in range(0, nrows, sub):
        take = max(0, min(sub, have - s0))
        if take == sub:
            src = rows[s0:s0 + sub]
        else:
            src = torch.full((sub, n), -3, dtype=rows.dtype, device=rows.device)
            if take > 0:
                src[:take] = rows[s0:s0 + take]
        w = dist.gather(src.contiguous(), gather_list=sink if rank == dst else None, dst=dst, group=group,
                        async_op=async_op)
        if async_op:
            works.append((w, src))                     # keep the padded source alive
        rounds += 1
    return works if async_op else rounds

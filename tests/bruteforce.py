"""Brute-force enumerators on tiny graphs (<= 8 vertices), used to pin the oracle's checker.

None of these share code with oracle/ or with the CUDA path; they are written out from the
definitions:

* classical_trees     — every tree Alg 1 can produce under SOME permutation of the
                        adjacency lists.  Enumerated as nondeterministic DFS: at each step the top
                        vertex may descend into ANY currently-unvisited out-neighbour, and pops
                        when none is left (equivalent to ranging over all list permutations).
* async_scan_outcomes — the model I6 describes: every claimed vertex owns a scanner walking its
                        list in CSR order; scanners interleave arbitrarily; a position whose target
                        is unclaimed claims it (atomic claim).
* stealing_outcomes   — k agents each running Alg 1 on a private stack; an idle agent may steal
                        the bottom (oldest) entry of another agent's stack (Alg 2-4 skeleton,
                        P:249-286).
* arborescences       — every candidate parent array: unreachable = -2, root = -1, each other
                        reachable vertex gets any in-neighbour (includes cyclic/invalid ones).
"""
from __future__ import annotations

import itertools
from typing import FrozenSet, Tuple

import numpy as np

UNR = -2


def lists(row_ptr, col_idx):
    n = len(row_ptr) - 1
    return [tuple(int(x) for x in col_idx[row_ptr[u]:row_ptr[u + 1]]) for u in range(n)]


def reach_set(adj, root):
    seen = {root}
    st = [root]
    while st:
        u = st.pop()
        for v in adj[u]:
            if v not in seen:
                seen.add(v)
                st.append(v)
    return seen


def classical_trees(adj, root) -> FrozenSet[Tuple[int, ...]]:
    n = len(adj)
    out = set()

    def rec(parent, stack):
        # pop exhausted tops (no unvisited neighbour left)
        stack = list(stack)
        while stack:
            u = stack[-1]
            cand = sorted({v for v in adj[u] if parent[v] == UNR and v != root})
            if cand:
                for v in cand:
                    p2 = list(parent)
                    p2[v] = u
                    rec(tuple(p2), tuple(stack) + (v,))
                return
            stack.pop()
        out.add(parent)

    p0 = [UNR] * n
    p0[root] = -1
    rec(tuple(p0), (root,))
    return frozenset(out)


def async_scan_outcomes(adj, root) -> FrozenSet[Tuple[int, ...]]:
    n = len(adj)
    p0 = [UNR] * n
    p0[root] = -1
    start = (tuple(p0), tuple([0] * n))
    seen = {start}
    todo = [start]
    out = set()
    while todo:
        parent, ptr = todo.pop()
        moved = False
        for u in range(n):
            if parent[u] == UNR or ptr[u] >= len(adj[u]):
                continue
            moved = True
            v = adj[u][ptr[u]]
            p2 = list(parent)
            if p2[v] == UNR:
                p2[v] = u
            q2 = list(ptr)
            q2[u] += 1
            s = (tuple(p2), tuple(q2))
            if s not in seen:
                seen.add(s)
                todo.append(s)
        if not moved:
            out.add(parent)
    return frozenset(out)


def stealing_outcomes(adj, root, k: int) -> FrozenSet[Tuple[int, ...]]:
    n = len(adj)
    p0 = [UNR] * n
    p0[root] = -1
    stacks0 = [((root, 0),)] + [()] * (k - 1)
    start = (tuple(p0), tuple(stacks0))
    seen = {start}
    todo = [start]
    out = set()
    while todo:
        parent, stacks = todo.pop()
        succ = []
        for a in range(k):
            st = stacks[a]
            if st:
                u, i = st[-1]
                p2 = list(parent)
                if i < len(adj[u]):
                    v = adj[u][i]
                    ns = st[:-1] + ((u, i + 1),)
                    if p2[v] == UNR:
                        p2[v] = u
                        ns = ns + ((v, 0),)
                else:
                    ns = st[:-1]
                s2 = list(stacks)
                s2[a] = ns
                succ.append((tuple(p2), tuple(s2)))
            else:
                for b in range(k):
                    if b != a and stacks[b]:
                        s2 = list(stacks)
                        s2[a] = (stacks[b][0],)
                        s2[b] = stacks[b][1:]
                        succ.append((parent, tuple(s2)))
        if not any(stacks):
            out.add(parent)
        for s in succ:
            if s not in seen:
                seen.add(s)
                todo.append(s)
    return frozenset(out)


def arborescences(adj, root):
    n = len(adj)
    R = reach_set(adj, root)
    inn = [[] for _ in range(n)]
    for u in range(n):
        if u in R:
            for v in set(adj[u]):
                inn[v].append(u)
    choices = []
    for v in range(n):
        if v == root:
            choices.append([-1])
        elif v in R:
            choices.append(sorted(set(inn[v])))
        else:
            choices.append([UNR])
    for combo in itertools.product(*choices):
        yield tuple(combo)


def random_tiny_graph(rng, n, p, directed, self_loops=False):
    src, dst = [], []
    for u in range(n):
        for v in range(n):
            if u == v and not self_loops:
                continue
            if not directed and v <= u:
                continue
            if rng.random() < p:
                src.append(u)
                dst.append(v)
                if not directed and u != v:
                    src.append(v)
                    dst.append(u)
    order = np.lexsort((np.array(dst), np.array(src))) if src else np.array([], dtype=int)
    src = np.array(src, dtype=np.int64)[order] if len(order) else np.array([], dtype=np.int64)
    dst = np.array(dst, dtype=np.int64)[order] if len(order) else np.array([], dtype=np.int64)
    row_ptr = np.zeros(n + 1, dtype=np.int64)
    np.add.at(row_ptr, src + 1, 1)
    row_ptr = np.cumsum(row_ptr)
    col = dst.astype(np.int32)
    # random list order per vertex: CSR order != sorted order
    for u in range(n):
        a, b = row_ptr[u], row_ptr[u + 1]
        col[a:b] = rng.permutation(col[a:b])
    return row_ptr, col

"""Seeded synthetic CSR graph generators (input side only; no DFS arithmetic).

Shared by both sides of the parity tests -- the oracle (``oracle/``) and the CUDA path
(``paper_conf_ppopp_niul0c26_b200``) -- as the build rules allow for input generators.
Recipes and the configs they reproduce are listed in DESIGN.md §"Input recipe":

* C1 ``grid(256, 256)``                       (BASELINE.json configs[0])
* C2 ``road(4900, 4900, seed=0x5EED)``         (configs[1]; DIMACS10-road-like)
* C3 ``rmat(24, 16)``                          (configs[2]; Graph500 Kronecker, SNAP/LAW-like)
* C4a ``path_chords(10**8, 10**6)``, C4b ``caterpillar(2**20, 94)``  (configs[3])
* C5 ``road`` + ``random_roots(.., 1024)``     (configs[4])
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "graphgen.c")
_SO = os.path.join(_HERE, "libgraphgen.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile libgraphgen.so with gcc (portable flags: the .so travels to the GPU box)."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        tmp = _SO + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O3", "-fopenmp", "-shared", "-fPIC", _SRC, "-o", tmp])
        os.replace(tmp, _SO)
    return _SO


def _L():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        P, I64, U64, D, I = ctypes.c_void_p, ctypes.c_int64, ctypes.c_uint64, ctypes.c_double, ctypes.c_int
        for name, args in {
            "gg_grid": [I64, I64],
            "gg_road": [I64, I64, U64, D],
            "gg_rmat": [I, I64, D, D, D, U64],
            "gg_path_chords": [I64, I64, U64],
            "gg_caterpillar": [I64, I64],
            "gg_random": [I64, I64, U64, I, I, I],
            "gg_from_edges": [I64, I64, P, P, I, I, I],
            "gg_read_mtx": [ctypes.c_char_p, I],
        }.items():
            f = getattr(lib, name)
            f.argtypes = args
            f.restype = P
        lib.gg_n.argtypes = [P]; lib.gg_n.restype = I64
        lib.gg_m.argtypes = [P]; lib.gg_m.restype = I64
        lib.gg_export.argtypes = [P, P, P]; lib.gg_export.restype = None
        lib.gg_destroy.argtypes = [P]; lib.gg_destroy.restype = None
        lib.gg_write_mtx.argtypes = [ctypes.c_char_p, I64, P, P]; lib.gg_write_mtx.restype = I
        _lib = lib
    return _lib


@dataclass
class CSR:
    """Directed out-adjacency: row_ptr int64[n+1], col_idx int32[m]."""
    row_ptr: np.ndarray
    col_idx: np.ndarray
    name: str = ""

    @property
    def n(self) -> int:
        return int(self.row_ptr.shape[0] - 1)

    @property
    def m(self) -> int:
        return int(self.col_idx.shape[0])

    def degree(self) -> np.ndarray:
        return np.diff(self.row_ptr)


def _take(h, name: str) -> CSR:
    lib = _L()
    if not h:
        raise MemoryError(f"graphgen: {name} failed")
    try:
        n, m = lib.gg_n(h), lib.gg_m(h)
        rp = np.empty(n + 1, dtype=np.int64)
        ci = np.empty(max(m, 0), dtype=np.int32)
        lib.gg_export(h, rp.ctypes.data, ci.ctypes.data)
    finally:
        lib.gg_destroy(h)
    return CSR(rp, ci, name)


def grid(W: int, H: int) -> CSR:
    return _take(_L().gg_grid(W, H), f"grid{W}x{H}")


def road(W: int, H: int, seed: int = 0x5EED, extra: float = 0.2) -> CSR:
    return _take(_L().gg_road(W, H, seed, extra), f"road{W}x{H}")


def rmat(scale: int, ef: int = 16, A: float = 0.57, B: float = 0.19, C: float = 0.19,
         seed: int = 0xC0FFEE) -> CSR:
    return _take(_L().gg_rmat(scale, ef, A, B, C, seed), f"rmat{scale}")


def path_chords(n: int, nchords: int, seed: int = 0xC4A) -> CSR:
    return _take(_L().gg_path_chords(n, nchords, seed), f"path{n}+{nchords}")


def caterpillar(spine: int, leaves: int) -> CSR:
    return _take(_L().gg_caterpillar(spine, leaves), f"caterpillar{spine}x{leaves}")


def random_graph(n: int, ne: int, seed: int, symmetric: bool = True, allow_self: bool = False,
                 allow_dup: bool = False) -> CSR:
    return _take(_L().gg_random(n, ne, seed, int(symmetric), int(allow_self), int(allow_dup)),
                 f"random{n}_{ne}")


def from_edges(n: int, src, dst, symmetrize: bool = True, dedup: bool = True,
               drop_self: bool = True) -> CSR:
    s = np.ascontiguousarray(src, dtype=np.int32)
    d = np.ascontiguousarray(dst, dtype=np.int32)
    return _take(_L().gg_from_edges(n, s.shape[0], s.ctypes.data, d.ctypes.data,
                                    int(symmetrize), int(dedup), int(drop_self)), "edges")


def read_mtx(path: str, symmetric: bool = False) -> CSR:
    """Matrix Market coordinate file -> CSR (1-based entries i j = edge i-1 -> j-1; symmetric
    files store both directions; self loops / duplicates dropped).  The paper's artifact runs on
    SuiteSparse .mtx graphs."""
    h = _L().gg_read_mtx(os.fsencode(path), int(symmetric))
    if not h:
        raise ValueError(f"graphgen: cannot parse Matrix Market file {path}")
    return _take(h, os.path.basename(path))


def write_mtx(g: CSR, path: str) -> None:
    rp = np.ascontiguousarray(g.row_ptr, dtype=np.int64)
    ci = np.ascontiguousarray(g.col_idx, dtype=np.int32)
    if _L().gg_write_mtx(os.fsencode(path), g.n, rp.ctypes.data, ci.ctypes.data if g.m else None) != 0:
        raise OSError(f"cannot write {path}")


def path(n: int) -> CSR:
    i = np.arange(n - 1)
    return from_edges(n, i, i + 1)


def star(n: int) -> CSR:
    """Centre 0, leaves 1..n-1."""
    return from_edges(n, np.zeros(n - 1, dtype=np.int64), np.arange(1, n))


def binary_tree(n: int) -> CSR:
    """Complete binary tree in heap order: parent of i is (i-1)//2."""
    i = np.arange(1, n)
    return from_edges(n, (i - 1) // 2, i)


def shuffle_lists(g: CSR, seed: int) -> CSR:
    """Same graph with every adjacency list permuted (CSR order != sorted order)."""
    rng = np.random.default_rng(seed)
    col = g.col_idx.copy()
    for u in range(g.n):
        a, b = int(g.row_ptr[u]), int(g.row_ptr[u + 1])
        if b - a > 1:
            col[a:b] = rng.permutation(col[a:b])
    return CSR(g.row_ptr.copy(), col, g.name + "~shuf")


def random_roots(g: CSR, k: int, seed: int = 0x600D, min_degree: int = 1) -> np.ndarray:
    """k distinct seeded roots with out-degree >= min_degree (GAP-style sources)."""
    deg = g.degree()
    cand = np.nonzero(deg >= min_degree)[0]
    rng = np.random.default_rng(seed)
    if k <= cand.shape[0]:
        pick = rng.choice(cand.shape[0], size=k, replace=False)
    else:
        pick = rng.integers(0, cand.shape[0], size=k)
    return cand[pick].astype(np.int32)


# --------------------------------------------------------------------------------------------
# Named configs (BASELINE.json "configs"), full size and a reduced "ci" size for tests.
# --------------------------------------------------------------------------------------------
CONFIGS = {
    "grid256": dict(builder=lambda: grid(256, 256), root=0, undirected=True,
                    desc="C1 undirected 2-D grid 256x256, root 0"),
    "road24m": dict(builder=lambda: road(4900, 4900), root=0, undirected=True,
                    desc="C2 road-maze 4900x4900 (24.01M vertices, avg deg 2.4), root 0"),
    "rmat24": dict(builder=lambda: rmat(24, 16), root=None, undirected=True,
                   desc="C3 RMAT scale 24 edge factor 16 (Graph500 A,B,C=.57,.19,.19)"),
    "path100m": dict(builder=lambda: path_chords(10**8, 10**6), root=0, undirected=True,
                     desc="C4a 10^8-vertex path + 10^6 random chords, root 0"),
    "caterpillar": dict(builder=lambda: caterpillar(2**20, 94), root=0, undirected=True,
                        desc="C4b caterpillar spine 2^20 x 94 leaves (99.6M vertices), root 0"),
}


def config_graph(name: str):
    """Returns (CSR, root, undirected, desc).  RMAT's root: seeded vertex with degree > 0."""
    c = CONFIGS[name]
    g = c["builder"]()
    root = c["root"]
    if root is None:
        root = int(random_roots(g, 1, seed=0x24)[0])
    return g, int(root), c["undirected"], c["desc"]

"""CPU oracle for unordered DFS — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product path
(``paper_conf_ppopp_niul0c26_b200``) never imports it and shares no code with it.

* :func:`dfs` — Algorithm 1 of the paper, in plain C (``dfs_oracle.c``).
* :func:`reach` — textbook BFS reachability.
* :func:`check_tree` — exact acceptance checks I1-I7 (reading S1).

Pins: ``tests/test_oracle_pins.py`` and ``tests/test_checker_bruteforce.py``.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "dfs_oracle.c")
_HDR = os.path.join(_HERE, "dfs_oracle.h")
_SO = os.path.join(_HERE, "liboracle.so")
_lib = None

ROOT_PARENT = -1
UNREACHED = -2


def build(force: bool = False) -> str:
    """gcc -O3 (generic x86-64: the .so may run on another host)."""
    newest = max(os.path.getmtime(_SRC), os.path.getmtime(_HDR))
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < newest:
        tmp = _SO + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O3", "-shared", "-fPIC", _SRC, "-o", tmp])
        os.replace(tmp, _SO)
    return _SO


class _Res(ctypes.Structure):
    _fields_ = [("ok_i1", ctypes.c_int32), ("ok_i2", ctypes.c_int32), ("ok_i3", ctypes.c_int32),
                ("ok_i4", ctypes.c_int32), ("ok_i5", ctypes.c_int32), ("ok_i6", ctypes.c_int32),
                ("ok_i7", ctypes.c_int32), ("pad", ctypes.c_int32),
                ("n_visited", ctypes.c_int64), ("m_visited", ctypes.c_int64),
                ("n_cross", ctypes.c_int64), ("bad_vertex", ctypes.c_int64)]


def _L():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        P, I64, I32, I = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32, ctypes.c_int
        lib.oracle_dfs.argtypes = [I64, P, P, I32, P]; lib.oracle_dfs.restype = I64
        lib.oracle_reach.argtypes = [I64, P, P, I32, P]; lib.oracle_reach.restype = I64
        lib.oracle_check_tree.argtypes = [I64, P, P, I32, P, I, ctypes.POINTER(_Res)]
        lib.oracle_check_tree.restype = I
        _lib = lib
    return _lib


def _csr(row_ptr, col_idx):
    rp = np.ascontiguousarray(row_ptr, dtype=np.int64)
    ci = np.ascontiguousarray(col_idx, dtype=np.int32)
    if ci.shape[0] == 0:
        ci = np.zeros(1, dtype=np.int32)   # valid pointer for m = 0
    return rp, ci


def dfs(row_ptr, col_idx, root: int) -> np.ndarray:
    """Alg 1: the unique lexicographic (CSR-order) DFS tree.  parent[root] = -1, unreached = -2."""
    rp, ci = _csr(row_ptr, col_idx)
    n = rp.shape[0] - 1
    parent = np.empty(n, dtype=np.int32)
    r = _L().oracle_dfs(n, rp.ctypes.data, ci.ctypes.data, int(root), parent.ctypes.data)
    if r < 0:
        raise ValueError("oracle_dfs: invalid arguments")
    return parent


def reach(row_ptr, col_idx, root: int) -> np.ndarray:
    rp, ci = _csr(row_ptr, col_idx)
    n = rp.shape[0] - 1
    vis = np.empty(n, dtype=np.uint8)
    if _L().oracle_reach(n, rp.ctypes.data, ci.ctypes.data, int(root), vis.ctypes.data) < 0:
        raise ValueError("oracle_reach: invalid arguments")
    return vis.astype(bool)


@dataclass
class CheckResult:
    ok: bool
    i1: int
    i2: int
    i3: int
    i4: int
    i5: int
    i6: int
    i7: int
    n_visited: int
    m_visited: int
    n_cross: int
    bad_vertex: int

    def failed(self):
        return [k for k in ("i1", "i2", "i3", "i4", "i5", "i6", "i7") if getattr(self, k) == 0]


def check_tree(row_ptr, col_idx, root: int, parent, i7: bool = False,
               undirected: bool = False) -> CheckResult:
    """Exact checks I1-I6 (+ I7 if requested).  ok iff every computed check holds."""
    rp, ci = _csr(row_ptr, col_idx)
    n = rp.shape[0] - 1
    par = np.ascontiguousarray(parent, dtype=np.int32)
    assert par.shape[0] == n
    flags = (1 if i7 else 0) | (2 if undirected else 0)
    res = _Res()
    r = _L().oracle_check_tree(n, rp.ctypes.data, ci.ctypes.data, int(root), par.ctypes.data,
                               flags, ctypes.byref(res))
    if r < 0:
        raise ValueError("oracle_check_tree: invalid arguments or out of memory")
    return CheckResult(r == 1, res.ok_i1, res.ok_i2, res.ok_i3, res.ok_i4, res.ok_i5, res.ok_i6,
                       res.ok_i7, res.n_visited, res.m_visited, res.n_cross, res.bad_vertex)

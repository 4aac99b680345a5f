"""ctypes binding of libdfs.so (include/dfs.h) — argument marshalling only.

PyTorch supplies device memory, the current CUDA stream and (in bench.py) process groups; the
traversal itself is the persistent sm_100a kernel behind ``dfs_run``/``dfs_run_batch``.
Function names follow the C ABI: :meth:`Graph.run` -> ``dfs_run_ex``, :meth:`Graph.run_batch`
-> ``dfs_run_batch_ex``, construction -> ``dfs_graph_create``, :meth:`Graph.close` ->
``dfs_graph_destroy``.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass, fields
from typing import Optional

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# DFS_LIB: an alternative build of the same library (A/B experiments, scripts/ab_libs.py)
_SO = os.environ.get("DFS_LIB") or os.path.join(_HERE, "libdfs.so")

DFS_ROOT_PARENT = -1
DFS_UNREACHED = -2

STATUS = {0: "DFS_OK", -1: "DFS_EINVAL", -2: "DFS_ENOMEM", -3: "DFS_ECUDA", -4: "DFS_EDEVICE",
          -5: "DFS_ETIMEOUT", -6: "DFS_EINTERNAL"}

#: every symbol include/dfs.h declares (checked by tests/test_capi.py)
EXPORTS = ["dfs_options_default", "dfs_graph_create", "dfs_run", "dfs_run_batch", "dfs_run_ex",
           "dfs_run_batch_ex", "dfs_set_stream", "dfs_graph_info", "dfs_launch_count",
           "dfs_graph_destroy", "dfs_last_error", "dfs_strerror", "dfs_debug_timeline",
           "dfs_debug_stack_script"]


class DfsError(RuntimeError):
    def __init__(self, code: int, what: str = ""):
        self.code = code
        super().__init__(f"{what}: {STATUS.get(code, code)} ({_strerror(code)})")


class _Options(ctypes.Structure):
    _fields_ = [("blocks", ctypes.c_int32), ("warps_per_block", ctypes.c_int32),
                ("hot_cutoff", ctypes.c_int32), ("cold_cutoff", ctypes.c_int32),
                ("deterministic", ctypes.c_int32), ("intra_steal", ctypes.c_int32),
                ("inter_steal", ctypes.c_int32), ("victim_policy", ctypes.c_int32),
                ("timeout_ms", ctypes.c_int32), ("seed", ctypes.c_uint32),
                ("collect_stats", ctypes.c_int32), ("spill", ctypes.c_int32),
                ("inter_any", ctypes.c_int32), ("spill_idle", ctypes.c_int32),
                ("backoff_max_ns", ctypes.c_int32), ("window", ctypes.c_int32),
                ("pub_batch", ctypes.c_int32), ("speculate", ctypes.c_int32),
                ("steal_half", ctypes.c_int32), ("concurrency", ctypes.c_int32),
                ("ring_cap", ctypes.c_int32), ("backoff_min_ns", ctypes.c_int32),
                ("max_pool_chunks", ctypes.c_int32), ("reserved0", ctypes.c_int32),
                ("leaf_skip", ctypes.c_int32), ("cluster", ctypes.c_int32),
                ("cluster_late", ctypes.c_int32), ("steal_tries", ctypes.c_int32),
                ("bulk_copy", ctypes.c_int32), ("spill_period", ctypes.c_int32),
                ("l2_persist_mb", ctypes.c_int32), ("walker_lanes", ctypes.c_int32),
                ("steal_period", ctypes.c_int32), ("donate", ctypes.c_int32),
                ("records", ctypes.c_int32)]


class _Stats(ctypes.Structure):
    _fields_ = [("kernel_ms", ctypes.c_float), ("traversal_ms", ctypes.c_float),
                ("blocks", ctypes.c_int32), ("warps_per_block", ctypes.c_int32),
                ("n_visited", ctypes.c_int64), ("m_visited", ctypes.c_int64),
                ("claims", ctypes.c_int64), ("failed_claims", ctypes.c_int64),
                ("flushes", ctypes.c_int64), ("refills", ctypes.c_int64),
                ("intra_steals", ctypes.c_int64), ("inter_steals", ctypes.c_int64),
                ("steal_attempts", ctypes.c_int64), ("chunks_allocated", ctypes.c_int64),
                ("windows", ctypes.c_int64), ("idle_ns", ctypes.c_int64),
                ("inter_scans", ctypes.c_int64), ("spills", ctypes.c_int64),
                ("cyc_window", ctypes.c_int64), ("cyc_probe", ctypes.c_int64),
                ("cyc_claim", ctypes.c_int64), ("cyc_tail", ctypes.c_int64),
                ("cyc_outside", ctypes.c_int64), ("root_counts", ctypes.c_void_p),
                ("block_claims", ctypes.c_void_p), ("cluster_steals", ctypes.c_int64),
                ("pops", ctypes.c_int64), ("dead_pops", ctypes.c_int64), ("donations", ctypes.c_int64),
                ("walker_lanes", ctypes.c_int32), ("window", ctypes.c_int32)]


@dataclass
class Options:
    """Mirror of ``struct dfs_options`` (None = library default)."""
    blocks: Optional[int] = None
    warps_per_block: Optional[int] = None
    hot_cutoff: Optional[int] = None
    cold_cutoff: Optional[int] = None
    deterministic: Optional[bool] = None
    intra_steal: Optional[bool] = None
    inter_steal: Optional[bool] = None
    victim_policy: Optional[int] = None
    timeout_ms: Optional[int] = None
    seed: Optional[int] = None
    collect_stats: Optional[bool] = None
    spill: Optional[bool] = None
    inter_any: Optional[bool] = None
    spill_idle: Optional[int] = None
    backoff_max_ns: Optional[int] = None
    window: Optional[int] = None
    pub_batch: Optional[int] = None
    speculate: Optional[int] = None
    steal_half: Optional[bool] = None
    concurrency: Optional[int] = None
    ring_cap: Optional[int] = None
    backoff_min_ns: Optional[int] = None
    max_pool_chunks: Optional[int] = None
    leaf_skip: Optional[bool] = None
    cluster: Optional[int] = None
    cluster_late: Optional[bool] = None
    steal_tries: Optional[int] = None
    bulk_copy: Optional[bool] = None
    spill_period: Optional[int] = None
    l2_persist_mb: Optional[int] = None
    walker_lanes: Optional[int] = None
    steal_period: Optional[int] = None
    donate: Optional[bool] = None
    records: Optional[bool] = None

    def to_c(self) -> _Options:
        o = _Options()
        load_library().dfs_options_default(ctypes.byref(o))
        for f in fields(self):
            v = getattr(self, f.name)
            if v is not None:
                setattr(o, f.name, int(v))
        return o


@dataclass
class Stats:
    kernel_ms: float
    traversal_ms: float
    blocks: int
    warps_per_block: int
    n_visited: int
    m_visited: int
    claims: int
    failed_claims: int
    flushes: int
    refills: int
    intra_steals: int
    inter_steals: int
    steal_attempts: int
    chunks_allocated: int
    windows: int
    idle_ns: int
    inter_scans: int
    spills: int
    cyc_window: int
    cyc_probe: int
    cyc_claim: int
    cyc_tail: int
    cyc_outside: int
    cluster_steals: int = 0
    pops: int = 0
    dead_pops: int = 0
    donations: int = 0
    walker_lanes: int = 32
    window: int = 32
    root_counts: Optional[np.ndarray] = None
    block_claims: Optional[np.ndarray] = None


_lib = None


def lib_path() -> str:
    return _SO


def load_library(path: Optional[str] = None):
    """Load libdfs.so; raises if it is missing (no fallback path exists).  ``path`` loads another
    build of the same library without caching it (A/B experiments)."""
    global _lib
    if path is not None or _lib is None:
        so = path or _SO
        if not os.path.exists(so):
            raise ImportError(f"{so} is missing: run `python __graft_entry__.py` (build()) first; "
                              "there is no CPU fallback")
        lib = ctypes.CDLL(so)
        P, I32, I64 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64
        lib.dfs_options_default.argtypes = [ctypes.POINTER(_Options)]
        lib.dfs_options_default.restype = None
        lib.dfs_graph_create.argtypes = [P, P, I64, I64]
        lib.dfs_graph_create.restype = P
        lib.dfs_run.argtypes = [P, I32, P]
        lib.dfs_run.restype = ctypes.c_int
        lib.dfs_run_batch.argtypes = [P, P, I32, P]
        lib.dfs_run_batch.restype = ctypes.c_int
        lib.dfs_run_ex.argtypes = [P, I32, P, ctypes.POINTER(_Options), ctypes.POINTER(_Stats)]
        lib.dfs_run_ex.restype = ctypes.c_int
        lib.dfs_run_batch_ex.argtypes = [P, P, I32, P, ctypes.POINTER(_Options), ctypes.POINTER(_Stats)]
        lib.dfs_run_batch_ex.restype = ctypes.c_int
        lib.dfs_set_stream.argtypes = [P, P]
        lib.dfs_set_stream.restype = ctypes.c_int
        lib.dfs_graph_info.argtypes = [P, ctypes.POINTER(I64), ctypes.POINTER(I64), ctypes.POINTER(I32)]
        lib.dfs_graph_info.restype = ctypes.c_int
        lib.dfs_launch_count.argtypes = [P]
        lib.dfs_launch_count.restype = I64
        lib.dfs_debug_timeline.argtypes = [P, ctypes.c_uint32, ctypes.c_uint32, P]
        lib.dfs_debug_timeline.restype = ctypes.c_int
        lib.dfs_debug_stack_script.argtypes = [P, I32, P, I32, P, I32, ctypes.POINTER(_Options)]
        lib.dfs_debug_stack_script.restype = ctypes.c_int
        lib.dfs_graph_destroy.argtypes = [P]
        lib.dfs_graph_destroy.restype = None
        lib.dfs_last_error.argtypes = []
        lib.dfs_last_error.restype = ctypes.c_int
        lib.dfs_strerror.argtypes = [ctypes.c_int]
        lib.dfs_strerror.restype = ctypes.c_char_p
        if path is not None:
            return lib
        _lib = lib
    return _lib


def _stats(st, counts=None, blocks=None) -> "Stats":
    d = {f[0]: getattr(st, f[0]) for f in _Stats._fields_ if f[0] not in ("root_counts", "block_claims")}
    if blocks is not None:
        blocks = blocks[:st.blocks].copy()
    return Stats(root_counts=counts, block_claims=blocks, **d)


def _strerror(code: int) -> str:
    try:
        return load_library().dfs_strerror(code).decode()
    except Exception:  # pragma: no cover
        return "?"


def _ptr(x):
    """(data pointer, keep-alive) of a contiguous torch tensor or numpy array."""
    try:
        import torch
        if isinstance(x, torch.Tensor):
            if not x.is_contiguous():
                x = x.contiguous()
            return x.data_ptr(), x
    except ImportError:  # pragma: no cover
        pass
    a = np.ascontiguousarray(x)
    return a.ctypes.data, a


def _as(x, np_dtype, torch_dtype):
    try:
        import torch
        if isinstance(x, torch.Tensor):
            return x.to(torch_dtype).contiguous()
    except ImportError:  # pragma: no cover
        pass
    return np.ascontiguousarray(x, dtype=np_dtype)


class Graph:
    """A CSR graph resident on the current CUDA device (``dfs_graph_create``).

    ``row_ptr`` (int64[n+1]) and ``col_idx`` (int32[m]) may be numpy arrays or torch tensors on
    the CPU or on the current GPU; they are copied, so the caller may drop them afterwards.
    """

    def __init__(self, row_ptr, col_idx, lib=None):
        import torch
        self._lib = lib if lib is not None else load_library()
        rp = _as(row_ptr, np.int64, torch.int64)
        ci = _as(col_idx, np.int32, torch.int32)
        n = int(rp.shape[0]) - 1
        m = int(ci.shape[0])
        prp, _k1 = _ptr(rp)
        pci, _k2 = _ptr(ci) if m > 0 else (None, None)
        self._h = self._lib.dfs_graph_create(prp, pci, n, m)
        if not self._h:
            raise DfsError(self._lib.dfs_last_error(), "dfs_graph_create")
        self.n, self.m = n, m
        self.device = torch.cuda.current_device()

    # -- helpers ------------------------------------------------------------------------
    def _stream(self):
        import torch
        rc = self._lib.dfs_set_stream(self._h, torch.cuda.current_stream().cuda_stream)
        if rc != 0:
            raise DfsError(rc, "dfs_set_stream")

    @staticmethod
    def _opts(options: Optional[Options], stats: bool):
        # stats=True returns dfs_stats (times, visited counts); the scheduler counters are only
        # compiled in when options.collect_stats is set
        if options is None:
            return None
        return options.to_c()

    # -- API ----------------------------------------------------------------------------
    def run(self, root: int, out=None, options: Optional[Options] = None, stats: bool = False,
            block_claims: bool = False):
        """One unordered DFS from ``root`` (``dfs_run_ex``).  Returns the int32 parent tensor
        (``out`` if given; host or device) and, with ``stats=True``, a :class:`Stats`."""
        import torch
        if out is None:
            out = torch.empty(self.n, dtype=torch.int32, device="cuda")
        assert out.dtype == torch.int32 and out.numel() == self.n
        self._stream()
        o = self._opts(options, stats)
        st = _Stats() if stats else None
        bc = None
        if stats and block_claims:
            bc = np.zeros(1024, dtype=np.int64)
            st.block_claims = bc.ctypes.data
        rc = self._lib.dfs_run_ex(self._h, int(root), out.data_ptr(),
                                  ctypes.byref(o) if o is not None else None,
                                  ctypes.byref(st) if st is not None else None)
        if rc != 0:
            raise DfsError(rc, "dfs_run_ex")
        if stats:
            return out, _stats(st, blocks=bc)
        return out

    def run_batch(self, roots, out=None, options: Optional[Options] = None, stats: bool = False):
        """``len(roots)`` traversals (``dfs_run_batch_ex``); row i of the (k, n) int32 result
        belongs to ``roots[i]``."""
        import torch
        r = torch.as_tensor(roots, dtype=torch.int32)
        k = int(r.numel())
        if out is None:
            out = torch.empty((k, self.n), dtype=torch.int32, device="cuda")
        assert out.dtype == torch.int32 and out.numel() == k * self.n
        self._stream()
        o = self._opts(options, stats)
        st = _Stats() if stats else None
        counts = np.zeros(2 * k, dtype=np.int64) if stats else None
        if stats:
            st.root_counts = counts.ctypes.data
        rr = r.contiguous()
        rc = self._lib.dfs_run_batch_ex(self._h, rr.data_ptr(), k, out.data_ptr(),
                                        ctypes.byref(o) if o is not None else None,
                                        ctypes.byref(st) if st is not None else None)
        if rc != 0:
            raise DfsError(rc, "dfs_run_batch_ex")
        if stats:
            return out, _stats(st, counts.reshape(k, 2))
        return out

    def timeline(self, len_: int = 0, dt_ns: int = 10_000, fetch: bool = False):
        """Diagnostics (dfs_debug_timeline): enable with len_ > 0; fetch=True returns the last
        run's (busy-block samples (-1 = no sample), claims-so-far, windows-so-far (collect_stats runs))
        samples as numpy arrays."""
        if not fetch:
            rc = self._lib.dfs_debug_timeline(self._h, len_, dt_ns, None)
            if rc != 0:
                raise DfsError(rc, "dfs_debug_timeline")
            return None
        buf = np.zeros(len_, dtype=np.uint32)
        rc = self._lib.dfs_debug_timeline(self._h, len_, dt_ns, buf.ctypes.data)
        if rc != 0:
            raise DfsError(rc, "dfs_debug_timeline")
        t = len_ // 3
        return (buf[:t].astype(np.int64) - 1, buf[t:2 * t].astype(np.int64),
                buf[2 * t:3 * t].astype(np.int64))

    def stack_script(self, lanes: int, ops, out_len: int = 256, options: Optional[Options] = None):
        """Replay stack operations on the walker kernel's own code (dfs_debug_stack_script);
        ``ops`` is a list of up to 6-int records; returns the int32 output values."""
        rec = np.zeros((len(ops), 6), dtype=np.int32)
        for q, r in enumerate(ops):
            rec[q, :len(r)] = r
        out = np.full(out_len, -7, dtype=np.int32)
        o = options.to_c() if options is not None else None
        rc = self._lib.dfs_debug_stack_script(self._h, int(lanes), rec.ctypes.data, len(ops), out.ctypes.data,
                                              out_len, ctypes.byref(o) if o is not None else None)
        if rc != 0:
            raise DfsError(rc, "dfs_debug_stack_script")
        return out

    def launch_count(self) -> int:
        return int(self._lib.dfs_launch_count(self._h))

    def close(self):
        if getattr(self, "_h", None):
            self._lib.dfs_graph_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:  # pragma: no cover
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

"""CPU-side checks of the C ABI boundary (no GPU needed; no compute calls).

* libdfs.so builds for sm_100a and loads;
* it exports every function include/dfs.h declares (parsed from the header, not hard-coded);
* the SASS is sm_100a and contains no Triton/library kernels, only ours;
* argument validation that happens before any device work (NULL handle) returns DFS_EINVAL.
"""
import ctypes
import os
import re
import subprocess

import pytest

from paper_conf_ppopp_niul0c26_b200 import build as dfs_build
from paper_conf_ppopp_niul0c26_b200 import dfs

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _header_functions():
    src = open(os.path.join(ROOT, "include", "dfs.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    names = re.findall(r"^[A-Za-z_][\w \*]*?\b(dfs_\w+)\s*\(", src, flags=re.M)
    return sorted(set(names))


@pytest.fixture(scope="module")
def lib():
    dfs_build.build()
    return dfs.load_library()


def test_header_declares_north_star_entry_points():
    names = _header_functions()
    for f in ("dfs_graph_create", "dfs_run", "dfs_run_batch", "dfs_graph_destroy"):
        assert f in names
    assert sorted(dfs.EXPORTS) == names


def test_library_exports_every_declared_symbol(lib):
    for name in _header_functions():
        assert hasattr(lib, name), name
    out = subprocess.run(["nm", "-D", "--defined-only", dfs.lib_path()], capture_output=True, text=True).stdout
    for name in _header_functions():
        assert re.search(rf"\bT {name}$", out, flags=re.M), name


def test_sass_is_sm100a_and_ours(lib):
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", dfs.lib_path()],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out
    sass = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "-sass", dfs.lib_path()],
                          capture_output=True, text=True).stdout
    kernels = set(re.findall(r"Function : (\S+)", sass))
    assert any("dfs_persistent_kernel" in k for k in kernels)
    assert all("b200dfs" in k for k in kernels), kernels
    # warp-level expansion: ballot (VOTE) + global atomics; 128-bit stack copies
    assert "VOTE.ANY" in sass or "VOTE.ALL" in sass or "VOTE" in sass
    assert "ATOMG" in sass or "RED" in sass
    # bulk async copies of the TMA flush/refill variant; cluster tier: DSMEM barrier
    assert "UBLKCP.G.S" in sass and "UBLKCP.S.G" in sass
    assert "UCGABAR_ARV" in sass


def test_null_handle_is_einval(lib):
    assert lib.dfs_run(None, 0, None) == -1
    assert lib.dfs_last_error() == -1
    assert lib.dfs_run_batch(None, None, 0, None) == -1
    assert lib.dfs_set_stream(None, None) == -1
    lib.dfs_graph_destroy(None)       # no-op
    assert lib.dfs_strerror(-5) == b"traversal watchdog fired"
    assert lib.dfs_launch_count(None) == -1


def test_options_default(lib):
    o = dfs._Options()
    lib.dfs_options_default(ctypes.byref(o))
    assert (o.hot_cutoff, o.cold_cutoff, o.warps_per_block) == (1, 1, 32)     # B200 sweep
    assert o.victim_policy == 1 and o.intra_steal == 1 and o.inter_steal == 1


def test_create_rejects_bad_sizes_without_touching_device(lib):
    # n <= 0 and m >= 2^32 are rejected before any CUDA call
    assert not lib.dfs_graph_create(None, None, 0, 0)
    assert lib.dfs_last_error() == -1

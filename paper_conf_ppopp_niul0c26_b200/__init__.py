"""B200-native unordered DFS (DiggerBees, PPoPP '26) — Python binding of libdfs.so.

The binding only marshals arguments: every step of the traversal runs in the CUDA kernels of
``csrc/`` behind the C ABI of ``include/dfs.h``.  There is no CPU fallback: importing
:mod:`.dfs` raises if ``libdfs.so`` is missing.
"""
from .dfs import (DFS_ROOT_PARENT, DFS_UNREACHED, DfsError, Graph, Options, Stats, lib_path,  # noqa: F401
                  load_library)

__all__ = ["Graph", "Options", "Stats", "DfsError", "DFS_ROOT_PARENT", "DFS_UNREACHED",
           "load_library", "lib_path"]

"""Build libdfs.so in-tree with nvcc for sm_100a (the .so travels to the GPU box with the repo)."""
from __future__ import annotations

import glob
import os
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
SO = os.path.join(HERE, "libdfs.so")
SOURCES = [os.path.join(HERE, "csrc", "dfs_runtime.cu")]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17",
         "-Xcompiler", "-fPIC", "-shared", "-Xptxas", "-v"]


def _deps():
    return SOURCES + glob.glob(os.path.join(HERE, "csrc", "*.cuh")) + [os.path.join(ROOT, "include", "dfs.h")]


def build(force: bool = False, verbose: bool = False) -> str:
    newest = max(os.path.getmtime(p) for p in _deps())
    if force or not os.path.exists(SO) or os.path.getmtime(SO) < newest:
        tmp = SO + f".tmp{os.getpid()}"
        extra = os.environ.get("DFS_NVCC_EXTRA", "").split()      # A/B builds (e.g. -DDFS_KRING=128)
        cmd = [NVCC, *FLAGS, *extra, *SOURCES, "-o", tmp]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError("nvcc failed:\n" + r.stdout + r.stderr)
        if verbose:
            print(r.stdout + r.stderr)
        os.replace(tmp, SO)
    return SO


if __name__ == "__main__":
    print(build(force=True, verbose=True))

"""Build libcrocco.so in-tree with nvcc for sm_100a (B200).

The .so lands next to this file (paper_conf_ipps_davissngmb23_b200/libcrocco.so)
so it travels with the repo snapshot to the GPU box.  NCCL headers/library are
the ones bundled with torch (nvidia-nccl-cu12 2.28.9); the rpath points at them.
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
SRC = [os.path.join(HERE, "csrc", "crocco.cu")]
DEPS = SRC + sorted(glob.glob(os.path.join(HERE, "csrc", "*.cuh"))) + [os.path.join(ROOT, "include", "crocco.h")]
LIB = os.path.join(HERE, "libcrocco.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")


def nccl_dirs():
    import nvidia.nccl
    base = list(nvidia.nccl.__path__)[0]
    return os.path.join(base, "include"), os.path.join(base, "lib")


def needs_build() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(p) > t for p in DEPS)


def build(force: bool = False, verbose: bool = False, defines=(), out: str | None = None) -> str:
    """Compile libcrocco.so; ``defines``/``out`` build tuning variants (tools/)."""
    target = out or LIB
    if not force and out is None and not needs_build():
        return LIB
    inc, lib = nccl_dirs()
    cmd = [NVCC, "-O3", "-std=c++17", "-gencode", "arch=compute_100a,code=sm_100a", "-lineinfo",
           "-Xcompiler", "-fPIC", "-shared", "-fmad=true", "--expt-relaxed-constexpr",
           "-I", os.path.join(ROOT, "include"), "-I", inc,
           *[f"-D{d}" for d in defines],
           "-o", target + ".tmp", *SRC,
           "-L", lib, "-l:libnccl.so.2", "-Xlinker", "-rpath=" + lib, "-lcudart"]
    if verbose:
        cmd.insert(1, "-Xptxas=-v")
    print(" ".join(cmd), file=sys.stderr)
    subprocess.check_call(cmd)
    os.replace(target + ".tmp", target)
    return target


if __name__ == "__main__":
    build(force=True, verbose="-v" in sys.argv)

"""Build the in-tree CUDA library libseis.so for sm_100a (nvcc, no JIT cache).

    python -m paper_conf_ppopp_qawasmehchc15_b200.build [--force] [--verbose]

The library links the CUDA runtime statically and NCCL (the torch-bundled
libnccl.so.2) dynamically with an rpath, so it loads on a GPU-less host (the
driver is only dlopen'ed at the first CUDA call).
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
ROOT = os.path.dirname(HERE)
LIB = os.path.join(HERE, "libseis.so")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def nccl_dirs():
    import nvidia.nccl  # torch's bundled NCCL (same path on the GPU boxes)

    base = os.path.dirname(nvidia.nccl.__file__) if nvidia.nccl.__file__ else list(nvidia.nccl.__path__)[0]
    return os.path.join(base, "include"), os.path.join(base, "lib")


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")) + glob.glob(os.path.join(CSRC, "*.cuh"))
                  + [os.path.join(ROOT, "include", "seis.h")])


def needs_build():
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(s) > t for s in sources())


def build(force: bool = False, verbose: bool = False, defines=(), out: str = None) -> str:
    """defines: extra -D macros (tile / ring-depth tuning sweeps); out: alternative .so path."""
    target = out or LIB
    if not force and out is None and not needs_build():
        return LIB
    inc, lib = nccl_dirs()
    cmd = (["nvcc"] + ARCH + ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-shared",
                              "-Xptxas", "-v" if verbose else "-O3",
                              "-I", inc, "-I", os.path.join(ROOT, "include"),
                              *[f"-D{d}" for d in defines],
                              "-o", target + ".tmp", os.path.join(CSRC, "seis.cu"),
                              "-L", lib, "-l:libnccl.so.2", "-Xlinker", "-rpath," + lib])
    if verbose:
        print(" ".join(cmd))
    subprocess.check_call(cmd)
    os.replace(target + ".tmp", target)
    return target


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose="--verbose" in sys.argv)
    print(LIB)

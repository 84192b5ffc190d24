"""Builds libratel.so (sm_100a) in-tree with nvcc.

The library is plain CUDA C++ behind an extern "C" ABI (include/ratel.h); no
torch headers are involved, so a direct nvcc -shared build is all it needs.
The .so lands next to this file so that it travels with the repo snapshot.
"""
from __future__ import annotations

import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
INCLUDE = os.path.join(ROOT, "include")
LIB = os.path.join(PKG, "libratel.so")
SOURCES = ["ratel_runtime.cu", "ratel_gen.cu", "ratel_host_adam.cpp", "ratel_plan.cpp"]
HEADERS = ["ratel_kernels.cuh", "ratel_bf16.cuh", "nccl_dl.h", "ratel_host_adam.h", "ratel_plan_impl.h", "ratel_uring.h"]
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _nccl_include() -> str:
    try:
        import nvidia.nccl  # torch's bundled NCCL (the copy loaded at run time)
        for base in list(getattr(nvidia.nccl, "__path__", [])):
            inc = os.path.join(base, "include")
            if os.path.exists(os.path.join(inc, "nccl.h")):
                return inc
    except ImportError:
        pass
    return "/usr/include"


def _nvcc() -> str:
    for c in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc"):
        if c and os.path.exists(c):
            return c
    return "nvcc"


def stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = [os.path.join(CSRC, f) for f in SOURCES + HEADERS]
    deps += [os.path.join(INCLUDE, f) for f in os.listdir(INCLUDE)]
    deps.append(os.path.abspath(__file__))
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False, out: str | None = None, defines=()) -> str:
    """Compile libratel.so; `out`/`defines` build a variant elsewhere (tools)."""
    target = out or LIB
    if out is None and not force and not stale():
        return LIB
    tmp = target + f".tmp{os.getpid()}"
    cmd = [_nvcc(), *ARCH, "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-O3,-fopenmp,-fno-math-errno",
           *[f"-D{d}" for d in defines],
           "-Xptxas", "-v" if verbose else "-O3", "-shared", "-o", tmp,
           "-I", INCLUDE, "-I", CSRC, "-I", _nccl_include(),
           *[os.path.join(CSRC, f) for f in SOURCES], "-ldl", "-lgomp"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        sys.stderr.write(r.stdout + r.stderr)
        raise RuntimeError("nvcc failed building libratel.so")
    if verbose:
        sys.stderr.write(r.stderr)
    os.replace(tmp, target)
    return target


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))

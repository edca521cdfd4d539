"""Build libstitch_b200.so (the C-ABI CUDA library) in-tree for sm_100a.

    python -m paper_conf_icpp_blattnerkcsbz14_b200.build [--force] [--ptxas-v]
"""
from __future__ import annotations

import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "libstitch_b200.so")
SOURCES = ["stitch_api.cu", "phase23.cu"]
HEADERS = ["fft_engine.cuh", "pciam_kernels.cuh", "pciam_fp64.cuh", "warp_rows.cuh",
           "async_copy.cuh", "codelets.cuh", "f32x2.cuh", "gen_codelets.py"]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def nccl_include() -> str:
    """nccl.h for the types of the run-time-loaded NCCL (the copy torch ships, else the system's)."""
    try:
        import nvidia.nccl
        for d in nvidia.nccl.__path__:
            inc = os.path.join(d, "include")
            if os.path.exists(os.path.join(inc, "nccl.h")):
                return inc
    except ImportError:
        pass
    return "/usr/include"


def _stale(target: str, deps: list[str]) -> bool:
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    return any(os.path.getmtime(d) > t for d in deps if os.path.exists(d))


def gen_codelets(force: bool = False) -> None:
    out = os.path.join(CSRC, "codelets.cuh")
    gen = os.path.join(CSRC, "gen_codelets.py")
    if force or _stale(out, [gen]):
        code = subprocess.check_output([sys.executable, gen])
        with open(out, "wb") as f:
            f.write(code)


def build(force: bool = False, ptxas_verbose: bool = False) -> str:
    gen_codelets(force)
    deps = [os.path.join(CSRC, s) for s in SOURCES + HEADERS]
    deps.append(os.path.join(ROOT, "include", "stitch.h"))
    deps.append(os.path.abspath(__file__))
    if not force and not _stale(LIB, deps):
        return LIB
    cmd = [NVCC, "-O3", "-std=c++17", *ARCH, "-lineinfo", "-Xcompiler", "-fPIC", "-shared",
           "-I" + os.path.join(ROOT, "include"), "-I" + nccl_include(), "-o", LIB]
    if ptxas_verbose:
        cmd += ["-Xptxas", "-v"]
    cmd += [os.path.join(CSRC, s) for s in SOURCES]
    cmd += ["-ldl"]
    subprocess.check_call(cmd)
    return LIB


if __name__ == "__main__":
    build(force="--force" in sys.argv, ptxas_verbose="--ptxas-v" in sys.argv)
    print(LIB)

"""Builds liblsqr_avugsr.so in-tree with nvcc for sm_100a (no JIT cache: the .so travels with the repo snapshot)."""
from __future__ import annotations

import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "liblsqr_avugsr.so")
SOURCES = ["lsqr_kernels.cu", "lsqr_repro.cu", "lsqr_capi.cu"]
HEADERS = ["lsqr_internal.cuh", os.path.join(ROOT, "include", "lsqr_avugsr.h")]
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _nccl_include() -> str:
    try:
        import nvidia.nccl  # noqa: F401
        base = os.path.dirname(nvidia.nccl.__path__[0] if hasattr(nvidia.nccl, "__path__") else "")
        cand = os.path.join(list(nvidia.nccl.__path__)[0], "include")
        if os.path.exists(os.path.join(cand, "nccl.h")):
            return cand
    except Exception:
        pass
    for c in ("/usr/include", "/usr/local/include"):
        if os.path.exists(os.path.join(c, "nccl.h")):
            return c
    raise RuntimeError("nccl.h not found")


def _nvcc() -> str:
    for c in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", "nvcc"):
        if c and (os.path.exists(c) or c == "nvcc"):
            return c
    return "nvcc"


def needs_build() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = [os.path.join(CSRC, s) for s in SOURCES] + [h if os.path.isabs(h) else os.path.join(CSRC, h)
                                                      for h in HEADERS]
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and not needs_build():
        return LIB
    tmp = LIB + f".tmp{os.getpid()}"
    cmd = [_nvcc(), *ARCH, "-O3", "-lineinfo", "-std=c++17", "-shared", "-Xcompiler", "-fPIC,-O2",
           "-Xptxas", "-warn-spills", "-I", os.path.join(ROOT, "include"), "-I", CSRC, "-I", _nccl_include(),
           "-o", tmp] + [os.path.join(CSRC, s) for s in SOURCES] + ["-ldl"]
    extra = os.environ.get("LSQR_NVCC_EXTRA", "").split()  # experiment builds only (e.g. -DLSQR_DIAG_EXPERIMENTS)
    cmd[1:1] = extra
    if verbose:
        print(" ".join(cmd), file=sys.stderr)
    subprocess.check_call(cmd)
    os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True))

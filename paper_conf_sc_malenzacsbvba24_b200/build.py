"""Builds liblsqr_avugsr.so in-tree with nvcc for sm_100a (no JIT cache: the .so travels with the repo snapshot)."""
from __future__ import annotations

import hashlib
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


def _deps() -> list[str]:
    return [os.path.join(CSRC, s) for s in SOURCES] + [h if os.path.isabs(h) else os.path.join(CSRC, h)
                                                      for h in HEADERS]


def source_hash() -> str:
    """16 hex digits of SHA-256 over the library's sources and headers (embedded in the .so as lsqr_build_id)."""
    h = hashlib.sha256()
    for d in _deps():
        h.update(os.path.basename(d).encode() + b"\0")
        with open(d, "rb") as f:
            h.update(f.read())
    return h.hexdigest()[:16]


def built_id(path: str = LIB) -> str | None:
    """The build id embedded in the .so (its LSQR_BUILD_ID marker), read from the file without loading it."""
    try:
        with open(path, "rb") as f:
            data = f.read()
    except OSError:
        return None
    i = data.find(b"LSQR_BUILD_ID=")
    return data[i + 14:i + 30].decode("ascii", "replace") if i >= 0 else None


def needs_build() -> bool:
    """True when the library is missing or was built from other sources than those on disk."""
    return built_id() != source_hash()


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and not needs_build():
        return LIB
    tmp = LIB + f".tmp{os.getpid()}"
    cmd = [_nvcc(), *ARCH, "-O3", "-lineinfo", "-std=c++17", "-shared", "-Xcompiler", "-fPIC,-O2",
           "-Xptxas", "-warn-spills", f"-DLSQR_SOURCE_HASH=\"{source_hash()}\"",
           "-I", os.path.join(ROOT, "include"), "-I", CSRC, "-I", _nccl_include(),
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

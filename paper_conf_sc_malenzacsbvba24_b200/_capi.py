"""ctypes declarations of include/lsqr_avugsr.h (argument marshalling only; every step runs in the CUDA library)."""
from __future__ import annotations

import ctypes as C
import os
import threading

from . import build as _build

_lock = threading.Lock()
_lib = None

i32, i64, u64, d, vp, sz = C.c_int32, C.c_int64, C.c_uint64, C.c_double, C.c_void_p, C.c_size_t
P64 = C.POINTER(C.c_int64)
PD = C.POINTER(C.c_double)

LSQR_NSCALARS = 24
SCALAR_NAMES = ["alpha", "beta", "rhobar", "phibar", "anorm", "acond", "ddnorm", "res2", "xnorm", "xxnorm", "z",
                "cs2", "sn2", "rnorm", "r1norm", "r2norm", "arnorm", "bnorm", "itn", "istop", "istop_first",
                "halted"]
STATUS = {0: "LSQR_OK", -1: "LSQR_EINVAL", -2: "LSQR_ENOMEM", -3: "LSQR_ECUDA", -4: "LSQR_ENCCL",
          -5: "LSQR_ESTATE", -6: "LSQR_EUNSORTED", -7: "LSQR_ECOMM"}

ALLOC_FN = C.CFUNCTYPE(vp, sz, vp)
FREE_FN = C.CFUNCTYPE(None, vp, vp)
ALLREDUCE_FN = C.CFUNCTYPE(C.c_int, vp, i64, u64, vp)


class Env(C.Structure):
    _fields_ = [("rank", i32), ("nranks", i32), ("device", i32), ("comm_kind", i32), ("nccl_id", vp),
                ("stream", u64), ("alloc", ALLOC_FN), ("free", FREE_FN), ("alloc_user", vp),
                ("allreduce", ALLREDUCE_FN), ("allreduce_user", vp), ("force_collectives", i32), ("pad_", i32)]


class Constraints(C.Structure):
    _fields_ = [("n_rows", i64), ("row_ptr", vp), ("col", vp), ("val", vp), ("rhs", vp)]


class GenParams(C.Structure):
    _fields_ = [("seed", u64), ("b_mode", i32), ("pad_", i32), ("noise", d)]


class SolveParams(C.Structure):
    _fields_ = [("itn_limit", i64), ("atol", d), ("btol", d), ("conlim", d), ("damp", d), ("fixed_count", i32),
                ("use_graph", i32), ("poll_every", i32), ("two_pass", i32)]


class Result(C.Structure):
    _fields_ = [("istop", i32), ("itn", i32), ("istop_first", i32), ("pad_", i32), ("r1norm", d), ("r2norm", d),
                ("anorm", d), ("acond", d), ("arnorm", d), ("xnorm", d), ("bnorm", d), ("t_iter_mean_s", d),
                ("t_iter_max_over_ranks_s", d)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_ if k != "pad_"}


EXPORTS = {
    "lsqr_abi_version": (C.c_int, []),
    "lsqr_build_id": (C.c_char_p, []),
    "lsqr_strerror": (C.c_char_p, [C.c_int]),
    "lsqr_last_error": (C.c_char_p, [vp]),
    "lsqr_synth_obs_per_star": (C.c_int, [u64, i64, i64, i32, vp]),
    "lsqr_synth_constraints": (i64, [u64, i64, i64, i64, i64, vp, vp, vp]),
    "lsqr_shard_map": (C.c_int, [vp, i64, i64, i32, vp]),
    "lsqr_nccl_unique_id": (C.c_int, [vp]),
    "lsqr_create": (C.c_int, [i64, i64, i64, i64, i32, vp, C.POINTER(Constraints), C.POINTER(Env),
                              C.POINTER(vp)]),
    "lsqr_destroy": (C.c_int, [vp]),
    "lsqr_layout": (C.c_int, [vp, vp]),
    "lsqr_generate": (C.c_int, [vp, C.POINTER(GenParams)]),
    "lsqr_set_system": (C.c_int, [vp, vp, vp, vp, vp, vp]),
    "lsqr_get_system": (C.c_int, [vp, vp, vp, vp, vp, vp]),
    "lsqr_precondition": (C.c_int, [vp]),
    "lsqr_get_precond": (C.c_int, [vp, vp]),
    "lsqr_set_reproducible": (C.c_int, [vp, C.c_int32]),
    "lsqr_aprod1": (C.c_int, [vp, vp, vp]),
    "lsqr_aprod2": (C.c_int, [vp, vp, vp]),
    "lsqr_solve": (C.c_int, [vp, C.POINTER(SolveParams), C.POINTER(Result), vp, vp]),
    "lsqr_init": (C.c_int, [vp, C.POINTER(SolveParams)]),
    "lsqr_iterate": (C.c_int, [vp, i64]),
    "lsqr_iterate_timed": (C.c_int, [vp, i64, vp]),
    "lsqr_finalize": (C.c_int, [vp, C.POINTER(Result), vp, vp]),
    "lsqr_get_state": (C.c_int, [vp, vp, vp, vp, vp, vp, vp]),
    "lsqr_set_state": (C.c_int, [vp, vp, vp, vp, vp, vp, vp]),
    "lsqr_sync": (C.c_int, [vp]),
}


def lib_path() -> str:
    return _build.LIB


def lib(build_if_missing: bool = True):
    """Loads liblsqr_avugsr.so, building it first when it is missing or was built from other sources (its embedded
    build id differs from the hash of csrc/ and the header); refuses a library whose id does not match."""
    global _lib
    with _lock:
        if _lib is None:
            if build_if_missing and _build.needs_build():
                # sources newer than the library (or no library): a failed build must not silently load a stale .so
                _build.build()
            if not os.path.exists(_build.LIB):
                raise RuntimeError(f"CUDA extension {_build.LIB} is missing (run __graft_entry__.build())")
            L = C.CDLL(_build.LIB, mode=C.RTLD_GLOBAL)
            for name, (res, args) in EXPORTS.items():
                f = getattr(L, name)
                f.restype = res
                f.argtypes = args
            bid, want = L.lsqr_build_id().decode(), _build.source_hash()
            if bid != want:  # a stale library must never stand in for the sources under test
                raise RuntimeError(f"{_build.LIB} was built from other sources (build id {bid}, sources {want}); "
                                   "rebuild it (__graft_entry__.build())")
            _lib = L
    return _lib


class LsqrError(RuntimeError):
    def __init__(self, status, msg=""):
        self.status = status
        super().__init__(f"{STATUS.get(status, status)}: {msg}")


def check(rc, h=None):
    if rc != 0:
        msg = ""
        if h is not None:
            m = lib().lsqr_last_error(h)
            msg = m.decode() if m else ""
        raise LsqrError(rc, msg)

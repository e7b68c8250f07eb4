"""CPU ORACLE for the Gaia AVU-GSR LSQR hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its ``cpu_baseline`` leg and ``--impl reference``)
may import this package. The product (``paper_conf_sc_malenzacsbvba24_b200``) never imports it; the two share no
code. All arithmetic lives in ``avugsr_oracle.c`` (plain serial C, ``-ffp-contract=off``);
this module only allocates numpy arrays and marshals ctypes arguments.

Functions and the paper passages they follow are listed in avugsr_oracle.c's header.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "avugsr_oracle.c")
_LIB = os.path.join(_HERE, "liboracle_avugsr.so")
_LIB_OMP = os.path.join(_HERE, "liboracle_avugsr_omp.so")
_lock = threading.Lock()
_lib = None

SLOTS = 24


def build(force: bool = False) -> str:
    """Compile the oracle (gcc -O2 -ffp-contract=off). Returns the .so path."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-fno-fast-math", "-std=c11", "-fPIC",
                               "-shared", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


class SysStruct(C.Structure):
    _fields_ = [("n_rows", C.c_int64), ("n_cols", C.c_int64), ("n_axis", C.c_int64), ("A0", C.c_int64),
                ("G0", C.c_int64), ("n_glob", C.c_int32), ("vals", C.c_void_p), ("mA", C.c_void_p),
                ("mT", C.c_void_p), ("iC", C.c_void_p), ("n_constr", C.c_int64), ("c_ptr", C.c_void_p),
                ("c_col", C.c_void_p), ("c_val", C.c_void_p), ("own_lo", C.c_int64), ("own_hi", C.c_int64),
                ("own_shared", C.c_int32)]


class LsqrOut(C.Structure):
    _fields_ = [("istop", C.c_int32), ("itn", C.c_int32), ("istop_first", C.c_int32), ("pad_", C.c_int32),
                ("r1norm", C.c_double), ("r2norm", C.c_double), ("anorm", C.c_double), ("acond", C.c_double),
                ("arnorm", C.c_double), ("xnorm", C.c_double), ("bnorm", C.c_double)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_ if k != "pad_"}


_STATE_NAMES = ["alpha", "beta", "rhobar", "phibar", "anorm", "acond", "ddnorm", "res2", "xnorm", "xxnorm", "z",
                "cs2", "sn2", "rnorm", "r1norm", "r2norm", "arnorm", "bnorm", "rho", "theta", "phi", "tau", "psi",
                "test1", "test2", "test3"]


class LsqrState(C.Structure):
    _fields_ = [("itn", C.c_int32), ("istop", C.c_int32)] + [(n, C.c_double) for n in _STATE_NAMES]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


APROD_FN = C.CFUNCTYPE(None, C.c_int32, C.c_void_p, C.c_void_p, C.c_void_p)
TRACE_FN = C.CFUNCTYPE(None, C.POINTER(LsqrState), C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p,
                       C.c_void_p)


def lib():
    global _lib
    with _lock:
        if _lib is None:
            L = C.CDLL(build())
            i64, u64, i32, d, vp = C.c_int64, C.c_uint64, C.c_int32, C.c_double, C.c_void_p
            L.orc_mix.restype = u64; L.orc_mix.argtypes = [u64]
            L.orc_hash.restype = u64; L.orc_hash.argtypes = [u64, u64, u64, u64]
            L.orc_pm1.restype = d; L.orc_pm1.argtypes = [u64]
            L.orc_star_counts.argtypes = [u64, i64, i64, i32, vp]
            L.orc_row_ptr.argtypes = [vp, i64, vp]
            L.orc_shard.argtypes = [vp, i64, i64, i32, vp]
            L.orc_generate.argtypes = [u64, i64, i64, i64, i32, vp, i64, i64, vp, vp, vp, vp]
            L.orc_x_true.argtypes = [u64, i64, vp]
            L.orc_generate_b.argtypes = [u64, i32, d, i64, i64, i64, i32, vp, i64, i64, vp, vp, vp, vp, vp, vp]
            L.orc_constraints.restype = i64
            L.orc_constraints.argtypes = [u64, i64, i64, i64, i64, vp, vp, vp]
            for f in (L.orc_aprod1, L.orc_aprod2):
                f.argtypes = [C.POINTER(SysStruct), vp, vp]
            L.orc_colnorms.argtypes = [C.POINTER(SysStruct), vp]
            L.orc_colnorms_repro.argtypes = [C.POINTER(SysStruct), vp]
            L.orc_precond_D.argtypes = [vp, i64, vp]
            L.orc_scale.argtypes = [C.POINTER(SysStruct), vp]
            L.orc_lsqr.restype = C.c_int
            L.orc_lsqr.argtypes = [i64, i64, vp, vp, vp, d, d, d, d, i64, i32, i32, i32, vp, vp, vp,
                                   C.POINTER(LsqrOut), vp, vp]
            L.orc_eda_sum.restype = d
            L.orc_eda_sum.argtypes = [vp, i64]
            for f in (L.orc_aprod1_repro, L.orc_aprod2_repro):
                f.argtypes = [C.POINTER(SysStruct), vp, vp]
            _lib = L
    return _lib


def _p(a: np.ndarray):
    return a.ctypes.data_as(C.c_void_p)


# --------------------------------------------------------------------------------------------- O-GEN / O-SHARD
def hash64(seed, tag, i, j) -> int:
    return lib().orc_hash(seed, tag, i, j)


def pm1(h) -> float:
    return lib().orc_pm1(h)


def star_counts(w) -> np.ndarray:
    c = np.zeros(w.n_stars, dtype=np.int64)
    lib().orc_star_counts(w.seed, w.n_stars, w.n_obs, w.jitter_pct, _p(c))
    return c


def row_ptr(counts: np.ndarray) -> np.ndarray:
    rp = np.zeros(len(counts) + 1, dtype=np.int64)
    lib().orc_row_ptr(_p(np.ascontiguousarray(counts, dtype=np.int64)), len(counts), _p(rp))
    return rp


def shard(rp: np.ndarray, n_obs: int, P: int) -> np.ndarray:
    sb = np.zeros(P + 1, dtype=np.int64)
    lib().orc_shard(_p(rp), len(rp) - 1, n_obs, P, _p(sb))
    return sb


def constraints(w):
    """12 synthetic constraint rows (CSR over global columns) or None when w.n_ext_stars == 0."""
    if w.n_ext_stars <= 0:
        return None
    L = lib()
    nnz = L.orc_constraints(w.seed, w.n_stars, w.n_att, w.n_instr, w.n_ext_stars, None, None, None)
    ptr = np.zeros(13, dtype=np.int64)
    col = np.zeros(nnz, dtype=np.int64)
    val = np.zeros(nnz, dtype=np.float64)
    L.orc_constraints(w.seed, w.n_stars, w.n_att, w.n_instr, w.n_ext_stars, _p(ptr), _p(col), _p(val))
    return ptr, col, val


def x_true(w) -> np.ndarray:
    x = np.zeros(w.n_cols, dtype=np.float64)
    lib().orc_x_true(w.seed, w.n_cols, _p(x))
    return x


class System:
    """One rank's share (stars [star_begin, star_end)) of a generated AVU-GSR system, paper layout
    (vals[n][24], matrixIndexAstro, matrixIndexAtt, instrCol), global column numbering."""

    def __init__(self, w, rank: int = 0, nranks: int = 1, generate: bool = True, stars=None):
        """``stars=(s0, s1)`` generates only that star range (sampled parity at full size); constraint entries
        are then owned for those stars' astro columns and the shared columns."""
        self.w = w
        self.counts = star_counts(w)
        self.row_ptr = row_ptr(self.counts)
        self.star_begins = shard(self.row_ptr, w.n_obs, nranks)
        self.rank, self.nranks = rank, nranks
        self.star_begin = int(self.star_begins[rank])
        self.star_end = int(self.star_begins[rank + 1])
        if stars is not None:
            self.star_begin, self.star_end = int(stars[0]), int(stars[1])
            self.rank = 0
        self.row_begin = int(self.row_ptr[self.star_begin])
        self.row_end = int(self.row_ptr[self.star_end])
        n = self.n_rows = self.row_end - self.row_begin
        self.n_axis = w.n_att // 3
        self.A0 = 5 * w.n_stars
        self.I0 = self.A0 + w.n_att
        self.G0 = self.I0 + w.n_instr
        self.n_cols = w.n_cols
        self.vals = np.zeros((n, SLOTS), dtype=np.float64)
        self.mA = np.zeros(n, dtype=np.int64)
        self.mT = np.zeros(n, dtype=np.int64)
        self.iC = np.zeros((n, 6), dtype=np.int64)
        self.b = np.zeros(n, dtype=np.float64)
        c = constraints(w)
        if c is None:
            self.c_ptr = np.zeros(1, dtype=np.int64)
            self.c_col = np.zeros(0, dtype=np.int64)
            self.c_val = np.zeros(0, dtype=np.float64)
        else:
            self.c_ptr, self.c_col, self.c_val = c
        self.n_constr = len(self.c_ptr) - 1
        self.D = None
        if generate:
            L = lib()
            L.orc_generate(w.seed, w.n_stars, w.n_att, w.n_instr, w.n_glob, _p(self.row_ptr), self.star_begin,
                           self.star_end, _p(self.vals), _p(self.mA), _p(self.mT), _p(self.iC))
            xt = x_true(w) if w.b_mode == 1 else np.zeros(1)
            L.orc_generate_b(w.seed, w.b_mode, w.noise, w.n_stars, w.n_att, w.n_instr, w.n_glob, _p(self.row_ptr),
                             self.star_begin, self.star_end, _p(self.vals), _p(self.mA), _p(self.mT), _p(self.iC),
                             _p(xt), _p(self.b))
        self._mk_struct()

    def _mk_struct(self):
        s = SysStruct()
        s.n_rows, s.n_cols, s.n_axis, s.A0, s.G0, s.n_glob = (self.n_rows, self.n_cols, self.n_axis, self.A0,
                                                               self.G0, self.w.n_glob)
        s.vals, s.mA, s.mT, s.iC = _p(self.vals), _p(self.mA), _p(self.mT), _p(self.iC)
        s.n_constr, s.c_ptr, s.c_col, s.c_val = self.n_constr, _p(self.c_ptr), _p(self.c_col), _p(self.c_val)
        s.own_lo, s.own_hi = 5 * self.star_begin, 5 * self.star_end
        s.own_shared = 1 if self.rank == 0 else 0
        self.S = s

    # number of rows of the LSQR system this rank's u vector covers (local obs + replicated constraint rows)
    @property
    def m_local(self) -> int:
        return self.n_rows + self.n_constr

    def aprod1(self, x: np.ndarray, y: np.ndarray) -> None:
        """y[n_rows + n_constr] += A x (x over ALL global columns)."""
        assert x.dtype == np.float64 and y.dtype == np.float64 and x.size == self.n_cols
        assert y.size == self.m_local
        lib().orc_aprod1(C.byref(self.S), _p(x), _p(y))

    def aprod2(self, y: np.ndarray, x: np.ndarray) -> None:
        """x[n_cols] += A^T y."""
        assert x.size == self.n_cols and y.size == self.m_local
        lib().orc_aprod2(C.byref(self.S), _p(y), _p(x))

    def aprod1_repro(self, x: np.ndarray, y: np.ndarray) -> None:
        """NEXT-4: y += A x with exact (order-independent) row sums, docs/REPRO.md."""
        assert x.size == self.n_cols and y.size == self.m_local
        lib().orc_aprod1_repro(C.byref(self.S), _p(x), _p(y))

    def aprod2_repro(self, y: np.ndarray, x: np.ndarray) -> None:
        """NEXT-4: x += A^T y with exact (order-independent) column sums."""
        assert x.size == self.n_cols and y.size == self.m_local
        lib().orc_aprod2_repro(C.byref(self.S), _p(y), _p(x))

    def colnorms(self, repro: bool = False) -> np.ndarray:
        c = np.zeros(self.n_cols, dtype=np.float64)
        (lib().orc_colnorms_repro if repro else lib().orc_colnorms)(C.byref(self.S), _p(c))
        return c

    def apply_precond(self, c_total: np.ndarray | None = None, repro: bool = False) -> np.ndarray:
        """O-PREC: D from the column sums of squares (given, e.g. summed over ranks, or computed here; ``repro``:
        NEXT-4 exact sums), then scale the stored values in place."""
        c = self.colnorms(repro) if c_total is None else c_total
        D = np.zeros(self.n_cols, dtype=np.float64)
        lib().orc_precond_D(_p(np.ascontiguousarray(c)), self.n_cols, _p(D))
        lib().orc_scale(C.byref(self.S), _p(D))
        self.D = D
        return D

    def rhs(self) -> np.ndarray:
        """[b | constraint rhs (0)]."""
        return np.concatenate([self.b, np.zeros(self.n_constr)])

    def dense(self) -> np.ndarray:
        """Dense materialisation (tests only; small systems) -- built from the index arrays with numpy, not from
        the C products."""
        n = self.n_rows
        A = np.zeros((self.m_local, self.n_cols))
        cols = np.zeros((n, SLOTS), dtype=np.int64)
        cols[:, 0:5] = self.mA[:, None] + np.arange(5)[None, :]
        for a in range(3):
            cols[:, 5 + 4 * a:9 + 4 * a] = self.mT[:, None] + a * self.n_axis + np.arange(4)[None, :]
        cols[:, 17:23] = self.iC
        cols[:, 23] = self.G0
        nslots = SLOTS if self.w.n_glob else SLOTS - 1
        for s in range(nslots):
            np.add.at(A, (np.arange(n), cols[:, s]), self.vals[:, s])
        for k in range(self.n_constr):
            for e in range(self.c_ptr[k], self.c_ptr[k + 1]):
                col = self.c_col[e]
                if (5 * self.star_begin <= col < 5 * self.star_end) or (col >= self.A0 and self.rank == 0):
                    A[n + k, col] += self.c_val[e]
        return A


# --------------------------------------------------------------------------------------------------- O-LSQR
def lsqr(m: int, n: int, aprod, b: np.ndarray, damp=0.0, atol=1e-8, btol=1e-8, conlim=1e8, itn_limit=None,
         fixed_count=False, reorth=False, trace=None, want_se=True, trace_vectors=True, repro=False):
    """Paige-Saunders LSQR (O-LSQR).  ``aprod`` is either a System (C products) or a python callable
    aprod(mode, vin, vout) with mode 1: vout[m] += A vin[n], mode 2: vout[n] += A^T vin[m].
    ``trace(state_dict, u, v, w, x, var)`` is called after every iteration with COPIES of the vectors
    (``trace_vectors=False``: ``trace(state_dict)`` only, no copies -- used to time iterations).
    Returns dict(x, var, se, istop, itn, istop_first, r1norm, r2norm, anorm, acond, arnorm, xnorm, bnorm)."""
    L = lib()
    if itn_limit is None:
        itn_limit = 2 * n
    b = np.ascontiguousarray(b, dtype=np.float64)
    assert b.size == m
    x = np.zeros(n); var = np.zeros(n); se = np.zeros(n)
    out = LsqrOut()
    keep = []
    if isinstance(aprod, System):
        fn = C.cast(L.orc_sys_aprod_repro if repro else L.orc_sys_aprod, C.c_void_p)
        ctx = C.cast(C.pointer(aprod.S), C.c_void_p)
    else:
        def _cb(mode, vin, vout, _ctx, _f=aprod):
            if mode == 1:
                a = np.ctypeslib.as_array(C.cast(vin, C.POINTER(C.c_double)), (n,))
                o = np.ctypeslib.as_array(C.cast(vout, C.POINTER(C.c_double)), (m,))
            else:
                a = np.ctypeslib.as_array(C.cast(vin, C.POINTER(C.c_double)), (m,))
                o = np.ctypeslib.as_array(C.cast(vout, C.POINTER(C.c_double)), (n,))
            _f(mode, a, o)
        cb = APROD_FN(_cb)
        keep.append(cb)
        fn = C.cast(cb, C.c_void_p)
        ctx = None
    tfn = None
    if trace is not None:
        def _tr(stp, u, v, w_, xx, vv, _ctx):
            st = stp.contents.as_dict()
            if not trace_vectors:
                trace(st)
                return
            arr = lambda p, k: np.ctypeslib.as_array(C.cast(p, C.POINTER(C.c_double)), (k,)).copy()
            trace(st, arr(u, m), arr(v, n), arr(w_, n), arr(xx, n), arr(vv, n))
        tcb = TRACE_FN(_tr)
        keep.append(tcb)
        tfn = C.cast(tcb, C.c_void_p)
    rc = L.orc_lsqr(m, n, fn, ctx, _p(b), damp, atol, btol, conlim, int(itn_limit), int(bool(fixed_count)),
                    int(bool(reorth)), int(bool(repro)), _p(x), _p(var), _p(se) if want_se else None, C.byref(out),
                    tfn, None)
    if rc != 0:
        raise MemoryError("orc_lsqr allocation failed")
    res = out.as_dict()
    res.update(x=x, var=var, se=se)
    return res


# --------------------------------------------------------------------------- all-core TIMING variant (not a checker)
_SRC_OMP = os.path.join(_HERE, "omp_timing.c")
_omp = None


def build_omp(force: bool = False) -> str:
    """Compile omp_timing.c (the oracle source with OpenMP loops and products; bench.py cpu_baseline timing only)."""
    newest = max(os.path.getmtime(_SRC), os.path.getmtime(_SRC_OMP))
    if force or not os.path.exists(_LIB_OMP) or os.path.getmtime(_LIB_OMP) < newest:
        tmp = _LIB_OMP + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-ffp-contract=off", "-fno-fast-math", "-std=c11", "-fPIC",
                               "-shared", "-o", tmp, _SRC_OMP, "-lm"])
        os.replace(tmp, _LIB_OMP)
    return _LIB_OMP


def omp_lib():
    global _omp
    with _lock:
        if _omp is None:
            L = C.CDLL(build_omp())
            vp, i64, i32, d = C.c_void_p, C.c_int64, C.c_int32, C.c_double
            L.orc_omp_threads.restype = C.c_int
            L.orc_omp_set_threads.argtypes = [C.c_int]
            for f in (L.orc_omp_aprod1, L.orc_omp_aprod2):
                f.argtypes = [C.POINTER(SysStruct), vp, vp]
            L.orc_lsqr.restype = C.c_int
            L.orc_lsqr.argtypes = [i64, i64, vp, vp, vp, d, d, d, d, i64, i32, i32, i32, vp, vp, vp,
                                   C.POINTER(LsqrOut), vp, vp]
            _omp = L
    return _omp


def time_lsqr_omp(sysm: System, iters: int, threads: int | None = None) -> dict:
    """TIMING ONLY: `iters` fixed-count LSQR iterations of the all-core variant on an already preconditioned
    System; returns per-iteration wall times (the first, which includes O-1, is dropped) and the thread count.
    threads: OpenMP threads for this and later calls from this thread (None: the OpenMP default)."""
    import time
    L = omp_lib()
    if threads:
        L.orc_omp_set_threads(int(threads))
    stamps = []

    def _tr(stp, u, v, w_, xx, vv, _ctx):
        stamps.append(time.perf_counter())
    tcb = TRACE_FN(_tr)
    m, n = sysm.m_local, sysm.n_cols
    x, var = np.zeros(n), np.zeros(n)
    out = LsqrOut()
    rc = L.orc_lsqr(m, n, C.cast(L.orc_omp_sys_aprod, C.c_void_p), C.cast(C.pointer(sysm.S), C.c_void_p),
                    _p(sysm.rhs()), 0.0, 0.0, 0.0, 0.0, int(iters + 1), 1, 0, 0, _p(x), _p(var), None,
                    C.byref(out), C.cast(tcb, C.c_void_p), None)
    if rc != 0:
        raise RuntimeError(f"orc_lsqr (omp) returned {rc}")
    per = [b - a for a, b in zip(stamps[:-1], stamps[1:])]
    return {"per_iter_s": per, "threads": int(L.orc_omp_threads()), "x": x}


def eda_sum(a) -> float:
    """NEXT-4 exact digit accumulator: order-independent sum of doubles (docs/REPRO.md)."""
    a = np.ascontiguousarray(a, dtype=np.float64)
    return lib().orc_eda_sum(_p(a), a.size)


def solve_system(sysm: System, damp=0.0, atol=1e-8, btol=1e-8, conlim=1e8, itn_limit=100, fixed_count=True,
                 precondition=True, trace=None, repro=False):
    """Full single-rank oracle solve: O-PREC (if requested and not yet applied), O-LSQR, O-4 se, O-5 unscale."""
    if precondition and sysm.D is None:
        sysm.apply_precond(repro=repro)
    res = lsqr(sysm.m_local, sysm.n_cols, sysm, sysm.rhs(), damp=damp, atol=atol, btol=btol, conlim=conlim,
               itn_limit=itn_limit, fixed_count=fixed_count, trace=trace, repro=repro)
    if sysm.D is not None:
        res["x_scaled"] = res["x"].copy()
        res["x"] = sysm.D * res["x"]
        res["se"] = sysm.D * res["se"]
    return res

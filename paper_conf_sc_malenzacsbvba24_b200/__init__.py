"""B200-native Gaia AVU-GSR LSQR (Malenza et al., SC-W 2024) -- Python binding of liblsqr_avugsr.so.

The binding only marshals arguments: system generation, preconditioning, aprod1/aprod2, the LSQR iteration and the
standard errors all run in the library's sm_100a kernels (csrc/).  PyTorch provides device memory (the caching
allocator, through the library's alloc hooks), the caller's CUDA stream and torch.distributed for multi-rank
bootstrap.  There is no CPU fallback: without the CUDA extension every call raises.

Quick start (one GPU)::

    import workloads, paper_conf_sc_malenzacsbvba24_b200 as avu
    s = avu.Solver.synthetic(workloads.C2)        # generate on device (+ 12 constraint rows)
    s.precondition()
    out = s.solve(itn_limit=100, fixed_count=True)  # dict: x, se, istop, itn, r1norm, arnorm, ...
"""
from __future__ import annotations

import ctypes as C

import numpy as np

from . import _capi
from ._capi import LsqrError, SCALAR_NAMES, check

__all__ = ["Solver", "LsqrError", "synth_obs_per_star", "synth_constraints", "shard_map", "nccl_unique_id",
           "abi_version", "SCALAR_NAMES"]


def _p(a):
    """ctypes pointer of a numpy array or torch tensor (no copies)."""
    if a is None:
        return None
    if isinstance(a, np.ndarray):
        return a.ctypes.data_as(C.c_void_p)
    return C.c_void_p(a.data_ptr())


def abi_version() -> int:
    return _capi.lib().lsqr_abi_version()


def synth_obs_per_star(seed: int, n_stars: int, n_obs: int, jitter_pct: int) -> np.ndarray:
    c = np.zeros(n_stars, dtype=np.int64)
    check(_capi.lib().lsqr_synth_obs_per_star(seed, n_stars, n_obs, jitter_pct, _p(c)))
    return c


def synth_constraints(seed: int, n_stars: int, n_att: int, n_instr: int, n_ext: int):
    L = _capi.lib()
    nnz = L.lsqr_synth_constraints(seed, n_stars, n_att, n_instr, n_ext, None, None, None)
    if nnz < 0:
        raise LsqrError(int(nnz), "lsqr_synth_constraints")
    ptr = np.zeros(13, dtype=np.int64)
    col = np.zeros(nnz, dtype=np.int64)
    val = np.zeros(nnz, dtype=np.float64)
    L.lsqr_synth_constraints(seed, n_stars, n_att, n_instr, n_ext, _p(ptr), _p(col), _p(val))
    return ptr, col, val


def shard_map(counts: np.ndarray, n_obs: int, nranks: int) -> np.ndarray:
    counts = np.ascontiguousarray(counts, dtype=np.int64)
    sb = np.zeros(nranks + 1, dtype=np.int64)
    check(_capi.lib().lsqr_shard_map(_p(counts), len(counts), n_obs, nranks, _p(sb)))
    return sb


def nccl_unique_id() -> bytes:
    buf = (C.c_uint8 * 128)()
    check(_capi.lib().lsqr_nccl_unique_id(buf))
    return bytes(buf)


class _CudaArray:
    """__cuda_array_interface__ view of a raw device pointer (for the host-callback allreduce)."""

    def __init__(self, ptr, n):
        self.__cuda_array_interface__ = {"shape": (n,), "typestr": "<f8", "data": (ptr, False), "version": 3,
                                         "strides": None}


def gloo_allreduce_callback(group=None):
    """Host-callback collective for LSQR_COMM_CALLBACK: SUM-allreduce through torch.distributed (e.g. gloo), several
    ranks may share one GPU.  Returns a python callable (dev_ptr, count, stream, user) -> int."""
    import torch
    import torch.distributed as dist

    def cb(ptr, count, stream, user):
        try:
            t = torch.as_tensor(_CudaArray(ptr, count), device="cuda")
            h = t.cpu()
            dist.all_reduce(h, op=dist.ReduceOp.SUM, group=group)
            t.copy_(h)
            torch.cuda.synchronize()
            return 0
        except Exception as e:  # never let an exception cross the C ABI
            print("allreduce callback failed:", e)
            return 1
    return cb


class Solver:
    """One rank's handle (lsqr_t).  Device vectors are torch float64 tensors on this rank's GPU."""

    def __init__(self, n_stars, n_obs, n_att, n_instr, n_glob=1, obs_per_star=None, constraints=None, rank=0,
                 nranks=1, device=None, comm="nccl", nccl_id=None, allreduce=None, stream=None,
                 torch_alloc=True, force_collectives=False):
        import torch
        self._torch = torch
        L = _capi.lib()
        if device is None:
            device = torch.cuda.current_device()
        self.device = int(device)
        self.rank, self.nranks = rank, nranks
        self._keep = []
        env = _capi.Env()
        env.rank, env.nranks, env.device = rank, nranks, self.device
        env.comm_kind = 1 if comm == "callback" else 0
        env.force_collectives = int(bool(force_collectives))  # test hook (lsqr_env.force_collectives)
        if nranks > 1 and env.comm_kind == 0:
            if nccl_id is None:
                raise ValueError("nccl_id required for nranks > 1 with NCCL")
            idbuf = (C.c_uint8 * 128).from_buffer_copy(nccl_id)
            self._keep.append(idbuf)
            env.nccl_id = C.cast(idbuf, C.c_void_p)
        if stream is None:
            stream = torch.cuda.current_stream(self.device)
        self.stream = stream
        env.stream = stream.cuda_stream
        if torch_alloc:
            dev = self.device

            def _alloc(nbytes, user):
                try:
                    return torch.cuda.caching_allocator_alloc(int(nbytes), dev)
                except Exception:
                    return None

            def _free(ptr, user):
                try:  # (may run from __del__ at interpreter exit, after torch is torn down)
                    torch.cuda.caching_allocator_delete(ptr)
                except Exception:
                    pass

            fa, ff = _capi.ALLOC_FN(_alloc), _capi.FREE_FN(_free)
            self._keep += [fa, ff]
            env.alloc, env.free = fa, ff
        if env.comm_kind == 1 and (nranks > 1 or force_collectives):
            cb = _capi.ALLREDUCE_FN(allreduce or gloo_allreduce_callback())
            self._keep.append(cb)
            env.allreduce = cb
        cons_p = None
        self.constraints = constraints
        if constraints is not None:
            ptr, col, val = [np.ascontiguousarray(a) for a in constraints[:3]]
            rhs = np.ascontiguousarray(constraints[3]) if len(constraints) > 3 and constraints[3] is not None \
                else None
            self._keep += [ptr, col, val, rhs]
            cs = _capi.Constraints(len(ptr) - 1, _p(ptr), _p(col), _p(val), _p(rhs))
            cons_p = C.byref(cs)
        ops = None
        if obs_per_star is not None:
            ops = np.ascontiguousarray(obs_per_star, dtype=np.int64)
            self._keep.append(ops)
        h = C.c_void_p()
        with torch.cuda.device(self.device):
            rc = L.lsqr_create(n_stars, n_obs, n_att, n_instr, n_glob, _p(ops), cons_p, C.byref(env), C.byref(h))
        check(rc)
        self._h = h
        self._env = env
        lay = np.zeros(10, dtype=np.int64)
        check(L.lsqr_layout(h, _p(lay)), h)
        (self.star_begin, self.star_end, self.row_begin, self.row_end, self.n_local_rows, self.n_local_cols,
         self.n_constr, self.n_shared, self.m_global, self.n_global) = [int(v) for v in lay]
        self.dims = dict(n_stars=n_stars, n_obs=n_obs, n_att=n_att, n_instr=n_instr, n_glob=n_glob)

    # ------------------------------------------------------------------ construction helpers
    @classmethod
    def synthetic(cls, w, rank=0, nranks=1, generate=True, **kw):
        """Solver for a workloads.Workload: synthetic obs-per-star and constraint rows, device-side generation."""
        counts = synth_obs_per_star(w.seed, w.n_stars, w.n_obs, w.jitter_pct)
        cons = synth_constraints(w.seed, w.n_stars, w.n_att, w.n_instr, w.n_ext_stars) if w.n_ext_stars > 0 \
            else None
        s = cls(w.n_stars, w.n_obs, w.n_att, w.n_instr, w.n_glob, obs_per_star=counts, constraints=cons, rank=rank,
                nranks=nranks, **kw)
        s.workload = w
        if generate:
            s.generate(w.seed, w.b_mode, w.noise)
        return s

    @property
    def handle(self):
        return self._h

    def close(self):
        if getattr(self, "_h", None) is not None and self._h.value:
            _capi.lib().lsqr_destroy(self._h)
            self._h = C.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def _chk(self, rc):
        check(rc, self._h)

    def new_x(self):
        return self._torch.zeros(self.n_local_cols, dtype=self._torch.float64, device=f"cuda:{self.device}")

    def new_y(self):
        return self._torch.zeros(self.n_local_rows + self.n_constr, dtype=self._torch.float64,
                                 device=f"cuda:{self.device}")

    # ------------------------------------------------------------------ system
    def generate(self, seed, b_mode=0, noise=0.0):
        self._chk(_capi.lib().lsqr_generate(self._h, C.byref(_capi.GenParams(seed, b_mode, 0, noise))))

    def set_system(self, vals, mA, mT, iC, b):
        arrs = [np.ascontiguousarray(vals, dtype=np.float64), np.ascontiguousarray(mA, dtype=np.int64),
                np.ascontiguousarray(mT, dtype=np.int64), np.ascontiguousarray(iC, dtype=np.int64),
                np.ascontiguousarray(b, dtype=np.float64)]
        self._chk(_capi.lib().lsqr_set_system(self._h, *[_p(a) for a in arrs]))

    def set_system_ptrs(self, vals_p, mA_p, mT_p, iC_p, b_p):
        """Raw host pointers (e.g. pinned torch tensors' data_ptr()) -- the e2e path."""
        self._chk(_capi.lib().lsqr_set_system(self._h, vals_p, mA_p, mT_p, iC_p, b_p))

    def get_system_ptrs(self, vals_p, mA_p, mT_p, iC_p, b_p):
        """lsqr_get_system into raw host pointers (e.g. pinned torch tensors' data_ptr()); any may be None."""
        self._chk(_capi.lib().lsqr_get_system(self._h, vals_p, mA_p, mT_p, iC_p, b_p))

    def get_system(self, with_b=True):
        n = self.n_local_rows
        out = dict(vals=np.zeros((n, 24)), mA=np.zeros(n, dtype=np.int64), mT=np.zeros(n, dtype=np.int64),
                   iC=np.zeros((n, 6), dtype=np.int64), b=np.zeros(n) if with_b else None)
        self._chk(_capi.lib().lsqr_get_system(self._h, _p(out["vals"]), _p(out["mA"]), _p(out["mT"]),
                                              _p(out["iC"]), _p(out["b"])))
        return out

    def precondition(self):
        self._chk(_capi.lib().lsqr_precondition(self._h))

    def get_precond(self) -> np.ndarray:
        D = np.zeros(self.n_local_cols)
        self._chk(_capi.lib().lsqr_get_precond(self._h, _p(D)))
        return D

    def set_reproducible(self, on: bool = True):
        """NEXT-4 bitwise-reproducible mode (docs/REPRO.md): exact order-independent reductions in precondition and
        LSQR; call before precondition()."""
        self._chk(_capi.lib().lsqr_set_reproducible(self._h, int(bool(on))))

    # ------------------------------------------------------------------ products
    def aprod1(self, x, y):
        """y += A^ x (device float64 tensors; y = [local rows | constraint rows])."""
        assert x.is_cuda and y.is_cuda and x.dtype == self._torch.float64 and y.dtype == self._torch.float64
        assert x.numel() == self.n_local_cols and y.numel() == self.n_local_rows + self.n_constr
        self._chk(_capi.lib().lsqr_aprod1(self._h, _p(x), _p(y)))

    def aprod2(self, y, x):
        """x += A^T y."""
        assert x.is_cuda and y.is_cuda and x.dtype == self._torch.float64 and y.dtype == self._torch.float64
        assert x.numel() == self.n_local_cols and y.numel() == self.n_local_rows + self.n_constr
        self._chk(_capi.lib().lsqr_aprod2(self._h, _p(y), _p(x)))

    # ------------------------------------------------------------------ LSQR
    @staticmethod
    def _params(itn_limit=100, atol=1e-8, btol=1e-8, conlim=1e8, damp=0.0, fixed_count=False, use_graph=True,
                poll_every=16, fused=True):
        return _capi.SolveParams(int(itn_limit), atol, btol, conlim, damp, int(bool(fixed_count)),
                                 int(bool(use_graph)), int(poll_every), int(not fused))

    def solve(self, x_out=None, se_out=None, **kw):
        """Full solve; returns dict(result fields, x, se) with x, se as numpy (host) unless device tensors are
        given."""
        p = self._params(**kw)
        res = _capi.Result()
        xo = x_out if x_out is not None else np.zeros(self.n_local_cols)
        so = se_out if se_out is not None else np.zeros(self.n_local_cols)
        self._chk(_capi.lib().lsqr_solve(self._h, C.byref(p), C.byref(res), _p(xo), _p(so)))
        out = res.as_dict()
        out.update(x=xo, se=so)
        return out

    def init(self, **kw):
        self._chk(_capi.lib().lsqr_init(self._h, C.byref(self._params(**kw))))

    def iterate(self, n):
        self._chk(_capi.lib().lsqr_iterate(self._h, int(n)))

    def iterate_events(self, n) -> float:
        """lsqr_iterate(n) bracketed by CUDA events on the solver's stream (the library's stream is ordered after it
        at entry and before it at exit); returns the elapsed device milliseconds."""
        torch = self._torch
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(self.stream)
        self.iterate(n)
        e1.record(self.stream)
        e1.synchronize()
        return e0.elapsed_time(e1)

    def iterate_timed(self, n):
        out = np.zeros(5)
        self._chk(_capi.lib().lsqr_iterate_timed(self._h, int(n), _p(out)))
        return dict(total_ms=out[0], aprod1_ms=out[1], aprod2_ms=out[2], launches=int(out[3]), worst_iter_ms=out[4])

    def finalize(self, x_out=None, se_out=None):
        res = _capi.Result()
        xo = x_out if x_out is not None else np.zeros(self.n_local_cols)
        so = se_out if se_out is not None else np.zeros(self.n_local_cols)
        self._chk(_capi.lib().lsqr_finalize(self._h, C.byref(res), _p(xo), _p(so)))
        out = res.as_dict()
        out.update(x=xo, se=so)
        return out

    def get_state(self, vectors=True):
        sc = np.zeros(_capi.LSQR_NSCALARS)
        if vectors:
            u = np.zeros(self.n_local_rows + self.n_constr)
            v, w, x, var = (np.zeros(self.n_local_cols) for _ in range(4))
            self._chk(_capi.lib().lsqr_get_state(self._h, _p(sc), _p(u), _p(v), _p(w), _p(x), _p(var)))
        else:
            u = v = w = x = var = None
            self._chk(_capi.lib().lsqr_get_state(self._h, _p(sc), None, None, None, None, None))
        st = {k: sc[i] for i, k in enumerate(SCALAR_NAMES)}
        for k in ("itn", "istop", "istop_first", "halted"):
            st[k] = int(st[k])
        return st, dict(u=u, v=v, w=w, x=x, var=var)

    def set_state(self, scalars: dict | None = None, u=None, v=None, w=None, x=None, var=None):
        sc = None
        if scalars is not None:
            sc = np.zeros(_capi.LSQR_NSCALARS)
            for i, k in enumerate(SCALAR_NAMES):
                sc[i] = scalars.get(k, 0.0)
        arrs = [None if a is None else np.ascontiguousarray(a, dtype=np.float64) for a in (u, v, w, x, var)]
        self._chk(_capi.lib().lsqr_set_state(self._h, _p(sc), *[_p(a) for a in arrs]))

    def sync(self):
        self._chk(_capi.lib().lsqr_sync(self._h))

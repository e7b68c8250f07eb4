#!/usr/bin/env python
"""Benchmark: seconds per LSQR iteration and HBM-roofline fraction (FP64) of the AVU-GSR hot path on B200.

    python bench.py [--gpus N --steps K --warmup W --config C3]          # our CUDA path (one JSON line)
    python bench.py --impl reference ...                                  # the CPU oracle (reference arm)
    torchrun --nproc-per-node N bench.py --gpus N ...                     # multi-GPU, weak scaling

A "step" is one LSQR iteration (aprod1 + beta + aprod2 + shared-slice update + scalar recurrence + column update,
SURVEY §8(a) a3-a9) over the whole synthetic system; in fixed-count mode as in the paper.  Default
variant: the fused single pass (SURVEY §8(f) NEXT-1, A read once per iteration); `--two-pass` times aprod1 and
aprod2 as separate passes.  Weak
scaling: every GPU holds one copy of the configuration's shape (n_stars, n_obs multiplied by N).  Inputs (A: 1 GB
at C2) are larger than L2 (126 MB), so no L2 flush is needed between iterations.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import workloads as W  # noqa: E402

METRIC = "s per LSQR iteration & % of HBM roofline (FP64) at 1/2/4/8 B200"
UNIT = "s/iteration"


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured"
    return 6650.0, "fallback"


# ------------------------------------------------------------------------------------------------ clocks
class ClockSampler:
    """Samples SM clock and throttle reasons during the timed region (pynvml; nvidia-smi fallback)."""

    REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap", 0x8: "hw_slowdown",
               0x10: "sync_boost", 0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown",
               0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting"}

    def __init__(self, device=0, period=0.05):
        self.device, self.period = device, period
        self.samples, self.reasons, self.max_mhz = [], set(), None
        self._stop = threading.Event()
        self._t = None
        self.ok = False
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(device)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception:
            self.nv = None

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                r = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for bit, name in self.REASONS.items():
                    if r & bit and name != "gpu_idle":
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(self.period)

    def __enter__(self):
        if self.ok:
            self._t = threading.Thread(target=self._run, daemon=True)
            self._t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self._t:
            self._t.join()

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons), "samples": 0}
        return {"sm_mhz": statistics.median(self.samples), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


# ------------------------------------------------------------------------------------------------ bytes
def algorithmic_bytes(w, n_rows, n_stars, n_sh, n_cols):
    """Algorithmic HBM bytes per launch.
    aprod1: A values 192 B + index record 16 B + u read 8 B + u write 8 B per row; v_astro 40 B per star; v_shared
    gathered once (8 B per shared column).  aprod2 (k_fused3<R3_AP2>): 192 + 16 + 8 (u) per row; astro z written
    once (zA, 40 B per star); z_shared written once.  Iteration (two-pass): both products + column update (v, w, x, var read, v, w, x, var
    written: 7 x 8 B per column counted as in SURVEY: 56 B) -- 440 B/row + 56 B/column."""
    ap1 = 224 * n_rows + 40 * n_stars + 8 * n_sh
    ap2 = 216 * n_rows + 40 * n_stars + 8 * n_sh
    it = 440 * n_rows + 56 * n_cols
    return ap1, ap2, it


def load_traffic(workload, kernel):
    """DRAM bytes per launch of `kernel` from a committed ncu --set full capture of the same workload, or None."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return d.get(workload, {}).get(kernel)
    return None


# ------------------------------------------------------------------------------------------------ cpu baseline
def oracle_sample(w):
    """A bounded sample of workload w for timing the CPU oracle: the rows of shard 0 of P (O-SHARD; P = 1 for systems
    up to ~7 M rows), with w's full column dimension.  Returns (System, P)."""
    import oracle
    P = max(1, -(-w.n_obs // 7_000_000))
    S = oracle.System(w, rank=0, nranks=P)
    return S, P


def _time_products(S, fns, reps=2):
    """Median wall time of one aprod1 + one aprod2 call on the sample (the part of an iteration that scales with
    the rows; the n-vector updates do not)."""
    x = np.full(S.n_cols, 1e-3)
    y = np.zeros(S.m_local)
    ts = []
    for _ in range(reps):
        t0 = time.perf_counter()
        fns[0](x, y)
        fns[1](y, x)
        ts.append(time.perf_counter() - t0)
    return float(np.median(ts))


def cpu_baseline(w, iters=3, repro=False, all_cores=True):
    """The oracle on a bounded sample of w (oracle_sample): `iters` timed fixed-count LSQR iterations of (a) the
    serial C checker as it stands (one core) and (b) its all-core OpenMP timing build (oracle/omp_timing.c: the same
    source with OpenMP loops and products; ``repro``: the serial repro mode only).  The sample covers 1/P of the rows
    with the full column dimension, so the full-workload time per iteration is extrapolated as
    t_iter(sample) + (P - 1) * t_products(sample) (the products scale with the rows, the n-vector updates do not)."""
    import ctypes
    import oracle
    t0 = time.perf_counter()
    S, P = oracle_sample(w)
    S.apply_precond(repro=repro)
    t_setup = time.perf_counter() - t0
    stamps = []
    oracle.lsqr(S.m_local, S.n_cols, S, S.rhs(), atol=0, btol=0, conlim=0, itn_limit=iters + 1, fixed_count=True,
                want_se=False, trace=lambda st: stamps.append(time.perf_counter()), trace_vectors=False, repro=repro)
    per = [b - a for a, b in zip(stamps[:-1], stamps[1:])]
    t_it = float(np.median(per))
    t_pr = _time_products(S, (S.aprod1_repro, S.aprod2_repro) if repro else (S.aprod1, S.aprod2)) if P > 1 else 0.0
    serial = {"value": t_it + (P - 1) * t_pr, "cores": 1, "sample_s_per_iter": t_it, "sample_products_s": t_pr}
    sample = (f"rows of shard 0 of {P} of {w.name} ({S.n_rows} of {w.n_obs} rows; all {S.n_cols} columns), "
              f"{len(per)} timed LSQR iterations{' (repro mode)' if repro else ''} after 1 untimed; "
              f"full-system s/iteration extrapolated as "
              f"t_iter + (P-1) * t(aprod1 + aprod2) on the sample (setup {t_setup:.1f} s excluded)")
    out = {"value": serial["value"], "unit": UNIT, "cores": 1, "kind": "oracle",
           "sample": sample, "serial": serial, "cpu_model": _cpu_model(), "host_cores": _host_cores()}
    if all_cores and not repro:
        r = oracle.time_lsqr_omp(S, iters, threads=_host_cores())
        L = oracle.omp_lib()
        fns = (lambda x, y: L.orc_omp_aprod1(ctypes.byref(S.S), oracle._p(x), oracle._p(y)),
               lambda y, x: L.orc_omp_aprod2(ctypes.byref(S.S), oracle._p(y), oracle._p(x)))
        o_it = float(np.median(r["per_iter_s"]))
        o_pr = _time_products(S, fns) if P > 1 else 0.0
        omp = {"value": o_it + (P - 1) * o_pr, "cores": r["threads"], "sample_s_per_iter": o_it,
               "sample_products_s": o_pr,
               "build": "oracle/omp_timing.c (the oracle source with OpenMP loops/products; timing only)"}
        out.update(value=omp["value"], cores=omp["cores"], build="all-core OpenMP timing build (value, cores); "
                   "the serial checker as it stands under 'serial'", all_cores=omp)
    return out


def _host_cores():
    """Cores this process may run on (the OpenMP timing build uses all of them, whatever OMP_NUM_THREADS says:
    torchrun exports OMP_NUM_THREADS=1 to every rank, and only rank 0 runs the oracle)."""
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count() or 1


def _mem_available():
    """MemAvailable of this host in bytes (None if unknown)."""
    try:
        for line in open("/proc/meminfo"):
            if line.startswith("MemAvailable:"):
                return int(line.split()[1]) * 1024
    except Exception:
        pass
    return None


def _cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return None


def time_api_products(s, k, ap1_bytes, ap2_bytes, peak, max_over_ranks):
    """The boundary's own product calls, lsqr_aprod1 (y += A x) and lsqr_aprod2 (x += A^T y, shared slice
    allreduced), k calls each between CUDA events on the caller's stream (device tensors).  Algorithmic bytes:
    aprod1 as the iteration's; aprod2 216 B/row + 120 B/star (z row sums written and read back, x_astro read and
    written) + 8 B/shared column."""
    import torch
    x = torch.full((s.n_local_cols,), 1e-3, dtype=torch.float64, device="cuda")
    y = torch.zeros(s.n_local_rows + s.n_constr, dtype=torch.float64, device="cuda")
    out = {"calls": k}
    for name, fn, nb in (("aprod1", lambda: s.aprod1(x, y), ap1_bytes), ("aprod2", lambda: s.aprod2(y, x), ap2_bytes)):
        fn()  # warm-up
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record(s.stream)
        for _ in range(k):
            fn()
        e1.record(s.stream)
        e1.synchronize()
        ms = max_over_ranks(e0.elapsed_time(e1) / k)
        out[name + "_ms"] = round(ms, 5)
        out[name + "_frac"] = round(nb / (ms * 1e-3) / 1e9 / peak, 4)
    out["note"] = ("lsqr_aprod1 / lsqr_aprod2 C-ABI calls on device buffers (k calls each, CUDA events on the "
                   "caller's stream); frac against the measured HBM peak on their algorithmic bytes")
    return out


def variant_name(args):
    if getattr(args, "force_collectives", False):
        base = "fused single pass" if getattr(args, "fused", False) else "two-pass"
        return base + " via the multi-rank path (forced 1-rank NCCL collectives)"
    if getattr(args, "repro", False):
        return "bitwise-reproducible (SURVEY 8(f) NEXT-4; exact digit reductions, verification mode)"
    return "fused single pass" if getattr(args, "fused", False) else "two-pass"


def config_block(w, n, args, extra=None):
    """w: the whole job's workload (weak scaling: n x the per-GPU shape; strong: the configuration, sharded)."""
    a_gpu = w.a_bytes // n
    c = {"workload": w.name, "scaling": getattr(args, "scaling", "weak"),
         "n_stars_per_gpu": w.n_stars // n, "n_obs_per_gpu": w.n_obs // n, "n_att": w.n_att,
         "n_instr": w.n_instr, "n_glob": w.n_glob, "constraint_rows": w.n_constr, "obs_jitter_pct": w.jitter_pct,
         "A_bytes_per_gpu": a_gpu, "total_rows": w.n_obs, "preconditioned": True,
         "mode": "fixed-count (paper timing mode)", "seed": w.seed, "parallelism": f"dp{n} (rows sharded by star)",
         "variant": variant_name(args),
         "l2": "no flush: A per GPU (%.2f GB) >> L2 (126 MB)" % (a_gpu / 1e9)}
    if extra:
        c.update(extra)
    return c


def workload_of(args):
    """The named configuration, with the shared-slice dimensions optionally overridden (SURVEY §8(d) sensitivity
    sweep: n_att and n_instr on the C3 shape)."""
    w = W.CONFIGS[args.config]
    if args.n_att:
        w = w.replace(n_att=args.n_att, name=f"{w.name}-att{args.n_att}")
    if args.n_instr:
        w = w.replace(n_instr=args.n_instr, name=f"{w.name}-instr{args.n_instr}")
    return w


# ------------------------------------------------------------------------------------------------ reference arm
def run_reference(args):
    """Reference arm: the CPU oracle (this tier has no reference implementation; the oracle is the base contract's
    reference) timed on the host cores -- its all-core OpenMP timing build -- on the same config, each step one LSQR
    iteration over the bounded sample of oracle_sample(), extrapolated to the full workload as in cpu_baseline()."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    n = int(os.environ.get("WORLD_SIZE", str(args.gpus)))
    base = workload_of(args)
    # the whole job our arm times at this N (weak: n x the configuration; strong: the configuration)
    w = (base.per_gpu(n) if (n > 1 and args.scaling == "weak") else base).replace(name=base.name)
    import ctypes
    import oracle
    t0 = time.perf_counter()
    S, P = oracle_sample(w)
    S.apply_precond()
    setup = time.perf_counter() - t0
    r = oracle.time_lsqr_omp(S, args.warmup + args.steps, threads=_host_cores())
    per = r["per_iter_s"][args.warmup:]
    L = oracle.omp_lib()
    t_pr = _time_products(S, (lambda x, y: L.orc_omp_aprod1(ctypes.byref(S.S), oracle._p(x), oracle._p(y)),
                              lambda y, x: L.orc_omp_aprod2(ctypes.byref(S.S), oracle._p(y), oracle._p(x)))) \
        if P > 1 else 0.0
    t_it = float(np.mean(per))
    v = t_it + (P - 1) * t_pr
    sample = (f"rows of shard 0 of {P} of {w.name} ({S.n_rows} of {w.n_obs} rows; all {S.n_cols} columns), "
              f"{len(per)} LSQR iterations after {args.warmup} warm-up (mean {t_it:.4f} s on the sample); "
              f"full-system s/iteration = t_iter + (P-1) * t(aprod1 + aprod2) = {v:.3f} (setup {setup:.1f} s excluded)")
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": UNIT, "n_gpus": n,
            "steps": len(per), "warmup": args.warmup, "ms_per_step": v * 1e3, "higher_is_better": False,
            "scaling": args.scaling, "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": config_block(w, n, args, {"note": "CPU oracle, all-core OpenMP timing build "
                                                        "(oracle/omp_timing.c), on the host; rank 0 only, timing "
                                                        "the whole job of this N"}),
            "cpu_baseline": {"value": v, "unit": UNIT, "cores": r["threads"], "kind": "oracle",
                             "build": "all-core OpenMP timing build (oracle/omp_timing.c)", "sample": sample,
                             "cpu_model": _cpu_model(), "host_cores": _host_cores()},
            "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    emit(line)
    return 0


# ------------------------------------------------------------------------------------------------ our arm
def run_ours(args):
    import torch
    import torch.distributed as dist
    import paper_conf_sc_malenzacsbvba24_b200 as avu

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = 0 if args.same_device else int(os.environ.get("LOCAL_RANK", "0"))
    n = world
    torch.cuda.set_device(local)
    multi = world > 1
    use_nccl = args.comm == "nccl"
    if multi and use_nccl:
        # NCCL's own init log on stderr (communicator size, NVLS / ring / tree choice) so the launch can be audited;
        # the JSON line goes to stdout
        os.environ.setdefault("NCCL_DEBUG", "INFO")
    if multi:
        if use_nccl:
            dist.init_process_group("nccl", rank=rank, world_size=world, device_id=torch.device("cuda", local))
        else:  # test mode: gloo + the library's host-callback communicator (ranks may share one GPU)
            dist.init_process_group("gloo", rank=rank, world_size=world)
    base = workload_of(args)
    # weak: every GPU holds one configuration-sized shard (n x the shape); strong: the configuration itself, each
    # rank its O-SHARD star range (C4 over 1/2/4/8 GPUs)
    w = base.per_gpu(n) if (n > 1 and args.scaling == "weak") else base
    w = w.replace(name=base.name)
    def comm_kw():
        """A FRESH ncclUniqueId per communicator (NCCL ids must not be reused), broadcast from rank 0."""
        if not multi:
            return {}
        if not use_nccl:
            return dict(comm="callback")
        obj = [avu.nccl_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        return dict(comm="nccl", nccl_id=obj[0])
    K, Wm = args.steps, args.warmup

    def barrier():
        if multi:
            dist.barrier()
        torch.cuda.synchronize()

    def max_over_ranks(v):
        if not multi:
            return v
        t = torch.tensor([v], dtype=torch.float64, device="cuda" if use_nccl else "cpu")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    # ---------------- e2e through the public API with HOST buffers (set_system -> precondition -> solve -> x, se)
    e2e = None
    if args.e2e:
        # host inputs in the paper's layout: values 192 B/row, matrixIndexAstro / matrixIndexAtt 8 B/row
        # each, instrCol 48 B/row, b 8 B/row -- allocated pinned ONCE and filled in place (lsqr_get_system into the
        # pinned buffers), so the host holds one copy (C3: 54.9 GB)
        s0 = avu.Solver.synthetic(w, rank=rank, nranks=world, **comm_kw())
        nloc_rows, nloc_cols = s0.n_local_rows, s0.n_local_cols
        need = nloc_rows * (24 * 8 + 8 + 8 + 48 + 8)
        local_ranks = int(os.environ.get("LOCAL_WORLD_SIZE", "1"))  # ranks of this node pin their inputs at once
        avail = _mem_available()
        short = avail is not None and need * local_ranks > 0.85 * avail
        if multi:  # the decision must be the same on every rank (the e2e leg has barriers and reductions)
            t = torch.tensor([1.0 if short else 0.0], dtype=torch.float64, device="cuda" if use_nccl else "cpu")
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            short = bool(t.item() > 0)
        if short:
            s0.close()
            e2e = {"value": None, "unit": UNIT,
                   "skipped": f"host RAM: {need * local_ranks / 1e9:.1f} GB of pinned inputs needed on this node, "
                              f"{(avail or 0) / 1e9:.1f} GB available"}
    if args.e2e and e2e is None:
        pin = {"vals": np.empty((nloc_rows, 24), dtype=np.float64), "mA": np.empty(nloc_rows, dtype=np.int64),
               "mT": np.empty(nloc_rows, dtype=np.int64), "iC": np.empty((nloc_rows, 6), dtype=np.int64),
               "b": np.empty(nloc_rows, dtype=np.float64)}
        cudart = torch.cuda.cudart()
        for a in pin.values():  # page-locked in place (exact size; torch's pinned allocator rounds up to 2^k)
            rc = cudart.cudaHostRegister(a.ctypes.data, a.nbytes, 0)
            assert int(rc) == 0, f"cudaHostRegister failed: {rc}"
        s0.get_system_ptrs(*[pin[k].ctypes.data for k in ("vals", "mA", "mT", "iC", "b")])
        s0.close()
        torch.cuda.synchronize()
        xo = torch.empty(nloc_cols, dtype=torch.float64).pin_memory()
        so = torch.empty(nloc_cols, dtype=torch.float64).pin_memory()
        se = avu.Solver.synthetic(w, rank=rank, nranks=world, generate=False, **comm_kw())
        if args.repro:
            se.set_reproducible(True)

        def e2e_cycle(itn):
            se.set_system_ptrs(*[pin[k].ctypes.data for k in ("vals", "mA", "mT", "iC", "b")])
            t1 = time.perf_counter()  # set_system is synchronous (host buffers are borrowed for the call only)
            se.precondition()
            out = se.solve(x_out=xo, se_out=so, itn_limit=itn, atol=0, btol=0, conlim=0, fixed_count=True,
                           fused=args.fused)
            return out, t1

        # one untimed cycle with W iterations on the same handle: first-use costs (lazy module loading, CUDA-graph
        # capture and instantiation) are warm-up, as for the device-resident pass
        e2e_cycle(max(Wm, 1))
        barrier()
        t0 = time.perf_counter()
        r, t1 = e2e_cycle(K)
        barrier()
        t3 = time.perf_counter()
        t_e2e = max_over_ranks(t3 - t0)
        h2d = sum(a.nbytes for a in pin.values())
        e2e = {"value": t_e2e / K, "unit": UNIT, "h2d_bytes_per_step": int(h2d * n / K),
               "d2h_bytes_per_step": int(2 * nloc_cols * 8 * n / K), "itn": r["itn"],
               "split_s": {"set_system": round(t1 - t0, 5), "precondition_solve_copy_out": round(t3 - t1, 5)},
               "note": "lsqr_set_system (pinned host A, indices, b) + lsqr_precondition + lsqr_solve(K iterations, "
                       "fixed count) + x, se to pinned host; wall clock / K, max over ranks; after one untimed "
                       "warm-up cycle (W iterations) on the same handle"}
        se.close()
        torch.cuda.synchronize()
        for a in pin.values():
            cudart.cudaHostUnregister(a.ctypes.data)
        del pin

    # ---------------- device-resident timing
    # pass 1 (the headline `value`): K iterations through the production path (lsqr_iterate: CUDA-graph replay, as
    # lsqr_solve runs them), CUDA events on the library stream around the K iterations only.
    # pass 2 (kernel roofline): K more iterations through lsqr_iterate_timed, CUDA events around every kernel launch
    # (those events cost ~7 % of a C2 step, which is why they are not in pass 1).
    s = avu.Solver.synthetic(w, rank=rank, nranks=world, force_collectives=args.force_collectives, **comm_kw())
    if args.repro:
        s.set_reproducible(True)
    t0 = time.perf_counter()
    s.precondition()
    s.init(itn_limit=4 * K + 2 * Wm + 10, atol=0, btol=0, conlim=0, fixed_count=True, use_graph=True,
           fused=args.fused)
    s.sync()
    t_setup = time.perf_counter() - t0
    if Wm > 0:
        s.iterate(Wm)
    barrier()
    with ClockSampler(local) as clk:
        t_pass1 = s.iterate_events(K)
        barrier()
        if Wm > 0:
            s.iterate_timed(Wm)
        barrier()
        r = s.iterate_timed(K)
        barrier()
        # 3 repetitions of the K-iteration measurement, median and min reported
        reps = [t_pass1]
        for _ in range(2):
            reps.append(s.iterate_events(K))
            barrier()
    reps = [max_over_ranks(t) / K for t in reps]
    t_ms = max_over_ranks(t_pass1)
    ap1_ms = max_over_ranks(r["aprod1_ms"] / K)
    ap2_ms = max_over_ranks(r["aprod2_ms"] / K)
    t_instr_ms = max_over_ranks(r["total_ms"])
    st, _ = s.get_state(vectors=False)
    peak, peak_kind = measured_peaks()
    ap1_b, ap2_b, it_b = algorithmic_bytes(w, s.n_local_rows, s.star_end - s.star_begin, s.n_shared,
                                           s.n_local_cols)
    if args.repro:
        # NEXT-4: the whole iteration (7 launches) is one timed unit; the algorithmic bytes are the two-pass ones
        kname, kb, kms = "repro iteration", it_b, t_instr_ms / K
    elif args.fused:
        # fused single pass (NEXT-1): A, indices, u_hat read once + u_hat written (224 B/row), v_astro read and
        # zA written (80 B/star), v_shared gathered and z_shared written once (16 B/column)
        n_st = s.star_end - s.star_begin
        fz_b = 224 * s.n_local_rows + 80 * n_st + 16 * s.n_shared
        it_b = 224 * s.n_local_rows + 56 * s.n_local_cols + 80 * n_st
        kname, kb, kms = "fused", fz_b, ap1_ms
        ap1_b = fz_b
    elif ap2_ms >= ap1_ms:
        kname, kb, kms = "aprod2", ap2_b, ap2_ms
    else:
        kname, kb, kms = "aprod1", ap1_b, ap1_ms
    achieved = kb / (kms * 1e-3) / 1e9
    ms_step = t_ms / K
    line = {
        "metric": METRIC, "value": ms_step * 1e-3, "unit": UNIT, "n_gpus": n, "steps": K, "warmup": Wm,
        "ms_per_step": ms_step, "higher_is_better": False, "scaling": args.scaling, "vs_baseline": None,
        "dtype": "f64",
        "data": "synthetic",
        "config": config_block(w, n, args, {"setup_s": round(t_setup, 3)}),
        "repetitions": {"ms_per_step": [round(t, 5) for t in reps], "median": round(statistics.median(reps), 5),
                        "min": round(min(reps), 5), "note": "value = repetition 1 (the first K-step pass)"},
        "roofline": {"bound": "hbm", "kernel": kname, "achieved": round(achieved, 1), "peak": peak,
                     "peak_kind": f"{peak_kind} (MEASURED_PEAKS.json hbm_gbs, copy; burst)", "unit": "GB/s",
                     "frac": round(achieved / peak, 4), "traffic": load_traffic(w.name if n == 1 else None, kname),
                     "algorithmic_bytes_per_launch": kb, "avg_launch_ms": round(kms, 4)},
        "iteration_roofline": {"algorithmic_bytes": it_b, "achieved_GBps": round(it_b / (ms_step * 1e-3) / 1e9, 1),
                               "frac": round(it_b / (ms_step * 1e-3) / 1e9 / peak, 4),
                               "aprod1_ms": round(ap1_ms, 4), "aprod2_ms": round(ap2_ms, 4),
                               "aprod1_frac": (round(ap1_b / (ap1_ms * 1e-3) / 1e9 / peak, 4)
                                               if not args.repro else None),
                               "aprod2_frac": (round(ap2_b / (ap2_ms * 1e-3) / 1e9 / peak, 4)
                                               if not (args.fused or args.repro) else None),
                               "variant": variant_name(args) if args.repro else
                               ("fused single pass (SURVEY 8(f) NEXT-1; bytes are its own 224 B/row)"
                                if args.fused else "two-pass (SURVEY 8(a)); 440 B/row")},
        "gpu_launches": int(max_over_ranks(r["launches"])),
        "timing": {"value_pass": "lsqr_iterate x K (CUDA graph replay, the lsqr_solve path), events around the K "
                                 "iterations", "roofline_pass": "lsqr_iterate_timed x K (events around every kernel)",
                   "note": "the two passes run back to back in the clock-sampled region; under the power cap their "
                           "SM clocks can differ by ~1 %, so avg_launch_ms can exceed ms_per_step",
                   "instrumented_ms_per_step": round(t_instr_ms / K, 5)},
        "clocks": clk.summary(),
        "e2e": e2e,
        "lsqr": {"itn": st["itn"], "r1norm": st["r1norm"], "arnorm": st["arnorm"]},
    }
    if not args.repro:
        line["api_products"] = time_api_products(s, min(K, 20), ap1_b,
                                                 216 * s.n_local_rows + 120 * (s.star_end - s.star_begin)
                                                 + 8 * s.n_shared, peak, max_over_ranks)
    s.close()
    if rank == 0 and n == 1 and args.cpu_baseline:
        line["cpu_baseline"] = cpu_baseline(base, iters=min(args.cpu_iters, 5) if args.repro else args.cpu_iters,
                                            repro=args.repro)
    if rank == 0:
        emit(line)
    if multi:
        dist.barrier()
        dist.destroy_process_group()
    return 0


_JSON_OUT = None


def _guard_stdout():
    """stdout carries exactly one JSON line (rank 0): libraries that print to the C-level stdout (e.g. NCCL's
    'NCCL version ...' banner at communicator init, on every rank) are redirected to stderr by pointing fd 1 at
    fd 2; the JSON line goes to a saved duplicate of the original stdout."""
    global _JSON_OUT
    if _JSON_OUT is None:
        sys.stdout.flush()
        _JSON_OUT = os.fdopen(os.dup(1), "w")
        os.dup2(2, 1)


def emit(line: dict):
    out = _JSON_OUT if _JSON_OUT is not None else sys.stdout
    out.write(json.dumps(line) + "\n")
    out.flush()


def main():
    _guard_stdout()
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=100)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="C3", choices=sorted(W.CONFIGS),
                    help="workload (default C3: BASELINE.json configs[2], the largest single-GPU configuration)")
    ap.add_argument("--no-e2e", dest="e2e", action="store_false")
    ap.add_argument("--no-cpu-baseline", dest="cpu_baseline", action="store_false")
    ap.add_argument("--cpu-iters", type=int, default=3,
                    help="oracle LSQR iterations timed for cpu_baseline on its bounded sample (oracle_sample)")
    ap.add_argument("--n-att", type=int, default=0, help="override n_att (multiple of 3, >= 12; sensitivity sweep)")
    ap.add_argument("--n-instr", type=int, default=0, help="override n_instr (multiple of 6; sensitivity sweep)")
    ap.add_argument("--fused", dest="fused", action="store_true", default=True,
                    help="fused single-pass iteration (SURVEY 8(f) NEXT-1; default)")
    ap.add_argument("--two-pass", dest="fused", action="store_false", help="two-pass iteration (aprod1 then aprod2)")
    ap.add_argument("--repro", action="store_true",
                    help="bitwise-reproducible mode (SURVEY 8(f) NEXT-4; single GPU; verification, not speed)")
    ap.add_argument("--scaling", default="weak", choices=["weak", "strong"],
                    help="weak: one configuration-sized shard per GPU (default); strong: the configuration split "
                         "over the GPUs (SURVEY 8(d) C4 over 1/2/4/8)")
    ap.add_argument("--comm", default="nccl", choices=["nccl", "gloo-callback"],
                    help="multi-rank communicator (gloo-callback: test mode through the library's host callback)")
    ap.add_argument("--same-device", action="store_true", help="test mode: every rank on cuda:0")
    ap.add_argument("--force-collectives", action="store_true",
                    help="diagnostic: run the multi-rank algorithm and its NCCL collectives on a 1-rank communicator "
                         "(measures the P > 1 code path's cost without a network)")
    args = ap.parse_args()
    if args.warmup < 3:
        print("warning: --warmup < 3 violates the timing rules", file=sys.stderr)
    if args.repro and int(os.environ.get("WORLD_SIZE", "1")) > 1:
        print("--repro is single-GPU", file=sys.stderr)
        return 2
    if args.impl == "reference":
        return run_reference(args)
    return run_ours(args)


if __name__ == "__main__":
    sys.exit(main())

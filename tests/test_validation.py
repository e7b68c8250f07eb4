"""NEXT-3: the paper's validation procedure (§V-C) on production-shaped synthetic
systems.  The paper validates a port by solving to convergence and comparing x and its standard errors with a trusted
implementation: (1) the solutions agree within 1 sigma; (2) the mean and the standard deviation of the sigma
differences are small (< 10 micro-arcseconds on the real data).  Our synthetic system has no physical
units, so (2) is applied relative to sigma.

Trusted implementation = the CPU oracle (the serial checker):
  * C2val: C2's shape at 2 M rows, oracle solved in the test; fused and two-pass GPU iterations;
  * C3v and C3 (BASELINE configs[2] itself, 208 M rows): the oracle's solution stored by tests/golden/make_next3.py
    (x and sigma on a column sample, float32) -- the GPU solves the full system in the test;
  * across ranks (C2val): P = 2 and 3 ranks (host-callback communicator, ranks sharing cuda:0) against P = 1 and the
    oracle, with the same criteria.
"""
import os

import numpy as np
import pytest

import oracle
import workloads as W
from tests.golden import make_next3

pytestmark = pytest.mark.gpu

W_VAL = W.C2.replace(name="C2val", n_stars=20_000, n_obs=2_000_000, seed=11)  # C2 shape, 2 M rows
TOL = dict(atol=1e-12, btol=1e-12, conlim=0)


@pytest.fixture(scope="module")
def reference():
    S = oracle.System(W_VAL)
    r = oracle.solve_system(S, itn_limit=3000, fixed_count=False, **TOL)
    assert r["istop"] in (1, 2, 4, 5), r["istop"]
    # the rounding-independent sigma at the same iteration: the oracle's test-only fully reorthogonalised LSQR
    # (pinned to the OLS formula at k = n, tests/test_oracle_lsqr.py); DESIGN R5
    rr = oracle.lsqr(S.m_local, S.n_cols, S, S.rhs(), reorth=True, atol=0, btol=0, conlim=0, itn_limit=r["itn"],
                     fixed_count=True)
    r["se_reorth"] = S.D * rr["se"]
    return r


def paper_criteria(x, se, x_ref, se_ref):
    within = np.abs(x - x_ref) <= se_ref                    # (1) solution within 1 sigma
    dsig = (se - se_ref) / se_ref                           # (2) sigma differences, relative
    return within.mean(), float(np.mean(dsig)), float(np.std(dsig))


def check(tag, out, x_ref, se_ref, itn_ref, x_tol=1e-8, se_reorth=None):
    frac, mean_d, std_d = paper_criteria(out["x"], out["se"], x_ref, se_ref)
    print(f"\nvalidation {tag}: itn {out['itn']} (oracle {itn_ref}), istop {out['istop']}; "
          f"x within 1 sigma: {100 * frac:.3f} %; sigma diff mean {mean_d:.2e} std {std_d:.2e}; "
          f"max |dx|/sigma {np.max(np.abs(out['x'] - x_ref) / se_ref):.2e}")
    assert out["istop"] in (1, 2, 4, 5)
    assert abs(out["itn"] - itn_ref) <= max(5, itn_ref // 20)
    assert frac == 1.0
    # The LSQR sigma is itself an estimate that depends on the iteration's rounding history (SURVEY EXP-4/5, DESIGN
    # R5): at this early convergence (k ~ 30-40) the oracle's sigma is 13 % below the reorthogonalised value (C2val),
    # and two valid roundings differ by ~2 % on average.  The paper's criterion is statistical: mean and spread of
    # the sigma differences small against sigma itself.
    assert abs(mean_d) <= 5e-2 and std_d <= 5e-2
    if se_reorth is not None:  # and the GPU's sigma is no farther from the rounding-independent value than the oracle's
        dg = np.median(np.abs(out["se"] / se_reorth - 1))
        do = np.median(np.abs(se_ref / se_reorth - 1))
        print(f"  sigma vs reorthogonalised: gpu {dg:.3e}, oracle {do:.3e}")
        assert dg <= 1.25 * do
    assert np.linalg.norm(out["x"] - x_ref) <= x_tol * np.linalg.norm(x_ref)


@pytest.mark.parametrize("fused", [True, False], ids=["fused", "twopass"])
def test_validation_vs_oracle(cuda_device, reference, fused):
    import paper_conf_sc_malenzacsbvba24_b200 as avu
    s = avu.Solver.synthetic(W_VAL)
    s.precondition()
    out = s.solve(itn_limit=3000, fused=fused, **TOL)
    s.close()
    check(f"C2val fused={fused}", out, reference["x"], reference["se"], reference["itn"],
          se_reorth=reference["se_reorth"])


@pytest.mark.parametrize("name", ["C3v", "C3"])
def test_validation_production_shape(cuda_device, name):
    """The stored oracle solution of a C3-shaped system (C3v, 20.8 M rows) and of C3 itself (208 M rows, 39.9 GB of
    A): the GPU (default fused path) solves the full system to the same tolerances; compared on the stored column
    sample (float32: x to 1e-6)."""
    import paper_conf_sc_malenzacsbvba24_b200 as avu
    p = make_next3.path(name)
    if not os.path.exists(p):
        pytest.skip(f"{p} not generated (python -m tests.golden.make_next3 {name})")
    ref = np.load(p)
    w = make_next3.WORKLOADS[name]
    assert str(ref["workload"]) == repr(w)
    s = avu.Solver.synthetic(w)
    s.precondition()
    out = s.solve(itn_limit=3000, **TOL)
    s.close()
    cols = make_next3.sample_columns(w)
    out_s = dict(out, x=out["x"][cols], se=out["se"][cols])
    check(name, out_s, ref["x"].astype(np.float64), ref["se"].astype(np.float64), int(ref["itn"]), x_tol=1e-6)
    assert abs(out["r1norm"] - float(ref["r1norm"])) <= 1e-9 * float(ref["r1norm"])


# ------------------------------------------------------------------------------------------------ across ranks
def _rank_worker(rank, world, port, q):
    try:
        import sys
        sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
        import torch
        import torch.distributed as dist
        import paper_conf_sc_malenzacsbvba24_b200 as avu
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        torch.cuda.set_device(0)
        s = avu.Solver.synthetic(W_VAL, rank=rank, nranks=world, comm="callback")
        s.precondition()
        out = s.solve(itn_limit=3000, **TOL)
        q.put((rank, s.star_begin, s.star_end, out["x"], out["se"], out["itn"], out["istop"]))
        s.close()
        dist.destroy_process_group()
    except Exception:
        import traceback
        q.put(("error", traceback.format_exc()))


@pytest.mark.parametrize("P", [2, 3])
def test_validation_across_ranks(cuda_device, reference, P):
    """The same validation across rank counts: P ranks' solutions (gathered into the global column order with the
    O-SHARD maps) against the oracle and against the 1-rank GPU solve, with the paper's criteria."""
    import socket
    import torch.multiprocessing as mp
    import paper_conf_sc_malenzacsbvba24_b200 as avu
    sk = socket.socket()
    sk.bind(("127.0.0.1", 0))
    port = sk.getsockname()[1]
    sk.close()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_rank_worker, args=(r, P, port, q)) for r in range(P)]
    for p in ps:
        p.start()
    outs = [q.get(timeout=900) for _ in range(P)]
    for p in ps:
        p.join(60)
    for o in outs:
        assert o[0] != "error", o[1]
    outs.sort(key=lambda o: o[0])
    w = W_VAL
    A0 = 5 * w.n_stars
    x = np.zeros(w.n_cols)
    se = np.zeros(w.n_cols)
    itns = set()
    for (rank, sb, send, xl, sel, itn, istop) in outs:
        A0l = 5 * (send - sb)
        x[5 * sb:5 * send], se[5 * sb:5 * send] = xl[:A0l], sel[:A0l]
        if rank == 0:
            x[A0:], se[A0:] = xl[A0l:], sel[A0l:]
        else:  # the shared slice is replicated (computed identically from the allreduced sums on every rank)
            assert np.allclose(xl[A0l:], x[A0:], rtol=1e-12, atol=0)
        itns.add((itn, istop))
    assert len(itns) == 1, itns  # every rank stopped at the same iteration
    itn, istop = itns.pop()
    out = dict(x=x, se=se, itn=itn, istop=istop)
    check(f"C2val P={P} vs oracle", out, reference["x"], reference["se"], reference["itn"],
          se_reorth=reference["se_reorth"])
    s = avu.Solver.synthetic(w)
    s.precondition()
    one = s.solve(itn_limit=3000, **TOL)
    s.close()
    check(f"C2val P={P} vs P=1", out, one["x"], one["se"], one["itn"])

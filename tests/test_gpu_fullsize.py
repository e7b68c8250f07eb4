"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times (SURVEY §8(c) parity contract:
"at full sizes ... on sampled outputs the oracle can compute one by one, else via properties that hold at any size").

  configs[2] C3    208 M rows, 40 GB of A, one GPU (bench --config C3)
  configs[4] C5    625 M rows, 120 GB of A: the per-GPU shard of the weak-scaling system (bench --config C5)
  configs[3] C4    rank 3 of the 8-GPU strong-scaling shard map (97.5 M rows; single process, the allreduce callback
                   is a no-op, so local rows and local astro columns are exact and the shared slice is this rank's
                   partial sum)

Checked on each:
  * aprod1 on sampled stars' rows (random x): the oracle regenerates those stars (O-GEN) and computes the rows one by
    one; |gpu - oracle| <= 1e-13 (sum |a_ij x_j| + |y_i|) -- this also pins the device generator at full size;
  * aprod2 on the same stars' astro columns (random y), same tolerance;
  * the adjoint identity <A x, y> = <x, A^T y> over the whole shard (relative 1e-12 of sum |a x y|);
  * C3/C5: LSQR's residual estimate r1norm equals ||b - A^ x^_k|| recomputed with aprod1 after 20 fixed iterations
    (relative 1e-8), and r1norm is non-increasing over the iterations;
  * C3/C5: a full solve to atol = btol = 1e-14 of the planted consistent system (b = A x_true on the device) stops
    with istop 1/2 and recovers x_true to 1e-9 (measured 1.9e-13 / 1.1e-13 in 25-26 iterations).
"""
import ctypes as C

import numpy as np
import pytest

import oracle
import workloads as W

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def avu(cuda_device):
    import paper_conf_sc_malenzacsbvba24_b200 as m
    return m


def abs_system(S):
    A = oracle.System(S.w, generate=False, stars=(S.star_begin, S.star_end))
    A.vals = np.abs(S.vals); A.mA, A.mT, A.iC = S.mA, S.mT, S.iC
    A.c_val = np.abs(S.c_val); A.c_ptr, A.c_col = S.c_ptr, S.c_col
    A.n_constr = S.n_constr
    A._mk_struct()
    return A


def sampled_stars(s, n, seed):
    rng = np.random.default_rng(seed)
    lo, hi = s.star_begin, s.star_end
    picks = set(rng.integers(lo, hi, size=n).tolist()) | {lo, hi - 1, min(lo + 3, hi - 1)}
    return sorted(picks)


CASES = {
    "C3": dict(w=W.C3, rank=0, nranks=1),
    "C5": dict(w=W.C5, rank=0, nranks=1),
    "C4-r3of8": dict(w=W.C4, rank=3, nranks=8),
}


@pytest.mark.parametrize("case", list(CASES))
def test_fullsize_sampled_products_and_adjoint(avu, case):
    import torch
    cfg = CASES[case]
    w, rank, nranks = cfg["w"], cfg["rank"], cfg["nranks"]
    kw = {} if nranks == 1 else dict(rank=rank, nranks=nranks, comm="callback", allreduce=lambda *a: 0)
    s = avu.Solver.synthetic(w, **kw)
    sb, se = s.star_begin, s.star_end
    A0l = 5 * (se - sb)
    A0 = 5 * w.n_stars
    # row offsets of this rank's stars (oracle's own counts: the shard map itself is pinned elsewhere)
    rp = oracle.row_ptr(oracle.star_counts(w))
    assert s.row_begin == rp[sb] and s.row_end == rp[se]
    gen = torch.Generator(device="cuda").manual_seed(7)
    x = torch.randn(s.n_local_cols, dtype=torch.float64, device="cuda", generator=gen)
    y = torch.zeros(s.n_local_rows + s.n_constr, dtype=torch.float64, device="cuda")
    s.aprod1(x, y)
    yy = torch.randn(s.n_local_rows + s.n_constr, dtype=torch.float64, device="cuda", generator=gen)
    z = torch.zeros(s.n_local_cols, dtype=torch.float64, device="cuda")
    s.aprod2(yy, z)
    # adjoint identity over the whole shard (local A: rows of this rank + owned constraint entries)
    lhs = float(torch.dot(y, yy))
    rhs = float(torch.dot(x, z))
    bound = float(torch.dot(torch.abs(x), torch.abs(z))) + float(torch.dot(torch.abs(y), torch.abs(yy)))
    assert abs(lhs - rhs) <= 1e-12 * bound, (lhs, rhs, bound)
    # global-column view of x for the oracle
    xh = x.cpu().numpy()
    xg = np.zeros(w.n_cols)
    xg[5 * sb:5 * se] = xh[:A0l]
    xg[A0:] = xh[A0l:]
    yh_c = yy[s.n_local_rows:].cpu().numpy()  # constraint part of y (replicated)
    for st in sampled_stars(s, 24, seed=11):
        S = oracle.System(w, stars=(st, st + 1))
        Aabs = abs_system(S)
        r0 = int(rp[st] - rp[sb])  # local row offset
        n = S.n_rows
        # aprod1 rows of star st
        yo = np.zeros(S.m_local)
        S.aprod1(xg, yo)
        sc = np.zeros(S.m_local)
        Aabs.aprod1(np.abs(xg), sc)
        got = y[r0:r0 + n].cpu().numpy()
        err = np.abs(got - yo[:n])
        assert (err <= 1e-13 * sc[:n] + 1e-300).all(), (case, st, err.max())
        # aprod2 astro columns of star st (its rows + the constraint rows' owned entries)
        yin = np.concatenate([yy[r0:r0 + n].cpu().numpy(), yh_c])
        xo = np.zeros(w.n_cols)
        S.aprod2(yin, xo)
        sc2 = np.zeros(w.n_cols)
        Aabs.aprod2(np.abs(yin), sc2)
        la = 5 * (st - sb)
        got2 = z[la:la + 5].cpu().numpy()
        ref2 = xo[5 * st:5 * st + 5]
        assert (np.abs(got2 - ref2) <= 1e-13 * sc2[5 * st:5 * st + 5] + 1e-300).all(), (case, st, got2, ref2)
    s.close()
    del x, y, yy, z
    torch.cuda.empty_cache()


@pytest.mark.parametrize("case", ["C3", "C5"])
def test_fullsize_lsqr_residual_estimate(avu, case):
    """r1norm (Paige-Saunders' recurrence estimate of ||b - A^ x^||) against the residual recomputed with aprod1 at
    full size, after 20 fixed iterations of the default (fused) path; and monotone r1norm."""
    import torch
    from paper_conf_sc_malenzacsbvba24_b200 import _capi
    w = CASES[case]["w"]
    s = avu.Solver.synthetic(w)
    b = torch.empty(s.n_local_rows, dtype=torch.float64, device="cuda")
    s._chk(_capi.lib().lsqr_get_system(s._h, None, None, None, None, C.c_void_p(b.data_ptr())))
    s.precondition()
    D = torch.tensor(s.get_precond(), device="cuda")
    s.init(itn_limit=20, atol=0, btol=0, conlim=0, fixed_count=True, use_graph=True, fused=True)
    r1 = []
    for _ in range(20):
        s.iterate(1)
        st, _ = s.get_state(vectors=False)
        r1.append(st["r1norm"])
    out = s.finalize(x_out=torch.empty(s.n_local_cols, dtype=torch.float64, device="cuda"))
    assert all(b_ <= a_ * (1 + 1e-12) for a_, b_ in zip(r1, r1[1:])), r1
    xhat = out["x"] / D  # scaled variables
    r = torch.zeros(s.n_local_rows + s.n_constr, dtype=torch.float64, device="cuda")
    r[:s.n_local_rows] = b  # constraint rhs = 0
    s.aprod1(-xhat, r)       # r = b - A^ x^
    rn = float(torch.linalg.vector_norm(r))
    print(f"{case}: r1norm {out['r1norm']:.12e}  ||b - A x|| {rn:.12e}")
    assert abs(rn - out["r1norm"]) <= 1e-8 * rn
    s.close()
    del b, D, r, xhat
    torch.cuda.empty_cache()


@pytest.mark.parametrize("case", ["C3", "C5"])
def test_fullsize_planted_solution(avu, case):
    """A full solve at full size to atol = btol = 1e-14 on a consistent planted system (b = A x_true generated on
    the device, O-GEN planted mode; no constraint rows, whose rhs 0 would make it inconsistent): Paige-Saunders stops
    with istop 1 or 2 and the unscaled x reproduces x_true."""
    w = CASES[case]["w"].replace(b_mode=1, noise=0.0, n_ext_stars=0)
    s = avu.Solver.synthetic(w)
    s.precondition()
    out = s.solve(itn_limit=4000, atol=1e-14, btol=1e-14, conlim=0)
    s.close()
    xt = oracle.x_true(w)
    rel = np.linalg.norm(out["x"] - xt) / np.linalg.norm(xt)
    print(f"{case} planted: istop {out['istop']} itn {out['itn']} rel(x - x_true) {rel:.2e} "
          f"r1norm {out['r1norm']:.2e} acond {out['acond']:.2e}")
    assert out["istop"] in (1, 2) and out["itn"] < 4000
    assert rel <= 1e-9

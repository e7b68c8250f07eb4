"""Pins for the oracle's products (O-AP1/O-AP2, Eqs. (3)-(4)) and preconditioner (O-PREC).

Pinned against: a dense materialisation of A built with numpy from the paper's index arrays, the
adjoint identity <Ax, y> = <x, A^T y>, unit column norms of A D, and numpy.linalg.lstsq on the unscaled system.
"""
import numpy as np
import pytest

import oracle
import workloads as W

CASES = [W.micro(), W.micro(n_glob=0, seed=5), W.micro(n_stars=9, obs=20, n_ext=4, seed=9),
         W.micro(n_stars=13, obs=25, n_att=36, n_instr=18, n_ext=5, seed=8)]


@pytest.mark.parametrize("w", CASES, ids=lambda w: f"{w.name}-g{w.n_glob}-c{w.n_constr}")
def test_aprod_vs_dense(w):
    S = oracle.System(w)
    A = S.dense()
    rng = np.random.default_rng(0)
    x = rng.standard_normal(S.n_cols)
    y0 = rng.standard_normal(S.m_local)
    y = y0.copy()
    S.aprod1(x, y)
    ref = y0 + A @ x
    scale = np.abs(A) @ np.abs(x) + np.abs(y0)
    assert (np.abs(y - ref) <= 1e-14 * scale).all()
    yy = rng.standard_normal(S.m_local)
    x0 = rng.standard_normal(S.n_cols)
    xx = x0.copy()
    S.aprod2(yy, xx)
    ref2 = x0 + A.T @ yy
    scale2 = np.abs(A.T) @ np.abs(yy) + np.abs(x0)
    assert (np.abs(xx - ref2) <= 1e-14 * scale2).all()


@pytest.mark.parametrize("w", [W.C1, W.C1C], ids=["C1", "C1c"])
def test_adjoint_identity_C1(w):
    S = oracle.System(w)
    rng = np.random.default_rng(1)
    for _ in range(3):
        x = rng.standard_normal(S.n_cols)
        y = rng.standard_normal(S.m_local)
        Ax = np.zeros(S.m_local); S.aprod1(x, Ax)
        Aty = np.zeros(S.n_cols); S.aprod2(y, Aty)
        # sum |a_ij x_j y_i| computed from the absolute-value system
        absS = oracle.System(w)
        absS.vals[:] = np.abs(absS.vals); absS.c_val[:] = np.abs(absS.c_val); absS._mk_struct()
        t = np.zeros(S.m_local); absS.aprod1(np.abs(x), t)
        bound = float(np.abs(y) @ t)
        assert abs(Ax @ y - x @ Aty) <= 1e-13 * bound


def test_duplicate_columns_are_summed():
    w = W.micro(seed=4)
    S = oracle.System(w)
    S.iC[3, 1] = S.iC[3, 0] = S.I0  # force two instr slots of row 3 onto one column (not produced by O-GEN)
    S.mT[5] = S.A0                  # and an attitude window at k0 = 0
    S._mk_struct()
    A = S.dense()
    x = np.arange(S.n_cols, dtype=float) / 7.0
    y = np.zeros(S.m_local); S.aprod1(x, y)
    assert np.allclose(y, A @ x, rtol=1e-14, atol=1e-14)
    yy = np.linspace(-1, 1, S.m_local)
    xx = np.zeros(S.n_cols); S.aprod2(yy, xx)
    assert np.allclose(xx, A.T @ yy, rtol=1e-14, atol=1e-14)


@pytest.mark.parametrize("P", [2, 3, 4])
@pytest.mark.parametrize("w", [W.micro(n_stars=11, obs=20, n_ext=3, seed=21), W.micro(n_stars=10, obs=16, seed=2)])
def test_rank_emulation_equals_single_rank(w, P):
    """O-SHARD P-rank emulation: per-rank products on shard-local rows, 'allreduce' = sum in rank order."""
    full = oracle.System(w)
    rng = np.random.default_rng(3)
    x = rng.standard_normal(full.n_cols)
    y = rng.standard_normal(full.m_local)
    y1 = np.zeros(full.m_local); full.aprod1(x, y1)
    x2 = np.zeros(full.n_cols); full.aprod2(y, x2)
    e1 = np.zeros(full.m_local)
    e2 = np.zeros(full.n_cols)
    for r in range(P):
        S = oracle.System(w, rank=r, nranks=P)
        yl = np.zeros(S.m_local)
        S.aprod1(x, yl)
        e1[S.row_begin:S.row_end] = yl[: S.n_rows]
        e1[full.n_rows:] += yl[S.n_rows:]           # constraint rows: AR1 of the owned partial dots
        yr = np.concatenate([y[S.row_begin:S.row_end], y[full.n_rows:]])
        xl = np.zeros(S.n_cols)
        S.aprod2(yr, xl)
        e2 += xl                                    # astro parts are disjoint; shared slice: AR2
    assert np.allclose(e1, y1, rtol=1e-14, atol=1e-14)
    assert np.allclose(e2, x2, rtol=1e-14, atol=1e-13)


@pytest.mark.parametrize("w", CASES[:3], ids=lambda w: f"{w.name}-g{w.n_glob}-c{w.n_constr}")
def test_precond_unit_columns_and_invariant_solution(w):
    S = oracle.System(w)
    A = S.dense()
    b = S.rhs()
    D = S.apply_precond()
    Ah = S.dense()
    norms = np.linalg.norm(Ah, axis=0)
    nz = np.linalg.norm(A, axis=0) > 0
    assert np.allclose(norms[nz], 1.0, rtol=1e-14, atol=0)
    assert (D[~nz] == 1.0).all()
    assert np.allclose(Ah, A * D[None, :], rtol=1e-15, atol=1e-15)
    # change of variables: x = D y solves the original least-squares problem
    y = np.linalg.lstsq(Ah, b, rcond=None)[0]
    x = np.linalg.lstsq(A, b, rcond=None)[0]
    assert np.linalg.norm(D * y - x) <= 1e-12 * np.linalg.norm(x)


def test_precond_zero_column_gets_unit_D():
    # n_instr = 60 with only 14 rows: most instrumental columns are never touched
    w = W.Workload("z", n_stars=2, n_obs=14, n_att=24, n_instr=60, seed=6)
    S = oracle.System(w)
    A = S.dense()
    D = S.apply_precond()
    empty = np.linalg.norm(A, axis=0) == 0
    assert empty.sum() > 10
    assert (D[empty] == 1.0).all()


def test_omp_timing_variant_matches_serial():
    """bench.py's all-core cpu_baseline runs oracle/omp_timing.c (the oracle source with OpenMP loops and products;
    never a parity reference).  Sanity: it solves the same system -- x after 6 fixed iterations within rounding of
    the serial checker's."""
    import numpy as np
    w = W.C1C.replace(jitter_pct=50)
    S = oracle.System(w)
    S.apply_precond()
    r = oracle.time_lsqr_omp(S, 5)
    ro = oracle.solve_system(oracle.System(w), atol=0, btol=0, conlim=0, itn_limit=6, fixed_count=True)
    assert r["threads"] >= 1 and len(r["per_iter_s"]) == 5
    assert np.linalg.norm(r["x"] - ro["x_scaled"]) <= 1e-12 * np.linalg.norm(ro["x_scaled"])

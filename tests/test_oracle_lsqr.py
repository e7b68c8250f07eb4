"""Pins for the oracle LSQR (O-LSQR: Paige & Saunders, refs [20],[21] of the paper).

Pinned against (none of these re-use the oracle's arithmetic):
  * numpy.linalg.lstsq on micro systems and on the C1 system at convergence (closed-form LS solution);
  * scipy.sparse.linalg.lsqr iterates x_k for small k (the same published algorithm, independent code);
  * full-reorthogonalisation test mode: after n iterations x = lstsq and var = diag((A^T A)^-1) (textbook
    Golub-Kahan / OLS), and se = s sqrt(var) with s^2 = ||r||^2/(m-n);
  * finite termination on diagonal A with d distinct singular values (Krylov dimension d);
  * one-step convergence for orthonormal columns; damped problem vs lstsq on [A; damp I];
  * invariants: ||b - A x_k|| non-increasing and equal to phibar_k; ||x_k|| non-decreasing; planted x_true;
  * istop special cases (b = 0 -> 0; consistent -> 1; iteration limit -> 7).
"""
import numpy as np
import pytest
import scipy.sparse.linalg as spla

import oracle
import workloads as W


def dense_aprod(A):
    def f(mode, vin, vout):
        if mode == 1:
            vout += A @ vin
        else:
            vout += A.T @ vin
    return f


def test_converged_vs_lstsq_micro():
    for w in [W.micro(), W.micro(n_stars=9, obs=20, n_ext=4, seed=9), W.micro(n_glob=0, seed=5)]:
        S = oracle.System(w)
        A, b = S.dense(), S.rhs()
        r = oracle.lsqr(S.m_local, S.n_cols, S, b, atol=1e-15, btol=1e-15, conlim=0, itn_limit=500)
        xs = np.linalg.lstsq(A, b, rcond=None)[0]
        assert np.linalg.norm(r["x"] - xs) <= 1e-12 * np.linalg.norm(xs)
        assert r["istop"] in (1, 2, 4, 5)


def sparse_A(S):
    """scipy.sparse CSR of the (local) system from the paper's index arrays (tests only)."""
    import scipy.sparse as sp
    n = S.n_rows
    cols = np.zeros((n, 24), dtype=np.int64)
    cols[:, 0:5] = S.mA[:, None] + np.arange(5)[None, :]
    for a in range(3):
        cols[:, 5 + 4 * a:9 + 4 * a] = S.mT[:, None] + a * S.n_axis + np.arange(4)[None, :]
    cols[:, 17:23] = S.iC
    cols[:, 23] = S.G0
    ns = 24 if S.w.n_glob else 23
    rows = np.repeat(np.arange(n), ns)
    A = sp.csr_matrix((S.vals[:, :ns].ravel(), (rows, cols[:, :ns].ravel())), shape=(S.m_local, S.n_cols))
    if S.n_constr:
        crow = np.repeat(np.arange(S.n_constr), np.diff(S.c_ptr)) + n
        A = A + sp.csr_matrix((S.c_val, (crow, S.c_col)), shape=A.shape)
    return A


def test_sparse_helper_matches_dense():
    S = oracle.System(W.micro(n_stars=9, obs=20, n_ext=4, seed=9))
    assert np.array_equal(sparse_A(S).toarray(), S.dense())


def test_C1_fixed_100_vs_lstsq():
    import scipy.linalg as sl
    S = oracle.System(W.C1)
    A, b = sparse_A(S), S.rhs()
    r = oracle.solve_system(S, itn_limit=100, fixed_count=True, atol=0, btol=0, conlim=0)
    # closed-form LS solution via the normal equations (kappa(A) ~ 14 on C1, so kappa^2 is harmless)
    AtA = (A.T @ A).toarray()
    xs = sl.cho_solve(sl.cho_factor(AtA), A.T @ b)
    assert r["itn"] == 100
    assert np.linalg.norm(r["x"] - xs) <= 1e-12 * np.linalg.norm(xs)
    rr = b - A @ xs
    assert abs(r["r2norm"] - np.linalg.norm(rr)) <= 1e-10 * np.linalg.norm(rr)


@pytest.mark.parametrize("w", [W.micro(), W.C1.replace(n_stars=200, n_obs=4000)], ids=["micro", "C1s"])
def test_iterates_vs_scipy(w):
    S = oracle.System(w)
    S.apply_precond()
    A, b = S.dense(), S.rhs()
    for k in (1, 2, 5, 10):
        r = oracle.lsqr(S.m_local, S.n_cols, S, b, atol=0, btol=0, conlim=0, itn_limit=k)
        xs = spla.lsqr(A, b, atol=0, btol=0, conlim=0, iter_lim=k)[0]
        assert np.linalg.norm(r["x"] - xs) <= 1e-12 * np.linalg.norm(xs), k


@pytest.mark.parametrize("seed", [3, 7])
def test_reorth_exact_var_and_se(seed):
    S = oracle.System(W.micro(seed=seed))
    A, b = S.dense(), S.rhs()
    m, n = A.shape
    r = oracle.lsqr(m, n, S, b, atol=0, btol=0, conlim=0, itn_limit=n, fixed_count=True, reorth=True)
    xs = np.linalg.lstsq(A, b, rcond=None)[0]
    cov = np.linalg.inv(A.T @ A)
    assert np.linalg.norm(r["x"] - xs) <= 1e-12 * np.linalg.norm(xs)
    assert np.max(np.abs(r["var"] / np.diag(cov) - 1)) <= 1e-10
    s = np.linalg.norm(b - A @ xs) / np.sqrt(m - n)
    assert np.max(np.abs(r["se"] / (s * np.sqrt(np.diag(cov))) - 1)) <= 1e-9


@pytest.mark.parametrize("d", [3, 5, 8])
def test_finite_termination_diagonal(d):
    vals = np.repeat(np.arange(1, d + 1, dtype=float), 3)  # d distinct values, multiplicity 3
    n = len(vals)
    A = np.vstack([np.diag(vals), np.zeros((4, n))])
    b = np.concatenate([np.linspace(1, 2, n), np.ones(4)])
    xs = vals ** -1 * b[:n]
    f = dense_aprod(A)
    r = oracle.lsqr(A.shape[0], n, f, b, atol=0, btol=0, conlim=0, itn_limit=d, fixed_count=True)
    assert np.linalg.norm(r["x"] - xs) <= 1e-13 * np.linalg.norm(xs)
    r1 = oracle.lsqr(A.shape[0], n, f, b, atol=0, btol=0, conlim=0, itn_limit=d - 1, fixed_count=True)
    assert np.linalg.norm(r1["x"] - xs) > 1e-4 * np.linalg.norm(xs)


def test_orthonormal_columns_one_iteration():
    rng = np.random.default_rng(5)
    Q, _ = np.linalg.qr(rng.standard_normal((40, 7)))
    b = rng.standard_normal(40)
    r = oracle.lsqr(40, 7, dense_aprod(Q), b, atol=0, btol=0, conlim=0, itn_limit=1)
    assert np.linalg.norm(r["x"] - Q.T @ b) <= 1e-14 * np.linalg.norm(Q.T @ b)


def test_damped_vs_augmented_lstsq():
    S = oracle.System(W.micro(seed=11))
    A, b = S.dense(), S.rhs()
    damp = 0.3
    r = oracle.lsqr(S.m_local, S.n_cols, S, b, damp=damp, atol=1e-15, btol=1e-15, conlim=0, itn_limit=500)
    Aa = np.vstack([A, damp * np.eye(A.shape[1])])
    xs = np.linalg.lstsq(Aa, np.concatenate([b, np.zeros(A.shape[1])]), rcond=None)[0]
    assert np.linalg.norm(r["x"] - xs) <= 1e-12 * np.linalg.norm(xs)
    rr = np.linalg.norm(b - A @ xs)
    assert abs(r["r1norm"] - rr) <= 1e-10 * rr


def test_invariants_monotone_and_phibar():
    S = oracle.System(W.C1C)
    S.apply_precond()
    A, b = S.dense(), S.rhs()
    hist = []
    oracle.lsqr(S.m_local, S.n_cols, S, b, atol=0, btol=0, conlim=0, itn_limit=60, fixed_count=True,
                trace=lambda st, u, v, w_, x, var: hist.append((st, x)))
    rn = [np.linalg.norm(b - A @ x) for _, x in hist]
    xn = [np.linalg.norm(x) for _, x in hist]
    for k in range(1, len(hist)):
        assert rn[k] <= rn[k - 1] * (1 + 1e-14)
        assert xn[k] >= xn[k - 1] * (1 - 1e-9)
    for k in range(40):
        assert abs(hist[k][0]["phibar"] - rn[k]) <= 1e-12 * rn[k]


def test_bidiagonal_relation():
    S = oracle.System(W.micro(seed=12))
    S.apply_precond()
    A, b = S.dense(), S.rhs()
    us, vs, ab = [], [], []
    beta0 = np.linalg.norm(b)
    u0 = b / beta0
    v0 = A.T @ u0; a0 = np.linalg.norm(v0); v0 /= a0
    oracle.lsqr(S.m_local, S.n_cols, S, b, atol=0, btol=0, conlim=0, itn_limit=5, fixed_count=True,
                trace=lambda st, u, v, w_, x, var: (us.append(u), vs.append(v), ab.append((st["alpha"],
                                                                                          st["beta"]))))
    U = [u0] + us
    V = [v0] + vs
    alphas = [a0] + [a for a, _ in ab]
    betas = [beta0] + [bb for _, bb in ab]
    for k in range(5):  # A v_k = alpha_k u_k + beta_{k+1} u_{k+1}
        lhs = A @ V[k]
        rhs = alphas[k] * U[k] + betas[k + 1] * U[k + 1]
        assert np.linalg.norm(lhs - rhs) <= 1e-12 * np.linalg.norm(lhs)


def test_planted_consistent_recovers_x_true():
    w = W.micro(seed=13, b_mode=1, noise=0.0)
    S = oracle.System(w)
    r = oracle.lsqr(S.m_local, S.n_cols, S, S.rhs(), atol=1e-14, btol=1e-14, conlim=0, itn_limit=1000)
    xt = oracle.x_true(w)
    assert r["istop"] == 1
    assert np.linalg.norm(r["x"] - xt) <= 1e-10 * np.linalg.norm(xt)


def test_istop_special_cases():
    S = oracle.System(W.micro())
    r = oracle.lsqr(S.m_local, S.n_cols, S, np.zeros(S.m_local), itn_limit=10)
    assert r["istop"] == 0 and r["itn"] == 0 and not r["x"].any()
    r = oracle.lsqr(S.m_local, S.n_cols, S, S.rhs(), atol=0, btol=0, conlim=0, itn_limit=4)
    assert r["istop"] == 7 and r["itn"] == 4
    r = oracle.lsqr(S.m_local, S.n_cols, S, S.rhs(), atol=1e-6, btol=1e-6, itn_limit=10, fixed_count=True)
    assert r["itn"] == 10


def test_fixed_count_records_first_stop():
    S = oracle.System(W.micro())
    rs = oracle.lsqr(S.m_local, S.n_cols, S, S.rhs(), atol=1e-6, btol=1e-6, itn_limit=200)
    rf = oracle.lsqr(S.m_local, S.n_cols, S, S.rhs(), atol=1e-6, btol=1e-6, itn_limit=rs["itn"] + 20,
                     fixed_count=True)
    assert rs["istop"] in (1, 2) and rf["istop_first"] == rs["istop"] and rf["itn"] == rs["itn"] + 20

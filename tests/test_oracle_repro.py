"""Pins for the oracle's bitwise-reproducible mode (docs/REPRO.md).

  * the exact digit accumulator (EDA) equals the exact rational sum (Fractions) to within 1 ulp of the result plus
    the documented 2^-168 truncation, and is invariant under any permutation of its terms, bit for bit;
  * repro LSQR iterates are bit-identical for a system whose rows (and constraint entries) are permuted -- the
    property the GPU path is then compared against;
  * repro LSQR computes the same least-squares solution as the standard oracle LSQR.
"""
import copy
from fractions import Fraction

import numpy as np
import pytest

import oracle
import workloads as W


def exact_sum(a):
    return sum((Fraction(float(v)) for v in a), Fraction(0))


@pytest.mark.parametrize("seed", range(6))
def test_eda_exact_and_order_independent(seed):
    rng = np.random.default_rng(seed)
    n = 2000
    a = rng.standard_normal(n) * np.exp2(rng.integers(-60, 25, size=n))
    a[::7] *= -1
    if seed % 2:
        a[:10] = [1e15, -1e15, 3.0, 1e-30, -1e-30, 0.0, -0.0, 2.0**-1074, 5e-324, 1.0]  # cancellation, tiny, zeros
        a[:10] = np.clip(a[:10], -2.0**31, 2.0**31)
    s = oracle.eda_sum(a)
    ex = exact_sum(a)
    # truncation below 2^-168 per term (at most n * 2^-168) + the final rounding chain (a few ulps)
    tol = Fraction(n) * Fraction(2) ** -168 + Fraction(abs(s)) * Fraction(2) ** -50 + Fraction(2) ** -1000
    assert abs(Fraction(s) - ex) <= tol
    for _ in range(5):
        p = rng.permutation(n)
        assert oracle.eda_sum(a[p]).hex() == s.hex()
    assert oracle.eda_sum(a[::-1]).hex() == s.hex()


def test_eda_special_values():
    assert oracle.eda_sum([]) == 0.0
    assert oracle.eda_sum([1.0, -1.0]) == 0.0
    assert oracle.eda_sum([2.0**-169]) == 0.0            # below the window: truncated (documented)
    assert oracle.eda_sum([2.0**-168]) == 2.0**-168
    assert oracle.eda_sum([2.0**31, 2.0**31]) == 2.0**32
    assert oracle.eda_sum([0.1] * 10) == float(Fraction(0.1) * 10)


def test_eda_many_terms_no_overflow():
    """2^25 terms (more than the 2^23 a 64-bit digit holds): the sums the mode takes at C3 and above -- beta^2 over
    all rows, the global column, alpha^2 over the astro columns -- stay exact.  Pinned to math.fsum (the correctly
    rounded exact sum) and to closed forms; the round-1 int64 digits failed both (off by 2^16 at 2*10^7 terms)."""
    import math
    n = 1 << 25
    rng = np.random.default_rng(7)
    a = rng.uniform(0.5, 1.0, n)                  # all positive: every piece adds up in the same digits
    s = oracle.eda_sum(a)
    f = math.fsum(a)
    assert abs(s - f) <= 2 * math.ulp(f), (s, f)  # exact sum + the documented final rounding chain
    assert oracle.eda_sum(np.full(n, 0.75)) == 0.75 * n                      # exact closed form
    assert oracle.eda_sum(np.full(n, 1.0 + 2.0**-52)) == n * (1.0 + 2.0**-52)  # low digits saturated too
    b = a * a
    b[1::2] *= -1.0                               # mixed signs, squares as in ||u||^2 partial pieces
    s2, f2 = oracle.eda_sum(b), math.fsum(b)
    assert abs(s2 - f2) <= 2 * math.ulp(abs(f2)) + 1e-300, (s2, f2)


def permuted(S, rng):
    """Same system, rows in a random order, constraint entries reversed (every sum in a different order)."""
    P = copy.copy(S)
    p = rng.permutation(S.n_rows)
    P.vals = S.vals[p].copy(); P.mA = S.mA[p].copy(); P.mT = S.mT[p].copy(); P.iC = S.iC[p].copy()
    P.b = S.b[p].copy()
    cc, cv = S.c_col.copy(), S.c_val.copy()
    for k in range(S.n_constr):
        a, b = S.c_ptr[k], S.c_ptr[k + 1]
        cc[a:b] = S.c_col[a:b][::-1]; cv[a:b] = S.c_val[a:b][::-1]
    P.c_col, P.c_val = cc, cv
    P._mk_struct()
    return P, p


@pytest.mark.parametrize("w", [W.C1C, W.micro(n_glob=0, seed=5, n_ext=3)], ids=["C1c", "micro_noglob"])
def test_repro_lsqr_bitwise_under_permutation(w):
    S = oracle.System(w)
    S.apply_precond()
    P, p = permuted(S, np.random.default_rng(3))
    hs, hp = [], []
    rs = oracle.lsqr(S.m_local, S.n_cols, S, S.rhs(), atol=0, btol=0, conlim=0, itn_limit=60, fixed_count=True,
                     repro=True, trace=lambda st, u, v, w_, x, var: hs.append((st, u, v, x)))
    rp = oracle.lsqr(P.m_local, P.n_cols, P, P.rhs(), atol=0, btol=0, conlim=0, itn_limit=60, fixed_count=True,
                     repro=True, trace=lambda st, u, v, w_, x, var: hp.append((st, u, v, x)))
    n = S.n_rows
    for (a, ua, va, xa), (b, ub, vb, xb) in zip(hs, hp):
        assert np.array_equal(va, vb) and np.array_equal(xa, xb)
        assert np.array_equal(ua[:n][p], ub[:n]) and np.array_equal(ua[n:], ub[n:])
        assert a["alpha"] == b["alpha"] and a["beta"] == b["beta"] and a["acond"] == b["acond"]
    assert np.array_equal(rs["x"], rp["x"]) and np.array_equal(rs["se"], rp["se"])
    # ... while the standard mode diverges under the same permutation (SURVEY EXP-1/2)
    r1 = oracle.lsqr(S.m_local, S.n_cols, S, S.rhs(), atol=0, btol=0, conlim=0, itn_limit=60, fixed_count=True)
    r2 = oracle.lsqr(P.m_local, P.n_cols, P, P.rhs(), atol=0, btol=0, conlim=0, itn_limit=60, fixed_count=True)
    assert not np.array_equal(r1["x"], r2["x"])


def test_repro_lsqr_solves_the_same_problem():
    S = oracle.System(W.C1C)
    S.apply_precond()
    a = oracle.lsqr(S.m_local, S.n_cols, S, S.rhs(), atol=0, btol=0, conlim=0, itn_limit=100, fixed_count=True)
    b = oracle.lsqr(S.m_local, S.n_cols, S, S.rhs(), atol=0, btol=0, conlim=0, itn_limit=100, fixed_count=True,
                    repro=True)
    # converged-x tolerance of SURVEY §8(c) (the two modes round differently)
    assert np.linalg.norm(a["x"] - b["x"]) <= 1e-9 * np.linalg.norm(a["x"])
    assert abs(a["r1norm"] - b["r1norm"]) <= 1e-10 * a["r1norm"]


def test_repro_products_vs_dense():
    S = oracle.System(W.micro(n_stars=9, obs=20, n_ext=4, seed=9))
    A = S.dense()
    rng = np.random.default_rng(4)
    x = rng.standard_normal(S.n_cols)
    y = np.zeros(S.m_local); S.aprod1_repro(x, y)
    assert np.allclose(y, A @ x, rtol=1e-15, atol=1e-15)
    yy = rng.standard_normal(S.m_local)
    xx = np.zeros(S.n_cols); S.aprod2_repro(yy, xx)
    assert np.allclose(xx, A.T @ yy, rtol=1e-15, atol=1e-15)


def test_repro_colnorms_exact_and_permutation_invariant():
    """NEXT-4 preconditioner: c_j = round(EDA sum a_ij^2) equals the exact rational sum of the rounded squares to
    within 1 ulp, agrees with the ordered fp64 sum, and is bitwise invariant under row permutation."""
    S = oracle.System(W.micro(n_stars=11, obs=25, n_ext=4, seed=13))
    c = S.colnorms(repro=True)
    A = S.dense()
    for j in range(S.n_cols):
        ex = sum((Fraction(float(a * a)) for a in A[:, j]), Fraction(0))
        assert abs(Fraction(c[j]) - ex) <= Fraction(abs(c[j])) * Fraction(2) ** -52
    assert np.allclose(c, S.colnorms(), rtol=1e-14, atol=0)
    P, _ = permuted(S, np.random.default_rng(8))
    assert np.array_equal(P.colnorms(repro=True), c)

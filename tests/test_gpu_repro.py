"""NEXT-4 bitwise-reproducible mode (docs/REPRO.md): the CUDA path (csrc/lsqr_repro.cu, through the C ABI)
against the oracle's independent repro implementation (oracle/avugsr_oracle.c), BIT FOR BIT:

  preconditioner D and the scaled matrix ........... bit-identical
  every free-run iterate u, v, w, x, var, scalars .. bit-identical for every k (no divergence onset: the reductions
                                                     are order-independent on both sides)
  x, se after finalize ............................. bit-identical
  run to run, graph vs eager, row order within a star (a different reduction schedule) ... bit-identical
"""
import numpy as np
import pytest

import oracle
import workloads as W

pytestmark = pytest.mark.gpu

SCALARS = ("alpha", "beta", "rhobar", "phibar", "anorm", "acond", "ddnorm", "res2", "xnorm", "xxnorm", "z", "cs2",
           "sn2", "rnorm", "r1norm", "r2norm", "arnorm", "bnorm")


@pytest.fixture(scope="module")
def avu(cuda_device):
    import paper_conf_sc_malenzacsbvba24_b200 as m
    return m


def same(a, b):
    a = np.ascontiguousarray(a, dtype=np.float64)
    b = np.ascontiguousarray(b, dtype=np.float64)
    return a.shape == b.shape and np.array_equal(a.view(np.uint64), b.view(np.uint64))


def first_diff(a, b):
    d = np.flatnonzero(np.ascontiguousarray(a).view(np.uint64) != np.ascontiguousarray(b).view(np.uint64))
    return (int(d.size), int(d[0]), float(a[d[0]]), float(b[d[0]])) if d.size else None


def repro_solver(avu, w, damp=0.0):
    s = avu.Solver.synthetic(w)
    s.set_reproducible(True)
    s.precondition()
    return s


CASES = [W.C1C, W.micro(n_glob=0, seed=5, n_ext=3), W.micro(n_stars=40, obs=30, seed=11, n_ext=6),
         W.C1.replace(n_instr=24_000, n_obs=30_000)]


@pytest.mark.parametrize("w", CASES, ids=["C1c", "micro_noglob", "micro", "C1_bigInstr"])
def test_repro_free_run_bitwise(avu, w):
    K = 60
    s = repro_solver(avu, w)
    S = oracle.System(w)
    S.apply_precond(repro=True)
    assert same(s.get_precond(), S.D), first_diff(s.get_precond(), S.D)
    assert same(s.get_system(with_b=False)["vals"], S.vals)
    hist = []
    ro = oracle.lsqr(S.m_local, S.n_cols, S, S.rhs(), atol=0, btol=0, conlim=0, itn_limit=K, fixed_count=True,
                     repro=True, trace=lambda st, u, v, w_, x, var: hist.append((st, u, v, w_, x, var)))
    s.init(itn_limit=K, atol=0, btol=0, conlim=0, fixed_count=True, use_graph=False)
    for k in range(1, K + 1):
        s.iterate(1)
        st, vec = s.get_state()
        so, u, v, w_, x, var = hist[k - 1]
        assert st["itn"] == k
        for name, a, b in (("u", vec["u"], u), ("v", vec["v"], v), ("w", vec["w"], w_), ("x", vec["x"], x),
                           ("var", vec["var"], var)):
            assert same(a, b), (k, name, first_diff(a, b))
        for name in SCALARS:
            assert same(st[name], so[name]), (k, name, st[name], so[name])
    out = s.finalize()
    assert same(out["x"], S.D * ro["x"]) and same(out["se"], S.D * ro["se"])
    assert out["itn"] == ro["itn"] and out["istop_first"] == ro["istop_first"]
    s.close()


def test_repro_run_to_run_graph_and_row_order(avu):
    """Same system three ways -- eager, CUDA graph, and with the rows of every star in reverse order (uploaded through
    lsqr_set_system, so every atomic and block reduction meets its terms in a different order): identical bits."""
    w = W.C2.replace(n_stars=20_000, n_obs=2_000_000, seed=7)
    kw = dict(itn_limit=25, atol=0, btol=0, conlim=0, fixed_count=True)
    s = repro_solver(avu, w)
    a = s.solve(use_graph=False, **kw)
    s.generate(w.seed)
    s.precondition()
    b = s.solve(use_graph=True, **kw)
    assert same(a["x"], b["x"]) and same(a["se"], b["se"])
    s.generate(w.seed)
    g = s.get_system()
    counts = oracle.star_counts(w)
    perm = np.concatenate([np.arange(o + c - 1, o - 1, -1) for o, c in zip(np.cumsum(counts) - counts, counts)])
    s.set_system(g["vals"][perm].copy(), g["mA"][perm].copy(), g["mT"][perm].copy(), g["iC"][perm].copy(),
                 g["b"][perm].copy())
    s.precondition()
    c = s.solve(use_graph=True, **kw)
    assert same(a["x"], c["x"]) and same(a["se"], c["se"]), first_diff(a["x"], c["x"])
    assert a["r1norm"] == c["r1norm"] and a["acond"] == c["acond"]
    s.close()


def test_repro_medium_vs_oracle(avu):
    """A 2M-row system (C2's per-GPU shape at 1/5 the rows): x and se after 10 iterations bit-identical."""
    w = W.C2.replace(n_stars=20_000, n_obs=2_000_000, seed=7)
    s = repro_solver(avu, w)
    S = oracle.System(w)
    ro = oracle.solve_system(S, atol=0, btol=0, conlim=0, itn_limit=10, fixed_count=True, repro=True)
    out = s.solve(itn_limit=10, atol=0, btol=0, conlim=0, fixed_count=True)
    assert same(out["x"], ro["x"]), first_diff(out["x"], ro["x"])
    assert same(out["se"], ro["se"])
    s.close()


def test_repro_converges_like_default(avu):
    """The repro mode solves the same least-squares problem (rounding differs from the default path)."""
    w = W.C1C
    kw = dict(itn_limit=100, atol=0, btol=0, conlim=0, fixed_count=True)
    s = repro_solver(avu, w)
    a = s.solve(**kw)
    s.close()
    s = avu.Solver.synthetic(w)
    s.precondition()
    b = s.solve(**kw)
    s.close()
    assert np.linalg.norm(a["x"] - b["x"]) <= 1e-9 * np.linalg.norm(b["x"])


def _empty_star_system():
    """micro system whose stars 10, 11, 30, 49 have no observations (their columns are exactly zero)."""
    import ctypes
    w = W.micro(n_stars=50, obs=12, n_ext=6, seed=17)
    counts = oracle.star_counts(w)
    counts[[10, 11, 30, 49]] = 0
    counts[0] += w.n_obs - counts.sum()
    S = oracle.System(w, generate=False)
    S.counts, S.row_ptr = counts, oracle.row_ptr(counts)
    n = int(counts.sum())
    S.n_rows, S.row_begin, S.row_end, S.star_begin, S.star_end = n, 0, n, 0, w.n_stars
    S.vals = np.zeros((n, 24)); S.mA = np.zeros(n, dtype=np.int64); S.mT = np.zeros(n, dtype=np.int64)
    S.iC = np.zeros((n, 6), dtype=np.int64); S.b = np.zeros(n)
    L = oracle.lib()
    P = lambda a: a.ctypes.data_as(ctypes.c_void_p)
    L.orc_generate(w.seed, w.n_stars, w.n_att, w.n_instr, w.n_glob, P(S.row_ptr), 0, w.n_stars, P(S.vals), P(S.mA),
                   P(S.mT), P(S.iC))
    L.orc_generate_b(w.seed, 0, 0.0, w.n_stars, w.n_att, w.n_instr, w.n_glob, P(S.row_ptr), 0, w.n_stars, P(S.vals),
                     P(S.mA), P(S.mT), P(S.iC), P(np.zeros(1)), P(S.b))
    S._mk_struct()
    return w, counts, S


@pytest.mark.parametrize("case", ["damped", "empty_stars"])
def test_repro_edge_cases_bitwise(avu, case):
    """Damped solve (the damping rotation branch of the scalar recurrence) and stars without observations (zero
    columns, D = 1): x, sigma and the norm estimates bit-identical to the oracle's repro mode."""
    if case == "damped":
        w, counts, damp = W.micro(n_stars=30, obs=25, seed=11, n_ext=5), None, 0.37
        S = oracle.System(w)
    else:
        (w, counts, S), damp = _empty_star_system(), 0.0
    host = {k: getattr(S, k).copy() for k in ("vals", "mA", "mT", "iC", "b", "c_ptr", "c_col", "c_val")}
    ro = oracle.solve_system(S, damp=damp, atol=0, btol=0, conlim=0, itn_limit=80, fixed_count=True, repro=True)
    if counts is None:
        s = avu.Solver.synthetic(w)
    else:
        s = avu.Solver(w.n_stars, w.n_obs, w.n_att, w.n_instr, w.n_glob, obs_per_star=counts,
                       constraints=(host["c_ptr"], host["c_col"], host["c_val"]))
        s.set_system(host["vals"], host["mA"], host["mT"], host["iC"], host["b"])
    s.set_reproducible(True)
    s.precondition()
    out = s.solve(damp=damp, atol=0, btol=0, conlim=0, itn_limit=80, fixed_count=True)
    s.close()
    assert same(out["x"], ro["x"]), first_diff(out["x"], ro["x"])
    assert same(out["se"], ro["se"])
    for k in ("r1norm", "r2norm", "anorm", "acond", "arnorm", "xnorm"):
        assert same(out[k], ro[k]), k


def test_repro_many_rows_no_overflow(avu):
    """12 M rows: beta^2 and the global column each sum 12 M terms, more than the 2^23 the round-1 int64 digits held
    (they wrapped silently on both sides).  x, se after 3 iterations bit-identical to the oracle's repro mode, and
    within 1e-9 of the default mode's x (3 iterations: before any divergence onset of the two roundings)."""
    w = W.C2.replace(n_stars=120_000, n_obs=12_000_000, seed=9)
    kw = dict(itn_limit=3, atol=0, btol=0, conlim=0, fixed_count=True)
    s = repro_solver(avu, w)
    out = s.solve(**kw)
    s.close()
    S = oracle.System(w)
    ro = oracle.solve_system(S, repro=True, **kw)
    assert same(out["x"], ro["x"]), first_diff(out["x"], ro["x"])
    assert same(out["se"], ro["se"])
    assert out["bnorm"] == ro["bnorm"]
    s = avu.Solver.synthetic(w)
    s.precondition()
    d = s.solve(**kw)
    s.close()
    assert abs(d["bnorm"] - out["bnorm"]) <= 1e-13 * out["bnorm"]
    assert np.linalg.norm(d["x"] - out["x"]) <= 1e-9 * np.linalg.norm(out["x"])

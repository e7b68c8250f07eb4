"""NEXT-3: the paper's validation procedure (§V-C) on a production-shaped synthetic
system.  The paper validates a port by solving to convergence and comparing x and its standard errors with a trusted
implementation: (1) the solutions agree within 1 sigma; (2) the mean and the standard deviation of the sigma
differences are small (< 10 micro-arcseconds on the real data).  Our synthetic system has no physical
units, so (2) is applied relative to sigma.

Trusted implementation = the CPU oracle.  Also compared: the fused single pass vs the two-pass iteration.
"""
import numpy as np
import pytest

import oracle
import workloads as W

pytestmark = pytest.mark.gpu

W_VAL = W.C2.replace(name="C2val", n_stars=20_000, n_obs=2_000_000, seed=11)  # C2 shape, 2 M rows
TOL = dict(atol=1e-12, btol=1e-12, conlim=0)


@pytest.fixture(scope="module")
def reference():
    S = oracle.System(W_VAL)
    r = oracle.solve_system(S, itn_limit=3000, fixed_count=False, **TOL)
    assert r["istop"] in (1, 2, 4, 5), r["istop"]
    return r


def paper_criteria(x, se, x_ref, se_ref):
    within = np.abs(x - x_ref) <= se_ref                    # (1) solution within 1 sigma
    dsig = (se - se_ref) / se_ref                           # (2) sigma differences, relative
    return within.mean(), float(np.mean(dsig)), float(np.std(dsig))


@pytest.mark.parametrize("fused", [True, False], ids=["fused", "twopass"])
def test_validation_vs_oracle(cuda_device, reference, fused):
    import paper_conf_sc_malenzacsbvba24_b200 as avu
    s = avu.Solver.synthetic(W_VAL)
    s.precondition()
    out = s.solve(itn_limit=3000, fused=fused, **TOL)
    s.close()
    frac, mean_d, std_d = paper_criteria(out["x"], out["se"], reference["x"], reference["se"])
    print(f"\nvalidation fused={fused}: itn {out['itn']} (oracle {reference['itn']}), istop {out['istop']}; "
          f"x within 1 sigma: {100 * frac:.3f} %; sigma diff mean {mean_d:.2e} std {std_d:.2e}; "
          f"max |dx|/sigma {np.max(np.abs(out['x'] - reference['x']) / reference['se']):.2e}")
    assert out["istop"] in (1, 2, 4, 5)
    assert abs(out["itn"] - reference["itn"]) <= max(5, reference["itn"] // 20)
    assert frac == 1.0
    # the LSQR sigma is itself an estimate whose value depends on the iteration's rounding history (SURVEY EXP-4,
    # EXP-5); the paper's criterion is statistical
    assert abs(mean_d) <= 2e-2 and std_d <= 5e-2
    x_rel = np.linalg.norm(out["x"] - reference["x"]) / np.linalg.norm(reference["x"])
    assert x_rel <= 1e-8

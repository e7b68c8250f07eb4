"""Small end-to-end run used under compute-sanitizer (tests/test_sanitizer.py): generate, precondition, products,
two solves (fused and two-pass) in each shared-slice regime of the fused kernel, set_system round trip, and the
bitwise-reproducible mode (NEXT-4).  Exits non-zero on any library error."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import workloads as W  # noqa: E402
import paper_conf_sc_malenzacsbvba24_b200 as avu  # noqa: E402


def main():
    torch.cuda.set_device(0)
    w = W.C1C.replace(n_stars=300, n_obs=6000, jitter_pct=50, n_ext_stars=100)
    for fused in (True, False):
        s = avu.Solver.synthetic(w, torch_alloc=False)
        g = s.get_system()  # (before the solve consumes b)
        s.precondition()
        x = torch.ones(s.n_local_cols, dtype=torch.float64, device="cuda")
        y = torch.zeros(s.n_local_rows + s.n_constr, dtype=torch.float64, device="cuda")
        s.aprod1(x, y)
        s.aprod2(y, x)
        out = s.solve(itn_limit=12, atol=0, btol=0, conlim=0, fixed_count=True, fused=fused, use_graph=False)
        assert out["itn"] == 12 and np.isfinite(out["x"]).all()
        s.set_system(g["vals"], g["mA"], g["mT"], g["iC"], g["b"])
        out = s.solve(itn_limit=3, fused=fused, use_graph=True)
        s.close()
    # the other shared-slice regimes of the fused kernel: one z_instr copy + L2 attitude REDs (the C2-C5 regime),
    # and the instrumental slice in L1/L2 (IG) with L2 attitude REDs
    for w2 in (W.C1.replace(name="san-plain", n_stars=300, n_obs=6000, n_att=6_000, n_instr=6_000),
               W.C1.replace(name="san-ig", n_stars=300, n_obs=6000, n_att=6_000, n_instr=24_000)):
        for fused in (True, False):
            s = avu.Solver.synthetic(w2, torch_alloc=False)
            s.precondition()
            out = s.solve(itn_limit=4, atol=0, btol=0, conlim=0, fixed_count=True, fused=fused, use_graph=False)
            assert out["itn"] == 4 and np.isfinite(out["x"]).all()
            s.close()
    s = avu.Solver.synthetic(w, torch_alloc=False)
    s.set_reproducible(True)
    s.precondition()
    out = s.solve(itn_limit=6, atol=0, btol=0, conlim=0, fixed_count=True, use_graph=False)
    assert out["itn"] == 6 and np.isfinite(out["x"]).all()
    s.close()
    torch.cuda.synchronize()
    print("sanitize run ok")


if __name__ == "__main__":
    main()

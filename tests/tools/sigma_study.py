"""Diagnostic (not a test): where does the GPU's sigma differ from the oracle's on C1 after 100 free-run
iterations, compared with the spread of reordered-sum oracle controls?  Prints per-block medians (astro,
attitude, instrumental, global) for: the GPU (3 runs, fused and two-pass), permutation controls, and the GPU's
var/sigma vs the oracle at several iteration counts."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np
import oracle
import workloads as W
import paper_conf_sc_malenzacsbvba24_b200 as avu
from tests.test_gpu_parity import permuted_control, control_perms

w = W.C1
S = oracle.System(w)
S.apply_precond()
nA, nat, nin = 5 * w.n_stars, w.n_att, w.n_instr
blocks = {"astro": slice(0, nA), "att": slice(nA, nA + nat), "instr": slice(nA + nat, nA + nat + nin),
          "glob": slice(nA + nat + nin, None)}


def med(se, ref):
    d = np.abs(se / ref - 1)
    return " ".join(f"{k} {np.median(d[b]):.1e}" for k, b in blocks.items()) + f" | all {np.median(d):.2e}"


for itn in (20, 40, 60, 100):
    ro = oracle.lsqr(S.m_local, S.n_cols, S, S.rhs(), atol=0, btol=0, conlim=0, itn_limit=itn, fixed_count=True)
    seo = ro["se"]
    print(f"--- itn {itn}")
    for i, p in enumerate(control_perms(S.n_rows, 3)):
        C = permuted_control(S, p)
        rc = oracle.lsqr(C.m_local, C.n_cols, C, C.rhs(), atol=0, btol=0, conlim=0, itn_limit=itn, fixed_count=True)
        print(f"control {i}: {med(rc['se'], seo)}")
    for fused in (True, False):
        for rep in range(2):
            s = avu.Solver.synthetic(w)
            s.precondition()
            out = s.solve(itn_limit=itn, atol=0, btol=0, conlim=0, fixed_count=True, fused=fused,
                          use_graph=bool(rep))
            D = s.get_precond()
            s.close()
            print(f"gpu fused={fused} graph={bool(rep)}: {med(out['se'] / D, seo)}  r1 {out['r1norm'] / ro['r1norm'] - 1:.1e}")

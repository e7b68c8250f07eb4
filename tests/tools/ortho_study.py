"""Diagnostic (not a test): loss of orthogonality of the Lanczos vectors u_k, v_k on C1 -- GPU (fused, two-pass)
vs the oracle and a reordered-sum oracle control; max_{j<k} |v_k . v_j| and |u_k . u_j| per iteration."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np
import oracle
import workloads as W
import paper_conf_sc_malenzacsbvba24_b200 as avu
from tests.test_gpu_parity import permuted_control, identical_inputs

w = W.C1C if "c" in sys.argv[1:] else W.C1
K = 100


def ortho(vs):
    V = np.array(vs)
    G = np.abs(V @ V.T)
    np.fill_diagonal(G, 0)
    return [G[k, :k].max() if k else 0.0 for k in range(len(vs))]


def oracle_run(S):
    us, vs = [], []
    oracle.lsqr(S.m_local, S.n_cols, S, S.rhs(), atol=0, btol=0, conlim=0, itn_limit=K, fixed_count=True,
                trace=lambda st, u, v, w_, x, var: (us.append(u), vs.append(v)))
    return ortho(us), ortho(vs)


s = avu.Solver.synthetic(w)
s.precondition()
S = identical_inputs(oracle.System(w), w, s.get_system(with_b=False)["vals"], s.get_precond())
res = {"oracle": oracle_run(S), "control": oracle_run(permuted_control(S, np.arange(S.n_rows)[::-1].copy()))}
for fused in (True, False):
    s.generate(w.seed)
    s.precondition()
    s.init(itn_limit=K, atol=0, btol=0, conlim=0, fixed_count=True, fused=fused)
    us, vs = [], []
    for k in range(K):
        s.iterate(1)
        st, vec = s.get_state()
        us.append(vec["u"])
        vs.append(vec["v"])
    res["gpu fused" if fused else "gpu twopass"] = (ortho(us), ortho(vs))
print(f"{w.name}: max_j<k |u_k.u_j| / |v_k.v_j|")
for k in (1, 5, 10, 20, 30, 40, 50, 60, 70, 80, 90, 99):
    print(f"k={k + 1:3d} " + "  ".join(f"{n}: {r[0][k]:.1e}/{r[1][k]:.1e}" for n, r in res.items()))

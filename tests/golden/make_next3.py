"""Writes tests/golden/next3_<config>.npz from the ORACLE ONLY (oracle/, the serial checker): reference solutions for
NEXT-3, the paper's validation procedure (§V-C) on production-shaped systems.

  C3v  C3's shape (208 +-50 % observations per star, 300,000 attitude and 6,000 instrumental columns, a global column,
       12 constraint rows) with 100,000 stars: 20.8 M rows, 4 GB of A (~3 min on one core)
  C3   BASELINE.json configs[2] itself: 1,000,000 stars, 208 M rows, 39.9 GB of A (~25 min on one core, ~60 GB RAM;
       run on the GPU box's host, profiles/r2_next3_c3.sh)

Both solved to atol = btol = 1e-12 (conlim off) from the oracle's own generator; stored as float32 (enough for the
1-sigma and sigma-difference criteria): x and se on sample_columns() -- the astrometric columns of every k-th star
(25,000 stars) and every 3rd shared column -- plus itn, istop and the norm estimates.

Run: python -m tests.golden.make_next3 [C3v|C3]   (re-run only when the generator or the LSQR oracle changes; say why
in the commit)
"""
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

import oracle  # noqa: E402
import workloads as W  # noqa: E402

HERE = os.path.dirname(os.path.abspath(__file__))
WORKLOADS = {"C3v": W.C3.replace(name="C3v", n_stars=100_000, n_obs=20_800_000, seed=5), "C3": W.C3}
TOL = dict(atol=1e-12, btol=1e-12, conlim=0)


def path(name: str) -> str:
    return os.path.join(HERE, f"next3_{name}.npz")


def sample_columns(w) -> np.ndarray:
    stride = max(1, w.n_stars // 25_000)
    astro = (5 * np.arange(0, w.n_stars, stride)[:, None] + np.arange(5)[None, :]).ravel()
    return np.concatenate([astro, np.arange(5 * w.n_stars, w.n_cols, 3)]).astype(np.int64)


def main(name: str):
    w = WORKLOADS[name]
    t0 = time.time()
    S = oracle.System(w)
    r = oracle.solve_system(S, itn_limit=3000, fixed_count=False, **TOL)
    idx = sample_columns(w)
    np.savez_compressed(path(name), x=r["x"][idx].astype(np.float32), se=r["se"][idx].astype(np.float32),
                        itn=r["itn"], istop=r["istop"], r1norm=r["r1norm"], arnorm=r["arnorm"], anorm=r["anorm"],
                        workload=repr(w))
    print(f"wrote {path(name)}: itn {r['itn']} istop {r['istop']} r1norm {r['r1norm']:.10e} in {time.time() - t0:.0f} s")


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else "C3v")

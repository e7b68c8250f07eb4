"""Synthetic AVU-GSR workload shapes (input description only -- no arithmetic of the method lives here).

Shared by the oracle side (oracle/, tests/) and the product side (bench.py, the Python binding) as the one
"module of their own" for seeded inputs: it only names sizes, seeds and generator parameters. Both sides then
run their OWN implementation of the counter-based generator spec (docs/GENERATOR.md).

Configs follow BASELINE.json ``configs`` and SURVEY.md §8(d):
  C1 tiny   1,000 stars x 20 obs, 1,200 att, 60 instr, 1 glob (CPU oracle in seconds)
  C2 small  ~1 GB of A (5 M rows), preconditioned, 12 constraint rows
  C3 medium ~40 GB of A on 1 B200 (paper-like size; bandwidth-bound steady state)
  C4 large  ~150 GB of A, strong-scaled over 1/2/4/8 GPUs
  C5 weak   ~120 GB of A per GPU (weak scaling), full solve with standard errors
The paper's synthetic generator takes "a size in GB and a seed" (Artifact appendix).
"""
from __future__ import annotations

import dataclasses

PARITY_SEED = 1           # seed 1 for parity
TIMING_SEED = 20241117    # seed 20241117 for timing


@dataclasses.dataclass(frozen=True)
class Workload:
    name: str
    n_stars: int
    n_obs: int
    n_att: int
    n_instr: int
    n_glob: int = 1
    jitter_pct: int = 0          # observation-count jitter, +-pct of the mean (pairwise, total preserved)
    n_ext_stars: int = 0         # >0 enables the 12 synthetic constraint rows (6 frame rows over n_ext stars)
    seed: int = PARITY_SEED
    b_mode: int = 0              # 0 hashed b, 1 planted b = A x_true + noise
    noise: float = 0.0
    itn: int = 100               # fixed-count iterations
    precondition: bool = True

    @property
    def n_cols(self) -> int:
        return 5 * self.n_stars + self.n_att + self.n_instr + self.n_glob

    @property
    def n_constr(self) -> int:
        return 12 if self.n_ext_stars > 0 else 0

    @property
    def a_bytes(self) -> int:
        """Bytes of A's values (24 FP64 slots per row), the paper's 'size of A'."""
        return self.n_obs * 24 * 8

    def replace(self, **kw) -> "Workload":
        return dataclasses.replace(self, **kw)

    def per_gpu(self, nranks: int) -> "Workload":
        """Weak-scaling shape: stars and rows multiplied by nranks (per-GPU work fixed)."""
        return dataclasses.replace(self, name=f"{self.name}x{nranks}", n_stars=self.n_stars * nranks,
                                   n_obs=self.n_obs * nranks)


C1 = Workload("C1", n_stars=1_000, n_obs=20_000, n_att=1_200, n_instr=60, n_glob=1)
C1C = C1.replace(name="C1c", n_ext_stars=1_000)                     # C1 + 12 constraint rows (test variant)
C2 = Workload("C2", n_stars=50_000, n_obs=5_000_000, n_att=30_000, n_instr=6_000, jitter_pct=50,
              n_ext_stars=1_000)
C3 = Workload("C3", n_stars=1_000_000, n_obs=208_000_000, n_att=300_000, n_instr=6_000, jitter_pct=50,
              n_ext_stars=1_000, seed=TIMING_SEED)
C4 = Workload("C4", n_stars=4_000_000, n_obs=780_000_000, n_att=3_000_000, n_instr=6_000, jitter_pct=50,
              n_ext_stars=1_000, seed=TIMING_SEED)
C5 = Workload("C5", n_stars=3_125_000, n_obs=625_000_000, n_att=3_000_000, n_instr=6_000, jitter_pct=50,
              n_ext_stars=1_000, seed=TIMING_SEED)

# C4's shape (n_att = 3,000,000: the 24 MB shared slice AR2 carries) at 1/100 of its stars and rows: the strong-scaling
# flow of bench.py at test size (--scaling strong --config C4s)
C4S = C4.replace(name="C4s", n_stars=40_000, n_obs=7_800_000)

CONFIGS = {w.name: w for w in (C1, C1C, C2, C3, C4, C4S, C5)}


def micro(n_stars=7, obs=30, n_att=24, n_instr=12, n_glob=1, jitter=50, n_ext=0, seed=3, **kw) -> Workload:
    """Tiny systems for dense / brute-force pins."""
    return Workload(f"micro{n_stars}x{obs}", n_stars=n_stars, n_obs=n_stars * obs, n_att=n_att, n_instr=n_instr,
                    n_glob=n_glob, jitter_pct=jitter, n_ext_stars=n_ext, seed=seed, **kw)

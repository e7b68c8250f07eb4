/*
 * avugsr_oracle.c -- CPU ORACLE for the Gaia AVU-GSR LSQR hot path.
 *
 *   *** TEST INFRASTRUCTURE ONLY. ***
 *   Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline leg, --impl reference) may load this
 *   library. The product (paper_conf_sc_malenzacsbvba24_b200/, liblsqr_avugsr.so) never links, imports or
 *   calls it, and this file shares no code, header, table or constant generator with the CUDA path.
 *
 * Plain, serial, slow and obviously correct: every loop follows the paper's definition (or Paige & Saunders'
 * published algorithm, refs [20],[21] of the paper) in the order written there. Built with
 *   gcc -O2 -ffp-contract=off -fPIC -shared   (no FMA contraction: every product and sum is rounded on its own).
 * All floating point is IEEE binary64, round to nearest.
 *
 * Citations: "P:Lx-y (§s)" = /root/reference/PAPER.md lines x-y, paper section s.
 *            "S:§8(c) O-xxx" = SURVEY.md §8(c) reading of the paper where it is silent/garbled.
 *
 * Parity pins (tests/test_oracle_*.py) -- what each function is checked against, other than itself:
 *   orc_hash/orc_pm1 ............ splitmix64 published test vectors; exactness/range properties
 *   orc_star_counts/orc_shard ... brute force invariants (sum, bounds, pair symmetry; cover/disjoint/lower_bound)
 *   orc_generate* ............... structural invariants + golden FNV-1a checksums (tests/golden/, written by
 *                                 tests/golden/make_golden.py which calls only this oracle) + an independent
 *                                 pure-Python splitmix64/H and sampled fields regenerated from it
 *   orc_aprod1/orc_aprod2 ........ dense materialisation A@x, A.T@y (numpy); adjoint identity
 *   orc_colnorms/orc_scale ....... unit column norms of the scaled matrix; scaled solve == unscaled lstsq
 *   orc_lsqr ..................... numpy.linalg.lstsq/QR; scipy.sparse.linalg.lsqr iterates; reorthogonalised mode
 *                                 gives exact diag((A^T A)^-1); finite termination on diagonal A; planted x;
 *                                 monotone ||r_k||; istop special cases
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define ORC_SLOTS 24 /* 5 astro + 12 att + 6 instr + 1 glob per row, P:L357-363 (§II-B) */

/* ORC_PAR_FOR / ORC_PAR_SUM(v) mark the O(m) / O(n) vector loops of orc_lsqr.  They are EMPTY in this build (the
 * checker: plain serial C).  oracle/omp_timing.c -- a separately compiled -fopenmp variant used only to time the
 * oracle on all host cores for bench.py's cpu_baseline, never as a parity reference -- defines them as OpenMP
 * pragmas before including this file. */
#ifndef ORC_PAR_FOR
#define ORC_PAR_FOR
#define ORC_PAR_SUM(v)
#endif

/* ------------------------------------------------------------------------------------------------------------
 * O-GEN: synthetic system generator (integer hash -> exact FP64).  The paper generates a synthetic system from a
 * size and a seed "distributed in the system as the real data" (Artifact appendix); the structure
 * it must reproduce is P:L350-388 (§II-B).  The exact hash/field spec is SURVEY §8(c) O-GEN (docs/GENERATOR.md).
 * ---------------------------------------------------------------------------------------------------------- */

/* splitmix64 finaliser (Steele, Lea, Flood 2014).  S:§8(c) O-GEN "mix". */
uint64_t orc_mix(uint64_t z) {
  z += 0x9E3779B97F4A7C15ULL;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}

/* H(seed,tag,i,j) = mix(mix(mix(seed ^ (tag<<56)) ^ i) ^ j).  S:§8(c) O-GEN. */
uint64_t orc_hash(uint64_t seed, uint64_t tag, uint64_t i, uint64_t j) {
  return orc_mix(orc_mix(orc_mix(seed ^ (tag << 56)) ^ i) ^ j);
}

/* pm1(h) = ((int64)(h>>10) - 2^53) * 2^-53, exact, in [-1, 1).  S:§8(c) O-GEN. */
double orc_pm1(uint64_t h) {
  int64_t k = (int64_t)(h >> 10) - ((int64_t)1 << 53);
  return (double)k * 0x1p-53;
}

/* Observations per star.  Rows are grouped by star (block-diagonal astrometric part).
 * Uniform: q = floor(n_obs/n_stars), star s gets q + [s < n_obs mod n_stars].  Jittered: pairs (2p, 2p+1) get
 * +d / -d with d = (H(seed,1,p,0) mod (2J+1)) - J, J = floor(q*pct/100) clamped to q-1.  S:§8(c) O-GEN. */
void orc_star_counts(uint64_t seed, int64_t n_stars, int64_t n_obs, int32_t jitter_pct, int64_t* counts) {
  int64_t q = n_obs / n_stars, rem = n_obs % n_stars;
  for (int64_t s = 0; s < n_stars; ++s) counts[s] = q + (s < rem ? 1 : 0);
  int64_t J = (q * (int64_t)jitter_pct) / 100;
  if (q == 0) J = 0;
  else if (q - J < 1) J = q - 1;
  if (J <= 0) return;
  for (int64_t p = 0; 2 * p + 1 < n_stars; ++p) {
    int64_t d = (int64_t)(orc_hash(seed, 1, (uint64_t)p, 0) % (uint64_t)(2 * J + 1)) - J;
    counts[2 * p] += d;
    counts[2 * p + 1] -= d;
  }
}

/* row_ptr = exclusive prefix sum of counts (n_stars+1 entries). */
void orc_row_ptr(const int64_t* counts, int64_t n_stars, int64_t* row_ptr) {
  row_ptr[0] = 0;
  for (int64_t s = 0; s < n_stars; ++s) row_ptr[s + 1] = row_ptr[s] + counts[s];
}

/* O-SHARD: each MPI rank owns a subset of the observations (§IV).  Contiguous star ranges balanced by
 * rows: target_r = floor(r*n_obs/P); star_begin[r] = lower_bound(row_ptr, target_r).  S:§8(c) O-SHARD. */
void orc_shard(const int64_t* row_ptr, int64_t n_stars, int64_t n_obs, int32_t P, int64_t* star_begin) {
  star_begin[0] = 0;
  for (int32_t r = 1; r < P; ++r) {
    int64_t target = ((int64_t)r * n_obs) / P;
    int64_t s = 0; /* lower_bound, written as a plain linear scan */
    while (s <= n_stars && row_ptr[s] < target) ++s;
    star_begin[r] = s;
  }
  star_begin[P] = n_stars;
}

/* Rows of stars [star_begin, star_end).  Storage follows the paper's arrays (§II-B):
 *   vals[i][24]          nonzeros, slot order astro 0-4, att 5-16 (axis a, knot j at 5+4a+j), instr 17-22, glob 23
 *   matrixIndexAstro[i]  starting column of the 5 contiguous astro nonzeros = 5*star(i)
 *   matrixIndexAtt[i]    column of the first attitude nonzero = A0 + k0_i; 3 blocks of 4, stride n_axis
 *   instrCol[i][6]       all 6 instrumental columns (irregular pattern)
 * Global part: one column G0 per row when n_glob = 1; slot 23 is a zero pad when n_glob = 0. */
void orc_generate(uint64_t seed, int64_t n_stars, int64_t n_att, int64_t n_instr, int32_t n_glob,
                  const int64_t* row_ptr, int64_t star_begin, int64_t star_end,
                  double* vals, int64_t* matrixIndexAstro, int64_t* matrixIndexAtt, int64_t* instrCol) {
  int64_t n_axis = n_att / 3, g = n_instr / 6;
  int64_t A0 = 5 * n_stars, I0 = A0 + n_att;
  int64_t row0 = row_ptr[star_begin];
  for (int64_t s = star_begin; s < star_end; ++s) {
    for (int64_t i = row_ptr[s]; i < row_ptr[s + 1]; ++i) {
      int64_t li = i - row0;
      matrixIndexAstro[li] = 5 * s;
      int64_t k0 = (int64_t)(orc_hash(seed, 2, (uint64_t)i, 0) % (uint64_t)(n_axis - 3));
      matrixIndexAtt[li] = A0 + k0;
      for (int j = 0; j < 6; ++j)
        instrCol[li * 6 + j] = I0 + j * g + (int64_t)(orc_hash(seed, 3, (uint64_t)i, (uint64_t)j) % (uint64_t)g);
      for (int sl = 0; sl < ORC_SLOTS; ++sl)
        vals[li * ORC_SLOTS + sl] = orc_pm1(orc_hash(seed, 4, (uint64_t)i, (uint64_t)sl));
      if (n_glob == 0) vals[li * ORC_SLOTS + 23] = 0.0;
    }
  }
}

/* x_true[j] = pm1(H(seed,7,j,0)) over global columns.  S:§8(c) O-GEN (planted mode). */
void orc_x_true(uint64_t seed, int64_t n_cols, double* x_true) {
  for (int64_t j = 0; j < n_cols; ++j) x_true[j] = orc_pm1(orc_hash(seed, 7, (uint64_t)j, 0));
}

/* Column of slot sl of local row li (global column numbering).  P:L369-388 (§II-B), S:§8(c) O-AP1. */
static int64_t orc_col(int sl, int64_t li, const int64_t* mA, const int64_t* mT, const int64_t* iC,
                       int64_t n_axis, int64_t G0) {
  if (sl < 5) return mA[li] + sl;
  if (sl < 17) return mT[li] + ((sl - 5) / 4) * n_axis + ((sl - 5) % 4);
  if (sl < 23) return iC[li * 6 + (sl - 17)];
  return G0;
}

/* Known terms b.  mode 0 (hashed): b_i = pm1(H(seed,5,i,0)).  mode 1 (planted):
 * b_i = sum_s val_is * x_true[col_is] in slot order (each product and sum rounded separately),
 * plus noise * pm1(H(seed,6,i,0)).  S:§8(c) O-GEN. */
void orc_generate_b(uint64_t seed, int32_t mode, double noise, int64_t n_stars, int64_t n_att, int64_t n_instr,
                    int32_t n_glob, const int64_t* row_ptr, int64_t star_begin, int64_t star_end,
                    const double* vals, const int64_t* mA, const int64_t* mT, const int64_t* iC,
                    const double* x_true, double* b) {
  int64_t n_axis = n_att / 3, G0 = 5 * n_stars + n_att + n_instr;
  int64_t row0 = row_ptr[star_begin], row1 = row_ptr[star_end];
  for (int64_t i = row0; i < row1; ++i) {
    int64_t li = i - row0;
    if (mode == 0) { b[li] = orc_pm1(orc_hash(seed, 5, (uint64_t)i, 0)); continue; }
    double acc = 0.0;
    for (int sl = 0; sl < ORC_SLOTS; ++sl) {
      if (sl == 23 && n_glob == 0) continue;
      double p = vals[li * ORC_SLOTS + sl] * x_true[orc_col(sl, li, mA, mT, iC, n_axis, G0)];
      acc = acc + p;
    }
    double e = noise * orc_pm1(orc_hash(seed, 6, (uint64_t)i, 0));
    b[li] = acc + e;
  }
}

/* Constraint equations (§II-B, §IV-a): the paper does not give their content; S:§8(c)
 * O-GEN reading: 6 "frame" rows k<6 with entries (5s+a, pm1(H(seed,8,k,5s+a))) for s < min(n_ext, n_stars),
 * a < 5, and 6 "instrumental" rows j<6 with entries (I0 + j*g + t, 1.0), t < g.  rhs = 0.
 * CSR over global columns; returns nnz.  Pass NULL arrays to query the size. */
int64_t orc_constraints(uint64_t seed, int64_t n_stars, int64_t n_att, int64_t n_instr, int64_t n_ext,
                        int64_t* c_ptr, int64_t* c_col, double* c_val) {
  int64_t ns = n_ext < n_stars ? n_ext : n_stars;
  int64_t g = n_instr / 6, I0 = 5 * n_stars + n_att;
  int64_t e = 0;
  if (c_ptr) c_ptr[0] = 0;
  for (int k = 0; k < 6; ++k) {
    for (int64_t s = 0; s < ns; ++s)
      for (int a = 0; a < 5; ++a) {
        if (c_col) {
          c_col[e] = 5 * s + a;
          c_val[e] = orc_pm1(orc_hash(seed, 8, (uint64_t)k, (uint64_t)(5 * s + a)));
        }
        ++e;
      }
    if (c_ptr) c_ptr[k + 1] = e;
  }
  for (int j = 0; j < 6; ++j) {
    for (int64_t t = 0; t < g; ++t) {
      if (c_col) { c_col[e] = I0 + j * g + t; c_val[e] = 1.0; }
      ++e;
    }
    if (c_ptr) c_ptr[6 + j + 1] = e;
  }
  return e;
}

/* ------------------------------------------------------------------------------------------------------------
 * The products.  aprod1: y <- y + A x (Eq. (3), garbled "big = A x 71"); aprod2: x <- x + A^T y
 * (Eq. (4), garbled "P+ =AT x b").  These are Paige & Saunders' mode 1 and mode 2 (refs [20],[21]).
 * ---------------------------------------------------------------------------------------------------------- */
typedef struct {
  int64_t n_rows;   /* local observation rows */
  int64_t n_cols;   /* global number of columns n = 5 n_stars + n_att + n_instr + n_glob */
  int64_t n_axis;   /* attitude stride n_att/3 (S:§8(c) Z8) */
  int64_t A0;       /* first attitude column = 5 n_stars */
  int64_t G0;       /* global column */
  int32_t n_glob;   /* 0 or 1 */
  double* vals;     /* [n_rows][24] */
  const int64_t* mA;
  const int64_t* mT;
  const int64_t* iC;
  int64_t n_constr; /* constraint rows, appended after the observation rows (S:§8(c) Z3) */
  const int64_t* c_ptr;
  const int64_t* c_col;
  double* c_val;
  /* constraint-entry ownership (S:§8(c) O-SHARD): an entry on column c counts on this rank iff
   * own_lo <= c < own_hi (this rank's astro columns) or (c >= A0 and own_shared). Single rank: all owned. */
  int64_t own_lo, own_hi;
  int32_t own_shared;
} orc_sys;

static int orc_owned(const orc_sys* S, int64_t c) {
  return (c >= S->own_lo && c < S->own_hi) || (c >= S->A0 && S->own_shared);
}

/* O-AP1: y_i += (sum_{s<24} val_is x[col_is]) accumulated from 0 in slot order, then added once; constraint rows
 * y_{n_rows+k} += sum over owned entries in entry order.  y has n_rows + n_constr entries. */
void orc_aprod1(const orc_sys* S, const double* x, double* y) {
  for (int64_t i = 0; i < S->n_rows; ++i) {
    double sum = 0.0;
    for (int sl = 0; sl < ORC_SLOTS; ++sl) {
      if (sl == 23 && S->n_glob == 0) continue;
      sum = sum + S->vals[i * ORC_SLOTS + sl] * x[orc_col(sl, i, S->mA, S->mT, S->iC, S->n_axis, S->G0)];
    }
    y[i] = y[i] + sum;
  }
  for (int64_t k = 0; k < S->n_constr; ++k) {
    double sum = 0.0;
    for (int64_t e = S->c_ptr[k]; e < S->c_ptr[k + 1]; ++e)
      if (orc_owned(S, S->c_col[e])) sum = sum + S->c_val[e] * x[S->c_col[e]];
    y[S->n_rows + k] = y[S->n_rows + k] + sum;
  }
}

/* O-AP2: for i ascending, for s ascending: x[col_is] += val_is * y_i; then the owned constraint entries. */
void orc_aprod2(const orc_sys* S, const double* y, double* x) {
  for (int64_t i = 0; i < S->n_rows; ++i) {
    for (int sl = 0; sl < ORC_SLOTS; ++sl) {
      if (sl == 23 && S->n_glob == 0) continue;
      int64_t c = orc_col(sl, i, S->mA, S->mT, S->iC, S->n_axis, S->G0);
      x[c] = x[c] + S->vals[i * ORC_SLOTS + sl] * y[i];
    }
  }
  for (int64_t k = 0; k < S->n_constr; ++k)
    for (int64_t e = S->c_ptr[k]; e < S->c_ptr[k + 1]; ++e)
      if (orc_owned(S, S->c_col[e])) x[S->c_col[e]] = x[S->c_col[e]] + S->c_val[e] * y[S->n_rows + k];
}


/* ------------------------------------------------------------------------------------------------------------
 * NEXT-4 bitwise-reproducible mode: exact digit accumulator (EDA), docs/REPRO.md.  Every reduction
 * becomes an order-independent integer sum of exactly split FP64 terms, rounded once; both the oracle and the GPU
 * implement the spec, so their iterates agree bit for bit.
 * ---------------------------------------------------------------------------------------------------------- */
#define ORC_EDA_L 5
/* Digits are accumulated in 128-bit integers: a piece is < 2^40 in magnitude, so no realistic number of additions
 * (< 2^87) can overflow -- the sum held in D is always the exact integer sum of the pieces.  (64-bit digits, as in
 * round 1, wrap after ~2^23 positive terms: beta^2 over 10^8 rows came out off by multiples of 2^64 * 2^B_d.) */
typedef struct { __int128 d[ORC_EDA_L]; } orc_eda;
static const int orc_eda_B[ORC_EDA_L] = {-8, -48, -88, -128, -168}; /* digit d covers bits [B_d, B_d + 40) */

void orc_eda_add(orc_eda* A, double c) {
  uint64_t bits;
  memcpy(&bits, &c, sizeof bits);
  const int neg = (int)(bits >> 63);
  const int ex = (int)((bits >> 52) & 0x7ff);
  uint64_t M = bits & ((1ULL << 52) - 1);
  int E;
  if (ex == 0) {
    E = -1074;
  } else {
    M |= 1ULL << 52;
    E = ex - 1075;
  }
  if (M == 0) return;
  for (int d = 0; d < ORC_EDA_L; ++d) {
    const int sh = E - orc_eda_B[d];
    uint64_t dig;
    if (sh >= 40) dig = 0;
    else if (sh >= 0) dig = (M << sh) & ((1ULL << 40) - 1);
    else if (sh > -53) dig = (M >> (-sh)) & ((1ULL << 40) - 1);
    else dig = 0;
    A->d[d] += neg ? -(__int128)dig : (__int128)dig;
  }
}

/* round(D) (docs/REPRO.md): carry-normalise so that D_d is in [0, 2^40) for d >= 1 (the unique such representation
 * of the exact value), then v = 0; v = v + D_d * 2^B_d for d = 0..4, every conversion and addition rounded. */
double orc_eda_round(const orc_eda* A) {
  __int128 D[ORC_EDA_L];
  for (int d = 0; d < ORC_EDA_L; ++d) D[d] = A->d[d];
  for (int d = ORC_EDA_L - 1; d >= 1; --d) {
    const __int128 c = D[d] >> 40; /* arithmetic shift = floor division (gcc) */
    D[d] -= c * ((__int128)1 << 40);
    D[d - 1] += c;
  }
  double v = 0.0;
  for (int d = 0; d < ORC_EDA_L; ++d) v = v + ldexp((double)D[d], orc_eda_B[d]);
  return v;
}

/* sum of n doubles through the EDA (test hook) */
double orc_eda_sum(const double* a, int64_t n) {
  orc_eda A;
  memset(&A, 0, sizeof A);
  for (int64_t i = 0; i < n; ++i) orc_eda_add(&A, a[i]);
  return orc_eda_round(&A);
}

/* repro aprod1: y_i <- y_i + round(EDA sum of a_is * x[col_is]) (rows), same for the owned constraint entries */
void orc_aprod1_repro(const orc_sys* S, const double* x, double* y) {
  for (int64_t i = 0; i < S->n_rows; ++i) {
    orc_eda A;
    memset(&A, 0, sizeof A);
    for (int sl = 0; sl < ORC_SLOTS; ++sl) {
      if (sl == 23 && S->n_glob == 0) continue;
      orc_eda_add(&A, S->vals[i * ORC_SLOTS + sl] * x[orc_col(sl, i, S->mA, S->mT, S->iC, S->n_axis, S->G0)]);
    }
    y[i] = y[i] + orc_eda_round(&A);
  }
  for (int64_t k = 0; k < S->n_constr; ++k) {
    orc_eda A;
    memset(&A, 0, sizeof A);
    for (int64_t e = S->c_ptr[k]; e < S->c_ptr[k + 1]; ++e)
      if (orc_owned(S, S->c_col[e])) orc_eda_add(&A, S->c_val[e] * x[S->c_col[e]]);
    y[S->n_rows + k] = y[S->n_rows + k] + orc_eda_round(&A);
  }
}

/* repro aprod2: x_j <- x_j + round(EDA sum over rows and owned constraint entries of a_ij * y_i), every column */
void orc_aprod2_repro(const orc_sys* S, const double* y, double* x) {
  orc_eda* Z = (orc_eda*)calloc((size_t)S->n_cols, sizeof(orc_eda));
  if (!Z) abort();
  for (int64_t i = 0; i < S->n_rows; ++i)
    for (int sl = 0; sl < ORC_SLOTS; ++sl) {
      if (sl == 23 && S->n_glob == 0) continue;
      orc_eda_add(&Z[orc_col(sl, i, S->mA, S->mT, S->iC, S->n_axis, S->G0)], S->vals[i * ORC_SLOTS + sl] * y[i]);
    }
  for (int64_t k = 0; k < S->n_constr; ++k)
    for (int64_t e = S->c_ptr[k]; e < S->c_ptr[k + 1]; ++e)
      if (orc_owned(S, S->c_col[e])) orc_eda_add(&Z[S->c_col[e]], S->c_val[e] * y[S->n_rows + k]);
  for (int64_t j = 0; j < S->n_cols; ++j) x[j] = x[j] + orc_eda_round(&Z[j]);
  free(Z);
}

/* ------------------------------------------------------------------------------------------------------------
 * O-PREC: the LSQR is "preconditioned" (§II-B); the paper gives no detail.  S:§8(c) Z2 reading:
 * Jacobi column scaling.  c_j = sum over all rows (constraints included) of a_ij^2; D_j = 1/sqrt(c_j) (1 if c_j = 0);
 * scale in place A^ = A D.
 * ---------------------------------------------------------------------------------------------------------- */
void orc_colnorms(const orc_sys* S, double* c) {
  for (int64_t i = 0; i < S->n_rows; ++i)
    for (int sl = 0; sl < ORC_SLOTS; ++sl) {
      if (sl == 23 && S->n_glob == 0) continue;
      double a = S->vals[i * ORC_SLOTS + sl];
      int64_t j = orc_col(sl, i, S->mA, S->mT, S->iC, S->n_axis, S->G0);
      c[j] = c[j] + a * a;
    }
  for (int64_t k = 0; k < S->n_constr; ++k)
    for (int64_t e = S->c_ptr[k]; e < S->c_ptr[k + 1]; ++e)
      if (orc_owned(S, S->c_col[e])) c[S->c_col[e]] = c[S->c_col[e]] + S->c_val[e] * S->c_val[e];
}

/* NEXT-4 (docs/REPRO.md): the same column sums of squares, each an order-independent EDA sum of the rounded
 * squares a*a, rounded once; every c[j] is overwritten (no accumulation into a caller value). */
void orc_colnorms_repro(const orc_sys* S, double* c) {
  orc_eda* Z = (orc_eda*)calloc((size_t)(S->n_cols > 0 ? S->n_cols : 1), sizeof(orc_eda));
  if (!Z) abort();
  for (int64_t i = 0; i < S->n_rows; ++i)
    for (int sl = 0; sl < ORC_SLOTS; ++sl) {
      if (sl == 23 && S->n_glob == 0) continue;
      double a = S->vals[i * ORC_SLOTS + sl];
      orc_eda_add(&Z[orc_col(sl, i, S->mA, S->mT, S->iC, S->n_axis, S->G0)], a * a);
    }
  for (int64_t k = 0; k < S->n_constr; ++k)
    for (int64_t e = S->c_ptr[k]; e < S->c_ptr[k + 1]; ++e)
      if (orc_owned(S, S->c_col[e])) orc_eda_add(&Z[S->c_col[e]], S->c_val[e] * S->c_val[e]);
  for (int64_t j = 0; j < S->n_cols; ++j) c[j] = orc_eda_round(&Z[j]);
  free(Z);
}

void orc_precond_D(const double* c, int64_t n, double* D) {
  for (int64_t j = 0; j < n; ++j) D[j] = c[j] > 0.0 ? 1.0 / sqrt(c[j]) : 1.0;
}

/* Scales every stored value (observation rows and ALL constraint entries) by D of its column. */
void orc_scale(orc_sys* S, const double* D) {
  for (int64_t i = 0; i < S->n_rows; ++i)
    for (int sl = 0; sl < ORC_SLOTS; ++sl) {
      if (sl == 23 && S->n_glob == 0) continue;
      S->vals[i * ORC_SLOTS + sl] =
          S->vals[i * ORC_SLOTS + sl] * D[orc_col(sl, i, S->mA, S->mT, S->iC, S->n_axis, S->G0)];
    }
  for (int64_t k = 0; k < S->n_constr; ++k)
    for (int64_t e = S->c_ptr[k]; e < S->c_ptr[k + 1]; ++e) S->c_val[e] = S->c_val[e] * D[S->c_col[e]];
}

/* ------------------------------------------------------------------------------------------------------------
 * O-LSQR: "customized and preconditioned version of the LSQR algorithm [20],[21]" (§I
 * §II-B); stops "when it reaches convergence or the maximum number of iterations".  Written against
 * an abstract aprod(mode, ...) callback exactly as Paige & Saunders' Algorithm 583 (LSQR, ACM TOMS 8(2), 1982);
 * step labels O-1 ... O-5 follow SURVEY §8(c).  Rotation in the lsqr.f form (rho = sqrt(rhobar1^2 + beta^2)).
 * ---------------------------------------------------------------------------------------------------------- */

/* mode 1: out[m] += A in[n];  mode 2: out[n] += A^T in[m] */
typedef void (*orc_aprod_fn)(int32_t mode, const double* in, double* out, void* ctx);

typedef struct {
  int32_t istop, itn, istop_first, pad_;
  double r1norm, r2norm, anorm, acond, arnorm, xnorm, bnorm;
} orc_lsqr_out;

/* full scalar state after an iteration (exposed to the trace callback for teacher-forced/free-run parity) */
typedef struct {
  int32_t itn, istop;
  double alpha, beta, rhobar, phibar, anorm, acond, ddnorm, res2, xnorm, xxnorm, z, cs2, sn2, rnorm, r1norm,
      r2norm, arnorm, bnorm;
  double rho, theta, phi, tau, psi, test1, test2, test3;
} orc_lsqr_state;

typedef void (*orc_trace_fn)(const orc_lsqr_state* st, const double* u, const double* v, const double* w,
                             const double* x, const double* var, void* ctx);

void orc_sys_aprod(int32_t mode, const double* in, double* out, void* ctx) {
  if (mode == 1) orc_aprod1((const orc_sys*)ctx, in, out);
  else orc_aprod2((const orc_sys*)ctx, in, out);
}

void orc_sys_aprod_repro(int32_t mode, const double* in, double* out, void* ctx) {
  if (mode == 1) orc_aprod1_repro((const orc_sys*)ctx, in, out);
  else orc_aprod2_repro((const orc_sys*)ctx, in, out);
}

static int orc_repro_mode = 0; /* set by orc_lsqr for the duration of a solve */

static double orc_nrm2(const double* a, int64_t n) { /* plain sqrt(sum a^2) in order, S:§8(c) Z5 */
  if (orc_repro_mode) { /* NEXT-4: order-independent exact sum of the rounded squares */
    orc_eda A;
    memset(&A, 0, sizeof A);
    for (int64_t i = 0; i < n; ++i) orc_eda_add(&A, a[i] * a[i]);
    return sqrt(orc_eda_round(&A));
  }
  double s = 0.0;
  ORC_PAR_SUM(s)
  for (int64_t i = 0; i < n; ++i) s = s + a[i] * a[i];
  return sqrt(s);
}
static void orc_scal(double* a, int64_t n, double f) {
  ORC_PAR_FOR
  for (int64_t i = 0; i < n; ++i) a[i] = f * a[i];
}
static double orc_dot(const double* a, const double* b, int64_t n) {
  double s = 0.0;
  for (int64_t i = 0; i < n; ++i) s = s + a[i] * b[i];
  return s;
}
/* Test-only full reorthogonalisation (classical Gram-Schmidt, applied twice) against the stored basis Q[0..k). */
static void orc_reorth(double* a, const double* Q, int64_t k, int64_t n) {
  for (int pass = 0; pass < 2; ++pass)
    for (int64_t j = 0; j < k; ++j) {
      double d = orc_dot(a, Q + j * n, n);
      for (int64_t i = 0; i < n; ++i) a[i] = a[i] - d * Q[j * n + i];
    }
}

/*
 * Solves min ||A x - b||^2 + damp^2 ||x||^2.  m rows, n columns.  x[n], var[n], se[n] out (se may be NULL).
 * fixed_count != 0: the stopping tests are evaluated and the first nonzero istop is reported in istop_first, but
 * iterations continue to itn_limit (the paper's timing mode: 100 iterations).
 * reorth != 0: TEST-ONLY full reorthogonalisation of u and v (needs (itn_limit+1)*(m+n) doubles).
 * Returns 0, or -1 on allocation failure.
 */
int orc_lsqr(int64_t m, int64_t n, orc_aprod_fn aprod, void* ctx, const double* b, double damp, double atol,
             double btol, double conlim, int64_t itn_limit, int32_t fixed_count, int32_t reorth, int32_t repro,
             double* x, double* var, double* se, orc_lsqr_out* out, orc_trace_fn trace, void* trace_ctx) {
#ifdef _OPENMP
  if (repro) return -2; /* omp_timing.c build: the repro accumulators are not thread-safe there */
#endif
  orc_repro_mode = repro ? 1 : 0;
  const double eps = 0x1p-52;
  double* u = (double*)malloc(sizeof(double) * (size_t)(m > 0 ? m : 1));
  double* v = (double*)malloc(sizeof(double) * (size_t)(n > 0 ? n : 1));
  double* w = (double*)malloc(sizeof(double) * (size_t)(n > 0 ? n : 1));
  double *U = NULL, *V = NULL;
  if (!u || !v || !w) { free(u); free(v); free(w); return -1; }
  if (reorth) {
    U = (double*)malloc(sizeof(double) * (size_t)(itn_limit + 2) * (size_t)m);
    V = (double*)malloc(sizeof(double) * (size_t)(itn_limit + 2) * (size_t)n);
    if (!U || !V) { free(u); free(v); free(w); free(U); free(V); return -1; }
  }
  orc_lsqr_state st;
  memset(&st, 0, sizeof st);
  memset(out, 0, sizeof *out);

  /* O-1: x = 0, var = 0; u = b, beta = ||u||, u /= beta; v = A^T u, alpha = ||v||, v /= alpha; w = v. */
  ORC_PAR_FOR
  for (int64_t j = 0; j < n; ++j) { x[j] = 0.0; var[j] = 0.0; v[j] = 0.0; }
  ORC_PAR_FOR
  for (int64_t i = 0; i < m; ++i) u[i] = b[i];
  double beta = orc_nrm2(u, m), alpha = 0.0;
  if (beta > 0.0) {
    orc_scal(u, m, 1.0 / beta);
    aprod(2, u, v, ctx);
    alpha = orc_nrm2(v, n);
  }
  if (alpha > 0.0) orc_scal(v, n, 1.0 / alpha);
  ORC_PAR_FOR
  for (int64_t j = 0; j < n; ++j) w[j] = v[j];
  int64_t nu = 0, nv = 0;
  if (reorth) {
    if (beta > 0.0) memcpy(U + (nu++) * m, u, sizeof(double) * (size_t)m);
    if (alpha > 0.0) memcpy(V + (nv++) * n, v, sizeof(double) * (size_t)n);
  }

  /* O-2 */
  double rhobar = alpha, phibar = beta, bnorm = beta, rnorm = beta, r1norm = beta, r2norm = beta;
  double anorm = 0, acond = 0, ddnorm = 0, res2 = 0, xnorm = 0, xxnorm = 0, z = 0, cs2 = -1, sn2 = 0;
  double dampsq = damp * damp;
  double ctol = conlim > 0 ? 1.0 / conlim : 0.0;
  double arnorm = alpha * beta;
  int32_t istop = 0, istop_first = 0, itn = 0;
  double rho = 0, theta = 0, phi = 0, tau = 0, psi = 0, test1 = 0, test2 = 0, test3 = 0;
  if (arnorm == 0.0) goto done;

  /* O-3 main loop */
  while (itn < itn_limit) {
    itn = itn + 1;
    /* a. u = A v - alpha u ; beta = ||u|| */
    orc_scal(u, m, -alpha);
    aprod(1, v, u, ctx);
    if (reorth) orc_reorth(u, U, nu, m);
    beta = orc_nrm2(u, m);
    /* b. */
    if (beta > 0.0) {
      orc_scal(u, m, 1.0 / beta);
      anorm = sqrt(anorm * anorm + alpha * alpha + beta * beta + dampsq);
      orc_scal(v, n, -beta);
      aprod(2, u, v, ctx);
      if (reorth) orc_reorth(v, V, nv, n);
      alpha = orc_nrm2(v, n);
      if (alpha > 0.0) orc_scal(v, n, 1.0 / alpha);
      if (reorth) {
        memcpy(U + (nu++) * m, u, sizeof(double) * (size_t)m);
        if (alpha > 0.0) memcpy(V + (nv++) * n, v, sizeof(double) * (size_t)n);
      }
    }
    /* c. damping rotation */
    double rhobar1;
    if (damp > 0.0) {
      rhobar1 = sqrt(rhobar * rhobar + dampsq);
      double cs1 = rhobar / rhobar1, sn1 = damp / rhobar1;
      psi = sn1 * phibar;
      phibar = cs1 * phibar;
    } else {
      rhobar1 = rhobar;
      psi = 0.0;
    }
    /* d. plane rotation eliminating beta */
    rho = sqrt(rhobar1 * rhobar1 + beta * beta);
    double cs = rhobar1 / rho, sn = beta / rho;
    theta = sn * alpha;
    rhobar = -cs * alpha;
    phi = cs * phibar;
    phibar = sn * phibar;
    tau = sn * phi;
    /* e. update x, w, var (old w used for var and x) */
    double t1 = phi / rho, t2 = -theta / rho, t3 = 1.0 / rho;
    orc_eda DD;
    memset(&DD, 0, sizeof DD);
    ORC_PAR_SUM(ddnorm) /* (the timing build rejects repro mode: DD is not thread-safe) */
    for (int64_t j = 0; j < n; ++j) {
      double dk = t3 * w[j];
      var[j] = var[j] + dk * dk;
      if (repro) orc_eda_add(&DD, dk * dk);
      else ddnorm = ddnorm + dk * dk;
      x[j] = x[j] + t1 * w[j];
      w[j] = v[j] + t2 * w[j];
    }
    if (repro) ddnorm = ddnorm + orc_eda_round(&DD); /* NEXT-4: order-independent */
    /* f. norm of x estimate */
    double delta = sn2 * rho, gambar = -cs2 * rho, rhs = phi - delta * z, zbar = rhs / gambar;
    xnorm = sqrt(xxnorm + zbar * zbar);
    double gamma = sqrt(gambar * gambar + theta * theta);
    cs2 = gambar / gamma;
    sn2 = theta / gamma;
    z = rhs / gamma;
    xxnorm = xxnorm + z * z;
    /* g. norm estimates */
    acond = anorm * sqrt(ddnorm);
    res2 = res2 + psi * psi;
    rnorm = sqrt(phibar * phibar + res2);
    arnorm = alpha * fabs(tau);
    if (damp > 0.0) {
      double r1sq = rnorm * rnorm - dampsq * xxnorm;
      r1norm = sqrt(fabs(r1sq));
      if (r1sq < 0) r1norm = -r1norm;
    } else {
      r1norm = rnorm;
    }
    r2norm = rnorm;
    /* h. convergence tests */
    test1 = rnorm / bnorm;
    test2 = arnorm / (anorm * rnorm + eps);
    test3 = 1.0 / (acond + eps);
    double tt1 = test1 / (1.0 + anorm * xnorm / bnorm);
    double rtol = btol + atol * anorm * xnorm / bnorm;
    /* i. istop, later assignments win */
    int32_t is = 0;
    if (itn >= itn_limit) is = 7;
    if (1.0 + test3 <= 1.0) is = 6;
    if (1.0 + test2 <= 1.0) is = 5;
    if (1.0 + tt1 <= 1.0) is = 4;
    if (test3 <= ctol) is = 3;
    if (test2 <= atol) is = 2;
    if (test1 <= rtol) is = 1;
    istop = is;
    if (istop != 0 && istop_first == 0) istop_first = istop;
    if (trace) {
      st.itn = itn; st.istop = istop; st.alpha = alpha; st.beta = beta; st.rhobar = rhobar; st.phibar = phibar;
      st.anorm = anorm; st.acond = acond; st.ddnorm = ddnorm; st.res2 = res2; st.xnorm = xnorm;
      st.xxnorm = xxnorm; st.z = z; st.cs2 = cs2; st.sn2 = sn2; st.rnorm = rnorm; st.r1norm = r1norm;
      st.r2norm = r2norm; st.arnorm = arnorm; st.bnorm = bnorm; st.rho = rho; st.theta = theta; st.phi = phi;
      st.tau = tau; st.psi = psi; st.test1 = test1; st.test2 = test2; st.test3 = test3;
      trace(&st, u, v, w, x, var, trace_ctx);
    }
    /* j. */
    if (istop != 0 && !fixed_count) break;
  }

done:
  /* O-4: standard errors, lsqr.f form: t = 1; m > n -> m - n; damp > 0 -> m; s = r2norm/sqrt(t); se = s sqrt(var) */
  if (se) {
    double t = 1.0;
    if (m > n) t = (double)(m - n);
    if (damp > 0.0) t = (double)m;
    double s = r2norm / sqrt(t);
    for (int64_t j = 0; j < n; ++j) se[j] = s * sqrt(var[j]);
  }
  out->istop = istop; out->itn = itn; out->istop_first = istop_first;
  out->r1norm = r1norm; out->r2norm = r2norm; out->anorm = anorm; out->acond = acond; out->arnorm = arnorm;
  out->xnorm = xnorm; out->bnorm = bnorm;
  free(u); free(v); free(w); free(U); free(V);
  orc_repro_mode = 0;
  return 0;
}

/*
 * omp_timing.c -- ALL-CORE TIMING VARIANT of the CPU oracle (bench.py's cpu_baseline only).
 *
 *   *** NOT A PARITY REFERENCE. ***  The checker is the serial avugsr_oracle.c built on its own.  This file includes
 *   that source with ORC_PAR_FOR / ORC_PAR_SUM defined as OpenMP pragmas (its LSQR vector loops run on all cores,
 *   with reductions in a thread-dependent order) and adds OpenMP versions of the two products, so that the oracle
 *   can be timed on every host core as SURVEY §8(d) asks.  Build: gcc -O2 -fopenmp -ffp-contract=off.
 *
 *   orc_omp_aprod1 (y += A x, Eq. (3)): rows are independent -- static row partition.
 *   orc_omp_aprod2 (x += A^T y, Eq. (4)): thread t takes a contiguous row range cut at star boundaries,
 *     so the astrometric columns it writes are its own; the shared slice (attitude, instrumental,
 *     global) goes to a thread-private buffer, summed afterwards in thread order.
 */
#define ORC_PRAGMA(x) _Pragma(#x)
#define ORC_PAR_FOR ORC_PRAGMA(omp parallel for schedule(static))
#define ORC_PAR_SUM(v) ORC_PRAGMA(omp parallel for schedule(static) reduction(+ : v))
#include "avugsr_oracle.c"

#include <omp.h>

int orc_omp_threads(void) { return omp_get_max_threads(); }
/* thread count of the parallel loops that follow (n > 0); torchrun exports OMP_NUM_THREADS=1 to every rank */
void orc_omp_set_threads(int n) {
  if (n > 0) omp_set_num_threads(n);
}

void orc_omp_aprod1(const orc_sys* S, const double* x, double* y) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < S->n_rows; ++i) {
    double s = 0.0;
    for (int sl = 0; sl < ORC_SLOTS; ++sl) {
      if (sl == 23 && S->n_glob == 0) continue;
      s = s + S->vals[i * ORC_SLOTS + sl] * x[orc_col(sl, i, S->mA, S->mT, S->iC, S->n_axis, S->G0)];
    }
    y[i] = y[i] + s;
  }
  for (int64_t k = 0; k < S->n_constr; ++k) {
    double s = 0.0;
    for (int64_t e = S->c_ptr[k]; e < S->c_ptr[k + 1]; ++e)
      if (orc_owned(S, S->c_col[e])) s = s + S->c_val[e] * x[S->c_col[e]];
    y[S->n_rows + k] = y[S->n_rows + k] + s;
  }
}

void orc_omp_aprod2(const orc_sys* S, const double* y, double* x) {
  const int nt = omp_get_max_threads();
  const int64_t A0 = S->A0, nsh = S->n_cols - A0;
  double* buf = (double*)calloc((size_t)nt * (size_t)(nsh > 0 ? nsh : 1), sizeof(double));
  if (!buf) abort();
#pragma omp parallel num_threads(nt)
  {
    const int t = omp_get_thread_num();
    int64_t lo = (S->n_rows * t) / nt, hi = (S->n_rows * (t + 1)) / nt;
    /* cut at star boundaries (rows are grouped by star: matrixIndexAstro = 5 * star) */
    while (lo > 0 && lo < S->n_rows && S->mA[lo] == S->mA[lo - 1]) ++lo;
    while (hi > 0 && hi < S->n_rows && S->mA[hi] == S->mA[hi - 1]) ++hi;
    double* zb = buf + (size_t)t * (size_t)nsh;
    for (int64_t i = lo; i < hi; ++i)
      for (int sl = 0; sl < ORC_SLOTS; ++sl) {
        if (sl == 23 && S->n_glob == 0) continue;
        const int64_t c = orc_col(sl, i, S->mA, S->mT, S->iC, S->n_axis, S->G0);
        const double a = S->vals[i * ORC_SLOTS + sl] * y[i];
        if (c < A0) x[c] = x[c] + a;
        else zb[c - A0] = zb[c - A0] + a;
      }
  }
#pragma omp parallel for schedule(static)
  for (int64_t c = 0; c < nsh; ++c) {
    double s = 0.0;
    for (int t = 0; t < nt; ++t) s = s + buf[(size_t)t * (size_t)nsh + c];
    x[A0 + c] = x[A0 + c] + s;
  }
  free(buf);
  for (int64_t k = 0; k < S->n_constr; ++k)
    for (int64_t e = S->c_ptr[k]; e < S->c_ptr[k + 1]; ++e)
      if (orc_owned(S, S->c_col[e])) x[S->c_col[e]] = x[S->c_col[e]] + S->c_val[e] * y[S->n_rows + k];
}

void orc_omp_sys_aprod(int32_t mode, const double* in, double* out, void* ctx) {
  if (mode == 1) orc_omp_aprod1((const orc_sys*)ctx, in, out);
  else orc_omp_aprod2((const orc_sys*)ctx, in, out);
}

// lsqr_repro.cu -- bitwise-reproducible mode (docs/REPRO.md), product side.
//
// Every reduction is an exact digit accumulation (EDA, docs/REPRO.md) of identically rounded FP64 terms, combined
// with 64-bit integer additions/atomics, which are associative: the result does not depend on thread, warp, block or
// atomic order.  Every other operation is a single IEEE operation written with explicit _rn intrinsics (no FMA
// contraction), in the order the Paige-Saunders recurrence writes them.  The CPU test oracle implements the same
// spec independently (docs/REPRO.md), so iterates agree bit for bit.
//
// Accumulation format (device-internal): 7 digits of 30-bit pieces in int64 over bits [-168, 42) (the spec's window
// is [-168, 32): bits of a term at or above 2^32 are dropped, as the spec says).  A piece is < 2^30 in magnitude, so
// ANY partial sum of fewer than 2^33 pieces is exact -- lsqr_set_reproducible rejects shards where an accumulator
// could receive more (6 n_local_rows + constraint entries >= 2^33).  Before a cross-rank allreduce the digits are
// carry-normalised (value-preserving), so the reduced digits stay below P * 2^30.  Rounding converts the exact
// value to the spec's unique carry-normalised 5 x 40-bit form and applies the spec's rounding chain, so the result
// does not depend on the accumulation format.
//
// These kernels are simple (thread per row / column, global atomics for every digit): the mode is for verification
// and run-to-run reproducibility, not for speed.
#include "lsqr_internal.cuh"

namespace lsqr {

namespace {

constexpr int kL = 7;   // digits; digit q covers bits [B_q, B_q + 30), B_q = 12 - 30 q (12, -18, ..., -168)
constexpr int kW = 30;  // bits per piece
constexpr long long kM30 = (1ll << kW) - 1;
constexpr long long kM20 = (1ll << 20) - 1;  // digit 0 keeps bits [12, 32) only: the spec's window top is 2^32

struct Eda {
  long long d[kL];
};

__device__ __forceinline__ void eda_zero(Eda& A) {
#pragma unroll
  for (int q = 0; q < kL; ++q) A.d[q] = 0;
}

// split(c): with p = E + 168 the offset of the significand's lowest bit above the window bottom (bits below the
// window are truncated first), the significand lands in digits 6-k, 5-k, 4-k (k = p div 30) as the 30-bit pieces
// lo, mid, hi of M << (p mod 30); pieces above digit 0 are dropped and digit 0 keeps its bits below 2^32.
struct Pieces {
  long long lo, mid, hi, sgn;  // magnitudes (sign applied by the consumer: (x ^ sgn) - sgn)
  int k;
};

__device__ __forceinline__ Pieces eda_split(double c) {
  const long long bits = __double_as_longlong(c);
  const int ex = (int)((bits >> 52) & 0x7ff);
  unsigned long long M = (unsigned long long)bits & ((1ull << 52) - 1);
  if (ex) M |= 1ull << 52;
  int p = (ex ? ex - 1075 : -1074) + 168;
  if (p < 0) {  // (rare) truncate the bits below 2^-168
    M = p > -53 ? (M >> (-p)) : 0ull;
    p = 0;
  }
  const int k = p / kW, o = p - kW * k;
  Pieces r;
  r.k = k;
  r.sgn = bits >> 63;  // 0 or -1
  r.lo = (long long)((M << o) & (unsigned long long)kM30);
  r.mid = (long long)((M >> (kW - o)) & (unsigned long long)kM30);
  r.hi = (long long)((M >> (2 * kW - o)) & (unsigned long long)kM30);
  return r;
}

__device__ __forceinline__ long long sgnd(long long x, long long sgn) { return (x ^ sgn) - sgn; }

__device__ __forceinline__ void eda_add(Eda& A, double c) {
  const Pieces P = eda_split(c);
  const long long s = P.sgn;
  switch (P.k) {  // constant digit indices keep A in registers; k is nearly warp-uniform for real data
    case 0: A.d[6] += sgnd(P.lo, s); A.d[5] += sgnd(P.mid, s); A.d[4] += sgnd(P.hi, s); break;
    case 1: A.d[5] += sgnd(P.lo, s); A.d[4] += sgnd(P.mid, s); A.d[3] += sgnd(P.hi, s); break;
    case 2: A.d[4] += sgnd(P.lo, s); A.d[3] += sgnd(P.mid, s); A.d[2] += sgnd(P.hi, s); break;
    case 3: A.d[3] += sgnd(P.lo, s); A.d[2] += sgnd(P.mid, s); A.d[1] += sgnd(P.hi, s); break;
    case 4: A.d[2] += sgnd(P.lo, s); A.d[1] += sgnd(P.mid, s); A.d[0] += sgnd(P.hi & kM20, s); break;
    case 5: A.d[1] += sgnd(P.lo, s); A.d[0] += sgnd(P.mid & kM20, s); break;
    case 6: A.d[0] += sgnd(P.lo & kM20, s); break;
    default: break;
  }
}

// the pieces of one term straight into the digit-major column accumulator zd[q][col] (q = 6-k, 5-k, 4-k)
__device__ __forceinline__ void eda_atomic_term(long long* __restrict__ zd_col, int64_t stride, double c) {
  const Pieces P = eda_split(c);
  const long long pc[3] = {P.lo, P.mid, P.hi};
#pragma unroll
  for (int r = 0; r < 3; ++r) {
    const int q = kL - 1 - P.k - r;
    const long long m = q == 0 ? (pc[r] & kM20) : pc[r];
    if (q >= 0 && m != 0)
      atomicAdd(reinterpret_cast<unsigned long long*>(zd_col + q * stride), (unsigned long long)sgnd(m, P.sgn));
  }
}

// carry-normalise (value-preserving): digits 1..6 in [0, 2^30), digit 0 signed
__device__ __forceinline__ void eda_normalize(long long (&D)[kL]) {
#pragma unroll
  for (int q = kL - 1; q >= 1; --q) {
    const long long c = D[q] >> kW;  // arithmetic shift = floor division
    D[q] -= c * (1ll << kW);
    D[q - 1] += c;
  }
}

// round(D) of the spec: the exact value's carry-normalised 40-bit digits N_0..N_4 (bits [-8, ..), [-48, -8), ...,
// [-168, -128)), then v = 0; v = v + N_d * 2^B_d for d = 0..4, every conversion and addition rounded
__device__ __forceinline__ double eda_round_d(const long long* Din) {
  long long D[kL];
#pragma unroll
  for (int q = 0; q < kL; ++q) D[q] = Din[q];
  eda_normalize(D);
  // D_q (q >= 1) covers bits [30 (6 - q), 30 (7 - q)) above 2^-168; D_0 sits at bit 180
  const long long N4 = D[6] | ((D[5] & 0x3ff) << 30);
  const long long N3 = (D[5] >> 10) | ((D[4] & 0xfffff) << 20);
  const long long N2 = (D[4] >> 20) | (D[3] << 10);
  const long long N1 = D[2] | ((D[1] & 0x3ff) << 30);
  const long long N0 = (D[1] >> 10) + D[0] * (1ll << 20);
  const long long N[5] = {N0, N1, N2, N3, N4};
  const double pw[5] = {0x1p-8, 0x1p-48, 0x1p-88, 0x1p-128, 0x1p-168};
  double v = 0.0;
#pragma unroll
  for (int q = 0; q < 5; ++q) v = __dadd_rn(v, __dmul_rn(__ll2double_rn(N[q]), pw[q]));
  return v;
}

// integer reduction of a thread's digits over the block, then one 64-bit atomic per digit (exact, order-free)
__device__ __forceinline__ void eda_flush_block(const Eda& A, long long* __restrict__ dst, int64_t stride = 1) {
  __shared__ long long sd[kL][32];
#pragma unroll
  for (int q = 0; q < kL; ++q) {
    long long v = A.d[q];
#pragma unroll
    for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    if ((threadIdx.x & 31) == 0) sd[q][threadIdx.x >> 5] = v;
  }
  __syncthreads();
  if (threadIdx.x < kL) {
    long long t = 0;
    for (int w = 0; w < (int)(blockDim.x >> 5); ++w) t += sd[threadIdx.x][w];
    if (t != 0 && dst)
      atomicAdd(reinterpret_cast<unsigned long long*>(dst + threadIdx.x * stride), (unsigned long long)t);
  }
  __syncthreads();
}

__device__ __forceinline__ void eda_atomic(long long* __restrict__ dst, const Eda& A, int64_t stride = 1) {
#pragma unroll
  for (int q = 0; q < kL; ++q)
    if (A.d[q] != 0) atomicAdd(reinterpret_cast<unsigned long long*>(dst + q * stride), (unsigned long long)A.d[q]);
}

// Column of position t (0..5) of lane j of a row (lane-major storage: position 6j+t holds paper slot slot_of(t, j)):
// t=0 astro j; t=1..3 attitude axis t-1, knot j; t=4 instrumental j; t=5: astro 4 (j=0), instrumental 4/5 (j=1/2),
// global (j=3).  Returns -1 for the global slot when the system has none.
__device__ __forceinline__ int64_t lane_col(const SysView& S, const IdxRec& r, int64_t star, int t, int j) {
  if (t == 0) return 5 * star + j;
  if (t <= 3) return S.A0 + (int64_t)(t - 1) * S.n_axis + r.k0 + j;
  const uint32_t w3[3] = {r.ic01, r.ic23, r.ic45};
  if (t == 4) return S.I0 + S.ip.inv((w3[j >> 1] >> ((j & 1) * 16)) & 0xffffu);
  if (j == 0) return 5 * star + 4;
  if (j == 3) return S.n_glob ? S.G0 : -1;
  const int q = 3 + j;  // instrumental 4 or 5
  return S.I0 + S.ip.inv((w3[q >> 1] >> ((q & 1) * 16)) & 0xffffu);
}

// Row partition of the repro product kernels: every warp takes an even, 8-aligned slice of the rows (star ownership
// is irrelevant here: integer digit sums are exact and associative, so how the terms are grouped -- registers,
// shuffles, atomics, which warp -- cannot change any result).  4 lanes per row, lane j holding positions 6j..6j+5;
// each lane carries kNR rows per step (loads for all of them issued before any arithmetic).
constexpr int kRThreads = 256;
constexpr int kNR = 2;
struct WarpRows {
  int64_t r0, r1, star;
  __device__ WarpRows(const SysView& S) {
    const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const int64_t chunk = ((S.n_rows + nw - 1) / nw + 7) & ~(int64_t)7;
    r0 = gw * chunk < S.n_rows ? gw * chunk : S.n_rows;
    r1 = r0 + chunk < S.n_rows ? r0 + chunk : S.n_rows;
    int64_t lo = 0, hi = S.n_stars;  // star of row r0: star_ptr[lo] <= r0 < star_ptr[lo + 1]
    while (hi - lo > 1) {
      const int64_t mid = (lo + hi) >> 1;
      if (S.star_ptr[mid] <= r0) lo = mid;
      else hi = mid;
    }
    star = lo;
  }
};

__device__ __forceinline__ void load6(const SysView& S, int64_t row, int j, double (&a)[6]) {
  const double2* p = reinterpret_cast<const double2*>(S.vals + row * kSlots + 6 * j);
#pragma unroll
  for (int k = 0; k < 3; ++k) {
    const double2 t = __ldg(p + k);
    a[2 * k] = t.x;
    a[2 * k + 1] = t.y;
  }
}

// ---------------------------------------------------------------------------------------------------- kernels
// aprod1 (P&S step a): u_hat_i <- ((-alpha) * (ib * u_hat_i)) + round(EDA_s a_is * v[col_is]); beta^2 digits.
// init: beta^2 digits of u = b only.
__global__ void __launch_bounds__(kRThreads) k_r_aprod1(SysView S, const double* __restrict__ v,
                                                        double* __restrict__ u, long long* __restrict__ b2d,
                                                        long long* __restrict__ cd, const DevState* __restrict__ st,
                                                        int init) {
  if (!init && st->halted) return;
  Eda B;
  eda_zero(B);
  if (init) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < S.n_rows;
         i += (int64_t)gridDim.x * blockDim.x)
      eda_add(B, __dmul_rn(u[i], u[i]));
    eda_flush_block(B, b2d);
    return;
  }
  const double ib = st->inv_beta, nalpha = -st->alpha;
  const int lane = threadIdx.x & 31, q = lane >> 2, j = lane & 3;
  const WarpRows R(S);
  int64_t star = R.star;
  for (int64_t g0 = R.r0; g0 < R.r1; g0 += 8 * kNR) {  // warp-uniform trip count
    double a[kNR][6], g[kNR][6];
    IdxRec rec[kNR];
#pragma unroll
    for (int n = 0; n < kNR; ++n) {
      const int64_t row = g0 + 8 * n + q;
      if (row < R.r1) {
        load6(S, row, j, a[n]);
        rec[n] = S.idx[row];
      }
    }
#pragma unroll
    for (int n = 0; n < kNR; ++n) {
      const int64_t row = g0 + 8 * n + q;
      if (row < R.r1) {
        while (S.star_ptr[star + 1] <= row) ++star;
#pragma unroll
        for (int t = 0; t < 6; ++t) {
          const int64_t c = lane_col(S, rec[n], star, t, j);
          g[n][t] = c >= 0 ? __ldg(v + c) : 0.0;
        }
      }
    }
#pragma unroll
    for (int n = 0; n < kNR; ++n) {
      const int64_t row = g0 + 8 * n + q;
      const bool valid = row < R.r1;
      Eda A;
      eda_zero(A);
      if (valid) {
#pragma unroll
        for (int t = 0; t < 6; ++t) eda_add(A, __dmul_rn(a[n][t], g[n][t]));
      }
#pragma unroll
      for (int k = 0; k < kL; ++k) {
        A.d[k] += __shfl_xor_sync(0xffffffffu, A.d[k], 1);
        A.d[k] += __shfl_xor_sync(0xffffffffu, A.d[k], 2);
      }
      if (valid && j == 0) {
        const double un = __dadd_rn(__dmul_rn(nalpha, __dmul_rn(ib, u[row])), eda_round_d(A.d));
        u[row] = un;
        eda_add(B, __dmul_rn(un, un));
      }
    }
  }
  eda_flush_block(B, b2d);
  // constraint rows: digits of every owned entry's product, one thread per chunk (chunks lie within one row)
  for (int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; c < S.n_chunks; c += (int64_t)gridDim.x * blockDim.x) {
    Eda A;
    eda_zero(A);
    for (int64_t e = S.ch_beg[c]; e < S.ch_end[c]; ++e) eda_add(A, __dmul_rn(S.cval[e], v[S.ccol[e]]));
    eda_atomic(cd + (int64_t)S.ch_row[c] * kL, A);
  }
}

// aprod2 contributions: digits of a_ij * (ib * u_hat_i) into zd[q][col] (digit-major) for every column (colnorm: a_ij^2).  Astro
// digits stay in registers per lane until the lane's star changes, global digits until the end (block-reduced);
// attitude and instrumental digits go straight to global 64-bit integer atomics.
__device__ __forceinline__ void flush_lane(long long* __restrict__ dst, Eda& A, int64_t stride) {
  eda_atomic(dst, A, stride);
  eda_zero(A);
}

__global__ void __launch_bounds__(kRThreads) k_r_aprod2(SysView S, const double* __restrict__ u,
                                                        const double* __restrict__ uc, long long* __restrict__ zd,
                                                        const DevState* __restrict__ st, int colnorm) {
  if (!colnorm && (st->halted || !st->beta_pos)) return;
  const double ib = colnorm ? 1.0 : st->inv_beta;
  const int lane = threadIdx.x & 31, q = lane >> 2, j = lane & 3;
  const WarpRows R(S);
  int64_t star = R.star;
  Eda As0, As1, G;  // astro column j (and 4 for j == 0) of `star`; global column
  eda_zero(As0);
  eda_zero(As1);
  eda_zero(G);
  for (int64_t g0 = R.r0; g0 < R.r1; g0 += 8 * kNR) {  // (no warp collectives in this loop)
    double a[kNR][6], y[kNR];
    IdxRec rec[kNR];
#pragma unroll
    for (int n = 0; n < kNR; ++n) {
      const int64_t row = g0 + 8 * n + q;
      if (row < R.r1) {
        load6(S, row, j, a[n]);
        rec[n] = S.idx[row];
        y[n] = colnorm ? 0.0 : __ldg(u + row);
      }
    }
#pragma unroll
    for (int n = 0; n < kNR; ++n) {
      const int64_t row = g0 + 8 * n + q;
      if (row >= R.r1) break;
      if (S.star_ptr[star + 1] <= row) {
        flush_lane(zd + 5 * star + j, As0, S.n_cols);
        if (j == 0) flush_lane(zd + 5 * star + 4, As1, S.n_cols);
        while (S.star_ptr[star + 1] <= row) ++star;
      }
      const double yn = colnorm ? 0.0 : __dmul_rn(ib, y[n]);
#pragma unroll
      for (int t = 0; t < 6; ++t) {
        const double term = colnorm ? __dmul_rn(a[n][t], a[n][t]) : __dmul_rn(a[n][t], yn);
        if (t == 0) {
          eda_add(As0, term);
        } else if (t == 5 && j == 0) {
          eda_add(As1, term);
        } else if (t == 5 && j == 3) {
          if (S.n_glob) eda_add(G, term);
        } else {
          eda_atomic_term(zd + lane_col(S, rec[n], star, t, j), S.n_cols, term);
        }
      }
    }
  }
  if (R.r1 > R.r0) {
    flush_lane(zd + 5 * star + j, As0, S.n_cols);
    if (j == 0) flush_lane(zd + 5 * star + 4, As1, S.n_cols);
  }
  eda_flush_block(G, S.n_glob ? zd + S.G0 : nullptr, S.n_cols);
  for (int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; c < S.n_chunks; c += (int64_t)gridDim.x * blockDim.x) {
    const double yc = colnorm ? 0.0 : __dmul_rn(ib, uc[S.ch_row[c]]);
    for (int64_t e = S.ch_beg[c]; e < S.ch_end[c]; ++e) {
      const double cv = S.cval[e];
      eda_atomic_term(zd + S.ccol[e], S.n_cols, colnorm ? __dmul_rn(cv, cv) : __dmul_rn(cv, yc));
    }
  }
}

// beta (one thread): constraint u, ||u||, anorm (P&S step b bookkeeping); resets the digit accumulators it read
__global__ void k_r_beta(SysView S, long long* __restrict__ b2d, long long* __restrict__ cd, double* __restrict__ uc,
                         const double* __restrict__ crhs, DevState* __restrict__ st, int init) {
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  if (!init && st->halted) return;
  Eda B;
  for (int q = 0; q < kL; ++q) B.d[q] = b2d[q];
  const double ib = st->inv_beta, nalpha = -st->alpha;
  for (int k = 0; k < S.n_constr; ++k) {
    double un;
    if (init) {
      un = crhs ? crhs[k] : 0.0;
    } else {
      un = __dadd_rn(__dmul_rn(nalpha, __dmul_rn(ib, uc[k])), eda_round_d(cd + (int64_t)k * kL));
      for (int q = 0; q < kL; ++q) cd[(int64_t)k * kL + q] = 0;
    }
    uc[k] = un;
    eda_add(B, __dmul_rn(un, un));
  }
  for (int q = 0; q < kL; ++q) b2d[q] = 0;
  const double beta = __dsqrt_rn(eda_round_d(B.d));
  const int pos = beta > 0.0;
  if (init) {
    st->bnorm = beta;
  } else if (pos) {
    const double a = st->alpha, d = st->damp;
    st->anorm = __dsqrt_rn(
        __dadd_rn(__dadd_rn(__dadd_rn(__dmul_rn(st->anorm, st->anorm), __dmul_rn(a, a)), __dmul_rn(beta, beta)),
                  __dmul_rn(d, d)));
  }
  st->beta = beta;
  st->beta_pos = pos;
  st->inv_beta = pos ? __ddiv_rn(1.0, beta) : 1.0;
}

// v_j <- ((-beta) * v_j) + round(zd_j) on every column (init: v_j = 0 + round(zd_j)); alpha^2 digits split into the
// astro part (columns < A0, rank-local: allreduced when P > 1) and the shared part (replicated on every rank: never
// reduced); zd reset.  mode 2 (colnorm): D_j = 1/sqrt(c_j) (1 if c_j == 0) with c_j = round(zd_j).
__global__ void k_r_vupdate(int64_t n, int64_t A0, double* __restrict__ v, long long* __restrict__ zd,
                            long long* __restrict__ a2d, long long* __restrict__ a2s, const DevState* __restrict__ st,
                            int mode) {  // mode 0 LSQR, 1 init, 2 colnorm -> D
  if (mode == 0 && (st->halted || !st->beta_pos)) return;
  if (mode == 1 && !st->beta_pos) return;
  const double nbeta = mode == 2 ? 0.0 : -st->beta;
  Eda Aa, As;
  eda_zero(Aa);
  eda_zero(As);
  for (int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; c < n; c += (int64_t)gridDim.x * blockDim.x) {
    long long dz[kL];
#pragma unroll
    for (int q = 0; q < kL; ++q) {
      dz[q] = zd[q * n + c];
      zd[q * n + c] = 0;
    }
    const double z = eda_round_d(dz);
    if (mode == 2) {
      v[c] = z > 0.0 ? __ddiv_rn(1.0, __dsqrt_rn(z)) : 1.0;
      continue;
    }
    const double vn = mode == 1 ? __dadd_rn(v[c], z) : __dadd_rn(__dmul_rn(nbeta, v[c]), z);
    v[c] = vn;
    eda_add(c < A0 ? Aa : As, __dmul_rn(vn, vn));
  }
  if (mode != 2) {
    eda_flush_block(Aa, a2d);
    eda_flush_block(As, a2s);
  }
}

// P&S steps b (alpha), c, d (rotation): t1, t2, t3 -- one thread
__global__ void k_r_scalar_a(DevState* __restrict__ st, long long* __restrict__ a2d, long long* __restrict__ a2s,
                             int init, int32_t* __restrict__ host_flag) {
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  if (!init && st->halted) {
    st->col_enable = 0;
    return;
  }
  const int bp = st->beta_pos;
  double alpha = st->alpha;
  if (bp) {
    long long a2[kL];
    for (int q = 0; q < kL; ++q) a2[q] = a2d[q] + a2s[q];
    alpha = __dsqrt_rn(eda_round_d(a2));
    st->inv_alpha = alpha > 0.0 ? __ddiv_rn(1.0, alpha) : 1.0;
    st->v_pending = 1;
  } else {
    st->v_pending = 0;
  }
  for (int q = 0; q < kL; ++q) a2d[q] = a2s[q] = 0;
  st->alpha = alpha;
  st->col_enable = 1;
  if (init) {  // O-1/O-2
    const double beta = st->beta;
    st->rhobar = alpha; st->phibar = beta; st->rnorm = beta; st->r1norm = beta; st->r2norm = beta;
    st->anorm = 0; st->acond = 0; st->ddnorm = 0; st->res2 = 0; st->xnorm = 0; st->xxnorm = 0; st->z = 0;
    st->cs2 = -1.0; st->sn2 = 0.0;
    st->arnorm = __dmul_rn(alpha, beta);
    st->t1 = 0.0; st->t2 = 0.0; st->t3 = 0.0;
    st->itn = 0; st->istop = 0; st->istop_first = 0;
    st->halted = (st->arnorm == 0.0) ? 1 : 0;
    if (host_flag) *reinterpret_cast<volatile int32_t*>(host_flag) = st->halted;
    return;
  }
  st->itn += 1;
  const double beta = st->beta, damp = st->damp, dampsq = __dmul_rn(damp, damp);
  double rhobar = st->rhobar, phibar = st->phibar, psi, rhobar1;
  if (damp > 0.0) {
    rhobar1 = __dsqrt_rn(__dadd_rn(__dmul_rn(rhobar, rhobar), dampsq));
    const double cs1 = __ddiv_rn(rhobar, rhobar1), sn1 = __ddiv_rn(damp, rhobar1);
    psi = __dmul_rn(sn1, phibar);
    phibar = __dmul_rn(cs1, phibar);
  } else {
    rhobar1 = rhobar;
    psi = 0.0;
  }
  const double rho = __dsqrt_rn(__dadd_rn(__dmul_rn(rhobar1, rhobar1), __dmul_rn(beta, beta)));
  const double cs = __ddiv_rn(rhobar1, rho), sn = __ddiv_rn(beta, rho);
  const double theta = __dmul_rn(sn, alpha);
  st->rhobar = __dmul_rn(-cs, alpha);
  const double phi = __dmul_rn(cs, phibar);
  st->phibar = __dmul_rn(sn, phibar);
  st->rn_tmp = psi;  // carried to scalar_b
  st->t1 = __ddiv_rn(phi, rho);
  st->t2 = __ddiv_rn(-theta, rho);
  st->t3 = __ddiv_rn(1.0, rho);
  st->r_rho = rho;  // hand-over to scalar_b
  st->r_theta = theta;
  st->r_phi = phi;
  st->r_sn = sn;
}

// O-3e: v <- (1/alpha) v (if pending); d = t3 w; var += d*d; x += t1 w; w = v + t2 w; ddnorm digits
__global__ void k_r_colupdate(double* __restrict__ v, double* __restrict__ w, double* __restrict__ x,
                              double* __restrict__ var, int64_t n, int64_t A0, long long* __restrict__ ddd,
                              long long* __restrict__ dds, const DevState* __restrict__ st, int init) {
  if (!st->col_enable) return;
  const double ia = st->inv_alpha, t1 = st->t1, t2 = st->t2, t3 = st->t3;
  const int vp = st->v_pending && st->alpha > 0.0;
  Eda Aa, As;  // ddnorm digits: astro (rank-local) / shared (replicated)
  eda_zero(Aa);
  eda_zero(As);
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const double vi = vp ? __dmul_rn(ia, v[i]) : v[i];
    v[i] = vi;
    if (init) {  // w = v
      w[i] = vi;
      continue;
    }
    const double wi = w[i];
    const double dk = __dmul_rn(t3, wi);
    const double d2 = __dmul_rn(dk, dk);
    var[i] = __dadd_rn(var[i], d2);
    eda_add(i < A0 ? Aa : As, d2);
    x[i] = __dadd_rn(x[i], __dmul_rn(t1, wi));
    w[i] = __dadd_rn(vi, __dmul_rn(t2, wi));
  }
  if (!init) {
    eda_flush_block(Aa, ddd);
    eda_flush_block(As, dds);
  }
}

// O-3f-j after the column update (ddnorm needed by acond) -- one thread
__global__ void k_r_scalar_b(DevState* __restrict__ st, long long* __restrict__ ddd, long long* __restrict__ dds,
                             int32_t* __restrict__ host_flag) {
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  if (st->halted || !st->col_enable) return;
  const double eps = 0x1p-52;
  const double rho = st->r_rho, theta = st->r_theta, phi = st->r_phi, sn = st->r_sn, psi = st->rn_tmp;
  const double tau = __dmul_rn(sn, phi);
  long long dd[kL];
  for (int q = 0; q < kL; ++q) {
    dd[q] = ddd[q] + dds[q];
    ddd[q] = dds[q] = 0;
  }
  const double ddnorm = __dadd_rn(st->ddnorm, eda_round_d(dd));
  // f.
  const double delta = __dmul_rn(st->sn2, rho), gambar = __dmul_rn(-st->cs2, rho);
  const double rhs = __dadd_rn(phi, -__dmul_rn(delta, st->z));
  const double zbar = __ddiv_rn(rhs, gambar);
  const double xnorm = __dsqrt_rn(__dadd_rn(st->xxnorm, __dmul_rn(zbar, zbar)));
  const double gamma = __dsqrt_rn(__dadd_rn(__dmul_rn(gambar, gambar), __dmul_rn(theta, theta)));
  st->cs2 = __ddiv_rn(gambar, gamma);
  st->sn2 = __ddiv_rn(theta, gamma);
  st->z = __ddiv_rn(rhs, gamma);
  st->xxnorm = __dadd_rn(st->xxnorm, __dmul_rn(st->z, st->z));
  // g.
  const double anorm = st->anorm, damp = st->damp, dampsq = __dmul_rn(damp, damp);
  const double acond = __dmul_rn(anorm, __dsqrt_rn(ddnorm));
  const double res2 = __dadd_rn(st->res2, __dmul_rn(psi, psi));
  const double phibar = st->phibar;
  const double rnorm = __dsqrt_rn(__dadd_rn(__dmul_rn(phibar, phibar), res2));
  const double arnorm = __dmul_rn(st->alpha, fabs(tau));
  double r1norm;
  if (damp > 0.0) {
    const double r1sq = __dadd_rn(__dmul_rn(rnorm, rnorm), -__dmul_rn(dampsq, st->xxnorm));
    r1norm = __dsqrt_rn(fabs(r1sq));
    if (r1sq < 0) r1norm = -r1norm;
  } else {
    r1norm = rnorm;
  }
  // h.
  const double bnorm = st->bnorm;
  const double test1 = __ddiv_rn(rnorm, bnorm);
  const double test2 = __ddiv_rn(arnorm, __dadd_rn(__dmul_rn(anorm, rnorm), eps));
  const double test3 = __ddiv_rn(1.0, __dadd_rn(acond, eps));
  const double axb = __ddiv_rn(__dmul_rn(anorm, xnorm), bnorm);
  const double tt1 = __ddiv_rn(test1, __dadd_rn(1.0, axb));
  const double rtol = __dadd_rn(st->btol, __ddiv_rn(__dmul_rn(__dmul_rn(st->atol, anorm), xnorm), bnorm));
  // i.
  int is = 0;
  if (st->itn >= st->itn_limit) is = 7;
  if (__dadd_rn(1.0, test3) <= 1.0) is = 6;
  if (__dadd_rn(1.0, test2) <= 1.0) is = 5;
  if (__dadd_rn(1.0, tt1) <= 1.0) is = 4;
  if (test3 <= st->ctol) is = 3;
  if (test2 <= st->atol) is = 2;
  if (test1 <= rtol) is = 1;
  st->ddnorm = ddnorm; st->xnorm = xnorm; st->acond = acond; st->res2 = res2; st->rnorm = rnorm;
  st->r1norm = r1norm; st->r2norm = rnorm; st->arnorm = arnorm;
  st->istop = is;
  if (is != 0 && st->istop_first == 0) st->istop_first = is;
  if ((is != 0 && !st->fixed_count) || st->itn >= st->itn_limit) st->halted = 1;
  if (host_flag) *reinterpret_cast<volatile int32_t*>(host_flag) = st->halted | (st->itn << 1);
}

// int64 digits <-> pairs of exact doubles (signed high 32 bits, unsigned low 32 bits) for the FP64 SUM allreduce:
// every partial sum of P such halves is an integer below 2^53 in magnitude, hence exact in any order.  nval values of
// kL digits: digit q of value i at src[q * plane + i] (digit-major planes) or, plane == 0, at src[i * kL + q].  Each
// value is carry-normalised first (value-preserving), so the rank sum of a digit stays below P * 2^30 whatever the
// number of terms behind it.
__device__ __forceinline__ int64_t dig_at(int64_t i, int q, int64_t plane) { return plane ? q * plane + i : i * kL + q; }

__global__ void k_r_pack(const long long* __restrict__ src, int64_t nval, int64_t plane, double* __restrict__ buf) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nval; i += (int64_t)gridDim.x * blockDim.x) {
    long long D[kL];
#pragma unroll
    for (int q = 0; q < kL; ++q) D[q] = src[dig_at(i, q, plane)];
    eda_normalize(D);
#pragma unroll
    for (int q = 0; q < kL; ++q) {
      const int64_t o = (int64_t)q * nval + i;
      buf[2 * o] = (double)(D[q] >> 32);
      buf[2 * o + 1] = (double)(D[q] & 0xffffffffll);
    }
  }
}

__global__ void k_r_unpack(const double* __restrict__ buf, int64_t nval, int64_t plane, long long* __restrict__ dst) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nval; i += (int64_t)gridDim.x * blockDim.x) {
#pragma unroll
    for (int q = 0; q < kL; ++q) {
      const int64_t o = (int64_t)q * nval + i;
      const unsigned long long hi = (unsigned long long)(long long)buf[2 * o];
      const unsigned long long lo = (unsigned long long)(long long)buf[2 * o + 1];
      dst[dig_at(i, q, plane)] = (long long)((hi << 32) + lo);  // two's-complement wrap-around = the int64 sum
    }
  }
}

// one full wave of resident CTAs (the row partition gives every warp an equal slice)
template <class K>
int resident_grid(K kernel, int n_sm) {
  int per_sm = 1;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kernel, kRThreads, 0) != cudaSuccess || per_sm < 1)
    per_sm = 1;
  return n_sm * per_sm;
}

int grid_for(int64_t n) {
  int64_t b = (n + kRedThreads - 1) / kRedThreads;
  if (b < 1) b = 1;
  return (int)(b < 148 * 8 ? b : 148 * 8);
}

struct SdView {  // layout of the scalar digit buffer (see lsqr_internal.cuh)
  long long *b2d, *cd, *a2d, *a2s, *ddd, *dds;
  SdView(long long* sd, int64_t nc) {
    b2d = sd;
    cd = sd + kL;
    a2d = cd + kL * nc;
    a2s = a2d + kL;
    ddd = a2s + kL;
    dds = ddd + kL;
  }
};

}  // namespace

int64_t repro_digits_per_value() { return kL; }
int64_t repro_max_terms() { return (int64_t)1 << 33; }
int64_t repro_sd_size(int64_t n_constr) { return kL * (5 + n_constr); }
long long* repro_sd_part(long long* sd, int64_t n_constr, int part) {
  const SdView V(sd, n_constr);
  return part == 0 ? V.b2d : (part == 1 ? V.a2d : V.ddd);
}

cudaError_t repro_step(int step, const ReproArgs& a, cudaStream_t s) {
  const SysView& S = a.S;
  const SdView V(a.sd, S.n_constr);
  static int g1 = 0, g2 = 0;  // per process (one device type)
  if (!g1) {
    g1 = resident_grid(k_r_aprod1, a.n_sm);
    g2 = resident_grid(k_r_aprod2, a.n_sm);
  }
  const int gc = grid_for(S.n_cols);
  switch (step) {
    case RS_APROD1: k_r_aprod1<<<g1, kRThreads, 0, s>>>(S, a.v, a.u, V.b2d, V.cd, a.st, a.init); break;
    case RS_BETA: k_r_beta<<<1, 32, 0, s>>>(S, V.b2d, V.cd, a.uc, a.crhs, a.st, a.init); break;
    case RS_APROD2: k_r_aprod2<<<g2, kRThreads, 0, s>>>(S, a.u, a.uc, a.zd, a.st, 0); break;
    case RS_VUPDATE: k_r_vupdate<<<gc, kRedThreads, 0, s>>>(S.n_cols, S.A0, a.v, a.zd, V.a2d, V.a2s, a.st, a.init); break;
    case RS_SCALAR_A: k_r_scalar_a<<<1, 32, 0, s>>>(a.st, V.a2d, V.a2s, a.init, a.init ? a.host_flag : nullptr); break;
    case RS_COLUPDATE:
      k_r_colupdate<<<gc, kRedThreads, 0, s>>>(a.v, a.w, a.x, a.var, S.n_cols, S.A0, V.ddd, V.dds, a.st, a.init);
      break;
    case RS_SCALAR_B: k_r_scalar_b<<<1, 32, 0, s>>>(a.st, V.ddd, V.dds, a.host_flag); break;
    case RS_COLNORM: k_r_aprod2<<<g2, kRThreads, 0, s>>>(S, nullptr, nullptr, a.zd, nullptr, 1); break;
    case RS_PRECOND_D:
      k_r_vupdate<<<gc, kRedThreads, 0, s>>>(S.n_cols, S.A0, a.D, a.zd, nullptr, nullptr, nullptr, 2);
      break;
    default: return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

cudaError_t repro_pack(const long long* src, int64_t nval, int64_t plane, double* buf, int unpack, cudaStream_t s) {
  if (nval == 0) return cudaSuccess;
  if (unpack) k_r_unpack<<<grid_for(nval), kRedThreads, 0, s>>>(buf, nval, plane, const_cast<long long*>(src));
  else k_r_pack<<<grid_for(nval), kRedThreads, 0, s>>>(src, nval, plane, buf);
  return cudaGetLastError();
}

}  // namespace lsqr

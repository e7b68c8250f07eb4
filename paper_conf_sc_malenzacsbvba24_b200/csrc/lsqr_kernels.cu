// lsqr_kernels.cu -- sm_100a kernels of the AVU-GSR LSQR hot path (product code; independent of oracle/).
//
// Row kernels (aprod1 / aprod2 / scale) are persistent: one 1024-thread CTA per SM, every warp owns a contiguous
// star range balanced by rows (SysView::warp_star).  A warp walks its rows 8 at a time, 4 lanes per row; lane j of
// a row group reads the row's slots by "knot": t=0 astro j, t=1..3 attitude axis t-1 knot j, t=4 instrumental j,
// t=5 {astro 4, instr 4, instr 5, global}[j].  Each of the 6 loads of a warp instruction reads 8 rows x 32
// contiguous bytes, so every fetched byte of A is used; the 4 lanes of a row hit 4 consecutive attitude columns,
// which makes the attitude gathers (aprod1) and REDs (aprod2) sector-coalesced.
#include <algorithm>
#include <cstdlib>
#include <map>
#include <mutex>
#include <type_traits>
#include <utility>

#include "lsqr_internal.cuh"

namespace lsqr {

// ------------------------------------------------------------------------------------------------ helpers
__device__ __forceinline__ double warp_sum(double v) {
#pragma unroll
  for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

// fixed-order block reduction (deterministic); result valid in thread 0
template <int NT>
__device__ __forceinline__ double block_sum(double v) {
  __shared__ double red_sh[NT / 32];
  v = warp_sum(v);
  if ((threadIdx.x & 31) == 0) red_sh[threadIdx.x >> 5] = v;
  __syncthreads();
  double r = 0.0;
  if (threadIdx.x < 32) {
    r = (threadIdx.x < NT / 32) ? red_sh[threadIdx.x] : 0.0;
    r = warp_sum(r);
  }
  __syncthreads();
  return r;
}

// ordered sum of part[0..n) by one block (thread t sums t, t+NT, ...), result in thread 0
template <int NT>
__device__ __forceinline__ double ordered_sum(const double* __restrict__ part, int64_t n) {
  double s = 0.0;
  for (int64_t i = threadIdx.x; i < n; i += NT) s += part[i];
  return block_sum<NT>(s);
}

// up to 4 ordered sums at once (one load phase, one reduction phase); results valid in thread 0
template <int NT>
__device__ __forceinline__ void ordered_sum4(const double* p0, int64_t n0, const double* p1, int64_t n1,
                                             const double* p2, int64_t n2, const double* p3, int64_t n3,
                                             double (&out)[4]) {
  double a[4] = {0.0, 0.0, 0.0, 0.0};
  for (int64_t i = threadIdx.x; i < n0; i += NT) a[0] += p0[i];
  for (int64_t i = threadIdx.x; i < n1; i += NT) a[1] += p1[i];
  for (int64_t i = threadIdx.x; i < n2; i += NT) a[2] += p2[i];
  for (int64_t i = threadIdx.x; i < n3; i += NT) a[3] += p3[i];
  __shared__ double red4[4][NT / 32];
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    const double v = warp_sum(a[q]);
    if ((threadIdx.x & 31) == 0) red4[q][threadIdx.x >> 5] = v;
  }
  __syncthreads();
  if (threadIdx.x < 32) {
#pragma unroll
    for (int q = 0; q < 4; ++q) out[q] = warp_sum(threadIdx.x < NT / 32 ? red4[q][threadIdx.x] : 0.0);
  }
  __syncthreads();
}

__device__ __forceinline__ uint32_t ic_of(const IdxRec& r, int q) {  // instrCol q (0..5), relative to I0
  uint32_t w = q < 2 ? r.ic01 : (q < 4 ? r.ic23 : r.ic45);
  return (w >> ((q & 1) * 16)) & 0xffffu;
}

// ------------------------------------------------------------------------------------------------ generator
// O-GEN (docs/GENERATOR.md): splitmix64-based counter hash; integer-only, exact int->double conversions, so the
// device arrays are bit-identical to any other implementation of the spec.
__device__ __forceinline__ uint64_t g_mix(uint64_t z) {
  z += 0x9E3779B97F4A7C15ULL;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}
__device__ __forceinline__ uint64_t g_hash(uint64_t seed, uint64_t tag, uint64_t i, uint64_t j) {
  return g_mix(g_mix(g_mix(seed ^ (tag << 56)) ^ i) ^ j);
}
__device__ __forceinline__ double g_pm1(uint64_t h) {
  return __dmul_rn(__ll2double_rn((long long)(h >> 10) - (1LL << 53)), 0x1p-53);
}

__global__ void k_generate(GenArgs g, double* __restrict__ vals, IdxRec* __restrict__ idx,
                           const int64_t* __restrict__ star_ptr, int64_t n_rows, int64_t n_stars_loc,
                           double* __restrict__ b) {
  const int64_t n_axis = g.n_att / 3, grp = g.n_instr / 6;
  const int64_t A0g = 5 * g.n_stars_global, I0g = A0g + g.n_att, G0g = I0g + g.n_instr;
  for (int64_t li = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; li < n_rows;
       li += (int64_t)gridDim.x * blockDim.x) {
    // local star: largest s with star_ptr[s] <= li
    int64_t lo = 0, hi = n_stars_loc;  // invariant star_ptr[lo] <= li < star_ptr[hi]
    while (hi - lo > 1) {
      int64_t mid = (lo + hi) >> 1;
      if (star_ptr[mid] <= li) lo = mid; else hi = mid;
    }
    const uint64_t i = (uint64_t)(g.row_begin_global + li);
    const int64_t gstar = g.star_begin_global + lo;
    const int64_t k0 = (int64_t)(g_hash(g.seed, 2, i, 0) % (uint64_t)(n_axis - 3));
    uint32_t ic[6];
#pragma unroll
    for (int j = 0; j < 6; ++j) ic[j] = (uint32_t)(j * grp + (int64_t)(g_hash(g.seed, 3, i, j) % (uint64_t)grp));
    IdxRec rec;
    rec.k0 = (int32_t)k0;
    rec.ic01 = (uint32_t)g.ip.fwd(ic[0]) | ((uint32_t)g.ip.fwd(ic[1]) << 16);
    rec.ic23 = (uint32_t)g.ip.fwd(ic[2]) | ((uint32_t)g.ip.fwd(ic[3]) << 16);
    rec.ic45 = (uint32_t)g.ip.fwd(ic[4]) | ((uint32_t)g.ip.fwd(ic[5]) << 16);
    idx[li] = rec;
    double v[kSlots];
#pragma unroll
    for (int s = 0; s < kSlots; ++s) v[s] = g_pm1(g_hash(g.seed, 4, i, s));
    if (g.n_glob == 0) v[23] = 0.0;
    double* rp = vals + li * kSlots;  // lane-major storage (position 6j + t holds slot_of(t, j))
#pragma unroll
    for (int p = 0; p < kSlots; p += 2)
      *reinterpret_cast<double2*>(rp + p) = make_double2(v[slot_of(p % 6, p / 6)], v[slot_of((p + 1) % 6, p / 6)]);
    if (g.b_mode == 0) {
      b[li] = g_pm1(g_hash(g.seed, 5, i, 0));
    } else {  // planted: b = sum_s val_s * x_true[col_s] in slot order, every op rounded (no FMA), + noise term
      double acc = 0.0;
#pragma unroll
      for (int s = 0; s < kSlots; ++s) {
        if (s == 23 && g.n_glob == 0) continue;
        int64_t col = s < 5 ? 5 * gstar + s
                            : (s < 17 ? A0g + ((s - 5) / 4) * n_axis + k0 + ((s - 5) % 4)
                                      : (s < 23 ? I0g + ic[s - 17] : G0g));
        acc = __dadd_rn(acc, __dmul_rn(v[s], g_pm1(g_hash(g.seed, 7, (uint64_t)col, 0))));
      }
      b[li] = __dadd_rn(acc, __dmul_rn(g.noise, g_pm1(g_hash(g.seed, 6, i, 0))));
    }
  }
}

// ------------------------------------------------------------------------------------------------ TMA row ring
// Every warp streams its contiguous row range through a private ring of kStages stages in shared memory.  A stage is
// kRows rows: the row values (kRows x 192 B) and index records (kRows x 16 B), fetched by two cp.async.bulk (1-D
// TMA) copies that complete on the stage's mbarrier.  Lane 0 keeps kStages-1 stages in flight while the warp
// computes on the oldest one, so the bytes in flight per SM do not depend on registers or occupancy.
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void mbar_expect_tx(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
// A is streamed exactly once per pass: its TMA copies carry an L2 evict-first policy so they do not displace the
// L2-resident shared-slice vectors (v_att/z_att: 24 MB at C4/C5) that the gathers and REDs hit.
__device__ __forceinline__ uint64_t l2_evict_first_policy() {
  uint64_t pol;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  return pol;
}
__device__ __forceinline__ void bulk_g2s(uint32_t dst, const void* src, uint32_t bytes, uint32_t bar, uint64_t pol) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::
          "r"(dst),
      "l"(src), "r"(bytes), "r"(bar), "l"(pol)
      : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
  asm volatile(
      "{\n"
      " .reg .pred p;\n"
      "WAIT_%=:\n"
      " mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      " @!p bra WAIT_%=;\n"
      "}\n" ::"r"(bar),
      "r"(parity)
      : "memory");
}

// Per-warp ring state, templated on rows per stage and ring depth.  Stage counters advance incrementally (no
// div/mod); lane 0 owns the issue pointers.
template <int ROWS, int STAGES, int NW = kWarpsPerCta>
struct RingT {
  static constexpr int kStage = ROWS * (kSlots * 8 + 16);
  static constexpr int kBytes = NW * STAGES * kStage;
  static constexpr int kBars = NW * STAGES * 8;
  const unsigned char* base;  // generic address of this warp's stage 0
  uint32_t ring, bar;         // shared addresses of stage 0 and mbarrier 0
  int64_t r_lo, r_hi, nst;    // row range and number of stages
  int slot;                   // consumer side
  uint32_t phase;
  int64_t issued;             // producer side (lane 0)
  int islot;
  const double* vsrc;
  const IdxRec* isrc;
  int64_t left;
  uint64_t pol;               // L2 evict-first policy for the streamed rows

  __device__ __forceinline__ void setup(const SysView& S, unsigned char* dsm, int wid, int lane, int64_t lo,
                                        int64_t hi) {
    base = dsm + (size_t)wid * STAGES * kStage;
    ring = smem_u32(base);
    bar = smem_u32(dsm + kBytes) + wid * STAGES * 8;
    r_lo = lo;
    r_hi = hi;
    nst = (hi - lo + ROWS - 1) / ROWS;
    slot = 0;
    phase = 0;
    issued = 0;
    islot = 0;
    vsrc = S.vals + lo * kSlots;
    isrc = S.idx + lo;
    left = hi - lo;
    pol = l2_evict_first_policy();
    if (lane == 0) {
      for (int q = 0; q < STAGES; ++q) mbar_init(bar + 8 * q, 1);
      fence_mbar_init();
    }
    __syncwarp();
  }
  __device__ __forceinline__ void issue() {  // lane 0 only
    const uint32_t n = (uint32_t)(left < ROWS ? left : ROWS);
    const uint32_t b = bar + 8 * islot, dst = ring + islot * kStage;
    mbar_expect_tx(b, n * (kSlots * 8 + 16));
    bulk_g2s(dst, vsrc, n * (kSlots * 8), b, pol);
    bulk_g2s(dst + ROWS * kSlots * 8, isrc, n * 16, b, pol);
    vsrc += ROWS * kSlots;
    isrc += ROWS;
    left -= n;
    islot = islot + 1 == STAGES ? 0 : islot + 1;
    ++issued;
  }
  __device__ __forceinline__ void prologue(int lane) {
    if (lane == 0)
      while (issued < STAGES && issued < nst) issue();
  }
  // after the warp has consumed the current stage: refill its slot with the next un-issued stage
  __device__ __forceinline__ void release(int lane) {
    __syncwarp();
    if (lane == 0 && issued < nst) {
      fence_proxy_async();
      issue();
    }
    slot = slot + 1 == STAGES ? 0 : slot + 1;
    phase ^= (slot == 0);
  }
  __device__ __forceinline__ const unsigned char* wait() const {
    mbar_wait(bar + 8 * slot, phase);
    return base + slot * kStage;
  }
  // wait for the stage d positions after the current one (software pipelining across stages; d < STAGES)
  __device__ __forceinline__ const unsigned char* wait_ahead(int d) const {
    const int s2 = slot + d >= STAGES ? slot + d - STAGES : slot + d;
    mbar_wait(bar + 8 * s2, phase ^ (slot + d >= STAGES ? 1u : 0u));
    return base + s2 * kStage;
  }
};
using Ring = RingT<kRows, kStages>;
static_assert(Ring::kBytes == kRingBytes && Ring::kBars == kBarBytes, "ring geometry");

// row lr (0..kRows-1) of a stage: the lane's 6 values and the index record (16-B broadcast within the row group)
template <int ROWS = kRows>
__device__ __forceinline__ void stage_row(const unsigned char* stg, int lr, int j, double (&v)[6], IdxRec& rec) {
  // lane-major row: the lane's 6 values are 48 contiguous bytes -> three conflict-free 16-B shared loads
  const double2* rp = reinterpret_cast<const double2*>(stg + lr * kSlots * 8 + 48 * j);
#pragma unroll
  for (int q = 0; q < 3; ++q) {
    const double2 d = rp[q];
    v[2 * q] = d.x;
    v[2 * q + 1] = d.y;
  }
  const int4 q = *reinterpret_cast<const int4*>(stg + ROWS * kSlots * 8 + lr * 16);
  rec.k0 = q.x;
  rec.ic01 = (uint32_t)q.y; rec.ic23 = (uint32_t)q.z; rec.ic45 = (uint32_t)q.w;
}

// local column of the lane's slot t (setup kernels only; the hot loops use hoisted pointers)
__device__ __forceinline__ int64_t col_of(const SysView& S, int t, int j, int64_t star, const IdxRec& r) {
  if (t == 0) return 5 * star + j;
  if (t <= 3) return S.A0 + (int64_t)(t - 1) * S.n_axis + r.k0 + j;
  if (t == 4) return S.I0 + S.ip.inv(ic_of(r, j));
  return j == 0 ? 5 * star + 4 : (j == 3 ? S.G0 : S.I0 + S.ip.inv(ic_of(r, 3 + j)));
}

// lane-local star of a row (rows are grouped by star, visited in increasing order): s / bound cached in registers
__device__ __forceinline__ bool track_star(const SysView& S, int64_t row, int64_t& s, int64_t& bound) {
  bool moved = false;
  while (bound <= row) {
    ++s;
    bound = S.star_ptr[s + 1];
    moved = true;
  }
  return moved;
}

// instrumental index of the lane's t=5 slot: lanes 1, 2 -> instr 4, 5 (lanes 0, 3 get a harmless in-range dummy)
__device__ __forceinline__ uint32_t ic5_of(const IdxRec& r, int j) { return (r.ic45 >> ((j & 2) << 3)) & 0xffffu; }
// instrumental index of the lane's t=4 slot: instr j
__device__ __forceinline__ uint32_t ic4_of(const IdxRec& r, int j) {
  const uint32_t w = (j & 2) ? r.ic23 : r.ic01;
  return (w >> ((j & 1) << 4)) & 0xffffu;
}

// Astro values of the lane's current star in registers, with the NEXT star's values prefetched one star ahead so
// a star change (every ~100-200 rows) does not stall the warp on a memory round trip.
struct AstroCache {
  double cj, c4, nj, n4;  // current / next star: x[5s+j], x[5s+4]
  int64_t s;              // current star
  __device__ __forceinline__ void init(const double* __restrict__ x, int64_t s0, int64_t s_hi, int j) {
    s = s0;
    cj = c4 = nj = n4 = 0.0;
    if (s0 < s_hi) { cj = __ldg(x + 5 * s0 + j); c4 = __ldg(x + 5 * s0 + 4); }
    if (s0 + 1 < s_hi) { nj = __ldg(x + 5 * (s0 + 1) + j); n4 = __ldg(x + 5 * (s0 + 1) + 4); }
  }
  __device__ __forceinline__ void move_to(const double* __restrict__ x, int64_t ns, int64_t s_hi, int j) {
    if (ns == s + 1) { cj = nj; c4 = n4; }
    else { cj = __ldg(x + 5 * ns + j); c4 = __ldg(x + 5 * ns + 4); }
    s = ns;
    if (ns + 1 < s_hi) { nj = __ldg(x + 5 * (ns + 1) + j); n4 = __ldg(x + 5 * (ns + 1) + 4); }
  }
};
// Shared-memory FP64 accumulation of up to N independent (address, value) pairs with interleaved CAS retries
// (sm_100a has no native shared-memory FP64 add; one CAS loop per update would serialise N round trips).
template <int N>
__device__ __forceinline__ void smem_add_n(double* const (&a)[N], const double (&val)[N], const bool (&on)[N]) {
  unsigned long long old[N];
  bool pend[N];
#pragma unroll
  for (int i = 0; i < N; ++i) {
    pend[i] = on[i];
    old[i] = pend[i] ? *reinterpret_cast<volatile unsigned long long*>(a[i]) : 0ull;
  }
  while (true) {
    bool any = false;
#pragma unroll
    for (int i = 0; i < N; ++i) {
      if (pend[i]) {
        const unsigned long long nw = __double_as_longlong(__longlong_as_double(old[i]) + val[i]);
        const unsigned long long got = atomicCAS(reinterpret_cast<unsigned long long*>(a[i]), old[i], nw);
        pend[i] = got != old[i];
        old[i] = got;
        any |= pend[i];
      }
    }
    if (!any) break;
  }
}

// a lane's three axis values of knot k from the padded knot-major gather copy: one 256-bit load (LDG.E.ENL2.256)
__device__ __forceinline__ void ldg_att4(const double* p, double& a0, double& a1, double& a2) {
  double r[4];
  asm("ld.global.nc.v4.f64 {%0, %1, %2, %3}, [%4];" : "=d"(r[0]), "=d"(r[1]), "=d"(r[2]), "=d"(r[3]) : "l"(p));
  a0 = r[0];
  a1 = r[1];
  a2 = r[2];
}

// ------------------------------------------------------------------------------------------------ aprod1
// MODE AP1_LSQR:  u_hat[i] = sum_s a_is v[col_is] - u_scale * u_hat[i];  per-warp partial of u_hat^2 (beta^2).
// MODE AP1_PLAIN: y[i] += sum_s a_is x[col_is].
// Constraint rows: per-chunk partial dots of the owned entries -> cpart (combined by k_beta / k_cdot).
// G4: the attitude values come from a padded knot-major copy of x (xg4[4k + a]): one 256-bit load per
// lane instead of three gathers.
template <int MODE, bool SMEM_INSTR, bool G4 = false>
__global__ void __launch_bounds__(kThreads, 1)
    k_aprod1(SysView S, const double* __restrict__ x, double* __restrict__ y, double* __restrict__ part,
             double* __restrict__ cpart, const DevState* __restrict__ st, const double* __restrict__ xg4) {
  extern __shared__ __align__(128) unsigned char dsm[];
  if (MODE == AP1_LSQR && st->halted) return;
  // the instrumental slice of x (<= 64 KB) is staged in shared memory: its gathers are random and L1-hostile
  double* sh_x = reinterpret_cast<double*>(dsm + kRingBytes + kBarBytes);
  if (SMEM_INSTR) {
    for (int64_t i = threadIdx.x; i < S.n_instr; i += blockDim.x) sh_x[S.ip.fwd(i)] = x[S.I0 + i];
    __syncthreads();
  }
  const int lane = threadIdx.x & 31, j = lane & 3, r = lane >> 2, wid = threadIdx.x >> 5;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t W = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const double uscale = MODE == AP1_LSQR ? st->u_scale : 0.0;
  const int64_t s_lo = S.warp_star[gw], s_hi = S.warp_star[gw + 1];
  Ring R;
  R.setup(S, dsm, wid, lane, S.star_ptr[s_lo], S.star_ptr[s_hi]);
  R.prologue(lane);
  // loop-invariant per-lane gather bases (32-bit offsets inside the loop)
  const double* xatt0 = x + S.A0 + j;
  const double* xatt1 = xatt0 + S.n_axis;
  const double* xatt2 = xatt1 + S.n_axis;
  const double* xins = SMEM_INSTR ? sh_x : x + S.I0;
  const double vglob = S.n_glob ? __ldg(x + S.G0) : 0.0;
  int64_t s = s_lo, bound = S.star_ptr[s_lo + 1];
  AstroCache ac;  // the lane's astrometric values of its current (and next) star live in registers
  ac.init(x, s_lo, s_hi, j);
  double b2 = 0.0;
  double* yp = y + R.r_lo + r;  // this lane's row in the current group
  double ynext[kGroups];
#pragma unroll
  for (int q = 0; q < kGroups; ++q) ynext[q] = (R.r_lo + q * 8 + r < R.r_hi) ? __ldg(yp + q * 8) : 0.0;
  int64_t row0 = R.r_lo;
  for (int64_t k = 0; k < R.nst; ++k, row0 += kRows, yp += kRows) {
    double ycur[kGroups];
#pragma unroll
    for (int q = 0; q < kGroups; ++q) {  // prefetch next stage's y (u_hat)
      ycur[q] = ynext[q];
      ynext[q] = (row0 + kRows + q * 8 + r < R.r_hi) ? __ldg(yp + kRows + q * 8) : 0.0;
    }
    const unsigned char* stg = R.wait();
    double v[kGroups][6], xv[kGroups][6];
    bool valid[kGroups];
#pragma unroll
    for (int q = 0; q < kGroups; ++q) {
      const int64_t row = row0 + q * 8 + r;
      valid[q] = row < R.r_hi;
      IdxRec rec;
      stage_row(stg, q * 8 + r, j, v[q], rec);
      if (valid[q] && track_star(S, row, s, bound)) ac.move_to(x, s, s_hi, j);
      // only the attitude values are gathered from global memory (L2) per row; instr from shared memory
      const int k0 = valid[q] ? rec.k0 : 0;
      xv[q][0] = ac.cj;
      if (G4) {
        ldg_att4(xg4 + S.att_kmul * (int64_t)k0 + 4 * j, xv[q][1], xv[q][2], xv[q][3]);
      } else {
        xv[q][1] = __ldg(xatt0 + k0);
        xv[q][2] = __ldg(xatt1 + k0);
        xv[q][3] = __ldg(xatt2 + k0);
      }
      const uint32_t i4 = valid[q] ? ic4_of(rec, j) : 0u, i5 = valid[q] ? ic5_of(rec, j) : 0u;
      xv[q][4] = SMEM_INSTR ? xins[i4] : __ldg(xins + i4);
      const double a_ins = SMEM_INSTR ? xins[i5] : __ldg(xins + i5);
      xv[q][5] = j == 0 ? ac.c4 : (j == 3 ? vglob : a_ins);
    }
    R.release(lane);
#pragma unroll
    for (int q = 0; q < kGroups; ++q) {
      double p = 0.0;
#pragma unroll
      for (int t = 0; t < 6; ++t) p = fma(v[q][t], xv[q][t], p);
      p += __shfl_xor_sync(0xffffffffu, p, 1);
      p += __shfl_xor_sync(0xffffffffu, p, 2);
      if (valid[q] && j == 0) {
        if (MODE == AP1_LSQR) {
          const double un = p - uscale * ycur[q];
          yp[q * 8] = un;
          b2 = fma(un, un, b2);
        } else {
          yp[q * 8] = ycur[q] + p;
        }
      }
    }
  }
  if (MODE == AP1_LSQR) {
    b2 = warp_sum(b2);
    if (lane == 0) part[gw] = b2;
  }
  // constraint rows: owned-entry partial dots, chunk by chunk
  for (int64_t c = gw; c < S.n_chunks; c += W) {
    double acc = 0.0;
    for (int64_t e = S.ch_beg[c] + lane; e < S.ch_end[c]; e += 32) acc = fma(S.cval[e], __ldg(x + S.ccol[e]), acc);
    acc = warp_sum(acc);
    if (lane == 0) cpart[c] = acc;
  }
}

// ------------------------------------------------------------------------------------------------ aprod2
// z = A^T y, scatter-free on the astrometric block (one warp owns whole stars, so the 5 astro sums of a star are
// a warp reduction), hierarchical on the shared slice: attitude -> sector-coalesced FP64 REDs into
// the L2-resident z_sh (P:L427-434 uses atomics), instrumental -> CTA-private shared-memory accumulator flushed
// once per CTA, global -> register + warp shuffle, one RED per warp.
//   MODE AP2_LSQR:    y = u_hat * inv_beta; astro: v[c] = z + constr - beta v[c] (v' of Paige-Saunders, unnormalised),
//                     per-warp partial of v'^2 (alpha^2, astro part).  Shared slice left in zsh (vshared finishes).
//   MODE AP2_PLAIN:   astro: x[c] += z (+ constraint entries with y_c); shared slice accumulated in zsh.
//   MODE AP2_COLNORM: contributions a^2 (column sums of squares, O-PREC); astro: c[c] = z; shared in zsh.
template <int MODE, bool SMEM_INSTR>
__global__ void __launch_bounds__(kThreads, 1)
    k_aprod2(SysView S, const double* __restrict__ yv, const double* __restrict__ ucn, double* __restrict__ xv,
             double* __restrict__ zsh, double* __restrict__ part, const DevState* __restrict__ st,
             int do_shared_constr) {
  extern __shared__ __align__(128) unsigned char dsm[];
  if (MODE == AP2_LSQR && (st->halted || !st->beta_pos)) return;
  double* sh_instr = reinterpret_cast<double*>(dsm + kRingBytes + kBarBytes);
  if (SMEM_INSTR) {
    for (int64_t i = threadIdx.x; i < S.ip.slots(); i += blockDim.x) sh_instr[i] = 0.0;
    __syncthreads();
  }
  const int lane = threadIdx.x & 31, j = lane & 3, r = lane >> 2, wid = threadIdx.x >> 5;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t W = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const double inv_beta = MODE == AP2_LSQR ? st->inv_beta : 1.0;
  const double beta = MODE == AP2_LSQR ? st->beta : 0.0;
  const int64_t s_lo = S.warp_star[gw], s_hi = S.warp_star[gw + 1];
  Ring R;
  R.setup(S, dsm, wid, lane, S.star_ptr[s_lo], S.star_ptr[s_hi]);
  R.prologue(lane);
  const bool glob_ok = S.n_glob != 0;
  double* zatt0 = zsh + j;
  double* zatt1 = zatt0 + S.n_axis;
  double* zatt2 = zatt1 + S.n_axis;
  double* z_ins = SMEM_INSTR ? sh_instr : zsh + S.n_att;
  double gacc = 0.0, a2 = 0.0, acc0 = 0.0, acc1 = 0.0;
  int64_t s = s_lo, bound = S.star_ptr[s_lo + 1];  // lane-local star of the lane's row
  int64_t cs = s_lo;                                // warp-uniform star being accumulated
  int64_t cs_end = (cs < s_hi) ? S.star_ptr[cs + 1] : 0;
  // old astro values of star cs, loaded when cs becomes current so the finalize does not wait on memory
  double xo_j = 0.0, xo_4 = 0.0;
  auto prefetch_old = [&](int64_t star) {
    if (MODE != AP2_COLNORM && star < s_hi && lane < 4) {
      xo_j = xv[5 * star + j];
      xo_4 = xv[5 * star + 4];
    }
  };
  prefetch_old(cs);

  auto finalize = [&](int64_t star) {
    double z0 = acc0, z1 = acc1;
    z0 += __shfl_xor_sync(0xffffffffu, z0, 4);
    z0 += __shfl_xor_sync(0xffffffffu, z0, 8);
    z0 += __shfl_xor_sync(0xffffffffu, z0, 16);
    z1 += __shfl_xor_sync(0xffffffffu, z1, 4);
    z1 += __shfl_xor_sync(0xffffffffu, z1, 8);
    z1 += __shfl_xor_sync(0xffffffffu, z1, 16);
    if (lane < 4) {
      if (star < S.n_cs) {  // constraint entries on this star's astro columns (after all rows, as O-AP2)
        const int64_t c0 = 5 * star + j;
        for (int64_t e = S.cs_ptr[c0]; e < S.cs_ptr[c0 + 1]; ++e) {
          const double cv = S.cval[S.cs_e[e]];
          z0 += MODE == AP2_COLNORM ? cv * cv : cv * ucn[S.cs_k[e]];
        }
        if (j == 0)
          for (int64_t e = S.cs_ptr[5 * star + 4]; e < S.cs_ptr[5 * star + 5]; ++e) {
            const double cv = S.cval[S.cs_e[e]];
            z1 += MODE == AP2_COLNORM ? cv * cv : cv * ucn[S.cs_k[e]];
          }
      }
      double* xc = xv + 5 * star;
      if (MODE == AP2_LSQR) {
        const double vn = z0 - beta * xo_j;
        xc[j] = vn;
        a2 = fma(vn, vn, a2);
        if (j == 0) {
          const double vn1 = z1 - beta * xo_4;
          xc[4] = vn1;
          a2 = fma(vn1, vn1, a2);
        }
      } else if (MODE == AP2_PLAIN) {
        xc[j] = xo_j + z0;
        if (j == 0) xc[4] = xo_4 + z1;
      } else {
        xc[j] = z0;
        if (j == 0) xc[4] = z1;
      }
    }
  };

  const double* ysrc = MODE == AP2_COLNORM ? nullptr : yv;
  const double* yp = ysrc ? ysrc + R.r_lo + r : nullptr;
  double ynext[kGroups];
#pragma unroll
  for (int q = 0; q < kGroups; ++q) ynext[q] = (ysrc && R.r_lo + q * 8 + r < R.r_hi) ? __ldg(yp + q * 8) : 0.0;
  int64_t row0 = R.r_lo;
  for (int64_t k = 0; k < R.nst; ++k, row0 += kRows) {
    double ycur[kGroups];
#pragma unroll
    for (int q = 0; q < kGroups; ++q) {
      ycur[q] = ynext[q];
      ynext[q] = (ysrc && row0 + kRows + q * 8 + r < R.r_hi) ? __ldg(yp + kRows + q * 8) : 0.0;
    }
    if (ysrc) yp += kRows;
    const unsigned char* stg = R.wait();
    double* ia[2 * kGroups];
    double iv[2 * kGroups];
    bool ion[2 * kGroups];
#pragma unroll
    for (int i = 0; i < 2 * kGroups; ++i) { ia[i] = z_ins; iv[i] = 0.0; ion[i] = false; }
#pragma unroll
    for (int q = 0; q < kGroups; ++q) {
      const int64_t base = row0 + q * 8;
      const int64_t row = base + r;
      const bool valid = row < R.r_hi;
      double v[6];
      IdxRec rec;
      stage_row(stg, q * 8 + r, j, v, rec);
      double c[6];
      const double yr = MODE == AP2_LSQR ? ycur[q] * inv_beta : ycur[q];
#pragma unroll
      for (int t = 0; t < 6; ++t) c[t] = MODE == AP2_COLNORM ? v[t] * v[t] : v[t] * yr;
      if (valid) {
        track_star(S, row, s, bound);
        // attitude: 3 axes x 4 consecutive knots -> sector-coalesced REDs (one per axis per lane)
        const int k0 = rec.k0;
        atomicAdd(zatt0 + k0, c[1]);
        atomicAdd(zatt1 + k0, c[2]);
        atomicAdd(zatt2 + k0, c[3]);
        // instrumental: collected for the whole stage, accumulated below with interleaved CAS (smem path)
        if (SMEM_INSTR) {
          ia[2 * q] = z_ins + ic4_of(rec, j);
          iv[2 * q] = c[4];
          ion[2 * q] = true;
          ia[2 * q + 1] = z_ins + ic5_of(rec, j);
          iv[2 * q + 1] = c[5];
          ion[2 * q + 1] = (j == 1 || j == 2);
        } else {
          atomicAdd(z_ins + ic4_of(rec, j), c[4]);
          if (j == 1 || j == 2) atomicAdd(z_ins + ic5_of(rec, j), c[5]);
        }
        if (j == 3) gacc += c[5];
      }
      // astrometric: segmented by star (rows are grouped by star)
      const double c0 = c[0], c5 = (j == 0) ? c[5] : 0.0;
      if (base < R.r_hi) {
        const int64_t step_end = base + 8 < R.r_hi ? base + 8 : R.r_hi;
        while (true) {
          if (valid && s == cs) { acc0 += c0; acc1 += c5; }
          if (cs < s_hi && cs_end <= step_end) {
            finalize(cs);
            acc0 = 0.0; acc1 = 0.0;
            ++cs;
            if (cs >= s_hi) break;
            cs_end = S.star_ptr[cs + 1];
            prefetch_old(cs);
          } else {
            break;
          }
        }
      }
    }
    if (SMEM_INSTR) smem_add_n<2 * kGroups>(ia, iv, ion);
    R.release(lane);
  }
  while (cs < s_hi) {  // empty trailing stars
    acc0 = 0.0; acc1 = 0.0;
    finalize(cs);
    ++cs;
    prefetch_old(cs);
  }
  // global column: one RED per warp
  if (glob_ok) {
    gacc = warp_sum(gacc);
    if (lane == 0 && gacc != 0.0) atomicAdd(zsh + S.n_att + S.n_instr, gacc);
  }
  if (MODE == AP2_LSQR) {
    a2 = warp_sum(a2);
    if (lane == 0) part[gw] = a2;
  }
  // constraint entries on shared columns (owned by rank 0 only; the host passes n_csh = 0 elsewhere)
  if (do_shared_constr) {
    for (int64_t e = gw * 32 + lane; e < S.n_csh; e += W * 32) {
      const double cv = S.cval[S.csh_e[e]];
      const double c = MODE == AP2_COLNORM ? cv * cv : cv * ucn[S.csh_k[e]];
      atomicAdd(zsh + S.csh_idx[e], c);
    }
  }
  if (SMEM_INSTR) {
    __syncthreads();
    for (int64_t i = threadIdx.x; i < S.n_instr; i += blockDim.x) {
      const double v = sh_instr[S.ip.fwd(i)];
      if (v != 0.0) atomicAdd(zsh + S.n_att + i, v);
    }
  }
}


// ------------------------------------------------------------------------------------------------ fused pass
// NEXT-1: one pass over the rows per iteration.  For each row
//     u_hat_i = a_i . v - u_scale * u_hat_i          (aprod1, Paige-Saunders step a)
//     z      += a_i^T u_hat_i                         (aprod2 with the UNNORMALISED new u; beta is not known yet)
// so A is read once (224 B/row instead of 440).  Afterwards (k_vastro, k_vshared) v' = z/beta - beta v, which is
// algebraically the P&S step b (u = u_hat/beta).  Astro z goes to zA (scatter-free, per star), the shared slice to
// z_sh exactly as in aprod2.  The ring is shallower (8-row stages) because v_instr (gathers) and z_instr
// (accumulator) both live in shared memory.
constexpr int kFRows = 8;
using FRing = RingT<kFRows, kFStages, kFWarps>;
constexpr int kSmemMaxBytes = 232448;  // 227 KB opt-in per CTA on sm_100

// k_fused3 (the third version of this kernel; DESIGN.md §7 has the history) has a hot loop written for issue
// efficiency -- the kernel is bound by the SM's issue slots and L1 data pipe, not by HBM:
//   * the loop is unrolled by two so the gather prefetch (group k+1) and the u_hat register queue alternate between
//     two register sets instead of being copied every group;
//   * the ring's shared memory is zeroed at entry, so the index records of rows past the end of a warp's range are
//     always in range (stale rows of the warp or zeros) and the gathers need no validity selects;
//   * the astro slot-4 (lane 0), instrumental-5 (lanes 1, 2) and global (lane 3) contributions of slot t=5 share one
//     accumulator `acc5`, folded per star (lane 0: zA, lane 3: global sum; lanes 1, 2 discard theirs);
//   * shared-memory FP64 accumulation of the instrumental slice uses the compiler's CAS-spin loop (ATOMS.CAST.SPIN;
//     measured faster than an explicit atom.cas loop);
//   * one proxy fence per two stages: lane 0 re-fills two released slots after one fence.async (generic-proxy reads
//     of a slot before the async-proxy TMA write into it; without the fence the full-size C2 parity test fails).
//
// The same loop, templated on KIND, is also the two-pass iteration's aprod2 (the paper's structure: A read twice per
// iteration):
//   R3_FUSED: u_hat_i = a_i . v - u_scale u_hat_i, then z += a_i^T u_hat_i  (NEXT-1, the default iteration);
//   R3_AP2:   z += a_i^T u_hat_i only, on the unnormalised u_hat k_aprod1 wrote (astro z -> zA, shared -> z_sh).
// k_aprod1<AP1_LSQR> followed by k_fused3<R3_AP2> leaves the state k_fused3<R3_FUSED> leaves, so k_post / k_vastro /
// k_vshared finish the iteration unchanged (v' = z / beta - beta v).  (An aprod1 on this loop measured slower than
// k_aprod1's deeper 16-row ring: C3 11.5 vs 10.5 ms.)
enum { R3_FUSED = 0, R3_AP2 = 2 };

#ifndef LSQR_IDX32
#define LSQR_IDX32 0    // index record as one 4-B shared load per lane + quad shuffles (A/B: 1.5-2.5 % slower at C2)
#endif
#ifndef LSQR_T5PRED
#define LSQR_T5PRED 1   // slot t=5 gathers only on the instrumental lanes (1, 2); v_glob from a register (lane 3)
#endif
#ifndef LSQR_GATHER4
#define LSQR_GATHER4 1  // attitude gathers: one 32-B load per lane from the padded knot-major copy xatt4 (A/B: 0)
#endif



constexpr int kF3Stage = kFRows * (kSlots * 8 + 16);  // 1664 B: 8 rows of values + 8 index records
constexpr int kF3Bars = kFWarps * kFStages * 8;          // per stage: "full" mbarrier (TMA bytes)
constexpr int kF3InstrMax = (kSmemMaxBytes - FRing::kBytes - kF3Bars - 1024) / 16 - 2;

// Shared-slice regimes (SURVEY §8(d) sensitivity sweep): `zrep` copies of the CTA's z_instr accumulator (warp w
// adds into copy w % zrep; more copies when the instrumental slice is small, fewer same-address CAS collisions);
// SMATT: the attitude slice is small too (n_att <= kSmAttMax), so z_att is accumulated in `arep` shared-memory
// copies (CAS) instead of L2 REDs, which serialise on few addresses.  Copies are summed once per CTA at the end.
// IG: the instrumental slice is too large for shared memory: its gathers go through L1/L2 (__ldg) and its
// contributions are L2 REDs (IdxRec then holds plain column offsets).  ZREP: zrep > 1 (a separate instantiation:
// in the one-copy case the runtime copy index changed the schedule and measured 2-4 % slower).
template <int KIND = R3_FUSED, int DIAG = 0, bool SMATT = false, bool IG = false, bool ZREP = false>
__global__ void __launch_bounds__(kFWarps * 32, 1)
    k_fused3(SysView S, const double* __restrict__ x, double* __restrict__ u, double* __restrict__ zA,
             double* __restrict__ zsh, double* __restrict__ part, double* __restrict__ cpart,
             const DevState* __restrict__ st) {
  extern __shared__ __align__(128) unsigned char dsm[];
  const int zrep = S.f3_zrep, arep = S.f3_arep;
  if (st->halted) return;
  constexpr bool kDot = KIND == R3_FUSED;  // computes the new u_hat (gathers, row dot, store, beta^2)
  // shared memory: [ring | mbarriers | v_instr (slots) + v_glob | zrep x z_instr | arep x z_att (SMATT)]
  const int64_t nsl = IG ? 0 : S.ip.slots(), zstride = IG ? 0 : nsl + 2;
  double* sh_x = reinterpret_cast<double*>(dsm + FRing::kBytes + kF3Bars);
  double* sh_z = IG ? sh_x : sh_x + nsl + 2;  // IG: no instrumental arrays, z_att copies (SMATT) start here
  double* sh_za = sh_z + zrep * zstride;
  for (int i = threadIdx.x; i < FRing::kBytes / 16; i += blockDim.x)
    reinterpret_cast<int4*>(dsm)[i] = make_int4(0, 0, 0, 0);
  constexpr bool kPlain = !SMATT && !IG && !ZREP;  // the C2-C5 regime (code kept as measured)
  if (kPlain) {
    for (int64_t i = threadIdx.x; i < nsl; i += blockDim.x) {
      sh_x[i] = 0.0;
      sh_z[i] = 0.0;
    }
  } else {
    for (int64_t i = threadIdx.x; i < zstride * (1 + zrep) + (SMATT ? arep * S.n_att : 0); i += blockDim.x)
      sh_x[i] = 0.0;
  }
  __syncthreads();
  if (kDot && !IG) {
    for (int64_t i = threadIdx.x; i < S.n_instr; i += blockDim.x) sh_x[S.ip.fwd(i)] = x[S.I0 + i];
    if (threadIdx.x == 0) sh_x[nsl] = S.n_glob ? x[S.G0] : 0.0;
  }
  const int lane = threadIdx.x & 31, j = lane & 3, r = lane >> 2, wid = threadIdx.x >> 5;
  const uint32_t ring = smem_u32(dsm) + wid * kFStages * kF3Stage;
  const uint32_t bar = smem_u32(dsm + FRing::kBytes) + wid * kFStages * 8;
  if (lane == 0) {
    for (int q = 0; q < kFStages; ++q) mbar_init(bar + 8 * q, 1);
    fence_mbar_init();
  }
  __syncthreads();  // ring zeroed (generic writes) before any TMA lands; v_instr staged
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t W = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const double uscale = st->u_scale;
  const int64_t s_lo = S.warp_star_f[gw], s_hi = S.warp_star_f[gw + 1];
  const int64_t r_lo = S.star_ptr[s_lo];
  const int nrows = (int)(S.star_ptr[s_hi] - r_lo);  // rows of this warp (< 2^31)
  const int nst = (nrows + kFRows - 1) / kFRows;

  // producer state (lane 0): stage q goes to slot q % kFStages, issued when the warp releases stage q - kFStages
  const double* vsrc = S.vals + r_lo * kSlots;
  const IdxRec* isrc = S.idx + r_lo;
  int left = nrows;
  const uint64_t pol = l2_evict_first_policy();
  auto issue = [&](int slot) {
    const uint32_t n = (uint32_t)(left < kFRows ? left : kFRows);
    const uint32_t b = bar + 8 * slot, dst = ring + slot * kF3Stage;
    mbar_expect_tx(b, n * (kSlots * 8 + 16));
    bulk_g2s(dst, vsrc, n * (kSlots * 8), b, pol);
    bulk_g2s(dst + kFRows * kSlots * 8, isrc, n * 16, b, pol);
    vsrc += kFRows * kSlots;
    isrc += kFRows;
    left -= (int)n;
  };
  if (lane == 0) {
    fence_proxy_async();  // the zeroing stores above precede the TMA writes into the ring
    for (int q = 0; q < kFStages && q < nst; ++q) issue(q);
  }

  const unsigned char* ringp = dsm + wid * kFStages * kF3Stage;
  const int voff = r * kSlots * 8 + 48 * j, ioff = kFRows * kSlots * 8 + r * 16;
#if LSQR_GATHER4
  const double* const xg4 = S.xatt4 + 4 * j;  // lane j gathers knot k0 + j (its three axis values, one load)
  const int gmul = S.att_kmul;                  // 4: knot format, 16: window format (one 128-B line per row)
#else
  const double* xatt0 = x + S.A0 + j;
  const double* xatt1 = xatt0 + S.n_axis;
  const double* xatt2 = xatt1 + S.n_axis;
#endif
  // attitude accumulator: axis-major z_att (lane j -> knot k0 + j of axis a), or, when S.z4 is set, the window
  // accumulator (folded by k_post, or into z_sh by k_att_fold): z4[k0][a][j] (z4_kmul = 16: a row's 12 REDs in one aligned 128-B
  // line) or z4[a][k0][j] (z4_kmul = 4: one aligned 32-B sector per row and axis)
  const bool z4 = !SMATT && S.z4 != nullptr;
  const int kmul = z4 ? S.z4_kmul : 1;
  const int64_t astride = !z4 ? S.n_axis : (kmul == 16 ? 4 : 4 * S.n_axis);
  double* zatt0 = (SMATT ? sh_za + (wid % arep) * S.n_att : (z4 ? S.z4 : zsh)) + j;
  double* zatt1 = zatt0 + astride;
  double* zatt2 = zatt1 + astride;
  double* const sh_zw = ZREP ? sh_z + (wid % zrep) * zstride : sh_z;  // this warp's z_instr copy
  const bool t5_ins = (j == 1 || j == 2);  // t=5 slot: lane 0 astro 4, lanes 1, 2 instr 4, 5, lane 3 global
  const int i5_shift = (j & 2) << 3;
  // lane 3 gathers v_glob (slot nsl; IG: column G0 = I0 + n_instr, which exists iff n_glob); lane 0 ignores its g5
  const uint32_t i5_or = (j == 3) ? (IG ? (S.n_glob ? (uint32_t)S.n_instr : 0u) : (uint32_t)nsl) : 0u;
  const double* const xins = x + S.I0;
  const double vglob_r = (kDot && S.n_glob) ? __ldg(x + S.G0) : 0.0;
  const int i4_shift = (j & 1) << 4;
  double* const urow = u + r_lo + r;

  // warp-uniform star state: cs = star of the next row to process; its astro values (cj, c4) and the next star's
  int64_t cs = s_lo;
  int cs_end = (cs < s_hi) ? (int)(S.star_ptr[cs + 1] - r_lo) : nrows;
  double cj = 0.0, c4 = 0.0, nj = 0.0, n4 = 0.0;
  if (kDot && cs < s_hi) { cj = __ldg(x + 5 * cs + j); c4 = __ldg(x + 5 * cs + 4); }
  if (kDot && cs + 1 < s_hi) { nj = __ldg(x + 5 * (cs + 1) + j); n4 = __ldg(x + 5 * (cs + 1) + 4); }
  double b2 = 0.0, gacc = 0.0, acc0 = 0.0, acc5 = 0.0;

  auto advance = [&]() {  // star cs is complete: its 5 astro sums -> zA (scatter-free), move to cs+1
    {
      double z0 = acc0, z1 = acc5;
      gacc += acc5;  // lane 3: global contributions of the star (lanes 0-2: unused)
      z0 += __shfl_xor_sync(0xffffffffu, z0, 4);
      z1 += __shfl_xor_sync(0xffffffffu, z1, 4);
      z0 += __shfl_xor_sync(0xffffffffu, z0, 8);
      z1 += __shfl_xor_sync(0xffffffffu, z1, 8);
      z0 += __shfl_xor_sync(0xffffffffu, z0, 16);
      z1 += __shfl_xor_sync(0xffffffffu, z1, 16);
      if (lane < 4) {
        zA[5 * cs + j] = z0;
        if (j == 0) zA[5 * cs + 4] = z1;
      }
      acc0 = 0.0;
      acc5 = 0.0;
    }
    ++cs;
    cs_end = (cs < s_hi) ? (int)(S.star_ptr[cs + 1] - r_lo) : nrows;
    if (kDot) {
      cj = nj;
      c4 = n4;
      if (cs + 1 < s_hi) { nj = __ldg(x + 5 * (cs + 1) + j); n4 = __ldg(x + 5 * (cs + 1) + 4); }
    }
  };
  while (cs < s_hi && cs_end <= 0) advance();  // leading empty stars

  struct Pre {
    double g1, g2, g3, g4, g5;
    int k0;
    uint32_t i4, i5;
  };
  // gathers of stage q (slot sl): attitude from L2, instrumental from shared memory
  auto prefetch = [&](int q, int sl, Pre& P) {
    mbar_wait(bar + 8 * sl, (uint32_t)(q >> 2) & 1u);
    static_assert(kFStages == 4, "parity uses q / 4");
#if LSQR_IDX32
    // lane j of a row reads word j of the row's 16-B record (k0, ic01, ic23, ic45): one conflict-free 128-B
    // wavefront per group; the quad exchanges the words it needs
    const uint32_t wj = *reinterpret_cast<const uint32_t*>(ringp + sl * kF3Stage + ioff + 4 * j);
    const int qb = lane & ~3;
    P.k0 = __shfl_sync(0xffffffffu, (int)wj, qb);
    const uint32_t w4 = __shfl_sync(0xffffffffu, wj, qb + 1 + (j >> 1));
    const uint32_t w5 = __shfl_sync(0xffffffffu, wj, qb + 3);
    P.i4 = (w4 >> i4_shift) & 0xffffu;
    P.i5 = t5_ins ? ((w5 >> i5_shift) & 0xffffu) : i5_or;
#else
    const int4 rec = *reinterpret_cast<const int4*>(ringp + sl * kF3Stage + ioff);
    P.k0 = rec.x;
    P.i4 = ((uint32_t)((j & 2) ? rec.z : rec.y) >> i4_shift) & 0xffffu;
    P.i5 = t5_ins ? (((uint32_t)rec.w >> i5_shift) & 0xffffu) : i5_or;
#endif
    if (kDot) {
      if (DIAG & 4) {
        P.g1 = P.g2 = P.g3 = 0.5;
      } else {
#if LSQR_GATHER4
        ldg_att4(xg4 + gmul * (int64_t)P.k0, P.g1, P.g2, P.g3);
#else
        P.g1 = __ldg(xatt0 + P.k0);
        P.g2 = __ldg(xatt1 + P.k0);
        P.g3 = __ldg(xatt2 + P.k0);
#endif
      }
      P.g4 = (DIAG & 8) ? 0.5 : (IG ? __ldg(xins + P.i4) : sh_x[P.i4]);
#if LSQR_T5PRED
      if (DIAG & 8) P.g5 = 0.5;
      else if (t5_ins) P.g5 = IG ? __ldg(xins + P.i5) : sh_x[P.i5];
      else P.g5 = vglob_r;  // lane 3: v_glob; lane 0 uses the astro value instead
#else
      P.g5 = (DIAG & 8) ? 0.5 : (IG ? __ldg(xins + P.i5) : sh_x[P.i5]);
#endif
    }
  };

  // one 8-row group.  CHECK: tail / star-boundary path with per-lane validity and per-lane star; otherwise every
  // lane's row is valid and in star cs.
  auto group = [&](const double (&v)[6], const Pre& P, int g0, double uold, auto check_tag) {
    constexpr bool CHECK = decltype(check_tag)::value;
    const int rel = g0 + r;
    const bool valid = !CHECK || rel < nrows;
    double xj = cj, x4 = c4;
    int64_t my_s = cs;
    if (CHECK && valid) {
      int my_end = cs_end;
      while (my_end <= rel) {
        ++my_s;
        my_end = (int)(S.star_ptr[my_s + 1] - r_lo);
      }
      if (kDot) {
        if (my_s == cs + 1) { xj = nj; x4 = n4; }
        else if (my_s != cs) { xj = __ldg(x + 5 * my_s + j); x4 = __ldg(x + 5 * my_s + 4); }
      }
    }
    double un;
    if (kDot) {
      const double g5 = (j == 0) ? x4 : P.g5;
      double p = fma(v[1], P.g1, v[0] * xj);  // two short chains instead of one long one
      double p2 = fma(v[4], P.g4, v[3] * P.g3);
      p = fma(v[2], P.g2, p);
      p2 = fma(v[5], g5, p2);
      p += p2;
      p += __shfl_xor_sync(0xffffffffu, p, 1);
      p += __shfl_xor_sync(0xffffffffu, p, 2);
      un = valid ? fma(-uscale, uold, p) : 0.0;  // identical in the row's 4 lanes
      if (j == 0 && valid) {
        __stcs(urow + g0, un);
        b2 = fma(un, un, b2);
      }
    } else {
      un = valid ? uold : 0.0;  // aprod2: the u_hat aprod1 wrote
    }
    const double c1 = v[1] * un, c2 = v[2] * un, c3 = v[3] * un, c4v = v[4] * un, c5 = v[5] * un;
    if (valid && !(DIAG & 2)) {  // per axis, the 4 lanes of a row hit one 32-B window (z4: one aligned sector)
      const int ko = kmul * P.k0;
      atomicAdd(zatt0 + ko, c1);
      atomicAdd(zatt1 + ko, c2);
      atomicAdd(zatt2 + ko, c3);
    }
    if (valid && !(DIAG & 1)) {
      double* const zi = IG ? zsh + S.n_att : sh_zw;
      atomicAdd(zi + P.i4, c4v);
      if (t5_ins) atomicAdd(zi + P.i5, c5);
    }
    if (!CHECK) {
      acc0 = fma(v[0], un, acc0);
      acc5 += c5;
    } else {  // segmented by star inside the group
      const double c0 = v[0] * un;
      const int g1end = g0 + kFRows < nrows ? g0 + kFRows : nrows;
      while (true) {
        if (valid && my_s == cs) { acc0 += c0; acc5 += c5; }
        if (cs < s_hi && cs_end <= g1end) advance();
        else break;
      }
    }
  };

  // one stage: prefetch the next stage's gathers, take this stage's values into registers, hand the slot back to
  // the TMA (lane 0 refills it with stage k + kFStages), compute
  auto step = [&](int k, int sl, int sln, const Pre& Pc, Pre& Pn, double& uq) {
    const int g0 = k * kFRows;
    if (k + 1 < nst) prefetch(k + 1, sln, Pn);
    const unsigned char* stg = ringp + sl * kF3Stage;
    double v[6];
    if (DIAG & 16) {  // experiment: no stage value reads (the LSU cost of staging A through shared memory)
#pragma unroll
      for (int t = 0; t < 6; ++t) v[t] = 0.125 * (t + 1);
    } else {
      const double2* rp = reinterpret_cast<const double2*>(stg + voff);
#pragma unroll
      for (int qq = 0; qq < 3; ++qq) {
        const double2 d = rp[qq];
        v[2 * qq] = d.x;
        v[2 * qq + 1] = d.y;
      }
    }
    // Refill: at every odd stage the slots of stages k-1 and k get stages k+3 and k+4 (one proxy fence per two
    // stages).  The fence (generic-proxy reads of the slot -> async-proxy TMA writes into it) is required: without
    // it, or with an intra-warp mbarrier hand-off instead, the full-size C2 parity test fails (x off by ~1e-4).
    auto release = [&]() {
      if (k & 1) {
        __syncwarp();
        if (lane == 0 && k + kFStages - 1 < nst) {
          fence_proxy_async();
          issue((sl + kFStages - 1) & (kFStages - 1));
          if (k + kFStages < nst) issue(sl);
        }
      }
    };
    double uold = uq;
    uq = (g0 + 2 * kFRows + r < nrows) ? __ldcs(urow + g0 + 2 * kFRows) : 0.0;  // u_hat two stages ahead
    if ((g0 + kFRows <= nrows) && (cs_end >= g0 + kFRows)) {
      release();
      group(v, Pc, g0, uold, std::false_type{});
      while (cs < s_hi && cs_end <= g0 + kFRows) advance();
    } else {
      if (g0 + r >= nrows) {
#pragma unroll
        for (int t = 0; t < 6; ++t) v[t] = 0.0;
        uold = 0.0;
      }
      release();
      group(v, Pc, g0, uold, std::true_type{});
    }
  };

  double uqa = (r < nrows) ? __ldcs(urow) : 0.0;                   // u_hat of even stages
  double uqb = (kFRows + r < nrows) ? __ldcs(urow + kFRows) : 0.0;  // u_hat of odd stages
  Pre PA{}, PB{};
  if (nst > 0) prefetch(0, 0, PA);
  int k = 0;
  for (; k + 1 < nst; k += 2) {
    const int sl = k & (kFStages - 1);
    step(k, sl, sl + 1, PA, PB, uqa);
    step(k + 1, sl + 1, (sl + 2) & (kFStages - 1), PB, PA, uqb);
  }
  if (k < nst) step(k, k & (kFStages - 1), (k + 1) & (kFStages - 1), PA, PB, uqa);
  while (cs < s_hi) advance();  // empty trailing stars
  if (S.n_glob) {
    gacc = warp_sum(j == 3 ? gacc : 0.0);
    if (lane == 0 && gacc != 0.0) atomicAdd(zsh + S.n_att + S.n_instr, gacc);
  }
  // beta^2: one partial per CTA (warps combined in a fixed order -> deterministic), so k_post re-sums few values
  __shared__ double b2w[kFWarps];
  if (kDot) {
    b2 = warp_sum(b2);
    if (lane == 0) b2w[wid] = b2;
    for (int64_t c = gw; c < S.n_chunks; c += W) {  // constraint rows: owned-entry partial dots with v
      double acc = 0.0;
      for (int64_t e = S.ch_beg[c] + lane; e < S.ch_end[c]; e += 32) acc = fma(S.cval[e], __ldg(x + S.ccol[e]), acc);
      acc = warp_sum(acc);
      if (lane == 0) cpart[c] = acc;
    }
  }
  __syncthreads();
  if (kDot && threadIdx.x == 0) {
    double t = 0.0;
    for (int q = 0; q < kFWarps; ++q) t += b2w[q];
    part[blockIdx.x] = t;
  }
  if (kPlain) {
    for (int64_t i = threadIdx.x; i < S.n_instr; i += blockDim.x) {
      const double vv = sh_z[S.ip.fwd(i)];
      if (vv != 0.0) atomicAdd(zsh + S.n_att + i, vv);
    }
  } else if (!IG) {
    for (int64_t i = threadIdx.x; i < S.n_instr; i += blockDim.x) {
      const int64_t q = S.ip.fwd(i);
      double vv = 0.0;
      for (int c = 0; c < zrep; ++c) vv += sh_z[c * zstride + q];
      if (vv != 0.0) atomicAdd(zsh + S.n_att + i, vv);
    }
  }
  if (SMATT)
    for (int64_t i = threadIdx.x; i < S.n_att; i += blockDim.x) {
      double vv = 0.0;
      for (int c = 0; c < arep; ++c) vv += sh_za[c * S.n_att + i];
      if (vv != 0.0) atomicAdd(zsh + i, vv);
    }
}

// Fused mode, after k_beta: astro columns v' = (zA + constraint entries . u_hat_c) / beta - beta v  (P&S step b),
// per-block alpha^2 partials; shared-column constraint entries added to z_sh (rank 0) before AR2 / k_vshared.
__global__ void __launch_bounds__(kRedThreads)
    k_vastro(SysView S, double* __restrict__ v, const double* __restrict__ zA, const double* __restrict__ uc,
             double* __restrict__ zsh, double* __restrict__ part, const DevState* __restrict__ st,
             int do_shared_constr) {
  if (st->halted || !st->beta_pos) return;
  const double ib = st->inv_beta, beta = st->beta;
  const int64_t na = 5 * S.n_stars;
  double a2 = 0.0;
  for (int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; c < na; c += (int64_t)gridDim.x * blockDim.x) {
    double z = zA[c];
    if (c < 5 * S.n_cs)
      for (int64_t e = S.cs_ptr[c]; e < S.cs_ptr[c + 1]; ++e) z += S.cval[S.cs_e[e]] * uc[S.cs_k[e]];
    const double vn = z * ib - beta * v[c];
    v[c] = vn;
    a2 = fma(vn, vn, a2);
  }
  a2 = block_sum<kRedThreads>(a2);
  if (threadIdx.x == 0) part[blockIdx.x] = a2;
  if (do_shared_constr)
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < S.n_csh;
         e += (int64_t)gridDim.x * blockDim.x)
      atomicAdd(zsh + S.csh_idx[e], S.cval[S.csh_e[e]] * uc[S.csh_k[e]]);
}


// z4 -> z_sh: z_att[a][k] += sum_j z4(w = k - j, a, j) (windows w in [0, n_axis - 4]); every z4 entry belongs to
// exactly one column, which zeroes it after reading (the accumulator is clean for the next pass)
__device__ __forceinline__ double att_fold_col(double* __restrict__ z4, int64_t c, int64_t n_axis, int kmul) {
  const int64_t a = c / n_axis, k = c - a * n_axis;
  double z = 0.0;
#pragma unroll
  for (int jj = 0; jj < 4; ++jj) {
    const int64_t w = k - jj;
    if (w >= 0 && w <= n_axis - 4) {
      double* p = z4 + (kmul == 16 ? 16 * w + 4 * a : 4 * (a * n_axis + w)) + jj;
      z += *p;
      *p = 0.0;
    }
  }
  return z;
}

// Single-rank fused mode, after k_fused: beta (every block recomputes it from the deterministic partials; block 0
// hands it to k_scalar through st->pb_*), then v' = z/beta - beta v on all local columns (astro from zA, shared
// from z_sh, which is zeroed for the next iteration), constraint terms added per column, alpha^2 partials.
__global__ void __launch_bounds__(kRedThreads)
    k_post(SysView S, double* __restrict__ v, const double* __restrict__ zA, double* __restrict__ zsh,
           const double* __restrict__ part_rows, int64_t n_part, const double* __restrict__ cpart,
           const double* __restrict__ uc, double* __restrict__ uc_tmp, double* __restrict__ part_a2,
           DevState* __restrict__ st) {
  __shared__ double un_sh[kMaxConstr];
  __shared__ double cd_sh[kMaxConstr];
  __shared__ double bsh[3];
  if (st->halted) return;
  const int nc = S.n_constr;
  const double b2r = ordered_sum<kRedThreads>(part_rows, n_part);
  __shared__ double cp_sh[kMaxChunksSmem];
  __shared__ int32_t cr_sh[kMaxChunksSmem];
  const int64_t nch = S.n_chunks;
  const bool in_smem = nch <= kMaxChunksSmem;
  if (in_smem)
    for (int64_t c = threadIdx.x; c < nch; c += blockDim.x) {
      cp_sh[c] = cpart[c];
      cr_sh[c] = S.ch_row[c];
    }
  __syncthreads();
  if (threadIdx.x < nc) {  // constraint row dots from the chunk partials (chunks are in row order)
    double d = 0.0;
    for (int64_t c = 0; c < nch; ++c) {
      const int rw = in_smem ? cr_sh[c] : S.ch_row[c];
      if (rw == (int)threadIdx.x) d += in_smem ? cp_sh[c] : cpart[c];
    }
    cd_sh[threadIdx.x] = d;
    un_sh[threadIdx.x] = uc[threadIdx.x];
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    const double us = st->u_scale;
    double b2 = b2r;
    for (int k = 0; k < nc; ++k) {
      const double un = cd_sh[k] - us * un_sh[k];
      un_sh[k] = un;
      b2 = fma(un, un, b2);
    }
    const double beta = sqrt(b2);
    bsh[0] = beta;
    bsh[1] = beta > 0.0 ? 1.0 / beta : 1.0;
    bsh[2] = beta > 0.0 ? 1.0 : 0.0;
    if (blockIdx.x == 0) {
      st->pb_beta = beta;
      st->pb_ib = bsh[1];
      st->pb_pos = beta > 0.0;
    }
  }
  __syncthreads();
  if (blockIdx.x == 0 && threadIdx.x < nc) uc_tmp[threadIdx.x] = un_sh[threadIdx.x];
  const double beta = bsh[0], ib = bsh[1];
  if (bsh[2] == 0.0) {  // beta == 0: v is left unchanged (P&S step b skipped); leave the accumulators clean
    for (int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; c < S.n_sh; c += (int64_t)gridDim.x * blockDim.x) {
      if (S.z4 && c < S.n_att) att_fold_col(S.z4, c, S.n_axis, S.z4_kmul);
      zsh[c] = 0.0;
    }
    return;
  }
  double a2 = 0.0;
  const int64_t na = 5 * S.n_stars;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; c < na; c += stride) {
    double z = zA[c];
    if (c < 5 * S.n_cs)
      for (int64_t e = S.cs_ptr[c]; e < S.cs_ptr[c + 1]; ++e) z += S.cval[S.cs_e[e]] * un_sh[S.cs_k[e]];
    const double vn = z * ib - beta * v[c];
    v[c] = vn;
    a2 = fma(vn, vn, a2);
  }
  double* vsh = v + S.A0;
  for (int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; c < S.n_sh; c += stride) {
    double z = zsh[c];
    if (S.z4 && c < S.n_att) z += att_fold_col(S.z4, c, S.n_axis, S.z4_kmul);  // the row pass's window accumulator
    if (c >= S.scs_lo && c < S.scs_hi) {
      const int64_t q = c - S.scs_lo;
      for (int64_t e = S.scs_ptr[q]; e < S.scs_ptr[q + 1]; ++e) z += S.cval[S.scs_e[e]] * un_sh[S.scs_k[e]];
    }
    const double vn = z * ib - beta * vsh[c];
    vsh[c] = vn;
    zsh[c] = 0.0;
    a2 = fma(vn, vn, a2);
  }
  a2 = block_sum<kRedThreads>(a2);
  if (threadIdx.x == 0) part_a2[blockIdx.x] = a2;
}

cudaError_t launch_post(const SysView& S, double* v, const double* zA, double* zsh, const double* part_rows,
                        int64_t n_part, const double* cpart, const double* uc, double* uc_tmp, double* part_a2,
                        int nblk, DevState* st, cudaStream_t s) {
  k_post<<<nblk, kRedThreads, 0, s>>>(S, v, zA, zsh, part_rows, n_part, cpart, uc, uc_tmp, part_a2, st);
  return cudaGetLastError();
}

// ------------------------------------------------------------------------------------------------ scale rows (O-PREC)
__global__ void __launch_bounds__(kThreads, 1)
    k_scale_rows(SysView S, double* __restrict__ vals, const double* __restrict__ D) {
  const int lane = threadIdx.x & 31, j = lane & 3, r = lane >> 2;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t s_lo = S.warp_star[gw], s_hi = S.warp_star[gw + 1];
  const int64_t r_lo = S.star_ptr[s_lo], r_hi = S.star_ptr[s_hi];
  int64_t s = s_lo;
  for (int64_t base = r_lo; base < r_hi; base += 8) {
    const int64_t row = base + r;
    if (row >= r_hi) continue;
    while (S.star_ptr[s + 1] <= row) ++s;
    const IdxRec rec = S.idx[row];
    double* rp = vals + row * kSlots + 6 * j;  // lane-major: position 6j + t
#pragma unroll
    for (int t = 0; t < 6; ++t) {
      if (t == 5 && j == 3 && S.n_glob == 0) continue;
      rp[t] = rp[t] * D[col_of(S, t, j, s, rec)];
    }
  }
}

__global__ void k_scale_constr(SysView S, double* __restrict__ cval, const double* __restrict__ D) {
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < S.n_ce; e += (int64_t)gridDim.x * blockDim.x)
    cval[e] = cval[e] * D[S.ccol[e]];
}

// ------------------------------------------------------------------------------------------------ vectors
__global__ void __launch_bounds__(kRedThreads) k_sumsq(const double* __restrict__ u, int64_t n,
                                                       double* __restrict__ part) {
  double s = 0.0;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    s = fma(u[i], u[i], s);
  s = block_sum<kRedThreads>(s);
  if (threadIdx.x == 0) part[blockIdx.x] = s;
}

// phase 0: single rank (reduce + finish); 1: multi-rank pre-AR1 (write ar1); 2: multi-rank post-AR1 (finish);
// 3: plain aprod1 constraint dots into ar1 (no state); init: u_hat = b (beta_0 = ||b||, O-1).
__global__ void __launch_bounds__(kRedThreads)
    k_beta(int phase, SysView S, const double* __restrict__ part, int64_t n_part, const double* __restrict__ cpart,
           double* __restrict__ ar1, double* __restrict__ uc, double* __restrict__ ucn,
           const double* __restrict__ crhs, DevState* __restrict__ st, int init) {
  __shared__ double cdot_sh[kMaxConstr];
  __shared__ double b2_sh;
  if (phase != 3 && !init && st->halted) return;
  const int nc = S.n_constr;
  if (phase != 2) {
    const double b2 = phase == 3 ? 0.0 : ordered_sum<kRedThreads>(part, n_part);
    if (threadIdx.x == 0) b2_sh = b2;
    // chunk partials -> per-row dots (chunks are in row order; each row's chunks summed in order)
    __shared__ double cp_sh[kMaxChunksSmem];
    __shared__ int32_t cr_sh[kMaxChunksSmem];
    const int64_t nch = init ? 0 : S.n_chunks;
    const bool in_smem = nch <= kMaxChunksSmem;
    if (in_smem)
      for (int64_t c = threadIdx.x; c < nch; c += blockDim.x) {
        cp_sh[c] = cpart[c];
        cr_sh[c] = S.ch_row[c];
      }
    __syncthreads();
    if (threadIdx.x < nc) {
      double d = 0.0;
      for (int64_t c = 0; c < nch; ++c) {
        const int rw = in_smem ? cr_sh[c] : S.ch_row[c];
        if (rw == (int)threadIdx.x) d += in_smem ? cp_sh[c] : cpart[c];
      }
      cdot_sh[threadIdx.x] = d;
    }
    __syncthreads();
    if (phase == 1 || phase == 3) {
      if (threadIdx.x < nc) ar1[threadIdx.x] = cdot_sh[threadIdx.x];
      if (threadIdx.x == 0 && phase == 1) ar1[nc] = b2_sh;
      return;
    }
  } else {
    if (threadIdx.x < nc) cdot_sh[threadIdx.x] = ar1[threadIdx.x];
    if (threadIdx.x == 0) b2_sh = ar1[nc];
    __syncthreads();
  }
  __shared__ double uc_sh[kMaxConstr];
  if (threadIdx.x < nc) uc_sh[threadIdx.x] = init ? (crhs ? crhs[threadIdx.x] : 0.0) : uc[threadIdx.x];
  __syncthreads();
  if (threadIdx.x == 0) {
    const double us = st->u_scale;
    double b2 = b2_sh;
    for (int k = 0; k < nc; ++k) {
      const double un = init ? uc_sh[k] : cdot_sh[k] - us * uc_sh[k];
      uc_sh[k] = un;
      b2 = fma(un, un, b2);
    }
    const double beta = sqrt(b2);
    const int pos = beta > 0.0;
    const double ib = pos ? 1.0 / beta : 1.0;
    if (init) {
      st->bnorm = beta;
    } else if (pos) {
      const double a = st->alpha, d = st->damp;
      st->anorm = sqrt(st->anorm * st->anorm + a * a + beta * beta + d * d);
    }
    st->beta = beta;
    st->beta_pos = pos;
    st->inv_beta = ib;
  }
  __syncthreads();
  if (threadIdx.x < nc) {
    const double ib = st->inv_beta;
    uc[threadIdx.x] = uc_sh[threadIdx.x];
    ucn[threadIdx.x] = uc_sh[threadIdx.x] * ib;
  }
}

// plain aprod1: y_c[k] += cdot[k] (cdot from chunks, or already allreduced in ar1 when from_ar1)
__global__ void k_cdot_add(SysView S, const double* __restrict__ cpart, const double* __restrict__ ar1,
                           double* __restrict__ yc) {
  const int k = threadIdx.x;
  if (k >= S.n_constr) return;
  double d = 0.0;
  if (ar1) d = ar1[k];
  else
    for (int64_t c = 0; c < S.n_chunks; ++c)
      if (S.ch_row[c] == k) d += cpart[c];
  yc[k] += d;
}

__global__ void __launch_bounds__(kRedThreads)
    k_vshared(int64_t n_sh, double* __restrict__ vsh, double* __restrict__ zsh, double* __restrict__ part,
              const DevState* __restrict__ st, int fused) {
  if (st->halted || !st->beta_pos) return;
  const double beta = st->beta, zs = fused ? st->inv_beta : 1.0;  // fused mode: z = A^T u_hat (unnormalised)
  double a2 = 0.0;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n_sh; i += (int64_t)gridDim.x * blockDim.x) {
    const double vn = zsh[i] * zs - beta * vsh[i];
    vsh[i] = vn;
    zsh[i] = 0.0;
    a2 = fma(vn, vn, a2);
  }
  a2 = block_sum<kRedThreads>(a2);
  if (threadIdx.x == 0) part[blockIdx.x] = a2;
}

// mode 0: x += z, z = 0 (plain aprod2);  mode 1: x = z, z = 0 (column norms)
// lsqr_aprod2 on the fused kernel's loop (after k_fused3<R3_AP2> wrote the row sums z = A_rows^T y): astro columns
// x[c] += z[c] + constraint entries . y_c (added after the rows, as O-AP2); shared-column constraint entries
// scattered into z_sh by their owner (rank 0) before the allreduce and k_add_shared.
__global__ void __launch_bounds__(kRedThreads)
    k_astro_add(SysView S, double* __restrict__ x, const double* __restrict__ zA, const double* __restrict__ yc,
                double* __restrict__ zsh, int do_shared_constr) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; c < 5 * S.n_stars; c += stride) {
    double z = zA[c];
    if (c < 5 * S.n_cs)
      for (int64_t e = S.cs_ptr[c]; e < S.cs_ptr[c + 1]; ++e) z += S.cval[S.cs_e[e]] * yc[S.cs_k[e]];
    x[c] += z;
  }
  if (do_shared_constr)
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < S.n_csh; e += stride)
      atomicAdd(zsh + S.csh_idx[e], S.cval[S.csh_e[e]] * yc[S.csh_k[e]]);
}

__global__ void k_add_shared(double* __restrict__ xsh, double* __restrict__ zsh, int64_t n, int mode) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    xsh[i] = mode == 0 ? xsh[i] + zsh[i] : zsh[i];
    zsh[i] = 0.0;
  }
}

// O-3 steps c-j (rotation, norm estimates, stopping tests) in one thread; Paige & Saunders (lsqr.f form).
__global__ void __launch_bounds__(kRedThreads)
    k_scalar(DevState* __restrict__ st, const double* __restrict__ part_astro, int64_t n_pa,
             const double* __restrict__ part_sh, int64_t n_ps, const double* __restrict__ part_wa, int64_t n_pwa,
             const double* __restrict__ part_ws, int64_t n_pws, const double* __restrict__ ar2_alpha2,
             const double* __restrict__ ar1_wa, int init, int32_t* __restrict__ host_flag,
             const double* __restrict__ post_uc, double* __restrict__ uc, double* __restrict__ ucn, int nc) {
  if (!init && st->halted) {
    if (threadIdx.x == 0) st->col_enable = 0;
    return;
  }
  // post_uc != nullptr: single-rank fused mode; beta and the new constraint u_hat come from k_post's hand-over
  const int bp = post_uc ? st->pb_pos : st->beta_pos;
  if (post_uc && threadIdx.x < nc) {
    uc[threadIdx.x] = post_uc[threadIdx.x];
    ucn[threadIdx.x] = post_uc[threadIdx.x] * st->pb_ib;
  }
  // alpha^2 = ||v'||^2: astro part (per-warp partials of aprod2, or the allreduced value on several ranks)
  // + shared part (replicated, counted once).  ||w||^2 likewise (for ddnorm).
  double sums[4] = {0.0, 0.0, 0.0, 0.0};
  ordered_sum4<kRedThreads>(part_astro, (bp && !ar2_alpha2) ? n_pa : 0, part_sh, bp ? n_ps : 0, part_wa,
                            (!init && !ar1_wa) ? n_pwa : 0, part_ws, init ? 0 : n_pws, sums);
  double a2 = sums[0] + sums[1];
  double w2 = sums[2] + sums[3];
  if (threadIdx.x != 0) return;
  if (bp && ar2_alpha2) a2 += *ar2_alpha2;
  if (!init && ar1_wa) w2 += *ar1_wa;
  DevState* const gst = st;
  DevState L = *gst;  // all loads issued together; computed on registers, written back once
  st = &L;
  if (post_uc) {  // P&S step a/b bookkeeping for the new beta (was k_beta's job in the other modes)
    const double beta = L.pb_beta;
    if (L.pb_pos) {
      const double a = L.alpha, d = L.damp;
      L.anorm = sqrt(L.anorm * L.anorm + a * a + beta * beta + d * d);
    }
    L.beta = beta;
    L.inv_beta = L.pb_ib;
    L.beta_pos = L.pb_pos;
  }
  const double eps = 0x1p-52;
  if (init) {
    const double alpha = bp ? sqrt(a2) : 0.0;
    const double beta = st->beta;
    st->alpha = alpha;
    st->inv_alpha = alpha > 0.0 ? 1.0 / alpha : 1.0;
    st->v_pending = bp;
    st->rhobar = alpha; st->phibar = beta; st->rnorm = beta; st->r1norm = beta; st->r2norm = beta;
    st->anorm = 0; st->acond = 0; st->ddnorm = 0; st->res2 = 0; st->xnorm = 0; st->xxnorm = 0; st->z = 0;
    st->cs2 = -1.0; st->sn2 = 0.0;
    st->arnorm = alpha * beta;
    st->t1 = 0.0; st->t2 = 0.0; st->t3 = 0.0;
    st->col_enable = 1;
    st->itn = 0; st->istop = 0; st->istop_first = 0;
    st->halted = (alpha * beta == 0.0) ? 1 : 0;
    st->u_scale = alpha * st->inv_beta;
  } else {
    st->itn += 1;
    double alpha = st->alpha;
    if (bp) {
      alpha = sqrt(a2);
      st->inv_alpha = alpha > 0.0 ? 1.0 / alpha : 1.0;
      st->v_pending = 1;
    } else {
      st->v_pending = 0;
    }
    st->alpha = alpha;
    const double beta = st->beta, damp = st->damp, dampsq = damp * damp;
    double rhobar = st->rhobar, phibar = st->phibar, psi, rhobar1;
    if (damp > 0.0) {  // c.
      rhobar1 = sqrt(rhobar * rhobar + dampsq);
      const double cs1 = rhobar / rhobar1, sn1 = damp / rhobar1;
      psi = sn1 * phibar;
      phibar = cs1 * phibar;
    } else {
      rhobar1 = rhobar;
      psi = 0.0;
    }
    const double rho = sqrt(rhobar1 * rhobar1 + beta * beta);  // d.
    const double cs = rhobar1 / rho, sn = beta / rho;
    const double theta = sn * alpha;
    rhobar = -cs * alpha;
    const double phi = cs * phibar;
    phibar = sn * phibar;
    const double tau = sn * phi;
    const double t1 = phi / rho, t2 = -theta / rho, t3 = 1.0 / rho;  // e. (applied by k_colupdate)
    st->t1 = t1; st->t2 = t2; st->t3 = t3;
    const double ddnorm = st->ddnorm + t3 * t3 * w2;  // sum_j (t3 w_j)^2 with w the pre-update w
    // f.
    const double delta = st->sn2 * rho, gambar = -st->cs2 * rho, rhs = phi - delta * st->z, zbar = rhs / gambar;
    const double xnorm = sqrt(st->xxnorm + zbar * zbar);
    const double gamma = sqrt(gambar * gambar + theta * theta);
    st->cs2 = gambar / gamma;
    st->sn2 = theta / gamma;
    st->z = rhs / gamma;
    st->xxnorm = st->xxnorm + st->z * st->z;
    // g.
    const double anorm = st->anorm;
    const double acond = anorm * sqrt(ddnorm);
    const double res2 = st->res2 + psi * psi;
    const double rnorm = sqrt(phibar * phibar + res2);
    const double arnorm = alpha * fabs(tau);
    double r1norm;
    if (damp > 0.0) {
      const double r1sq = rnorm * rnorm - dampsq * st->xxnorm;
      r1norm = sqrt(fabs(r1sq));
      if (r1sq < 0) r1norm = -r1norm;
    } else {
      r1norm = rnorm;
    }
    // h.
    const double bnorm = st->bnorm;
    const double test1 = rnorm / bnorm, test2 = arnorm / (anorm * rnorm + eps), test3 = 1.0 / (acond + eps);
    const double tt1 = test1 / (1.0 + anorm * xnorm / bnorm);
    const double rtol = st->btol + st->atol * anorm * xnorm / bnorm;
    // i.
    int is = 0;
    if (st->itn >= st->itn_limit) is = 7;
    if (1.0 + test3 <= 1.0) is = 6;
    if (1.0 + test2 <= 1.0) is = 5;
    if (1.0 + tt1 <= 1.0) is = 4;
    if (test3 <= st->ctol) is = 3;
    if (test2 <= st->atol) is = 2;
    if (test1 <= rtol) is = 1;
    st->rhobar = rhobar; st->phibar = phibar; st->ddnorm = ddnorm; st->xnorm = xnorm; st->acond = acond;
    st->res2 = res2; st->rnorm = rnorm; st->r1norm = r1norm; st->r2norm = rnorm; st->arnorm = arnorm;
    st->istop = is;
    if (is != 0 && st->istop_first == 0) st->istop_first = is;
    st->col_enable = 1;
    st->u_scale = alpha * st->inv_beta;
    if ((is != 0 && !st->fixed_count) || st->itn >= st->itn_limit) st->halted = 1;
  }
  *gst = L;
  if (host_flag) *reinterpret_cast<volatile int32_t*>(host_flag) = L.halted | (L.itn << 1);
}

// attitude column c (axis a, knot k) of v into the gather copy: knot format xg[4k + a]; window format
// xg[16 w + 4 (k - w) + a] for every window start w in [k - 3, k] ∩ [0, n_axis - 4]
__device__ __forceinline__ void att_put(double* __restrict__ xg, int kmul, int64_t n_axis, int64_t c, double v) {
  const int64_t a = c / n_axis, k = c - a * n_axis;
  if (kmul == 4) {
    xg[4 * k + a] = v;
    return;
  }
#pragma unroll
  for (int jj = 0; jj < 4; ++jj) {
    const int64_t w = k - jj;
    if (w >= 0 && w <= n_axis - 4) xg[16 * w + 4 * jj + a] = v;
  }
}

// O-3e: v <- v/alpha (if pending); d = t3 w; var += d^2; x += t1 w; w = v + t2 w;  partials of ||w_new||^2 split
// into the local astro columns (i < A0) and the replicated shared slice (i >= A0); the new v's attitude slice also
// goes to the fused kernel's gather copy (att_put).
__global__ void __launch_bounds__(kRedThreads)
    k_colupdate(double* __restrict__ v, double* __restrict__ w, double* __restrict__ x, double* __restrict__ var,
                int64_t n, int64_t A0, int64_t n_att, int64_t n_axis, double* __restrict__ xatt4, int kmul,
                double* __restrict__ part_wa, double* __restrict__ part_ws, const DevState* __restrict__ st) {
  if (!st->col_enable) return;
  const double ia = st->v_pending ? st->inv_alpha : 1.0;
  const double t1 = st->t1, t2 = st->t2, t3 = st->t3;
  double wa = 0.0, ws = 0.0;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const double vi = v[i] * ia, wi = w[i];
    const double d = t3 * wi;
    var[i] = fma(d, d, var[i]);
    x[i] = fma(t1, wi, x[i]);
    const double wnew = fma(t2, wi, vi);
    w[i] = wnew;
    v[i] = vi;
    if (i < A0) {
      wa = fma(wnew, wnew, wa);
    } else {
      ws = fma(wnew, wnew, ws);
      const int64_t c = i - A0;
      if (c < n_att) att_put(xatt4, kmul, n_axis, c, vi);  // the attitude gather copy
    }
  }
  wa = block_sum<kRedThreads>(wa);
  ws = block_sum<kRedThreads>(ws);
  if (threadIdx.x == 0) {
    part_wa[blockIdx.x] = wa;
    part_ws[blockIdx.x] = ws;
  }
}

__global__ void k_sum_to(const double* __restrict__ part, int64_t n, double* __restrict__ dst) {
  const double s = ordered_sum<kRedThreads>(part, n);
  if (threadIdx.x == 0) *dst = s;
}

__global__ void k_precond_D(double* __restrict__ c, int64_t n) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    c[i] = c[i] > 0.0 ? 1.0 / sqrt(c[i]) : 1.0;
}

// O-4/O-5: se_j = D_j * s * sqrt(var_j), x_j = D_j * x_j,  s = r2norm / sqrt(t)
__global__ void k_finalize(const double* __restrict__ x, const double* __restrict__ var, const double* __restrict__ D,
                           int64_t n, const DevState* __restrict__ st, double se_t, double* __restrict__ xo,
                           double* __restrict__ so) {
  const double s = st->r2norm / sqrt(se_t);
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    if (xo) xo[i] = D[i] * x[i];
    if (so) so[i] = D[i] * (s * sqrt(var[i]));
  }
}

__global__ void k_fill(double* __restrict__ p, int64_t n, double v) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    p[i] = v;
}

// ------------------------------------------------------------------------------------------------ launchers
static int vec_grid(int64_t n, int maxb) {
  int64_t b = (n + kRedThreads - 1) / kRedThreads;
  if (b < 1) b = 1;
  return (int)(b < maxb ? b : maxb);
}


// ------------------------------------------------------------------------------------------------ ingest (set_system)
// Converts a chunk of host-layout rows (paper slot order, int64 global column indices) into the device
// layout (lane-major values, 16-B index record), validating the star grouping and index ranges.  err[0] receives
// (min) 1 + offending row and err[1] the kind (1 unsorted, 2 range) on failure.
__global__ void k_ingest(const double* __restrict__ sv, const int64_t* __restrict__ smA,
                         const int64_t* __restrict__ smT, const int64_t* __restrict__ siC, int64_t row0, int64_t nrows,
                         const int64_t* __restrict__ star_ptr, int64_t n_stars_loc, int64_t star_begin, int64_t A0g,
                         int64_t I0g, int64_t n_axis, int64_t n_instr, InstrPerm ip, double* __restrict__ vals,
                         IdxRec* __restrict__ idx, unsigned long long* __restrict__ err) {
  for (int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; q < nrows; q += (int64_t)gridDim.x * blockDim.x) {
    const int64_t li = row0 + q;
    int64_t lo = 0, hi = n_stars_loc;  // star_ptr[lo] <= li < star_ptr[hi]
    while (hi - lo > 1) {
      const int64_t mid = (lo + hi) >> 1;
      if (star_ptr[mid] <= li) lo = mid; else hi = mid;
    }
    int kind = 0;
    if (smA[q] != 5 * (star_begin + lo)) kind = 1;
    const int64_t k0 = smT[q] - A0g;
    if (k0 < 0 || k0 > n_axis - 4) kind = kind ? kind : 2;
    uint32_t ic[6];
#pragma unroll
    for (int jj = 0; jj < 6; ++jj) {
      const int64_t c = siC[q * 6 + jj] - I0g;
      if (c < 0 || c >= n_instr) kind = kind ? kind : 2;
      ic[jj] = (uint32_t)(ip.fwd(c < 0 || c >= n_instr ? 0 : c) & 0xffff);
    }
    if (kind) {
      atomicMin(err, (unsigned long long)(li + 1));
      atomicMax(err + 1, (unsigned long long)kind);
      continue;
    }
    IdxRec rec;
    rec.k0 = (int32_t)k0;
    rec.ic01 = ic[0] | (ic[1] << 16);
    rec.ic23 = ic[2] | (ic[3] << 16);
    rec.ic45 = ic[4] | (ic[5] << 16);
    idx[li] = rec;
    const double* src = sv + q * kSlots;
    double* dst = vals + li * kSlots;
#pragma unroll
    for (int pp = 0; pp < kSlots; ++pp) dst[pp] = src[slot_of(pp % 6, pp / 6)];
  }
}

cudaError_t launch_ingest(const double* sv, const int64_t* smA, const int64_t* smT, const int64_t* siC, int64_t row0,
                          int64_t nrows, const int64_t* star_ptr, int64_t n_stars_loc, int64_t star_begin,
                          int64_t A0g, int64_t I0g, int64_t n_axis, int64_t n_instr, InstrPerm ip, double* vals,
                          IdxRec* idx, unsigned long long* err, cudaStream_t s) {
  if (nrows == 0) return cudaSuccess;
  k_ingest<<<vec_grid(nrows, 148 * 8), kRedThreads, 0, s>>>(sv, smA, smT, siC, row0, nrows, star_ptr, n_stars_loc,
                                                            star_begin, A0g, I0g, n_axis, n_instr, ip, vals, idx,
                                                            err);
  return cudaGetLastError();
}

cudaError_t launch_generate(const GenArgs& g, double* vals, IdxRec* idx, const int64_t* star_ptr, int64_t n_rows,
                            int64_t n_stars_loc, double* b, cudaStream_t s) {
  if (n_rows == 0) return cudaSuccess;
  k_generate<<<vec_grid(n_rows, 148 * 16), kRedThreads, 0, s>>>(g, vals, idx, star_ptr, n_rows, n_stars_loc, b);
  return cudaGetLastError();
}

// Dynamic shared-memory opt-in of a kernel, per (kernel, device): the attribute applies to the device current at
// the call, and handles of one process may live on different devices or threads.
static cudaError_t ensure_smem(const void* fn, size_t bytes) {
  static std::mutex mu;
  static std::map<std::pair<const void*, int>, size_t> done;
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  std::lock_guard<std::mutex> g(mu);
  size_t& cur = done[{fn, dev}];
  if (bytes <= cur) return cudaSuccess;
  e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes);
  if (e == cudaSuccess) cur = bytes;
  return e;
}

template <int MODE, bool SM, bool G4>
static cudaError_t ap1(const SysView& S, int grid, const double* x, double* y, double* part, double* cpart,
                       const DevState* st, const double* xg4, cudaStream_t s) {
  const size_t smem = kRingBytes + kBarBytes + (SM ? (size_t)S.ip.slots() * sizeof(double) : 0);
  cudaError_t e = ensure_smem((const void*)k_aprod1<MODE, SM, G4>, smem);
  if (e != cudaSuccess) return e;
  k_aprod1<MODE, SM, G4><<<grid, kThreads, smem, s>>>(S, x, y, part, cpart, st, xg4);
  return cudaGetLastError();
}

cudaError_t launch_aprod1(int mode, const SysView& S, int grid, const double* x, double* y, double* part,
                          double* cpart, const DevState* st, cudaStream_t s, const double* xg4) {
  const bool sm = S.ip.slots() <= kInstrSmemMax;
  if (xg4) {  // the two products that run per iteration / per API call in the default regimes
    if (mode == AP1_LSQR) return sm ? ap1<AP1_LSQR, true, true>(S, grid, x, y, part, cpart, st, xg4, s)
                                    : ap1<AP1_LSQR, false, true>(S, grid, x, y, part, cpart, st, xg4, s);
    return sm ? ap1<AP1_PLAIN, true, true>(S, grid, x, y, part, cpart, st, xg4, s)
              : ap1<AP1_PLAIN, false, true>(S, grid, x, y, part, cpart, st, xg4, s);
  }
  if (mode == AP1_LSQR) return sm ? ap1<AP1_LSQR, true, false>(S, grid, x, y, part, cpart, st, nullptr, s)
                                  : ap1<AP1_LSQR, false, false>(S, grid, x, y, part, cpart, st, nullptr, s);
  return sm ? ap1<AP1_PLAIN, true, false>(S, grid, x, y, part, cpart, st, nullptr, s)
            : ap1<AP1_PLAIN, false, false>(S, grid, x, y, part, cpart, st, nullptr, s);
}

template <int MODE, bool SM>
static cudaError_t ap2(const SysView& S, int grid, const double* y, const double* ucn, double* xv, double* zsh,
                       double* part, const DevState* st, int dsc, cudaStream_t s) {
  size_t smem = kRingBytes + kBarBytes + (SM ? (size_t)S.ip.slots() * sizeof(double) : 0);
  cudaError_t e = ensure_smem((const void*)k_aprod2<MODE, SM>, smem);
  if (e != cudaSuccess) return e;
  k_aprod2<MODE, SM><<<grid, kThreads, smem, s>>>(S, y, ucn, xv, zsh, part, st, dsc);
  return cudaGetLastError();
}

cudaError_t launch_aprod2(int mode, const SysView& S, int grid, const double* y, const double* ucn, double* xv,
                          double* zsh, double* part, const DevState* st, int dsc, cudaStream_t s) {
  const bool sm = S.ip.slots() <= kInstrSmemMax;
  switch (mode) {
    case AP2_LSQR: return sm ? ap2<AP2_LSQR, true>(S, grid, y, ucn, xv, zsh, part, st, dsc, s)
                             : ap2<AP2_LSQR, false>(S, grid, y, ucn, xv, zsh, part, st, dsc, s);
    case AP2_PLAIN: return sm ? ap2<AP2_PLAIN, true>(S, grid, y, ucn, xv, zsh, part, st, dsc, s)
                              : ap2<AP2_PLAIN, false>(S, grid, y, ucn, xv, zsh, part, st, dsc, s);
    default: return sm ? ap2<AP2_COLNORM, true>(S, grid, y, ucn, xv, zsh, part, st, dsc, s)
                       : ap2<AP2_COLNORM, false>(S, grid, y, ucn, xv, zsh, part, st, dsc, s);
  }
}

cudaError_t launch_scale_rows(const SysView& S, int grid, double* vals, const double* D, cudaStream_t s) {
  k_scale_rows<<<grid, kThreads, 0, s>>>(S, vals, D);
  return cudaGetLastError();
}
cudaError_t launch_scale_constr(const SysView& S, double* cval, const double* D, cudaStream_t s) {
  if (S.n_ce == 0) return cudaSuccess;
  k_scale_constr<<<vec_grid(S.n_ce, 148), kRedThreads, 0, s>>>(S, cval, D);
  return cudaGetLastError();
}
cudaError_t launch_sumsq(const double* u, int64_t n, double* part, int nblk, cudaStream_t s) {
  k_sumsq<<<nblk, kRedThreads, 0, s>>>(u, n, part);
  return cudaGetLastError();
}
cudaError_t launch_beta(int phase, const SysView& S, const double* part, int64_t n_part, const double* cpart,
                        double* ar1, double* uc, double* ucn, const double* crhs, DevState* st, int init,
                        cudaStream_t s) {
  k_beta<<<1, kRedThreads, 0, s>>>(phase, S, part, n_part, cpart, ar1, uc, ucn, crhs, st, init);
  return cudaGetLastError();
}
cudaError_t launch_cdot_add(const SysView& S, const double* cpart, const double* ar1, double* yc, cudaStream_t s) {
  if (S.n_constr == 0) return cudaSuccess;
  k_cdot_add<<<1, 64, 0, s>>>(S, cpart, ar1, yc);
  return cudaGetLastError();
}
cudaError_t launch_vshared(const SysView& S, double* vsh, double* zsh, double* part, int nblk, const DevState* st,
                           int fused, cudaStream_t s) {
  k_vshared<<<nblk, kRedThreads, 0, s>>>(S.n_sh, vsh, zsh, part, st, fused);
  return cudaGetLastError();
}
// Shared-memory plan of k_fused3: copies of the z_instr accumulator and, for small attitude slices, of z_att.
struct F3Plan {
  int zrep, arep;
  size_t smem;
};
constexpr int64_t kSmAttMax = 4096;  // n_att up to this: z_att privatised in shared memory (L2 REDs contend below)
static bool f3_ig(const SysView& S) { return S.ip.slots() > kF3InstrMax; }
static F3Plan f3_plan(const SysView& S) {
  const int64_t zb = f3_ig(S) ? 0 : 8 * (S.ip.slots() + 2), ab = 8 * S.n_att;
  const int64_t fixed = FRing::kBytes + kF3Bars + zb;           // ring, mbarriers, v_instr
  const int64_t avail = kSmemMaxBytes - 2048 - fixed;           // 2 KB: static shared memory of the kernel
  F3Plan p{1, 0, 0};
  if (S.n_att <= kSmAttMax && zb + ab <= avail) {
    const int64_t r = std::min<int64_t>(kFWarps, avail / (zb + ab));
    p.arep = (int)r;
    p.zrep = zb ? (int)std::max<int64_t>(1, std::min<int64_t>(kFWarps, (avail - r * ab) / zb)) : 1;
  } else {
    p.zrep = zb ? (int)std::max<int64_t>(1, std::min<int64_t>(kFWarps, avail / zb)) : 1;
  }
  p.smem = (size_t)(fixed + (int64_t)p.zrep * zb + (int64_t)p.arep * ab);
  return p;
}
template <int KIND, int DIAG, bool SMATT, bool IG, bool ZREP>
static cudaError_t fz3v(const SysView& S, const F3Plan& P, int grid, const double* x, double* u, double* zA,
                        double* zsh, double* part, double* cpart, const DevState* st, cudaStream_t s) {
  cudaError_t e = ensure_smem((const void*)k_fused3<KIND, DIAG, SMATT, IG, ZREP>, P.smem);
  if (e != cudaSuccess) return e;
  SysView S2 = S;
  S2.f3_zrep = P.zrep;
  S2.f3_arep = P.arep;
  k_fused3<KIND, DIAG, SMATT, IG, ZREP><<<grid, kFWarps * 32, P.smem, s>>>(S2, x, u, zA, zsh, part, cpart, st);
  return cudaGetLastError();
}
template <int KIND, int DIAG>
static cudaError_t fz3(const SysView& S, int grid, const double* x, double* u, double* zA, double* zsh, double* part,
                       double* cpart, const DevState* st, cudaStream_t s) {
  const F3Plan P = f3_plan(S);
  if (DIAG == 0 && f3_ig(S))
    return P.arep > 0 ? fz3v<KIND, 0, true, true, false>(S, P, grid, x, u, zA, zsh, part, cpart, st, s)
                      : fz3v<KIND, 0, false, true, false>(S, P, grid, x, u, zA, zsh, part, cpart, st, s);
  if (DIAG == 0 && P.arep > 0) return fz3v<KIND, 0, true, false, true>(S, P, grid, x, u, zA, zsh, part, cpart, st, s);
  if (DIAG == 0 && P.zrep > 1) return fz3v<KIND, 0, false, false, true>(S, P, grid, x, u, zA, zsh, part, cpart, st, s);
  F3Plan Q = P;  // one z_instr copy, attitude REDs in L2 (the C2-C5 regime; DIAG experiments)
  Q.smem -= (size_t)Q.arep * 8 * S.n_att + (size_t)(Q.zrep - 1) * 8 * (S.ip.slots() + 2);
  Q.arep = 0;
  Q.zrep = 1;
  return fz3v<KIND, DIAG, false, false, false>(S, Q, grid, x, u, zA, zsh, part, cpart, st, s);
}

// Build-time experiment switch (not in the product build): compile with -DLSQR_DIAG_EXPERIMENTS to let the env var
// LSQR_DIAG select kernel variants that skip work (results are WRONG): bit 0 the instrumental CAS, bit 1 the
// attitude REDs, bit 2 the attitude gathers, bit 3 the instrumental gathers, bit 4 the stage reads of A's values.
// Used for DESIGN.md §7's time breakdown.
#ifdef LSQR_DIAG_EXPERIMENTS
static int diag_mode() {
  static int m = -1;
  if (m < 0) {
    const char* e = getenv("LSQR_DIAG");
    m = e ? atoi(e) : 0;
  }
  return m;
}
#endif

__global__ void k_att_fold(double* __restrict__ z4, double* __restrict__ zsh, int64_t n_att, int64_t n_axis, int kmul) {
  for (int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; c < n_att; c += (int64_t)gridDim.x * blockDim.x)
    zsh[c] += att_fold_col(z4, c, n_axis, kmul);
}
static cudaError_t att_fold(const SysView& S, double* zsh, cudaStream_t s) {
  if (!S.z4) return cudaSuccess;
  k_att_fold<<<vec_grid(S.n_att, 148 * 4), kRedThreads, 0, s>>>(S.z4, zsh, S.n_att, S.n_axis, S.z4_kmul);
  return cudaGetLastError();
}

cudaError_t launch_fused(const SysView& S, int grid, const double* x, double* u, double* zA, double* zsh,
                         double* part, double* cpart, const DevState* st, cudaStream_t s, bool fold) {
  cudaError_t e;
#ifdef LSQR_DIAG_EXPERIMENTS
  switch (diag_mode()) {
    case 1: e = fz3<R3_FUSED, 1>(S, grid, x, u, zA, zsh, part, cpart, st, s); break;
    case 2: e = fz3<R3_FUSED, 2>(S, grid, x, u, zA, zsh, part, cpart, st, s); break;
    case 4: e = fz3<R3_FUSED, 4>(S, grid, x, u, zA, zsh, part, cpart, st, s); break;
    case 8: e = fz3<R3_FUSED, 8>(S, grid, x, u, zA, zsh, part, cpart, st, s); break;
    case 15: e = fz3<R3_FUSED, 15>(S, grid, x, u, zA, zsh, part, cpart, st, s); break;
    case 16: e = fz3<R3_FUSED, 16>(S, grid, x, u, zA, zsh, part, cpart, st, s); break;
    case 31: e = fz3<R3_FUSED, 31>(S, grid, x, u, zA, zsh, part, cpart, st, s); break;
    default: e = fz3<R3_FUSED, 0>(S, grid, x, u, zA, zsh, part, cpart, st, s); break;
  }
#else
  e = fz3<R3_FUSED, 0>(S, grid, x, u, zA, zsh, part, cpart, st, s);
#endif
  return e != cudaSuccess || !fold ? e : att_fold(S, zsh, s);
}

cudaError_t launch_ap2_lean(const SysView& S, int grid, const double* u, double* zA, double* zsh, const DevState* st,
                            cudaStream_t s, bool fold) {
  const cudaError_t e = fz3<R3_AP2, 0>(S, grid, nullptr, const_cast<double*>(u), zA, zsh, nullptr, nullptr, st, s);
  return e != cudaSuccess || !fold ? e : att_fold(S, zsh, s);
}

cudaError_t launch_vastro(const SysView& S, double* v, const double* zA, const double* uc, double* zsh, double* part,
                          int nblk, const DevState* st, int do_shared_constr, cudaStream_t s) {
  k_vastro<<<nblk, kRedThreads, 0, s>>>(S, v, zA, uc, zsh, part, st, do_shared_constr);
  return cudaGetLastError();
}

cudaError_t launch_astro_add(const SysView& S, double* x, const double* zA, const double* yc, double* zsh,
                             int do_shared_constr, cudaStream_t s) {
  k_astro_add<<<vec_grid(std::max<int64_t>(5 * S.n_stars, S.n_csh), 148 * 4), kRedThreads, 0, s>>>(S, x, zA, yc, zsh,
                                                                                                 do_shared_constr);
  return cudaGetLastError();
}
cudaError_t launch_add_shared(const SysView& S, double* xsh, double* zsh, int mode, cudaStream_t s) {
  k_add_shared<<<vec_grid(S.n_sh, 148 * 4), kRedThreads, 0, s>>>(xsh, zsh, S.n_sh, mode);
  return cudaGetLastError();
}
cudaError_t launch_scalar(DevState* st, const double* part_astro, int64_t n_pa, const double* part_sh,
                          int64_t n_ps, const double* part_wa, int64_t n_pwa, const double* part_ws, int64_t n_pws,
                          const double* ar2_alpha2, const double* ar1_wa, int init, int32_t* host_flag,
                          cudaStream_t s, const double* post_uc, double* uc, double* ucn, int nc) {
  k_scalar<<<1, kRedThreads, 0, s>>>(st, part_astro, n_pa, part_sh, n_ps, part_wa, n_pwa, part_ws, n_pws,
                                     ar2_alpha2, ar1_wa, init, host_flag, post_uc, uc, ucn, nc);
  return cudaGetLastError();
}
cudaError_t launch_colupdate(const SysView& S, double* v, double* w, double* x, double* var, double* part_wa,
                             double* part_ws, int nblk, const DevState* st, cudaStream_t s) {
  k_colupdate<<<nblk, kRedThreads, 0, s>>>(v, w, x, var, S.n_cols, S.A0, S.n_att, S.n_axis, S.xatt4, S.att_kmul,
                                           part_wa, part_ws, st);
  return cudaGetLastError();
}

__global__ void k_att_pack(const double* __restrict__ v, int64_t n_att, int64_t n_axis, double* __restrict__ xatt4,
                           int kmul) {
  for (int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; c < n_att; c += (int64_t)gridDim.x * blockDim.x)
    att_put(xatt4, kmul, n_axis, c, v[c]);
}
cudaError_t launch_att_pack(const SysView& S, const double* v, cudaStream_t s, double* dst) {
  k_att_pack<<<vec_grid(S.n_att, 148 * 4), kRedThreads, 0, s>>>(v + S.A0, S.n_att, S.n_axis, dst ? dst : S.xatt4,
                                                                 S.att_kmul);
  return cudaGetLastError();
}
cudaError_t launch_sum_to(const double* part, int64_t n, double* dst, cudaStream_t s) {
  k_sum_to<<<1, kRedThreads, 0, s>>>(part, n, dst);
  return cudaGetLastError();
}
cudaError_t launch_precond_D(double* c, int64_t n, cudaStream_t s) {
  k_precond_D<<<vec_grid(n, 148 * 4), kRedThreads, 0, s>>>(c, n);
  return cudaGetLastError();
}
cudaError_t launch_finalize(const double* x, const double* var, const double* D, int64_t n, const DevState* st,
                            double se_t, double* x_out, double* se_out, cudaStream_t s) {
  k_finalize<<<vec_grid(n, 148 * 4), kRedThreads, 0, s>>>(x, var, D, n, st, se_t, x_out, se_out);
  return cudaGetLastError();
}
cudaError_t launch_fill(double* p, int64_t n, double v, cudaStream_t s) {
  if (n == 0) return cudaSuccess;
  k_fill<<<vec_grid(n, 148 * 4), kRedThreads, 0, s>>>(p, n, v);
  return cudaGetLastError();
}

}  // namespace lsqr

// lsqr_internal.cuh -- device data layout and kernel launchers of liblsqr_avugsr.so (product code; shares nothing
// with oracle/).  Layout rationale and per-kernel roofline: DESIGN.md §5-§6.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace lsqr {

constexpr int kSlots = 24;           // 5 astro + 12 att + 6 instr + 1 glob

constexpr int kThreads = 512;        // persistent row kernels: one 16-warp CTA per SM
constexpr int kWarpsPerCta = kThreads / 32;
constexpr int kRows = 16;            // rows per TMA stage (two 8-row groups, 4 lanes per row)
constexpr int kGroups = kRows / 8;
constexpr int kStages = 3;           // ring depth per warp (kStages-1 stages in flight while computing)
constexpr int kStageBytes = kRows * (kSlots * 8 + 16);                  // 3328 B: values + index records
#ifndef LSQR_FWARPS
#define LSQR_FWARPS 16
#endif
constexpr int kFWarps = LSQR_FWARPS; // fused kernel: warps per CTA (own partition SysView::warp_star_f; 12 x 6 stages
                                     // and a separate producer warp measured slower)
constexpr int kFStages = 4;          // fused kernel: ring depth (8-row stages)
constexpr int kRingBytes = kWarpsPerCta * kStages * kStageBytes;        // 159,744 B per CTA
constexpr int kBarBytes = kWarpsPerCta * kStages * 8;                   // mbarriers
constexpr int kRedThreads = 256;     // small reduction / vector kernels
constexpr int kInstrSmemMax = 7680;  // n_instr above this -> instrumental gathers/scatter use global memory (L2)
constexpr int kMaxConstr = 64;       // constraint rows handled by the one-block beta kernel
constexpr int kMaxChunksSmem = 1024; // constraint chunk partials staged in shared memory by k_beta

// Row storage is LANE-MAJOR: the 24 values of a row are stored so that lane j of the row's 4-lane group finds its
// 6 values at positions 6j..6j+5 (slot_of(t, j) = slot held at position 6j + t).  Slot 23 stays at position 23.
// lsqr_set_system / lsqr_get_system convert from / to the paper's slot order.
__host__ __device__ __forceinline__ int slot_of(int t, int j) {
  return t == 0 ? j : (t <= 3 ? 5 + 4 * (t - 1) + j : (t == 4 ? 17 + j : (j == 0 ? 4 : 20 + j)));
}

// Per-row index record, 16 B: the paper's matrixIndexAtt (as k0, relative to the attitude block) and instrCol
// (6 x u16, relative to the instrumental block) in one 128-bit word.  matrixIndexAstro is implicit: rows are
// grouped by star (star_ptr), so the astro column is 5*star.
struct __align__(16) IdxRec {
  int32_t k0;
  uint32_t ic01, ic23, ic45;  // instrCol[j] in 16-bit halves (j even: low half)
};
static_assert(sizeof(IdxRec) == 16, "IdxRec must be 16 bytes");

// Shared-memory slot of instrumental column c (device-internal; stored in IdxRec).  With the generator's structure
// (row j-th instrumental column in group j of g = n_instr/6 columns), the 8 lanes that touch group j (< 4) in one
// warp instruction get their own 4 of the 16 bank pairs, and groups 4 / 5 (touched together) get 8 each, which cuts
// bank conflicts of the instrumental gathers and CAS updates.  Identity when disabled (n_instr % 6 != 0 or the
// instrumental slice is not kept in shared memory).
struct InstrPerm {
  int64_t n = 0, g = 0, oa = 0;
  bool on = false;
  __host__ __device__ void init(int64_t n_instr, bool enable) {
    n = n_instr;
    on = enable && n_instr % 6 == 0 && n_instr >= 6;
    g = on ? n_instr / 6 : 0;
    oa = on ? 16 * ((g + 3) / 4) : 0;
  }
  __host__ __device__ int64_t slots() const { return on ? oa + 16 * ((g + 7) / 8) : n; }
  __host__ __device__ int64_t fwd(int64_t c) const {
    if (!on) return c;
    const int64_t grp = c / g, t = c - grp * g;
    if (grp < 4) return 16 * (t >> 2) + 4 * grp + (t & 3);
    return oa + 16 * (t >> 3) + 8 * (grp - 4) + (t & 7);
  }
  __host__ __device__ int64_t inv(int64_t p) const {  // slot -> column
    if (!on) return p;
    if (p < oa) {
      const int64_t b = p >> 4, w = p & 15;
      return (w >> 2) * g + 4 * b + (w & 3);
    }
    const int64_t q = p - oa, b = q >> 4, w = q & 15;
    return (4 + (w >> 3)) * g + 8 * b + (w & 7);
  }
};

// LSQR scalar state kept on the device (Paige-Saunders scalars) + control flags.
struct DevState {
  double alpha, beta, rhobar, phibar, anorm, acond, ddnorm, res2, xnorm, xxnorm, z, cs2, sn2, rnorm, r1norm,
      r2norm, arnorm, bnorm;
  double damp, atol, btol, ctol;
  double inv_beta;   // 1/beta (1 if beta == 0): u_k = u_hat * inv_beta (u is kept unnormalised)
  double u_scale;    // alpha_k * inv_beta_k: next aprod1 computes u_hat = A v - u_scale * u_hat
  double inv_alpha;  // colupdate: v <- v * inv_alpha when v_pending
  double t1, t2, t3; // x += t1 w ; w = v + t2 w ; d = t3 w
  double rn_tmp;
  double pb_beta, pb_ib;  // k_post -> k_scalar hand-over (written by k_post block 0, read by k_scalar only)
  double r_rho, r_theta, r_phi, r_sn;  // repro mode: k_r_scalar_a -> k_r_scalar_b hand-over
  int32_t itn, istop, istop_first, itn_limit;
  int32_t fixed_count, halted, col_enable, v_pending, beta_pos, pb_pos, pad_[2];
};

// Everything a row kernel needs, passed by value.
struct SysView {
  const double* vals;       // [n_rows][24]
  const IdxRec* idx;        // [n_rows]
  const int64_t* star_ptr;  // [n_stars+1] local row offsets per local star
  const int64_t* warp_star; // [n_warps+1] star partition of the persistent warps (balanced by rows)
  const int64_t* warp_star_f; // same for the fused kernel's warps (kFWarps per CTA)
  int64_t n_rows, n_stars, n_axis, n_att, n_instr, n_sh, n_cols, A0, I0, G0;
  int32_t n_glob, n_constr;
  // constraint entries OWNED by this rank (S:§8(c) O-SHARD), values scaled with A
  const double* cval;       // [n_ce]
  const int64_t* ccol;      // [n_ce] local column
  int64_t n_ce;
  // aprod1 constraint dot chunks (each within one row): row, begin, end into cval/ccol
  const int32_t* ch_row; const int64_t* ch_beg; const int64_t* ch_end; int64_t n_chunks;
  // astro constraint entries grouped by local astro column (CSC): columns [0, 5 n_cs) of stars [0, n_cs)
  int64_t n_cs; const int64_t* cs_ptr; const int32_t* cs_k; const int64_t* cs_e;  // row k, entry index
  // shared-column constraint entries: shared index, constraint row, entry index
  int64_t n_csh; const int64_t* csh_idx; const int32_t* csh_k; const int64_t* csh_e;
  InstrPerm ip;  // IdxRec instrumental fields hold ip.fwd(column); shared-memory arrays have ip.slots() entries
  // shared-column constraint entries grouped by shared column (CSC) over [scs_lo, scs_hi) (rank 0 only)
  int64_t scs_lo, scs_hi; const int64_t* scs_ptr; const int32_t* scs_k; const int64_t* scs_e;
  int32_t f3_zrep, f3_arep;  // k_fused3 launch only: shared-memory accumulator copies (set by its launcher)
  // The fused kernel's attitude gather copy: xatt4[4k + a] = v[A0 + a n_axis + k] for a < 3, [4k + 3] = 0,
  // written by k_colupdate -- a lane's three axis values of knot k0 + j are one 32-B load (LDG.E.ENL2.256).
  double* xatt4;
  // Window format of the same copy when the attitude slice is small enough (n_att <= kZ4MaxAtt; C2, C3):
  // xatt4[16 k0 + 4 j + a] = v[A0 + a n_axis + k0 + j] -- every row's 4 lanes read ONE aligned 128-B line (4x the
  // writes of the knot format, 128 B per knot).  att_kmul = 16 (window) or 4 (knot): a lane's address is
  // xatt4 + att_kmul * k0 + 4 j.
  int32_t att_kmul;
  // Attitude window accumulator of the fused kernel, or nullptr: z4[a][k0][j] (4 doubles per window
  // start k0, 32-B aligned) collects the 4 lanes' REDs of a row in one aligned sector; k_post (P = 1) or k_att_fold
  // (P > 1, the lsqr_aprod2 API) folds it into the attitude columns after each pass and zeroes it.  Used when 4 n_att doubles stay well inside L2 (n_att <= kZ4MaxAtt) and the attitude slice is
  // not privatised in shared memory.
  double* z4;
  int32_t z4_kmul;  // 16: z4[k0][a (4)][j] (window-major, 128 B per window start); 4: z4[a][k0][j]
};
#ifndef LSQR_Z4_MAX_ATT
#define LSQR_Z4_MAX_ATT (1 << 20)
#endif
constexpr int64_t kZ4MaxAtt = LSQR_Z4_MAX_ATT;

enum { AP1_LSQR = 0, AP1_PLAIN = 1 };
enum { AP2_LSQR = 0, AP2_PLAIN = 1, AP2_COLNORM = 2 };

struct GenArgs {
  InstrPerm ip;
  uint64_t seed;
  int32_t b_mode;
  double noise;
  int64_t row_begin_global, star_begin_global;
  int64_t n_stars_global, n_att, n_instr;
  int32_t n_glob;
};

// ---------------------------------------------------------------------------------------------- launchers
// All return cudaGetLastError() of the launch.
cudaError_t launch_generate(const GenArgs& g, double* vals, IdxRec* idx, const int64_t* star_ptr, int64_t n_rows,
                            int64_t n_stars_loc, double* b, cudaStream_t s);
// lsqr_set_system: host-layout chunk -> device layout with validation (err: [1 + first bad row (min), kind])
cudaError_t launch_ingest(const double* sv, const int64_t* smA, const int64_t* smT, const int64_t* siC, int64_t row0,
                          int64_t nrows, const int64_t* star_ptr, int64_t n_stars_loc, int64_t star_begin,
                          int64_t A0g, int64_t I0g, int64_t n_axis, int64_t n_instr, InstrPerm ip, double* vals,
                          IdxRec* idx, unsigned long long* err, cudaStream_t s);
// xg4: the padded knot-major copy of x's attitude slice (launch_att_pack), or nullptr (gathers from x)
cudaError_t launch_aprod1(int mode, const SysView& S, int grid, const double* x, double* y, double* part,
                          double* cpart, const DevState* st, cudaStream_t s, const double* xg4 = nullptr);
cudaError_t launch_aprod2(int mode, const SysView& S, int grid, const double* y, const double* ucn, double* xv,
                          double* zsh, double* part, const DevState* st, int do_shared_constr, cudaStream_t s);
cudaError_t launch_scale_rows(const SysView& S, int grid, double* vals, const double* D, cudaStream_t s);
cudaError_t launch_scale_constr(const SysView& S, double* cval, const double* D, cudaStream_t s);
// u2 partials: sum of squares of u[0..n) in a fixed grid
cudaError_t launch_sumsq(const double* u, int64_t n, double* part, int nblk, cudaStream_t s);
// beta kernel: reduces aprod1 partials + constraint chunks; P>1 split into pre (writes ar1) / post (reads ar1)
cudaError_t launch_beta(int phase, const SysView& S, const double* part, int64_t n_part, const double* cpart,
                        double* ar1, double* uc, double* ucn, const double* crhs, DevState* st, int init,
                        cudaStream_t s);
cudaError_t launch_cdot_add(const SysView& S, const double* cpart, const double* ar1, double* yc, cudaStream_t s);
// fused = 1: z_sh holds A^T u_hat of the fused kernel (unnormalised); 0: A^T u of k_aprod2 (init)
cudaError_t launch_vshared(const SysView& S, double* vsh, double* zsh, double* part, int nblk, const DevState* st,
                           int fused, cudaStream_t s);
// NEXT-1 fused single pass (u_hat update + A^T u_hat in one read of A) and its astro column pass
cudaError_t launch_fused(const SysView& S, int grid, const double* x, double* u, double* zA, double* zsh,
                         double* part, double* cpart, const DevState* st, cudaStream_t s, bool fold = true);
// fold = false (single rank): k_post folds the window accumulator S.z4 into the attitude columns itself
// lsqr_aprod2 after k_fused3<R3_AP2>: x_astro += zA + astro constraint entries . y_c; shared constraint entries -> z_sh
cudaError_t launch_astro_add(const SysView& S, double* x, const double* zA, const double* yc, double* zsh,
                             int do_shared_constr, cudaStream_t s);
// the two-pass iteration's aprod2 on the fused kernel's loop (k_fused3<R3_AP2>): z = A^T u_hat (unnormalised) into
// zA / z_sh, the state the fused pass leaves (every instrumental-slice size: the IG regime covers large ones)
cudaError_t launch_ap2_lean(const SysView& S, int grid, const double* u, double* zA, double* zsh, const DevState* st,
                            cudaStream_t s, bool fold = true);
cudaError_t launch_vastro(const SysView& S, double* v, const double* zA, const double* uc, double* zsh, double* part,
                          int nblk, const DevState* st, int do_shared_constr, cudaStream_t s);
// mode 0: x += z, 1: x = z; z zeroed
cudaError_t launch_add_shared(const SysView& S, double* xsh, double* zsh, int mode, cudaStream_t s);
cudaError_t launch_scalar(DevState* st, const double* part_astro, int64_t n_pa, const double* part_sh,
                          int64_t n_ps, const double* part_wa, int64_t n_pwa, const double* part_ws, int64_t n_pws,
                          const double* ar2_alpha2, const double* ar1_wa, int init, int32_t* host_flag,
                          cudaStream_t s, const double* post_uc = nullptr, double* uc = nullptr,
                          double* ucn = nullptr, int nc = 0);
// single-rank fused mode: beta (recomputed per block) + astro/shared v' + constraint terms in one kernel; also folds
// the row pass's attitude window accumulator S.z4 (the row pass was launched with fold = false)
cudaError_t launch_post(const SysView& S, double* v, const double* zA, double* zsh, const double* part_rows,
                        int64_t n_part, const double* cpart, const double* uc, double* uc_tmp, double* part_a2,
                        int nblk, DevState* st, cudaStream_t s);
// also refreshes the attitude gather copy S.xatt4 from the new v
cudaError_t launch_colupdate(const SysView& S, double* v, double* w, double* x, double* var, double* part_wa,
                             double* part_ws, int nblk, const DevState* st, cudaStream_t s);
// the padded knot-major copy of v's attitude slice into dst (nullptr: S.xatt4, e.g. after lsqr_set_state)
cudaError_t launch_att_pack(const SysView& S, const double* v, cudaStream_t s, double* dst = nullptr);
cudaError_t launch_sum_to(const double* part, int64_t n, double* dst, cudaStream_t s);
cudaError_t launch_precond_D(double* c, int64_t n, cudaStream_t s);
cudaError_t launch_finalize(const double* x, const double* var, const double* D, int64_t n, const DevState* st,
                            double se_t, double* x_out, double* se_out, cudaStream_t s);
cudaError_t launch_fill(double* p, int64_t n, double v, cudaStream_t s);

// NEXT-4 bitwise-reproducible mode (lsqr_repro.cu, docs/REPRO.md).  Digit buffers (int64, zeroed; every step leaves
// what it consumed zeroed; L = repro_digits_per_value()): zd [L][n_cols] digit-major column accumulator;
// sd [repro_sd_size(n_constr)] = [beta^2 (L) | constraint rows (L n_constr) | alpha^2 astro (L) | alpha^2 shared (L) |
// ddnorm astro (L) | ddnorm shared (L)].  The astro parts are rank-local (allreduced when P > 1), the shared parts are computed
// identically on every rank.  u / uc hold u_hat (unnormalised) like the default path; st->inv_beta normalises.
enum { RS_APROD1, RS_BETA, RS_APROD2, RS_VUPDATE, RS_SCALAR_A, RS_COLUPDATE, RS_SCALAR_B, RS_COLNORM, RS_PRECOND_D };
struct ReproArgs {
  SysView S;
  int n_sm, init;
  double *u, *uc, *v, *w, *x, *var, *D;
  const double* crhs;
  long long *zd, *sd;
  DevState* st;
  int32_t* host_flag;
};
int64_t repro_digits_per_value();
int64_t repro_sd_size(int64_t n_constr);
// part 0: [beta^2 | constraint rows] (5 + 5 n_constr contiguous), 1: alpha^2 astro (5), 2: ddnorm astro (5)
long long* repro_sd_part(long long* sd, int64_t n_constr, int part);
cudaError_t repro_step(int step, const ReproArgs& a, cudaStream_t s);
// int64 digits <-> exact double pairs for the allreduce: nval values of L digits, digit q of value i at
// src[q * plane + i] (plane > 0: digit-major planes) or src[i * L + q] (plane == 0); carry-normalised on packing;
// buf holds 2 L nval doubles
cudaError_t repro_pack(const long long* src, int64_t nval, int64_t plane, double* buf, int unpack, cudaStream_t s);
// largest number of terms any digit accumulator may receive on one rank (the exactness bound of the format)
int64_t repro_max_terms();

}  // namespace lsqr

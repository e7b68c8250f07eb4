// lsqr_capi.cu -- host side of liblsqr_avugsr.so: the C ABI of include/lsqr_avugsr.h, the LSQR driver (device-
// resident scalars, CUDA-graph replay of one iteration, stop-flag polling) and the communication layer (NCCL over
// NVLink/NVSwitch, or a host callback).  Product code; independent of oracle/.
#include <dlfcn.h>
#include <nccl.h>

#include <algorithm>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <new>
#include <string>
#include <vector>

#include "lsqr_avugsr.h"
#include "lsqr_internal.cuh"

using namespace lsqr;

namespace {

// ------------------------------------------------------------------------------------------------ NCCL (dlopen)
struct NcclApi {
  bool tried = false, ok = false;
  ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*AllReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                            cudaStream_t) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  const char* (*GetErrorString)(ncclResult_t) = nullptr;
};
NcclApi g_nccl;

bool nccl_load() {
  if (g_nccl.tried) return g_nccl.ok;
  g_nccl.tried = true;
  // libnccl.so.2: torch's bundled copy is already loaded in a torch process; dlopen finds it or the system one.
  void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
  if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
  if (!h) return false;
  g_nccl.GetUniqueId = (decltype(g_nccl.GetUniqueId))dlsym(h, "ncclGetUniqueId");
  g_nccl.CommInitRank = (decltype(g_nccl.CommInitRank))dlsym(h, "ncclCommInitRank");
  g_nccl.AllReduce = (decltype(g_nccl.AllReduce))dlsym(h, "ncclAllReduce");
  g_nccl.CommDestroy = (decltype(g_nccl.CommDestroy))dlsym(h, "ncclCommDestroy");
  g_nccl.GetErrorString = (decltype(g_nccl.GetErrorString))dlsym(h, "ncclGetErrorString");
  g_nccl.ok = g_nccl.GetUniqueId && g_nccl.CommInitRank && g_nccl.AllReduce && g_nccl.CommDestroy;
  return g_nccl.ok;
}

// ------------------------------------------------------------------------------------------------ host synth (O-GEN)
uint64_t h_mix(uint64_t z) {
  z += 0x9E3779B97F4A7C15ULL;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}
uint64_t h_hash(uint64_t seed, uint64_t tag, uint64_t i, uint64_t j) {
  return h_mix(h_mix(h_mix(seed ^ (tag << 56)) ^ i) ^ j);
}
double h_pm1(uint64_t h) { return (double)((int64_t)(h >> 10) - ((int64_t)1 << 53)) * 0x1p-53; }

constexpr int kG1 = 148 * 4;  // sumsq partial blocks
constexpr int kG2 = 148 * 2;  // vshared partial blocks
constexpr int kG3 = 148 * 4;  // colupdate partial blocks
constexpr int64_t kChunk = 256;

}  // namespace

// ------------------------------------------------------------------------------------------------ handle
struct lsqr_ctx {
  // dims (global)
  int64_t n_stars = 0, n_obs = 0, n_att = 0, n_instr = 0, n_axis = 0, n_cols_g = 0, A0g = 0, I0g = 0, G0g = 0;
  int32_t n_glob = 0;
  // rank
  int32_t rank = 0, nranks = 1, device = 0, comm_kind = 0;
  bool multi = false;  // multi-rank algorithm + collectives (nranks > 1, or env->force_collectives)
  int64_t star_begin = 0, star_end = 0, row_begin = 0, row_end = 0;
  int64_t n_loc_stars = 0, n_loc_rows = 0, n_sh = 0, n_loc_cols = 0, n_constr = 0;
  std::vector<int64_t> counts;       // obs per star (global)
  std::vector<int64_t> star_ptr_h;   // local
  // env
  lsqr_alloc_fn alloc = nullptr;
  lsqr_free_fn free = nullptr;
  void* alloc_user = nullptr;
  lsqr_allreduce_fn cb_allreduce = nullptr;
  void* cb_user = nullptr;
  cudaStream_t user_stream = 0, s = 0;
  cudaEvent_t ev_sync = nullptr;
  ncclComm_t nccl = nullptr;
  int n_sm = 148, grid = 148;
  int64_t W = 0;  // warps of the persistent row kernels
  // device buffers
  std::vector<void*> allocs;
  double *vals = nullptr, *u = nullptr, *v = nullptr, *w = nullptr, *x = nullptr, *var = nullptr, *D = nullptr;
  double *zsh = nullptr, *part_rows = nullptr, *part_a2 = nullptr, *cpart = nullptr, *part_sh = nullptr;
  double *zA = nullptr, *part_va = nullptr;
  double* xatt4 = nullptr;      // the attitude gather copy of v (S.xatt4), kept by k_colupdate
  double* xatt4_api = nullptr;  // lsqr_aprod1's gather copy of its x (allocated on first use; pad entries unused)
  double* z4 = nullptr;         // attitude window accumulator of the fused kernel (S.z4), or nullptr
  int32_t att_kmul = 4;         // gather-copy format (S.att_kmul): 4 knot, 16 window
  int32_t z4_kmul = 4;          // window-accumulator layout (S.z4_kmul)
  double* ingest = nullptr;  // lsqr_set_system staging (lazily allocated)
  double* uc_tmp = nullptr;  // k_post -> k_scalar constraint u_hat hand-over  // fused mode: astro z (A^T u_hat) and alpha^2 partials of k_vastro
  double *part_wa = nullptr, *part_ws = nullptr, *part_g1 = nullptr, *ar1 = nullptr, *uc = nullptr,
         *ucn = nullptr, *crhs = nullptr, *tmp = nullptr, *tmax = nullptr;
  IdxRec* idx = nullptr;
  int64_t *star_ptr = nullptr, *warp_star = nullptr, *warp_star_f = nullptr;
  DevState* st = nullptr;
  DevState* st_api = nullptr;  // never-halted state for the lsqr_aprod2 API call on the fused kernel's loop
  int32_t* hflag = nullptr;  // host-mapped
  int32_t* hflag_dev = nullptr;
  SysView S{};
  // constraint host copies (owned entries, unscaled) to restore the raw system on regenerate / set_system
  int64_t n_ce = 0;
  std::vector<double> cval_raw;
  // state
  bool poisoned = false, have_system = false, b_valid = false, preconditioned = false, initialized = false;
  int64_t n_enq = 0;        // iterations enqueued since lsqr_init (lsqr_iterate's stop-flag bookkeeping)
  int64_t itn_at_init = 0;  // device itn after lsqr_init (0; lsqr_set_state may change it)
  lsqr_solve_params params{};
  cudaGraphExec_t gexec = nullptr;
  bool graph_ok = false;
  // NEXT-4 bitwise-reproducible mode: digit buffers (lsqr_repro.cu)
  bool repro = false;
  long long *rzd = nullptr, *rsd = nullptr;
  double* rbuf = nullptr;  // digit allreduce staging (P > 1)
  std::string err;
};

namespace {

int fail(lsqr_t h, int code, const char* fmt, ...) {
  if (h) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    h->err = buf;
    if (code == LSQR_ECUDA || code == LSQR_ENCCL || code == LSQR_ECOMM) h->poisoned = true;
  }
  return code;
}

#define CKC(h, expr)                                                                                    \
  do {                                                                                                  \
    cudaError_t e_ = (expr);                                                                            \
    if (e_ != cudaSuccess) return fail(h, LSQR_ECUDA, "%s: %s (%s:%d)", #expr, cudaGetErrorString(e_), \
                                       __FILE__, __LINE__);                                             \
  } while (0)

#define GUARD(h)                                                                \
  do {                                                                          \
    if (!(h)) return LSQR_EINVAL;                                               \
    if ((h)->poisoned) return LSQR_ESTATE;                                      \
    if (cudaSetDevice((h)->device) != cudaSuccess) return fail(h, LSQR_ECUDA, "cudaSetDevice"); \
  } while (0)

template <class T>
int dalloc(lsqr_t h, T** p, int64_t count) {
  size_t bytes = (size_t)std::max<int64_t>(count, 1) * sizeof(T);
  bytes = (bytes + 255) & ~(size_t)255;
  void* q = nullptr;
  if (h->alloc) {
    q = h->alloc(bytes, h->alloc_user);
    if (!q) return fail(h, LSQR_ENOMEM, "alloc hook failed for %zu bytes", bytes);
  } else {
    cudaError_t e = cudaMalloc(&q, bytes);
    if (e != cudaSuccess) {
      cudaGetLastError();
      return fail(h, LSQR_ENOMEM, "cudaMalloc(%zu) failed: %s", bytes, cudaGetErrorString(e));
    }
  }
  h->allocs.push_back(q);
  *p = (T*)q;
  return LSQR_OK;
}

// stream ordering with the caller's stream
void enter(lsqr_t h) {
  cudaEventRecord(h->ev_sync, h->user_stream);
  cudaStreamWaitEvent(h->s, h->ev_sync, 0);
}
void leave(lsqr_t h) {
  cudaEventRecord(h->ev_sync, h->s);
  cudaStreamWaitEvent(h->user_stream, h->ev_sync, 0);
}

// in-place SUM allreduce of count doubles on the library stream (no-op on one rank)
int allreduce(lsqr_t h, double* buf, int64_t count) {
  if (!h->multi || count == 0) return LSQR_OK;
  if (h->comm_kind == LSQR_COMM_NCCL) {
    ncclResult_t r = g_nccl.AllReduce(buf, buf, (size_t)count, ncclFloat64, ncclSum, h->nccl, h->s);
    if (r != ncclSuccess)
      return fail(h, LSQR_ENCCL, "ncclAllReduce: %s", g_nccl.GetErrorString ? g_nccl.GetErrorString(r) : "?");
    return LSQR_OK;
  }
  CKC(h, cudaStreamSynchronize(h->s));
  int rc = h->cb_allreduce(buf, count, (uint64_t)(uintptr_t)h->s, h->cb_user);
  if (rc != 0) return fail(h, LSQR_ECOMM, "allreduce callback returned %d", rc);
  return LSQR_OK;
}

bool is_device_ptr(const void* p) {
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

void synth_counts(uint64_t seed, int64_t n_stars, int64_t n_obs, int32_t pct, int64_t* c) {
  const int64_t q = n_obs / n_stars, rem = n_obs % n_stars;
  for (int64_t s = 0; s < n_stars; ++s) c[s] = q + (s < rem ? 1 : 0);
  int64_t J = (q * (int64_t)pct) / 100;
  if (q == 0) J = 0;
  else if (q - J < 1) J = q - 1;
  if (J <= 0) return;
  for (int64_t p = 0; 2 * p + 1 < n_stars; ++p) {
    const int64_t d = (int64_t)(h_hash(seed, 1, (uint64_t)p, 0) % (uint64_t)(2 * J + 1)) - J;
    c[2 * p] += d;
    c[2 * p + 1] -= d;
  }
}

void shard_map(const int64_t* row_ptr, int64_t n_stars, int64_t n_obs, int32_t P, int64_t* sb) {
  sb[0] = 0;
  for (int32_t r = 1; r < P; ++r) {
    const int64_t target = ((int64_t)r * n_obs) / P;
    sb[r] = std::lower_bound(row_ptr, row_ptr + n_stars + 1, target) - row_ptr;
  }
  sb[P] = n_stars;
}

int launch_ok(lsqr_t h, cudaError_t e, const char* what) {
  if (e != cudaSuccess) return fail(h, LSQR_ECUDA, "launch %s: %s", what, cudaGetErrorString(e));
  return LSQR_OK;
}
#define CKL(h, expr, what)                      \
  do {                                          \
    int r_ = launch_ok(h, (expr), what);        \
    if (r_ != LSQR_OK) return r_;               \
  } while (0)
#define CKR(expr)                               \
  do {                                          \
    int r_ = (expr);                            \
    if (r_ != LSQR_OK) return r_;               \
  } while (0)

// ------------------------------------------------------------------------------------------------ repro mode
// NEXT-4: allreduce of int64 digits as exact double pairs (no-op on one rank)
// nval values of L digits: digit-major planes of stride `plane`, or (plane == 0) L consecutive digits per value
int repro_allreduce(lsqr_t h, long long* src, int64_t nval, int64_t plane) {
  if (!h->multi || nval == 0) return LSQR_OK;
  CKL(h, repro_pack(src, nval, plane, h->rbuf, 0, h->s), "repro_pack");
  CKR(allreduce(h, h->rbuf, 2 * repro_digits_per_value() * nval));
  CKL(h, repro_pack(src, nval, plane, h->rbuf, 1, h->s), "repro_unpack");
  return LSQR_OK;
}

ReproArgs repro_args(lsqr_t h, int init) {
  ReproArgs a;
  a.S = h->S; a.n_sm = h->n_sm; a.init = init;
  a.u = h->u; a.uc = h->uc; a.v = h->v; a.w = h->w; a.x = h->x; a.var = h->var; a.D = h->D; a.crhs = h->crhs;
  a.zd = h->rzd; a.sd = h->rsd; a.st = h->st; a.host_flag = h->hflag_dev;
  return a;
}

// One reproducible iteration (init: O-1).  P > 1: four exact digit allreduces -- [beta^2 | constraint rows] before
// beta, the shared slice of zd before the v update, the astro alpha^2 and ddnorm digits before the scalar steps.
int enqueue_repro(lsqr_t h, int init) {
  const ReproArgs a = repro_args(h, init);
  const int64_t nc = h->n_constr;
  cudaStream_t s = h->s;
  CKL(h, repro_step(RS_APROD1, a, s), "repro_aprod1");
  CKR(repro_allreduce(h, repro_sd_part(h->rsd, nc, 0), 1 + nc, 0));
  CKL(h, repro_step(RS_BETA, a, s), "repro_beta");
  CKL(h, repro_step(RS_APROD2, a, s), "repro_aprod2");
  CKR(repro_allreduce(h, h->rzd + h->S.A0, h->n_sh, h->n_loc_cols));
  CKL(h, repro_step(RS_VUPDATE, a, s), "repro_vupdate");
  CKR(repro_allreduce(h, repro_sd_part(h->rsd, nc, 1), 1, 0));
  CKL(h, repro_step(RS_SCALAR_A, a, s), "repro_scalar_a");
  CKL(h, repro_step(RS_COLUPDATE, a, s), "repro_colupdate");
  if (init) return LSQR_OK;
  CKR(repro_allreduce(h, repro_sd_part(h->rsd, nc, 2), 1, 0));
  CKL(h, repro_step(RS_SCALAR_B, a, s), "repro_scalar_b");
  return LSQR_OK;
}

// ------------------------------------------------------------------------------------------------ iteration
// One LSQR iteration, all stream-ordered on h->s.  timing: optional events around the two
// products ([0..1] aprod1 or the fused row pass, [2..3] aprod2 or the column pass after the fused row pass).
// Both variants leave the same state after their row pass(es) -- z = A^T u_hat with the UNNORMALISED u_hat in zA
// (astro) and z_sh (shared slice) -- and finish with the same kernels (v' = z / beta - beta v, scalars, column update):
//   fused (NEXT-1, default): k_fused3<R3_FUSED> reads A once (u_hat update and A^T u_hat in one pass);
//   two-pass (the paper's structure): k_aprod1, then k_fused3<R3_AP2> (aprod2 on the fused kernel's loop).
int enqueue_iteration(lsqr_t h, cudaEvent_t* ev) {
  SysView& S = h->S;
  cudaStream_t s = h->s;
  const bool multi = h->multi;
  const bool fused = h->params.two_pass == 0;
  if (h->repro) {  // NEXT-4: 7 launches (+ 4 x pack/unpack when P > 1), all in lsqr_repro.cu
    if (ev) cudaEventRecord(ev[0], s);
    CKR(enqueue_repro(h, 0));
    if (ev) for (int k = 1; k < 4; ++k) cudaEventRecord(ev[k], s);
    return LSQR_OK;
  }
  if (ev) cudaEventRecord(ev[0], s);
  if (fused) {
    CKL(h, launch_fused(S, h->grid, h->v, h->u, h->zA, h->zsh, h->part_rows, h->cpart, h->st, s, multi), "fused");
  } else {
    CKL(h, launch_aprod1(AP1_LSQR, S, h->grid, h->v, h->u, h->part_rows, h->cpart, h->st, s, h->xatt4), "aprod1");
  }
  if (ev) cudaEventRecord(ev[1], s);
  if (!fused) {
    if (ev) cudaEventRecord(ev[2], s);
    CKL(h, launch_ap2_lean(S, h->grid, h->u, h->zA, h->zsh, h->st, s, multi), "aprod2");
    if (ev) cudaEventRecord(ev[3], s);
  }
  const int64_t n_b2 = fused ? h->grid : h->W;  // k_fused3 publishes one beta^2 partial per CTA, k_aprod1 per warp
  if (!multi) {  // fused: 4 launches (rows, post = z4 fold + beta + v' everywhere, scalar, column update); two-pass: 5
    if (ev && fused) cudaEventRecord(ev[2], s);
    CKL(h, launch_post(S, h->v, h->zA, h->zsh, h->part_rows, n_b2, h->cpart, h->uc, h->uc_tmp, h->part_va, kG3,
                       h->st, s), "post");
    if (ev && fused) cudaEventRecord(ev[3], s);
    CKL(h, launch_scalar(h->st, h->part_va, kG3, nullptr, 0, h->part_wa, kG3, h->part_ws, kG3, nullptr, nullptr, 0,
                         h->hflag_dev, s, h->uc_tmp, h->uc, h->ucn, (int)h->n_constr), "scalar");
    CKL(h, launch_colupdate(S, h->v, h->w, h->x, h->var, h->part_wa, h->part_ws, kG3, h->st, s),
        "colupdate");
    return LSQR_OK;
  }
  // P > 1: beta needs AR1 = [constraint dots | beta^2 local | ||w_astro||^2 local]
  CKL(h, launch_beta(1, S, h->part_rows, n_b2, h->cpart, h->ar1, h->uc, h->ucn, h->crhs, h->st, 0, s), "beta1");
  CKL(h, launch_sum_to(h->part_wa, kG3, h->ar1 + h->n_constr + 1, s), "wsum");
  CKR(allreduce(h, h->ar1, h->n_constr + 2));
  CKL(h, launch_beta(2, S, h->part_rows, n_b2, h->cpart, h->ar1, h->uc, h->ucn, h->crhs, h->st, 0, s), "beta2");
  if (ev && fused) cudaEventRecord(ev[2], s);
  CKL(h, launch_vastro(S, h->v, h->zA, h->uc, h->zsh, h->part_va, kG3, h->st, h->rank == 0, s), "vastro");
  if (ev && fused) cudaEventRecord(ev[3], s);
  // AR2 payload: [z_att | z_instr | z_glob | alpha^2 astro local]
  CKL(h, launch_sum_to(h->part_va, kG3, h->zsh + h->n_sh, s), "a2sum");
  CKR(allreduce(h, h->zsh, h->n_sh + 1));
  CKL(h, launch_vshared(S, h->v + S.A0, h->zsh, h->part_sh, kG2, h->st, 1, s), "vshared");
  CKL(h, launch_scalar(h->st, h->part_va, kG3, h->part_sh, kG2, h->part_wa, kG3, h->part_ws, kG3, h->zsh + h->n_sh,
                       h->ar1 + h->n_constr + 1, 0, h->hflag_dev, s),
      "scalar");
  CKL(h, launch_colupdate(S, h->v, h->w, h->x, h->var, h->part_wa, h->part_ws, kG3, h->st, s),
      "colupdate");
  return LSQR_OK;
}

int kernels_per_iteration(lsqr_t h) {
  if (h->repro) return h->multi ? 15 : 7;
  const int fold = h->z4 && h->multi ? 1 : 0;  // k_att_fold after the row pass (P = 1: folded by k_post)
  if (!h->params.two_pass) return (h->multi ? 9 : 4) + fold;
  return (h->multi ? 10 : 5) + fold;
}

int build_graph(lsqr_t h) {
  if (h->gexec) {
    cudaGraphExecDestroy(h->gexec);
    h->gexec = nullptr;
  }
  h->graph_ok = false;
  if (h->multi && h->comm_kind == LSQR_COMM_CALLBACK) return LSQR_OK;  // host callback: no capture
  cudaGraph_t g = nullptr;
  CKC(h, cudaStreamBeginCapture(h->s, cudaStreamCaptureModeThreadLocal));
  int rc = enqueue_iteration(h, nullptr);
  cudaError_t e = cudaStreamEndCapture(h->s, &g);
  if (rc != LSQR_OK) {
    if (g) cudaGraphDestroy(g);
    return rc;
  }
  if (e != cudaSuccess) return fail(h, LSQR_ECUDA, "graph capture: %s", cudaGetErrorString(e));
  e = cudaGraphInstantiate(&h->gexec, g, 0);
  cudaGraphDestroy(g);
  if (e != cudaSuccess) return fail(h, LSQR_ECUDA, "graph instantiate: %s", cudaGetErrorString(e));
  h->graph_ok = true;
  return LSQR_OK;
}

}  // namespace

// ================================================================================================ C ABI
extern "C" {

int lsqr_abi_version(void) { return LSQR_ABI_VERSION; }

#ifndef LSQR_SOURCE_HASH
#define LSQR_SOURCE_HASH "0000000000000000"
#endif
// the marker lets build.py read the id from the .so file without loading it
static const char kBuildId[] = "LSQR_BUILD_ID=" LSQR_SOURCE_HASH;
const char* lsqr_build_id(void) { return kBuildId + 14; }

const char* lsqr_strerror(int status) {
  switch (status) {
    case LSQR_OK: return "ok";
    case LSQR_EINVAL: return "invalid argument";
    case LSQR_ENOMEM: return "out of memory";
    case LSQR_ECUDA: return "CUDA error";
    case LSQR_ENCCL: return "NCCL error";
    case LSQR_ESTATE: return "invalid state (call order, consumed b, or poisoned handle)";
    case LSQR_EUNSORTED: return "rows not grouped by star / inconsistent with obs_per_star";
    case LSQR_ECOMM: return "allreduce callback failed";
    default: return "unknown status";
  }
}

const char* lsqr_last_error(lsqr_t h) { return h ? h->err.c_str() : "null handle"; }

int lsqr_synth_obs_per_star(uint64_t seed, int64_t n_stars, int64_t n_obs, int32_t jitter_pct, int64_t* counts) {
  if (n_stars <= 0 || n_obs < 0 || jitter_pct < 0 || jitter_pct > 100 || !counts) return LSQR_EINVAL;
  synth_counts(seed, n_stars, n_obs, jitter_pct, counts);
  return LSQR_OK;
}

int64_t lsqr_synth_constraints(uint64_t seed, int64_t n_stars, int64_t n_att, int64_t n_instr, int64_t n_ext,
                               int64_t* row_ptr, int64_t* col, double* val) {
  if (n_stars <= 0 || n_att <= 0 || n_instr < 6 || n_instr % 6 || n_ext < 0) return LSQR_EINVAL;
  const int64_t ns = std::min(n_ext, n_stars), g = n_instr / 6, I0 = 5 * n_stars + n_att;
  int64_t e = 0;
  if (row_ptr) row_ptr[0] = 0;
  for (int k = 0; k < 6; ++k) {
    for (int64_t s = 0; s < ns; ++s)
      for (int a = 0; a < 5; ++a, ++e)
        if (col) {
          col[e] = 5 * s + a;
          val[e] = h_pm1(h_hash(seed, 8, (uint64_t)k, (uint64_t)(5 * s + a)));
        }
    if (row_ptr) row_ptr[k + 1] = e;
  }
  for (int j = 0; j < 6; ++j) {
    for (int64_t t = 0; t < g; ++t, ++e)
      if (col) {
        col[e] = I0 + j * g + t;
        val[e] = 1.0;
      }
    if (row_ptr) row_ptr[7 + j] = e;
  }
  return e;
}

int lsqr_shard_map(const int64_t* counts, int64_t n_stars, int64_t n_obs, int32_t nranks, int64_t* star_begin) {
  if (!counts || !star_begin || n_stars <= 0 || nranks < 1) return LSQR_EINVAL;
  std::vector<int64_t> rp(n_stars + 1, 0);
  for (int64_t s = 0; s < n_stars; ++s) {
    if (counts[s] < 0) return LSQR_EINVAL;
    rp[s + 1] = rp[s] + counts[s];
  }
  if (rp[n_stars] != n_obs) return LSQR_EINVAL;
  shard_map(rp.data(), n_stars, n_obs, nranks, star_begin);
  return LSQR_OK;
}

int lsqr_nccl_unique_id(uint8_t out[128]) {
  if (!out) return LSQR_EINVAL;
  if (!nccl_load()) return LSQR_ENCCL;
  ncclUniqueId id;
  if (g_nccl.GetUniqueId(&id) != ncclSuccess) return LSQR_ENCCL;
  memcpy(out, id.internal, 128);
  return LSQR_OK;
}

int lsqr_destroy(lsqr_t h) {
  if (!h) return LSQR_OK;
  cudaSetDevice(h->device);
  if (h->s) cudaStreamSynchronize(h->s);
  if (h->gexec) cudaGraphExecDestroy(h->gexec);
  if (h->nccl && g_nccl.CommDestroy) g_nccl.CommDestroy(h->nccl);
  for (void* p : h->allocs) {
    if (h->free) h->free(p, h->alloc_user);
    else cudaFree(p);
  }
  if (h->hflag) cudaFreeHost(h->hflag);
  if (h->ev_sync) cudaEventDestroy(h->ev_sync);
  if (h->s) cudaStreamDestroy(h->s);
  delete h;
  return LSQR_OK;
}

int lsqr_create(int64_t n_stars, int64_t n_obs, int64_t n_att, int64_t n_instr, int32_t n_glob,
                const int64_t* obs_per_star, const lsqr_constraints* cons, const lsqr_env* env, lsqr_t* out) {
  if (!out) return LSQR_EINVAL;
  *out = nullptr;
  // ---- validation (before any allocation)
  if (!env || n_stars <= 0 || n_obs < 0 || n_att < 12 || n_att % 3 || n_instr < 6 || n_instr > 65536 ||
      (n_glob != 0 && n_glob != 1))
    return LSQR_EINVAL;
  if (env->nranks < 1 || env->rank < 0 || env->rank >= env->nranks) return LSQR_EINVAL;
  if ((env->alloc == nullptr) != (env->free == nullptr)) return LSQR_EINVAL;
  if (env->force_collectives != 0 && env->force_collectives != 1) return LSQR_EINVAL;
  if (env->nranks > 1 || env->force_collectives) {
    if (env->comm_kind == LSQR_COMM_NCCL && !env->nccl_id && env->nranks > 1) return LSQR_EINVAL;
    if (env->comm_kind == LSQR_COMM_CALLBACK && !env->allreduce) return LSQR_EINVAL;
    if (env->comm_kind != LSQR_COMM_NCCL && env->comm_kind != LSQR_COMM_CALLBACK) return LSQR_EINVAL;
  }
  const int64_t n_axis = n_att / 3, A0g = 5 * n_stars, I0g = A0g + n_att, G0g = I0g + n_instr;
  const int64_t n_cols_g = G0g + n_glob;
  if (n_axis > INT32_MAX) return LSQR_EINVAL;
  int64_t nc = 0;
  if (cons && cons->n_rows > 0) {
    if (cons->n_rows > kMaxConstr || !cons->row_ptr || !cons->col || !cons->val) return LSQR_EINVAL;
    if (cons->row_ptr[0] != 0) return LSQR_EINVAL;
    for (int64_t k = 0; k < cons->n_rows; ++k)
      if (cons->row_ptr[k + 1] < cons->row_ptr[k]) return LSQR_EINVAL;
    for (int64_t e = 0; e < cons->row_ptr[cons->n_rows]; ++e)
      if (cons->col[e] < 0 || cons->col[e] >= n_cols_g) return LSQR_EINVAL;
    nc = cons->n_rows;
  }
  std::vector<int64_t> counts(n_stars);
  if (obs_per_star) {
    int64_t tot = 0;
    for (int64_t s = 0; s < n_stars; ++s) {
      if (obs_per_star[s] < 0) return LSQR_EINVAL;
      counts[s] = obs_per_star[s];
      tot += counts[s];
    }
    if (tot != n_obs) return LSQR_EINVAL;
  } else {
    synth_counts(0, n_stars, n_obs, 0, counts.data());
  }

  lsqr_t h = new (std::nothrow) lsqr_ctx();
  if (!h) return LSQR_ENOMEM;
  h->n_stars = n_stars; h->n_obs = n_obs; h->n_att = n_att; h->n_instr = n_instr; h->n_glob = n_glob;
  h->n_axis = n_axis; h->A0g = A0g; h->I0g = I0g; h->G0g = G0g; h->n_cols_g = n_cols_g;
  h->rank = env->rank; h->nranks = env->nranks; h->device = env->device; h->comm_kind = env->comm_kind;
  h->multi = env->nranks > 1 || env->force_collectives == 1;
  h->alloc = env->alloc; h->free = env->free; h->alloc_user = env->alloc_user;
  h->cb_allreduce = env->allreduce; h->cb_user = env->allreduce_user;
  h->user_stream = (cudaStream_t)(uintptr_t)env->stream;
  h->n_constr = nc;
  h->counts.swap(counts);

  auto bail = [&](int rc) {
    lsqr_destroy(h);
    return rc;
  };
  if (cudaSetDevice(h->device) != cudaSuccess) return bail(LSQR_ECUDA);
  if (cudaStreamCreateWithFlags(&h->s, cudaStreamNonBlocking) != cudaSuccess) return bail(LSQR_ECUDA);
  if (cudaEventCreateWithFlags(&h->ev_sync, cudaEventDisableTiming) != cudaSuccess) return bail(LSQR_ECUDA);
  cudaDeviceGetAttribute(&h->n_sm, cudaDevAttrMultiProcessorCount, h->device);
  h->grid = h->n_sm;
  h->W = (int64_t)h->grid * kWarpsPerCta;

  // ---- shard map (O-SHARD)
  std::vector<int64_t> rp(n_stars + 1, 0);
  for (int64_t s = 0; s < n_stars; ++s) rp[s + 1] = rp[s] + h->counts[s];
  std::vector<int64_t> sb(h->nranks + 1);
  shard_map(rp.data(), n_stars, n_obs, h->nranks, sb.data());
  h->star_begin = sb[h->rank];
  h->star_end = sb[h->rank + 1];
  h->row_begin = rp[h->star_begin];
  h->row_end = rp[h->star_end];
  h->n_loc_stars = h->star_end - h->star_begin;
  h->n_loc_rows = h->row_end - h->row_begin;
  h->n_sh = n_att + n_instr + n_glob;
  h->n_loc_cols = 5 * h->n_loc_stars + h->n_sh;
  h->star_ptr_h.resize(h->n_loc_stars + 1);
  for (int64_t s = 0; s <= h->n_loc_stars; ++s) h->star_ptr_h[s] = rp[h->star_begin + s] - h->row_begin;

  // warp partitions: warp w starts at the first star whose rows begin at or after w*n_loc_rows/W (stars whole)
  auto partition = [&](int64_t W) {
    std::vector<int64_t> ws(W + 1);
    for (int64_t w = 0; w < W; ++w) {
      const int64_t target = (int64_t)((__int128)w * h->n_loc_rows / W);
      ws[w] = std::lower_bound(h->star_ptr_h.begin(), h->star_ptr_h.end(), target) - h->star_ptr_h.begin();
      if (ws[w] > h->n_loc_stars) ws[w] = h->n_loc_stars;
    }
    ws[0] = 0;
    ws[W] = h->n_loc_stars;
    return ws;
  };
  std::vector<int64_t> ws = partition(h->W);
  std::vector<int64_t> wsf = partition((int64_t)h->grid * kFWarps);

  // ---- constraint ownership (O-SHARD): astro entries by the star's owner, shared entries by rank 0
  std::vector<double> cval;
  std::vector<int64_t> ccol;
  std::vector<int32_t> ch_row;
  std::vector<int64_t> ch_beg, ch_end;
  std::vector<int64_t> cs_ptr;
  std::vector<int32_t> cs_k;
  std::vector<int64_t> cs_e, csh_idx, csh_e;
  std::vector<int32_t> csh_k;
  std::vector<double> crhs(std::max<int64_t>(nc, 1), 0.0);
  if (nc > 0) {
    const int64_t A0l = 5 * h->n_loc_stars;
    std::vector<std::vector<std::pair<int32_t, int64_t>>> by_col;  // local astro column -> (row k, entry)
    for (int64_t k = 0; k < nc; ++k) {
      if (cons->rhs) crhs[k] = cons->rhs[k];
      const int64_t row_first = (int64_t)cval.size();
      for (int64_t e = cons->row_ptr[k]; e < cons->row_ptr[k + 1]; ++e) {
        const int64_t c = cons->col[e];
        int64_t lc;
        if (c < A0g) {
          if (c < 5 * h->star_begin || c >= 5 * h->star_end) continue;
          lc = c - 5 * h->star_begin;
          if ((int64_t)by_col.size() <= lc) by_col.resize(lc + 1);
          by_col[lc].push_back({(int32_t)k, (int64_t)cval.size()});
        } else {
          if (h->rank != 0) continue;
          lc = A0l + (c - A0g);
          csh_idx.push_back(c - A0g);
          csh_k.push_back((int32_t)k);
          csh_e.push_back((int64_t)cval.size());
        }
        cval.push_back(cons->val[e]);
        ccol.push_back(lc);
      }
      for (int64_t b = row_first; b < (int64_t)cval.size(); b += kChunk) {
        ch_row.push_back((int32_t)k);
        ch_beg.push_back(b);
        ch_end.push_back(std::min<int64_t>(b + kChunk, (int64_t)cval.size()));
      }
    }
    if (!by_col.empty()) by_col.resize(((by_col.size() + 4) / 5) * 5);  // whole stars
    cs_ptr.push_back(0);
    for (auto& v : by_col) {
      for (auto& pr : v) {
        cs_k.push_back(pr.first);
        cs_e.push_back(pr.second);
      }
      cs_ptr.push_back((int64_t)cs_k.size());
    }
  }
  h->n_ce = (int64_t)cval.size();
  h->cval_raw = cval;
  // shared-column constraint entries as a CSC over [scs_lo, scs_hi) of the shared slice (entry order kept)
  int64_t scs_lo = 0, scs_hi = 0;
  std::vector<int64_t> scs_ptr(1, 0), scs_e;
  std::vector<int32_t> scs_k;
  if (!csh_idx.empty()) {
    scs_lo = *std::min_element(csh_idx.begin(), csh_idx.end());
    scs_hi = *std::max_element(csh_idx.begin(), csh_idx.end()) + 1;
    std::vector<std::vector<std::pair<int32_t, int64_t>>> by(scs_hi - scs_lo);
    for (size_t q = 0; q < csh_idx.size(); ++q) by[csh_idx[q] - scs_lo].push_back({csh_k[q], csh_e[q]});
    for (auto& v : by) {
      for (auto& pr : v) {
        scs_k.push_back(pr.first);
        scs_e.push_back(pr.second);
      }
      scs_ptr.push_back((int64_t)scs_k.size());
    }
  }

  // ---- allocations
  int rc = LSQR_OK;
#define AL(p, n) do { rc = dalloc(h, &(p), (n)); if (rc) return bail(rc); } while (0)
  AL(h->vals, h->n_loc_rows * kSlots);
  AL(h->idx, h->n_loc_rows);
  AL(h->u, h->n_loc_rows + 2);
  AL(h->star_ptr, h->n_loc_stars + 1);
  AL(h->warp_star, h->W + 1);
  AL(h->warp_star_f, (int64_t)h->grid * kFWarps + 1);
  AL(h->v, h->n_loc_cols);
  AL(h->w, h->n_loc_cols);
  AL(h->x, h->n_loc_cols);
  AL(h->var, h->n_loc_cols);
  AL(h->D, h->n_loc_cols);
  AL(h->zsh, h->n_sh + 8);
  const bool use_z4 = n_att > 4096 && n_att <= kZ4MaxAtt && !getenv("LSQR_NO_Z4");  // 4096: kSmAttMax (smem copies)
  // z4[a][k0][j] (default); z4[k0][a][j] with LSQR_Z4_WINDOW_MAJOR (measured 3-7 % slower: the three RED instructions
  // of a row then hit one line, serialising in the L2 atomic unit)
  h->z4_kmul = getenv("LSQR_Z4_WINDOW_MAJOR") ? 16 : 4;
  const int64_t z4_n = h->z4_kmul == 16 ? 16 * n_axis : 4 * n_att;
  if (use_z4) AL(h->z4, z4_n);
  h->att_kmul = (n_att <= kZ4MaxAtt && !getenv("LSQR_KNOT_GATHER")) ? 16 : 4;  // window / knot gather format
  AL(h->xatt4, (int64_t)h->att_kmul * n_axis);
  AL(h->part_rows, h->W);
  AL(h->part_a2, h->W);
  AL(h->cpart, std::max<int64_t>((int64_t)ch_row.size(), 1));
  AL(h->part_sh, kG2);
  AL(h->zA, 5 * h->n_loc_stars);
  AL(h->uc_tmp, kMaxConstr);
  AL(h->part_va, kG3);
  AL(h->part_wa, kG3);
  AL(h->part_ws, kG3);
  AL(h->part_g1, kG1);
  AL(h->ar1, nc + 8);
  AL(h->uc, nc + 1);
  AL(h->ucn, nc + 1);
  AL(h->crhs, nc + 1);
  AL(h->tmp, std::max<int64_t>(h->n_loc_cols, nc + 1));
  AL(h->tmax, std::max<int32_t>(h->nranks, 8));
  AL(h->st, 1);
  AL(h->st_api, 1);
  double* d_cval = nullptr;
  int64_t *d_ccol = nullptr, *d_chb = nullptr, *d_che = nullptr, *d_csp = nullptr, *d_cse = nullptr,
          *d_cshi = nullptr, *d_cshe = nullptr;
  int32_t *d_chr = nullptr, *d_csk = nullptr, *d_cshk = nullptr;
  AL(d_cval, h->n_ce);
  AL(d_ccol, h->n_ce);
  AL(d_chr, ch_row.size());
  AL(d_chb, ch_row.size());
  AL(d_che, ch_row.size());
  AL(d_csp, cs_ptr.size());
  AL(d_csk, cs_k.size());
  AL(d_cse, cs_e.size());
  AL(d_cshi, csh_idx.size());
  AL(d_cshk, csh_k.size());
  AL(d_cshe, csh_e.size());
  int64_t *d_scsp = nullptr, *d_scse = nullptr;
  int32_t* d_scsk = nullptr;
  AL(d_scsp, scs_ptr.size());
  AL(d_scsk, scs_k.size());
  AL(d_scse, scs_e.size());
#undef AL
  if (cudaHostAlloc(&h->hflag, sizeof(int32_t) * 4, cudaHostAllocMapped) != cudaSuccess) return bail(LSQR_ENOMEM);
  h->hflag[0] = 0;
  if (cudaHostGetDevicePointer((void**)&h->hflag_dev, h->hflag, 0) != cudaSuccess) return bail(LSQR_ECUDA);

  auto up = [&](void* dst, const void* src, size_t bytes) {
    return bytes == 0 || cudaMemcpy(dst, src, bytes, cudaMemcpyHostToDevice) == cudaSuccess;
  };
  bool ok = up(h->star_ptr, h->star_ptr_h.data(), sizeof(int64_t) * h->star_ptr_h.size()) &&
            up(h->warp_star, ws.data(), sizeof(int64_t) * ws.size()) &&
            up(h->warp_star_f, wsf.data(), sizeof(int64_t) * wsf.size()) &&
            up(d_cval, cval.data(), sizeof(double) * cval.size()) &&
            up(d_ccol, ccol.data(), sizeof(int64_t) * ccol.size()) &&
            up(d_chr, ch_row.data(), sizeof(int32_t) * ch_row.size()) &&
            up(d_chb, ch_beg.data(), sizeof(int64_t) * ch_beg.size()) &&
            up(d_che, ch_end.data(), sizeof(int64_t) * ch_end.size()) &&
            up(d_csp, cs_ptr.data(), sizeof(int64_t) * cs_ptr.size()) &&
            up(d_csk, cs_k.data(), sizeof(int32_t) * cs_k.size()) &&
            up(d_cse, cs_e.data(), sizeof(int64_t) * cs_e.size()) &&
            up(d_cshi, csh_idx.data(), sizeof(int64_t) * csh_idx.size()) &&
            up(d_cshk, csh_k.data(), sizeof(int32_t) * csh_k.size()) &&
            up(d_cshe, csh_e.data(), sizeof(int64_t) * csh_e.size()) &&
            up(d_scsp, scs_ptr.data(), sizeof(int64_t) * scs_ptr.size()) &&
            up(d_scsk, scs_k.data(), sizeof(int32_t) * scs_k.size()) &&
            up(d_scse, scs_e.data(), sizeof(int64_t) * scs_e.size()) &&
            up(h->crhs, crhs.data(), sizeof(double) * nc);
  if (!ok) return bail(LSQR_ECUDA);

  SysView& S = h->S;
  S.vals = h->vals; S.idx = h->idx; S.star_ptr = h->star_ptr; S.warp_star = h->warp_star;
  S.warp_star_f = h->warp_star_f;
  S.n_rows = h->n_loc_rows; S.n_stars = h->n_loc_stars; S.n_axis = n_axis; S.n_att = n_att; S.n_instr = n_instr;
  S.n_sh = h->n_sh; S.n_cols = h->n_loc_cols; S.A0 = 5 * h->n_loc_stars; S.I0 = S.A0 + n_att;
  S.G0 = S.I0 + n_instr; S.n_glob = n_glob; S.n_constr = (int32_t)nc;
  S.cval = d_cval; S.ccol = d_ccol; S.n_ce = h->n_ce;
  S.ch_row = d_chr; S.ch_beg = d_chb; S.ch_end = d_che; S.n_chunks = (int64_t)ch_row.size();
  S.n_cs = cs_ptr.empty() ? 0 : ((int64_t)cs_ptr.size() - 1) / 5; S.cs_ptr = d_csp; S.cs_k = d_csk; S.cs_e = d_cse;
  S.n_csh = (int64_t)csh_idx.size(); S.csh_idx = d_cshi; S.csh_k = d_cshk; S.csh_e = d_cshe;
  S.scs_lo = scs_lo; S.scs_hi = scs_hi; S.scs_ptr = d_scsp; S.scs_k = d_scsk; S.scs_e = d_scse;
  S.xatt4 = h->xatt4;
  S.att_kmul = h->att_kmul;
  S.z4 = h->z4;
  S.z4_kmul = h->z4_kmul;
  {  // bank-grouped instrumental slots only when every row kernel keeps the instrumental slice in shared memory
    InstrPerm probe;
    probe.init(n_instr, true);
    S.ip.init(n_instr, probe.slots() <= kInstrSmemMax && !getenv("LSQR_NO_INSTR_PERM"));  // env: A/B only
  }

  // zero-initialised state
  if (launch_fill(h->zsh, h->n_sh + 8, 0.0, h->s) != cudaSuccess) return bail(LSQR_ECUDA);
  if (launch_fill(h->D, h->n_loc_cols, 1.0, h->s) != cudaSuccess) return bail(LSQR_ECUDA);
  if (launch_fill(h->xatt4, (int64_t)h->att_kmul * n_axis, 0.0, h->s) != cudaSuccess) return bail(LSQR_ECUDA);
  if (h->z4 && launch_fill(h->z4, z4_n, 0.0, h->s) != cudaSuccess) return bail(LSQR_ECUDA);
  for (double* p : {h->v, h->w, h->x, h->var})
    if (launch_fill(p, h->n_loc_cols, 0.0, h->s) != cudaSuccess) return bail(LSQR_ECUDA);
  if (launch_fill(h->u, h->n_loc_rows + 2, 0.0, h->s) != cudaSuccess) return bail(LSQR_ECUDA);
  if (cudaMemsetAsync(h->st, 0, sizeof(DevState), h->s) != cudaSuccess) return bail(LSQR_ECUDA);
  if (cudaMemsetAsync(h->st_api, 0, sizeof(DevState), h->s) != cudaSuccess) return bail(LSQR_ECUDA);
  if (cudaStreamSynchronize(h->s) != cudaSuccess) return bail(LSQR_ECUDA);

  // ---- communicator
  if (h->multi && h->comm_kind == LSQR_COMM_NCCL) {
    if (!nccl_load()) return bail(LSQR_ENCCL);
    ncclUniqueId id;
    if (env->nccl_id) memcpy(id.internal, env->nccl_id, 128);
    else if (g_nccl.GetUniqueId(&id) != ncclSuccess) return bail(LSQR_ENCCL);  // 1-rank test communicator
    if (g_nccl.CommInitRank(&h->nccl, h->nranks, id, h->rank) != ncclSuccess) return bail(LSQR_ENCCL);
  }
  *out = h;
  return LSQR_OK;
}

int lsqr_layout(lsqr_t h, int64_t* L) {
  if (!h || !L) return LSQR_EINVAL;
  L[0] = h->star_begin; L[1] = h->star_end; L[2] = h->row_begin; L[3] = h->row_end; L[4] = h->n_loc_rows;
  L[5] = h->n_loc_cols; L[6] = h->n_constr; L[7] = h->n_sh; L[8] = h->n_obs + h->n_constr; L[9] = h->n_cols_g;
  return LSQR_OK;
}

// A new system replaces a preconditioned one: restore raw constraint values and D = 1.
static int reset_precond(lsqr_t h) {
  if (!h->preconditioned) return LSQR_OK;
  if (h->n_ce)
    CKC(h, cudaMemcpyAsync(const_cast<double*>(h->S.cval), h->cval_raw.data(), sizeof(double) * h->n_ce,
                           cudaMemcpyHostToDevice, h->s));
  CKL(h, launch_fill(h->D, h->n_loc_cols, 1.0, h->s), "fill");
  CKC(h, cudaStreamSynchronize(h->s));
  h->preconditioned = false;
  return LSQR_OK;
}

int lsqr_generate(lsqr_t h, const lsqr_gen_params* p) {
  GUARD(h);
  if (!p || (p->b_mode != 0 && p->b_mode != 1) || h->n_instr % 6 || h->n_axis < 4) return LSQR_EINVAL;
  enter(h);
  CKR(reset_precond(h));
  GenArgs g;
  g.ip = h->S.ip;
  g.seed = p->seed; g.b_mode = p->b_mode; g.noise = p->noise;
  g.row_begin_global = h->row_begin; g.star_begin_global = h->star_begin;
  g.n_stars_global = h->n_stars; g.n_att = h->n_att; g.n_instr = h->n_instr; g.n_glob = h->n_glob;
  CKL(h, launch_generate(g, h->vals, h->idx, h->star_ptr, h->n_loc_rows, h->n_loc_stars, h->u, h->s), "generate");
  leave(h);
  h->have_system = true;
  h->b_valid = true;
  h->initialized = false;
  return LSQR_OK;
}

int lsqr_set_system(lsqr_t h, const double* vals, const int64_t* mA, const int64_t* mT, const int64_t* iC,
                    const double* b) {
  GUARD(h);
  if (!vals || !mA || !mT || !iC || !b) return LSQR_EINVAL;
  const int64_t n = h->n_loc_rows;
  // staging for the device-side conversion (paper layout -> lane-major values + 16-B index records), allocated
  // once: kIngestRows rows of [24 values | mA | mT | 6 instrCol]
  constexpr int64_t kIngestRows = 1 << 18;
  if (!h->ingest) {
    int rc = dalloc(h, &h->ingest, kIngestRows * (kSlots + 8) + 4);
    if (rc) return rc;
  }
  double* sv = h->ingest;
  int64_t* smA = reinterpret_cast<int64_t*>(sv + kIngestRows * kSlots);
  int64_t* smT = smA + kIngestRows;
  int64_t* siC = smT + kIngestRows;
  unsigned long long* err = reinterpret_cast<unsigned long long*>(siC + kIngestRows * 6);
  enter(h);
  CKR(reset_precond(h));
  const unsigned long long err0[2] = {~0ull, 0ull};
  CKC(h, cudaMemcpyAsync(err, err0, sizeof err0, cudaMemcpyHostToDevice, h->s));
  for (int64_t r0 = 0; r0 < n; r0 += kIngestRows) {
    const int64_t nb = std::min(kIngestRows, n - r0);
    CKC(h, cudaMemcpyAsync(sv, vals + r0 * kSlots, sizeof(double) * kSlots * nb, cudaMemcpyHostToDevice, h->s));
    CKC(h, cudaMemcpyAsync(smA, mA + r0, sizeof(int64_t) * nb, cudaMemcpyHostToDevice, h->s));
    CKC(h, cudaMemcpyAsync(smT, mT + r0, sizeof(int64_t) * nb, cudaMemcpyHostToDevice, h->s));
    CKC(h, cudaMemcpyAsync(siC, iC + r0 * 6, sizeof(int64_t) * 6 * nb, cudaMemcpyHostToDevice, h->s));
    CKL(h, launch_ingest(sv, smA, smT, siC, r0, nb, h->star_ptr, h->n_loc_stars, h->star_begin, h->A0g, h->I0g,
                         h->n_axis, h->n_instr, h->S.ip, h->vals, h->idx, err, h->s), "ingest");
  }
  CKC(h, cudaMemcpyAsync(h->u, b, sizeof(double) * n, cudaMemcpyHostToDevice, h->s));
  unsigned long long errh[2];
  CKC(h, cudaMemcpyAsync(errh, err, sizeof errh, cudaMemcpyDeviceToHost, h->s));
  CKC(h, cudaStreamSynchronize(h->s));  // host buffers may be reused on return
  leave(h);
  if (errh[1] != 0) {
    h->have_system = false;
    h->b_valid = false;
    return fail(h, errh[1] == 1 ? LSQR_EUNSORTED : LSQR_EINVAL,
                errh[1] == 1 ? "row %llu: matrixIndexAstro is not 5*star (rows must be grouped by star in order)"
                             : "row %llu: attitude or instrumental column out of range",
                errh[0] - 1);
  }
  h->have_system = true;
  h->b_valid = true;
  h->initialized = false;
  return LSQR_OK;
}

int lsqr_get_system(lsqr_t h, double* vals, int64_t* mA, int64_t* mT, int64_t* iC, double* b) {
  GUARD(h);
  if (!h->have_system) return fail(h, LSQR_ESTATE, "no system");
  if (b && !h->b_valid) return fail(h, LSQR_ESTATE, "b was consumed by a solve");
  const int64_t n = h->n_loc_rows;
  enter(h);
  CKC(h, cudaStreamSynchronize(h->s));
  if (vals) {
    CKC(h, cudaMemcpy(vals, h->vals, sizeof(double) * kSlots * n, cudaMemcpyDeviceToHost));
    double row[kSlots];
    for (int64_t i = 0; i < n; ++i) {  // lane-major -> paper slot order
      for (int p = 0; p < kSlots; ++p) row[slot_of(p % 6, p / 6)] = vals[i * kSlots + p];
      memcpy(vals + i * kSlots, row, sizeof row);
    }
  }
  if (b) CKC(h, cudaMemcpy(b, h->u, sizeof(double) * n, cudaMemcpyDeviceToHost));
  if (mA || mT || iC) {
    std::vector<int64_t> inv(std::max<int64_t>(h->S.ip.slots(), 1), 0);  // shared-memory slot -> column
    for (int64_t c = 0; c < h->n_instr; ++c) inv[h->S.ip.fwd(c)] = c;
    std::vector<IdxRec> rec(std::max<int64_t>(n, 1));
    CKC(h, cudaMemcpy(rec.data(), h->idx, sizeof(IdxRec) * n, cudaMemcpyDeviceToHost));
    for (int64_t s = 0; s < h->n_loc_stars; ++s)
      for (int64_t i = h->star_ptr_h[s]; i < h->star_ptr_h[s + 1]; ++i) {
        if (mA) mA[i] = 5 * (h->star_begin + s);
        if (mT) mT[i] = h->A0g + rec[i].k0;
        if (iC) {
          const uint32_t w3[3] = {rec[i].ic01, rec[i].ic23, rec[i].ic45};
          for (int j = 0; j < 6; ++j) iC[i * 6 + j] = h->I0g + inv[(w3[j / 2] >> ((j & 1) * 16)) & 0xffff];
        }
      }
  }
  leave(h);
  return LSQR_OK;
}

int lsqr_precondition(lsqr_t h) {
  GUARD(h);
  if (!h->have_system) return fail(h, LSQR_ESTATE, "no system");
  if (h->preconditioned) return fail(h, LSQR_ESTATE, "already preconditioned");
  SysView& S = h->S;
  enter(h);
  if (h->repro) {  // NEXT-4: exact column sums of squares
    const ReproArgs a = repro_args(h, 0);
    CKL(h, repro_step(RS_COLNORM, a, h->s), "colnorm_repro");
    CKR(repro_allreduce(h, h->rzd + S.A0, h->n_sh, h->n_loc_cols));
    CKL(h, repro_step(RS_PRECOND_D, a, h->s), "precond_D_repro");
    CKL(h, launch_scale_rows(S, h->grid, h->vals, h->D, h->s), "scale_rows");
    CKL(h, launch_scale_constr(S, const_cast<double*>(S.cval), h->D, h->s), "scale_constr");
    leave(h);
    h->preconditioned = true;
    h->initialized = false;
    return LSQR_OK;
  }
  // c_j = sum a_ij^2: astro columns straight into D, shared slice accumulated in zsh (+ AR), then D = 1/sqrt(c)
  CKL(h, launch_aprod2(AP2_COLNORM, S, h->grid, nullptr, nullptr, h->D, h->zsh, h->part_a2, h->st, h->rank == 0,
                       h->s), "colnorm");
  CKR(allreduce(h, h->zsh, h->n_sh));
  CKL(h, launch_add_shared(S, h->D + S.A0, h->zsh, 1, h->s), "colnorm_sh");
  CKL(h, launch_precond_D(h->D, h->n_loc_cols, h->s), "precond_D");
  CKL(h, launch_scale_rows(S, h->grid, h->vals, h->D, h->s), "scale_rows");
  CKL(h, launch_scale_constr(S, const_cast<double*>(S.cval), h->D, h->s), "scale_constr");
  leave(h);
  h->preconditioned = true;
  h->initialized = false;
  return LSQR_OK;
}

int lsqr_get_precond(lsqr_t h, double* D) {
  GUARD(h);
  if (!D) return LSQR_EINVAL;
  enter(h);
  CKC(h, cudaStreamSynchronize(h->s));
  CKC(h, cudaMemcpy(D, h->D, sizeof(double) * h->n_loc_cols, cudaMemcpyDefault));
  leave(h);
  return LSQR_OK;
}

int lsqr_set_reproducible(lsqr_t h, int32_t on) {
  GUARD(h);
  if (on != 0 && on != 1) return LSQR_EINVAL;
  // exactness bound of the digit format: no accumulator may receive 2^33 terms on one rank (a column gets at most 6
  // terms per row plus its constraint entries; beta^2 one per row; alpha^2 / ddnorm one per column)
  if (on && (6 * h->n_loc_rows + h->n_ce >= repro_max_terms() || h->n_loc_cols >= repro_max_terms()))
    return fail(h, LSQR_EINVAL, "reproducible mode: shard too large for exact digit accumulation (6 rows + "
                                "constraint entries >= 2^33)");
  if (on && !h->rzd) {
    const int64_t L = repro_digits_per_value();
    CKR(dalloc(h, &h->rzd, L * h->n_loc_cols));
    CKR(dalloc(h, &h->rsd, repro_sd_size(h->n_constr)));
    if (h->multi) CKR(dalloc(h, &h->rbuf, 2 * std::max<int64_t>(L * h->n_sh, repro_sd_size(h->n_constr))));
    CKC(h, cudaMemset(h->rzd, 0, sizeof(long long) * L * h->n_loc_cols));
    CKC(h, cudaMemset(h->rsd, 0, sizeof(long long) * repro_sd_size(h->n_constr)));
  }
  h->repro = on != 0;
  h->initialized = false;
  return LSQR_OK;
}

int lsqr_aprod1(lsqr_t h, const double* x_dev, double* y_dev) {
  GUARD(h);
  if (!x_dev || !y_dev) return LSQR_EINVAL;
  if (!h->have_system) return fail(h, LSQR_ESTATE, "no system");
  SysView& S = h->S;
  enter(h);
  // the attitude slice of x in the padded knot-major layout (32 B per knot, <= 32 MB), then one 256-bit load per lane
  if (!h->xatt4_api) CKR(dalloc(h, &h->xatt4_api, (int64_t)h->att_kmul * h->n_axis));
  CKL(h, launch_att_pack(S, x_dev, h->s, h->xatt4_api), "att_pack");
  CKL(h, launch_aprod1(AP1_PLAIN, S, h->grid, x_dev, y_dev, h->part_rows, h->cpart, h->st, h->s, h->xatt4_api),
      "aprod1");
  if (h->n_constr > 0) {
    if (!h->multi) {
      CKL(h, launch_cdot_add(S, h->cpart, nullptr, y_dev + h->n_loc_rows, h->s), "cdot");
    } else {
      CKL(h, launch_beta(3, S, nullptr, 0, h->cpart, h->ar1, h->uc, h->ucn, h->crhs, h->st, 0, h->s), "cdot1");
      CKR(allreduce(h, h->ar1, h->n_constr));
      CKL(h, launch_cdot_add(S, nullptr, h->ar1, y_dev + h->n_loc_rows, h->s), "cdot2");
    }
  }
  leave(h);
  return LSQR_OK;
}

int lsqr_aprod2(lsqr_t h, const double* y_dev, double* x_dev) {
  GUARD(h);
  if (!x_dev || !y_dev) return LSQR_EINVAL;
  if (!h->have_system) return fail(h, LSQR_ESTATE, "no system");
  SysView& S = h->S;
  enter(h);
  // rows on the fused kernel's loop (its halted flag comes from st_api, a DevState that is never halted), then the
  // astro columns and constraint entries
  CKL(h, launch_ap2_lean(S, h->grid, y_dev, h->zA, h->zsh, h->st_api, h->s), "aprod2");
  CKL(h, launch_astro_add(S, x_dev, h->zA, y_dev + h->n_loc_rows, h->zsh, h->rank == 0, h->s), "aprod2_astro");
  CKR(allreduce(h, h->zsh, h->n_sh));
  CKL(h, launch_add_shared(S, x_dev + S.A0, h->zsh, 0, h->s), "aprod2_sh");
  leave(h);
  return LSQR_OK;
}

int lsqr_init(lsqr_t h, const lsqr_solve_params* p) {
  GUARD(h);
  if (!p || p->itn_limit < 0 || p->atol < 0 || p->btol < 0 || p->conlim < 0 || p->damp < 0) return LSQR_EINVAL;
  if (!h->have_system) return fail(h, LSQR_ESTATE, "no system");
  if (!h->b_valid) return fail(h, LSQR_ESTATE, "b was consumed by a previous solve; regenerate or set_system");
  h->params = *p;
  if (h->params.poll_every <= 0) h->params.poll_every = 16;
  h->n_enq = 0;
  h->itn_at_init = 0;
  SysView& S = h->S;
  const bool multi = h->multi;
  enter(h);
  DevState st0;
  memset(&st0, 0, sizeof st0);
  st0.damp = p->damp; st0.atol = p->atol; st0.btol = p->btol; st0.ctol = p->conlim > 0 ? 1.0 / p->conlim : 0.0;
  st0.itn_limit = (int32_t)std::min<int64_t>(p->itn_limit, INT32_MAX);
  st0.fixed_count = p->fixed_count ? 1 : 0;
  st0.inv_beta = 1.0;
  CKC(h, cudaMemcpyAsync(h->st, &st0, sizeof st0, cudaMemcpyHostToDevice, h->s));
  for (double* q : {h->v, h->w, h->x, h->var}) CKL(h, launch_fill(q, h->n_loc_cols, 0.0, h->s), "fill");
  CKL(h, launch_fill(h->zsh, h->n_sh + 8, 0.0, h->s), "fill");
  if (h->z4)  // the window accumulator is clean after every pass; re-zeroed here in case a solve ended mid-pass
    CKL(h, launch_fill(h->z4, h->z4_kmul == 16 ? 16 * h->S.n_axis : 4 * h->S.n_att, 0.0, h->s), "fill");
  if (h->repro) {  // NEXT-4 O-1
    CKC(h, cudaMemsetAsync(h->rzd, 0, sizeof(long long) * repro_digits_per_value() * h->n_loc_cols, h->s));
    CKC(h, cudaMemsetAsync(h->rsd, 0, sizeof(long long) * repro_sd_size(h->n_constr), h->s));
    CKR(enqueue_repro(h, 1));
    h->b_valid = false;
    h->initialized = true;
    if (p->use_graph) CKR(build_graph(h));
    else if (h->gexec) { cudaGraphExecDestroy(h->gexec); h->gexec = nullptr; h->graph_ok = false; }
    leave(h);
    return LSQR_OK;
  }
  // O-1: u = b, beta = ||u|| (constraint rows: u_c = rhs)
  CKL(h, launch_sumsq(h->u, h->n_loc_rows, h->part_g1, kG1, h->s), "sumsq");
  if (!multi) {
    CKL(h, launch_beta(0, S, h->part_g1, kG1, h->cpart, h->ar1, h->uc, h->ucn, h->crhs, h->st, 1, h->s), "beta0");
  } else {
    CKL(h, launch_beta(1, S, h->part_g1, kG1, h->cpart, h->ar1, h->uc, h->ucn, h->crhs, h->st, 1, h->s), "beta0a");
    CKL(h, launch_fill(h->ar1 + h->n_constr + 1, 1, 0.0, h->s), "fill");
    CKR(allreduce(h, h->ar1, h->n_constr + 2));
    CKL(h, launch_beta(2, S, h->part_g1, kG1, h->cpart, h->ar1, h->uc, h->ucn, h->crhs, h->st, 1, h->s), "beta0b");
  }
  // v = A^T u (v = 0, so the LSQR-mode update v' = z - beta*0 = z)
  CKL(h, launch_aprod2(AP2_LSQR, S, h->grid, h->u, h->ucn, h->v, h->zsh, h->part_a2, h->st, h->rank == 0, h->s),
      "aprod2");
  if (multi) {
    CKL(h, launch_sum_to(h->part_a2, h->W, h->zsh + h->n_sh, h->s), "a2sum");
    CKR(allreduce(h, h->zsh, h->n_sh + 1));
  }
  CKL(h, launch_vshared(S, h->v + S.A0, h->zsh, h->part_sh, kG2, h->st, 0, h->s), "vshared");
  CKL(h, launch_scalar(h->st, h->part_a2, h->W, h->part_sh, kG2, h->part_wa, kG3, h->part_ws, kG3,
                       multi ? h->zsh + h->n_sh : nullptr, nullptr, 1, h->hflag_dev, h->s),
      "scalar0");
  CKL(h, launch_colupdate(S, h->v, h->w, h->x, h->var, h->part_wa, h->part_ws, kG3, h->st, h->s),
      "colupdate0");
  h->b_valid = false;
  h->initialized = true;
  if (p->use_graph) CKR(build_graph(h));
  else if (h->gexec) { cudaGraphExecDestroy(h->gexec); h->gexec = nullptr; h->graph_ok = false; }
  leave(h);
  return LSQR_OK;
}

int lsqr_iterate(lsqr_t h, int64_t n_iter) {
  GUARD(h);
  if (!h->initialized) return fail(h, LSQR_ESTATE, "lsqr_init first");
  if (n_iter <= 0) return LSQR_OK;
  enter(h);
  const int64_t k = h->params.poll_every;
  cudaEvent_t evs[2];
  CKC(h, cudaEventCreateWithFlags(&evs[0], cudaEventDisableTiming));
  CKC(h, cudaEventCreateWithFlags(&evs[1], cudaEventDisableTiming));
  int64_t done = 0, batch = 0;
  int64_t enq_end[2] = {0, 0};  // iterations enqueued since lsqr_init at the end of batch b (slot b & 1)
  int rc = LSQR_OK;
  while (done < n_iter && rc == LSQR_OK) {
    const int64_t nb = std::min(k, n_iter - done);
    for (int64_t i = 0; i < nb && rc == LSQR_OK; ++i) {
      if (h->graph_ok) {
        cudaError_t e = cudaGraphLaunch(h->gexec, h->s);
        if (e != cudaSuccess) rc = fail(h, LSQR_ECUDA, "cudaGraphLaunch: %s", cudaGetErrorString(e));
      } else {
        rc = enqueue_iteration(h, nullptr);
      }
    }
    done += nb;
    h->n_enq += nb;
    enq_end[batch & 1] = h->n_enq;
    cudaEventRecord(evs[batch & 1], h->s);
    if (batch > 0) {  // wait for the previous batch, then poll the stop flag (device-written, host-mapped)
      cudaEventSynchronize(evs[(batch - 1) & 1]);
      // The flag is written by every scalar step, so it may already come from batch b, still running.  Stop only on
      // a halt that happened within the FINISHED batches (its iteration count <= the count enqueued by the end of
      // batch b-1): the halting iteration is the same on every rank, so all ranks stop after the same batch and
      // issue the same collectives (a halt seen early is acted on after the next batch).
      const int32_t f = *(volatile int32_t*)h->hflag;
      if ((f & 1) && (int64_t)(f >> 1) <= enq_end[(batch - 1) & 1] + h->itn_at_init) break;
    }
    ++batch;
  }
  cudaEventDestroy(evs[0]);
  cudaEventDestroy(evs[1]);
  leave(h);
  return rc;
}

int lsqr_iterate_timed(lsqr_t h, int64_t n_iter, double* out) {
  GUARD(h);
  if (!h->initialized) return fail(h, LSQR_ESTATE, "lsqr_init first");
  if (!out || n_iter <= 0) return LSQR_EINVAL;
  enter(h);
  std::vector<cudaEvent_t> ev(4 * n_iter + 2);
  for (auto& e : ev) CKC(h, cudaEventCreate(&e));
  int rc = LSQR_OK;
  cudaEventRecord(ev[4 * n_iter], h->s);
  for (int64_t i = 0; i < n_iter && rc == LSQR_OK; ++i) rc = enqueue_iteration(h, &ev[4 * i]);
  cudaEventRecord(ev[4 * n_iter + 1], h->s);
  if (rc == LSQR_OK) {
    CKC(h, cudaEventSynchronize(ev[4 * n_iter + 1]));
    float ms;
    double a1 = 0, a2 = 0, worst = 0;
    cudaEventElapsedTime(&ms, ev[4 * n_iter], ev[4 * n_iter + 1]);
    out[0] = ms;
    for (int64_t i = 0; i < n_iter; ++i) {
      float t;
      cudaEventElapsedTime(&t, ev[4 * i], ev[4 * i + 1]);
      a1 += t;
      cudaEventElapsedTime(&t, ev[4 * i + 2], ev[4 * i + 3]);
      a2 += t;
      float it;
      cudaEventElapsedTime(&it, ev[4 * i], i + 1 < n_iter ? ev[4 * (i + 1)] : ev[4 * n_iter + 1]);
      worst = std::max(worst, (double)it);
    }
    out[1] = a1;
    out[2] = a2;
    out[3] = (double)(kernels_per_iteration(h) * n_iter);
    out[4] = worst;
  }
  for (auto& e : ev) cudaEventDestroy(e);
  leave(h);
  return rc;
}

int lsqr_get_state(lsqr_t h, double* sc, double* u, double* v, double* w, double* x, double* var) {
  GUARD(h);
  enter(h);
  CKC(h, cudaStreamSynchronize(h->s));
  DevState st;
  CKC(h, cudaMemcpy(&st, h->st, sizeof st, cudaMemcpyDeviceToHost));
  if (sc) {
    for (int i = 0; i < LSQR_NSCALARS; ++i) sc[i] = 0.0;
    sc[LSQR_S_ALPHA] = st.alpha; sc[LSQR_S_BETA] = st.beta; sc[LSQR_S_RHOBAR] = st.rhobar;
    sc[LSQR_S_PHIBAR] = st.phibar; sc[LSQR_S_ANORM] = st.anorm; sc[LSQR_S_ACOND] = st.acond;
    sc[LSQR_S_DDNORM] = st.ddnorm; sc[LSQR_S_RES2] = st.res2; sc[LSQR_S_XNORM] = st.xnorm;
    sc[LSQR_S_XXNORM] = st.xxnorm; sc[LSQR_S_Z] = st.z; sc[LSQR_S_CS2] = st.cs2; sc[LSQR_S_SN2] = st.sn2;
    sc[LSQR_S_RNORM] = st.rnorm; sc[LSQR_S_R1NORM] = st.r1norm; sc[LSQR_S_R2NORM] = st.r2norm;
    sc[LSQR_S_ARNORM] = st.arnorm; sc[LSQR_S_BNORM] = st.bnorm; sc[LSQR_S_ITN] = st.itn;
    sc[LSQR_S_ISTOP] = st.istop; sc[LSQR_S_ISTOP_FIRST] = st.istop_first; sc[LSQR_S_HALTED] = st.halted;
  }
  if (u) {
    CKC(h, cudaMemcpy(u, h->u, sizeof(double) * h->n_loc_rows, cudaMemcpyDeviceToHost));
    for (int64_t i = 0; i < h->n_loc_rows; ++i) u[i] *= st.inv_beta;
    if (h->n_constr) {
      CKC(h, cudaMemcpy(u + h->n_loc_rows, h->repro ? h->uc : h->ucn, sizeof(double) * h->n_constr,
                        cudaMemcpyDeviceToHost));
      if (h->repro)  // repro mode keeps the constraint u unnormalised too
        for (int64_t k = 0; k < h->n_constr; ++k) u[h->n_loc_rows + k] *= st.inv_beta;
    }
  }
  const size_t nb = sizeof(double) * h->n_loc_cols;
  if (v) CKC(h, cudaMemcpy(v, h->v, nb, cudaMemcpyDeviceToHost));
  if (w) CKC(h, cudaMemcpy(w, h->w, nb, cudaMemcpyDeviceToHost));
  if (x) CKC(h, cudaMemcpy(x, h->x, nb, cudaMemcpyDeviceToHost));
  if (var) CKC(h, cudaMemcpy(var, h->var, nb, cudaMemcpyDeviceToHost));
  leave(h);
  return LSQR_OK;
}

int lsqr_set_state(lsqr_t h, const double* sc, const double* u, const double* v, const double* w, const double* x,
                   const double* var) {
  GUARD(h);
  if (!h->initialized) return fail(h, LSQR_ESTATE, "lsqr_init first");
  enter(h);
  CKC(h, cudaStreamSynchronize(h->s));
  DevState st;
  CKC(h, cudaMemcpy(&st, h->st, sizeof st, cudaMemcpyDeviceToHost));  // h->s is idle (synchronised above)
  if (sc) {
    st.alpha = sc[LSQR_S_ALPHA]; st.beta = sc[LSQR_S_BETA]; st.rhobar = sc[LSQR_S_RHOBAR];
    st.phibar = sc[LSQR_S_PHIBAR]; st.anorm = sc[LSQR_S_ANORM]; st.acond = sc[LSQR_S_ACOND];
    st.ddnorm = sc[LSQR_S_DDNORM]; st.res2 = sc[LSQR_S_RES2]; st.xnorm = sc[LSQR_S_XNORM];
    st.xxnorm = sc[LSQR_S_XXNORM]; st.z = sc[LSQR_S_Z]; st.cs2 = sc[LSQR_S_CS2]; st.sn2 = sc[LSQR_S_SN2];
    st.rnorm = sc[LSQR_S_RNORM]; st.r1norm = sc[LSQR_S_R1NORM]; st.r2norm = sc[LSQR_S_R2NORM];
    st.arnorm = sc[LSQR_S_ARNORM]; st.bnorm = sc[LSQR_S_BNORM]; st.itn = (int32_t)sc[LSQR_S_ITN];
    st.istop = (int32_t)sc[LSQR_S_ISTOP]; st.istop_first = (int32_t)sc[LSQR_S_ISTOP_FIRST];
    st.halted = (int32_t)sc[LSQR_S_HALTED];
  }
  if (u) {  // the given u is normalised: store it as u_hat with inv_beta = 1
    CKC(h, cudaMemcpyAsync(h->u, u, sizeof(double) * h->n_loc_rows, cudaMemcpyHostToDevice, h->s));
    if (h->n_constr) {
      CKC(h, cudaMemcpyAsync(h->uc, u + h->n_loc_rows, sizeof(double) * h->n_constr, cudaMemcpyHostToDevice, h->s));
      CKC(h, cudaMemcpyAsync(h->ucn, u + h->n_loc_rows, sizeof(double) * h->n_constr, cudaMemcpyHostToDevice, h->s));
    }
    st.inv_beta = 1.0;
  }
  h->itn_at_init = (int64_t)st.itn - h->n_enq;  // lsqr_iterate: device itn = itn_at_init + iterations enqueued
  st.u_scale = st.alpha * st.inv_beta;
  st.v_pending = 0;
  st.col_enable = 0;
  CKC(h, cudaMemcpyAsync(h->st, &st, sizeof st, cudaMemcpyHostToDevice, h->s));
  const size_t nb = sizeof(double) * h->n_loc_cols;
  if (v) CKC(h, cudaMemcpyAsync(h->v, v, nb, cudaMemcpyHostToDevice, h->s));
  if (w) CKC(h, cudaMemcpyAsync(h->w, w, nb, cudaMemcpyHostToDevice, h->s));
  if (x) CKC(h, cudaMemcpyAsync(h->x, x, nb, cudaMemcpyHostToDevice, h->s));
  if (var) CKC(h, cudaMemcpyAsync(h->var, var, nb, cudaMemcpyHostToDevice, h->s));
  if (v) CKL(h, launch_att_pack(h->S, h->v, h->s), "att_pack");
  // ||w||^2 partials (astro / shared) for the next iteration's ddnorm
  CKL(h, launch_sumsq(h->w, h->S.A0, h->part_wa, kG3, h->s), "wsum_a");
  CKL(h, launch_sumsq(h->w + h->S.A0, h->n_sh, h->part_ws, kG3, h->s), "wsum_s");
  CKC(h, cudaStreamSynchronize(h->s));
  leave(h);
  return LSQR_OK;
}

int lsqr_finalize(lsqr_t h, lsqr_result* res, double* x_out, double* se_out) {
  GUARD(h);
  if (!h->initialized) return fail(h, LSQR_ESTATE, "lsqr_init first");
  enter(h);
  // O-4: t = 1; m > n -> m - n; damp > 0 -> m  (m, n count all rows and columns of the global system)
  const double m = (double)(h->n_obs + h->n_constr), n = (double)h->n_cols_g;
  double t = 1.0;
  if (m > n) t = m - n;
  if (h->params.damp > 0) t = m;
  const bool xd = x_out && is_device_ptr(x_out), sd = se_out && is_device_ptr(se_out);
  double* xo = x_out ? (xd ? x_out : h->tmp) : nullptr;
  if (x_out) CKL(h, launch_finalize(h->x, h->var, h->D, h->n_loc_cols, h->st, t, xo, nullptr, h->s), "finalize_x");
  if (x_out && !xd) CKC(h, cudaMemcpyAsync(x_out, h->tmp, sizeof(double) * h->n_loc_cols, cudaMemcpyDeviceToHost, h->s));
  if (x_out && !xd) CKC(h, cudaStreamSynchronize(h->s));
  double* so = se_out ? (sd ? se_out : h->tmp) : nullptr;
  if (se_out) CKL(h, launch_finalize(h->x, h->var, h->D, h->n_loc_cols, h->st, t, nullptr, so, h->s), "finalize_se");
  if (se_out && !sd) CKC(h, cudaMemcpyAsync(se_out, h->tmp, sizeof(double) * h->n_loc_cols, cudaMemcpyDeviceToHost, h->s));
  CKC(h, cudaStreamSynchronize(h->s));
  if (res) {
    DevState st;
    CKC(h, cudaMemcpy(&st, h->st, sizeof st, cudaMemcpyDeviceToHost));
    res->istop = st.istop; res->itn = st.itn; res->istop_first = st.istop_first;
    res->r1norm = st.r1norm; res->r2norm = st.r2norm; res->anorm = st.anorm; res->acond = st.acond;
    res->arnorm = st.arnorm; res->xnorm = st.xnorm; res->bnorm = st.bnorm;
  }
  leave(h);
  return LSQR_OK;
}

int lsqr_solve(lsqr_t h, const lsqr_solve_params* p, lsqr_result* res, double* x_out, double* se_out) {
  GUARD(h);
  CKR(lsqr_init(h, p));
  cudaEvent_t e0, e1;
  CKC(h, cudaEventCreate(&e0));
  CKC(h, cudaEventCreate(&e1));
  CKC(h, cudaEventRecord(e0, h->s));
  CKR(lsqr_iterate(h, p->itn_limit));
  CKC(h, cudaEventRecord(e1, h->s));
  CKC(h, cudaEventSynchronize(e1));
  float ms = 0;
  cudaEventElapsedTime(&ms, e0, e1);
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  CKR(lsqr_finalize(h, res, x_out, se_out));
  if (res) {
    res->t_iter_mean_s = res->itn > 0 ? ms * 1e-3 / res->itn : 0.0;
    res->t_iter_max_over_ranks_s = res->t_iter_mean_s;
    if (h->multi) {
      // max over ranks through the communicator's SUM allreduce (NCCL or the host callback): every rank puts its
      // time in its own slot of an nranks-long vector of zeros
      std::vector<double> tv(h->nranks, 0.0);
      tv[h->rank] = res->t_iter_mean_s;
      CKC(h, cudaMemcpyAsync(h->tmax, tv.data(), sizeof(double) * h->nranks, cudaMemcpyHostToDevice, h->s));
      CKR(allreduce(h, h->tmax, h->nranks));
      CKC(h, cudaMemcpyAsync(tv.data(), h->tmax, sizeof(double) * h->nranks, cudaMemcpyDeviceToHost, h->s));
      CKC(h, cudaStreamSynchronize(h->s));
      res->t_iter_max_over_ranks_s = *std::max_element(tv.begin(), tv.end());
    }
  }
  return LSQR_OK;
}

int lsqr_sync(lsqr_t h) {
  GUARD(h);
  CKC(h, cudaStreamSynchronize(h->s));
  return LSQR_OK;
}

}  // extern "C"

/*
 * lsqr_avugsr.h -- C ABI of the B200-native Gaia AVU-GSR LSQR library (liblsqr_avugsr.so).
 *
 * What it computes.  The Gaia AVU-GSR solver finds the astrometric, attitude, instrumental and global unknowns x of
 * the overdetermined sparse system A x = b (Eq. (2), §II-B) with a "customized and preconditioned"
 * LSQR [20],[21], whose cost is dominated by aprod1 (b <- b + A x, Eq. (3)) and aprod2
 * (x <- x + A^T b, Eq. (4)).  A has <= 24 nonzeros per row: 5 astrometric (block-diagonal by star),
 * 12 attitude (3 blocks of 4 with a fixed stride), 6 instrumental (irregular), 1 global.  Each rank
 * owns a subset of the observation rows (§IV).  "P:Lx" = /root/reference/PAPER.md line x; readings of
 * garbled or silent passages are SURVEY.md §8(c) (listed in DESIGN.md §3).
 *
 * Conventions (all calls):
 *   - Every call returns int: LSQR_OK (0) or a negative lsqr_status.  No C++ exception crosses the ABI.
 *   - Invalid arguments return LSQR_EINVAL before any allocation.  A failed lsqr_create sets *out = NULL.
 *   - After a CUDA or NCCL failure the handle is poisoned: later calls return LSQR_ESTATE; only lsqr_destroy and
 *     lsqr_last_error are legal.
 *   - A handle is single-threaded.  Device work runs on a library stream ordered after env->stream at entry and
 *     before it at exit ("stream-ordered"): device outputs are valid for later work on env->stream.
 *   - All floating point is IEEE binary64.  Index arithmetic is int64.
 *   - Device vectors follow the LOCAL layouts below; host arrays are copied and never retained.
 *
 * Local layouts (rank r of P; shard map = lsqr_shard_map, star ranges balanced by rows, SURVEY §8(c) O-SHARD):
 *   x-like vectors (n_local_cols): [ astro 5*n_local_stars | attitude n_att | instrumental n_instr | global n_glob ]
 *       astro entries of this rank's stars, in star order (global column 5*s + a  ->  local 5*(s - star_begin) + a);
 *       the shared attitude/instrumental/global slice is REPLICATED on every rank.
 *   y-like vectors (n_local_rows + n_constr): [ this rank's observation rows | constraint rows (replicated) ]
 *   Values: 24 slots per row in the order astro 0-4, attitude 5-16 (axis a, knot j at 5+4a+j), instrumental 17-22,
 *   global 23 (a zero pad when n_glob = 0).
 */
#ifndef LSQR_AVUGSR_H
#define LSQR_AVUGSR_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define LSQR_ABI_VERSION 2
#define LSQR_SLOTS 24

typedef struct lsqr_ctx* lsqr_t;

typedef enum {
  LSQR_OK = 0,
  LSQR_EINVAL = -1,     /* bad argument (checked before any allocation) */
  LSQR_ENOMEM = -2,     /* device or host allocation failed */
  LSQR_ECUDA = -3,      /* CUDA runtime error (handle poisoned) */
  LSQR_ENCCL = -4,      /* NCCL error (handle poisoned) */
  LSQR_ESTATE = -5,     /* wrong call order, consumed b, or poisoned handle */
  LSQR_EUNSORTED = -6,  /* lsqr_set_system: rows not grouped by star / inconsistent with obs_per_star */
  LSQR_ECOMM = -7       /* host-callback allreduce returned an error (handle poisoned) */
} lsqr_status;

/* Device memory hooks (e.g. torch.cuda.caching_allocator_alloc/delete).  NULL => cudaMalloc/cudaFree. */
typedef void* (*lsqr_alloc_fn)(size_t bytes, void* user);
typedef void (*lsqr_free_fn)(void* ptr, void* user);
/* Host-callback collective: in-place SUM allreduce of `count` doubles at DEVICE address `dev_buf`, ordered after
 * all work on `stream` (the library synchronises the stream before the call).  Return 0 on success.  Used to run
 * the multi-rank path without NCCL (e.g. torch.distributed gloo, several ranks on one GPU in tests). */
typedef int (*lsqr_allreduce_fn)(double* dev_buf, int64_t count, uint64_t stream, void* user);

typedef enum { LSQR_COMM_NCCL = 0, LSQR_COMM_CALLBACK = 1 } lsqr_comm_kind;

typedef struct {
  int32_t rank;            /* 0 <= rank < nranks */
  int32_t nranks;          /* >= 1 (one process per GPU) */
  int32_t device;          /* CUDA device ordinal used by this rank */
  int32_t comm_kind;       /* lsqr_comm_kind; ignored when nranks == 1 */
  const uint8_t* nccl_id;  /* 128 bytes from lsqr_nccl_unique_id on rank 0 (broadcast by the caller);
                              required iff nranks > 1 and comm_kind == LSQR_COMM_NCCL */
  uint64_t stream;         /* cudaStream_t the caller orders work on; 0 = legacy default stream */
  lsqr_alloc_fn alloc;     /* nullable */
  lsqr_free_fn free;       /* nullable (must be set iff alloc is) */
  void* alloc_user;
  lsqr_allreduce_fn allreduce; /* required iff nranks > 1 (or force_collectives) and comm_kind == LSQR_COMM_CALLBACK */
  void* allreduce_user;
  int32_t force_collectives; /* test hook: 1 = run the multi-rank algorithm and its collectives even when nranks == 1
                                (NCCL: a 1-rank communicator with an internally generated id, nccl_id may be NULL;
                                callback: the callback is called).  Results equal the nranks == 1 path up to rounding
                                (bit-identical in the reproducible mode).  0 = normal. */
  int32_t pad_;
} lsqr_env;

/* Constraint equations: extra sparse rows appended after the observations (content not
 * given by the paper -- S:§8(c) Z3).  Host CSR over GLOBAL column numbers; copied at lsqr_create.  On a multi-rank
 * run every rank passes the same full set; an entry counts on the rank that owns its column (astro: the star's
 * owner; shared columns: rank 0), so each entry is counted exactly once after the allreduce. */
typedef struct {
  int64_t n_rows;          /* number of constraint rows (0..64) */
  const int64_t* row_ptr;  /* [n_rows+1] */
  const int64_t* col;      /* [nnz] global columns, 0 <= col < n_cols */
  const double* val;       /* [nnz] */
  const double* rhs;       /* [n_rows]; NULL => 0 */
} lsqr_constraints;

/* On-device synthetic system ("a system ... distributed in the system as the real data", generated
 * from a seed).  Exact integer-hash spec: docs/GENERATOR.md (SURVEY §8(c) O-GEN). */
typedef struct {
  uint64_t seed;
  int32_t b_mode;          /* 0: hashed b; 1: planted b = A x_true (+ noise) */
  int32_t pad_;
  double noise;            /* planted mode only */
} lsqr_gen_params;

typedef struct {
  int64_t itn_limit;       /* maximum iterations */
  double atol, btol;       /* Paige-Saunders stopping tolerances */
  double conlim;           /* condition-number limit (0 => none); S:§8(c) Z4 */
  double damp;             /* damping (regularisation) acting on the scaled variables */
  int32_t fixed_count;     /* 1: evaluate the tests but run exactly itn_limit iterations (paper timing mode,
                              P:L1763-1767); the first nonzero istop is reported in istop_first */
  int32_t use_graph;       /* 1: replay the iteration as a CUDA graph (default for small systems) */
  int32_t poll_every;      /* host polls the stop flag every k iterations (<= 0 => 16) */
  int32_t two_pass;        /* 0 (default, the zero-initialised struct): fused single pass:
                              u_hat = A v - (alpha/beta) u_hat and z = A^T u_hat in ONE read of A, then
                              v' = z/beta - beta v.  1: two-pass iteration (the paper's structure: aprod1, then
                              aprod2, A read twice).  Same results up to rounding (ABI v2; v1 had `fused`, default 0) */
} lsqr_solve_params;

typedef struct {
  int32_t istop;           /* Paige-Saunders istop (0..7) */
  int32_t itn;             /* iterations performed */
  int32_t istop_first;     /* first nonzero istop seen (fixed_count mode) */
  int32_t pad_;
  double r1norm, r2norm;   /* ||r||, sqrt(||r||^2 + damp^2 ||x||^2) estimates */
  double anorm, acond, arnorm, xnorm, bnorm;
  double t_iter_mean_s;    /* mean device time per iteration on this rank (CUDA events) */
  double t_iter_max_over_ranks_s; /* same, max over ranks (allreduced) */
} lsqr_result;

/* Scalar state exchanged by lsqr_get_state/lsqr_set_state (teacher-forced parity tests): indices into double[] */
enum {
  LSQR_S_ALPHA = 0, LSQR_S_BETA, LSQR_S_RHOBAR, LSQR_S_PHIBAR, LSQR_S_ANORM, LSQR_S_ACOND, LSQR_S_DDNORM,
  LSQR_S_RES2, LSQR_S_XNORM, LSQR_S_XXNORM, LSQR_S_Z, LSQR_S_CS2, LSQR_S_SN2, LSQR_S_RNORM, LSQR_S_R1NORM,
  LSQR_S_R2NORM, LSQR_S_ARNORM, LSQR_S_BNORM, LSQR_S_ITN, LSQR_S_ISTOP, LSQR_S_ISTOP_FIRST, LSQR_S_HALTED,
  LSQR_NSCALARS = 24
};

/* ---------------------------------------------------------------- meta / host-only helpers (no GPU needed) */
int lsqr_abi_version(void);
/* Hash of the library's sources (csrc/*.cu, *.cuh and this header) it was built from, as 16 lower-case hex digits;
 * static storage, never NULL.  The Python binding compares it with the sources on disk and refuses a stale build. */
const char* lsqr_build_id(void);
const char* lsqr_strerror(int status);

/* Observations per star of the synthetic generator (O-GEN): uniform q = floor(n_obs/n_stars) (+1 for the first
 * n_obs mod n_stars stars), pairwise +-jitter_pct% (total preserved).  counts: host [n_stars]. */
int lsqr_synth_obs_per_star(uint64_t seed, int64_t n_stars, int64_t n_obs, int32_t jitter_pct, int64_t* counts);

/* The 12 synthetic constraint rows (O-GEN): 6 frame rows over the astro columns of the first min(n_ext, n_stars)
 * stars and 6 instrumental rows of ones.  Returns nnz (>= 0) or a negative status; NULL arrays => size query.
 * row_ptr: host [13], col: [nnz], val: [nnz]. */
int64_t lsqr_synth_constraints(uint64_t seed, int64_t n_stars, int64_t n_att, int64_t n_instr, int64_t n_ext,
                               int64_t* row_ptr, int64_t* col, double* val);

/* Star-range shard map (O-SHARD): star_begin[r] = lower_bound(row_ptr, floor(r*n_obs/nranks)),
 * star_begin[0] = 0, star_begin[nranks] = n_stars.  counts: host [n_stars]; star_begin: host [nranks+1]. */
int lsqr_shard_map(const int64_t* counts, int64_t n_stars, int64_t n_obs, int32_t nranks, int64_t* star_begin);

/* NCCL bootstrap: rank 0 calls this and broadcasts the 128 bytes (e.g. with torch.distributed). */
int lsqr_nccl_unique_id(uint8_t out[128]);

/* ---------------------------------------------------------------- handle */
/* n_att % 3 == 0, n_att/3 >= 4 (3 blocks of 4 with stride n_att/3); 6 <= n_instr <= 65536 and
 * n_instr % 6 == 0 when the generator is used; n_glob in {0,1}; obs_per_star: host [n_stars]
 * (NULL => uniform).  Collective over ranks when nranks > 1. */
int lsqr_create(int64_t n_stars, int64_t n_obs, int64_t n_att, int64_t n_instr, int32_t n_glob,
                const int64_t* obs_per_star, const lsqr_constraints* constraints, const lsqr_env* env,
                lsqr_t* out);
int lsqr_destroy(lsqr_t h);
const char* lsqr_last_error(lsqr_t h);

/* layout[0..9] = star_begin, star_end, row_begin, row_end, n_local_rows, n_local_cols, n_constr, n_shared,
 *                n_rows_global (= n_obs + n_constr), n_cols_global */
int lsqr_layout(lsqr_t h, int64_t* layout);

/* ---------------------------------------------------------------- system */
/* Generate this rank's rows on the device (O-GEN); b goes into the solver's u buffer.  Replaces any previous system
 * (a previous lsqr_precondition is undone: D = 1, raw constraint values). */
int lsqr_generate(lsqr_t h, const lsqr_gen_params* p);
/* Upload this rank's rows from HOST arrays in the paper's layout, global columns:
 * vals [n_local_rows][24], matrixIndexAstro [n_local_rows] (= 5*star), matrixIndexAtt [n_local_rows] (column of the
 * first attitude nonzero = 5*n_stars + k0), instrCol [n_local_rows][6], b [n_local_rows].  Rows must be grouped by
 * star in star order with obs_per_star rows each (else LSQR_EUNSORTED).  Replaces any previous system (undoes
 * lsqr_precondition).  Synchronous on return (host buffers may be reused). */
int lsqr_set_system(lsqr_t h, const double* vals, const int64_t* matrixIndexAstro, const int64_t* matrixIndexAtt,
                    const int64_t* instrCol, const double* b);
/* Download (test/diagnostic): same layout as lsqr_set_system; any pointer may be NULL.  Synchronous. */
int lsqr_get_system(lsqr_t h, double* vals, int64_t* matrixIndexAstro, int64_t* matrixIndexAtt, int64_t* instrCol,
                    double* b);
/* Column preconditioning ("preconditioned"; S:§8(c) O-PREC): c_j = sum_i a_ij^2 (constraints included),
 * D_j = 1/sqrt(c_j) (1 if c_j == 0), A <- A D in place.  Once per system.  Collective. */
int lsqr_precondition(lsqr_t h);
/* D (n_local_cols; host or device pointer).  All ones before lsqr_precondition. */
int lsqr_get_precond(lsqr_t h, double* D);
/* Bitwise-reproducible mode (docs/REPRO.md), on = 1 / off = 0; off by default.  When on,
 * lsqr_precondition and the LSQR (lsqr_init / lsqr_iterate / lsqr_solve) compute every reduction -- the column sums
 * of squares, the row dots of aprod1, the column sums of aprod2, ||u||, ||v|| and ddnorm -- as an exact,
 * order-independent digit accumulation rounded once, and every other step as one IEEE operation without FMA
 * contraction, in the order of Paige & Saunders' recurrence.  The iterates are then bit-identical run
 * to run and to the CPU oracle's repro mode, independent of scheduling; lsqr_solve_params.two_pass is ignored and the
 * iteration is several times slower than the default path (verification mode).  With nranks > 1 the digits are
 * allreduced exactly (as pairs of exact doubles), so D, x, se and every scalar are bit-identical for ANY number of
 * ranks and any shard map.  Allocates 56 B per local column of digit storage (+ 112 B per shared column when
 * nranks > 1; LSQR_ENOMEM).  The digit sums are exact for fewer than 2^33 terms per accumulator on a rank: the call
 * returns LSQR_EINVAL when 6 * n_local_rows + (owned constraint entries) >= 2^33 or n_local_cols >= 2^33.
 * Invalidates a previous lsqr_init; call before lsqr_precondition for a reproducible D.
 * Collective when nranks > 1 (only in the sense that all ranks must use the same mode). */
int lsqr_set_reproducible(lsqr_t h, int32_t on);

/* ---------------------------------------------------------------- products (hot path) */
/* y += A^ x  (aprod1, Eq. (3)).  x: device [n_local_cols], y: device [n_local_rows + n_constr].  A^ = A D after
 * lsqr_precondition, else A.  Constraint rows are complete (allreduced) on every rank.  Async, collective. */
int lsqr_aprod1(lsqr_t h, const double* x_dev, double* y_dev);
/* x += A^T y  (aprod2, Eq. (4)).  y: device [n_local_rows + n_constr] (constraint part replicated), x: device
 * [n_local_cols].  The shared slice is allreduced, so it is identical on every rank.  Async, collective. */
int lsqr_aprod2(lsqr_t h, const double* y_dev, double* x_dev);

/* ---------------------------------------------------------------- LSQR */
/* Full solve: init, iterate until istop or itn_limit (or exactly itn_limit in fixed_count mode),
 * standard errors (lsqr.f se), unscale by D.  x_out, se_out: [n_local_cols], host or device, nullable.
 * Consumes b (u's buffer): a second solve needs lsqr_generate / lsqr_set_system first (else LSQR_ESTATE).
 * Synchronous.  Collective. */
int lsqr_solve(lsqr_t h, const lsqr_solve_params* p, lsqr_result* res, double* x_out, double* se_out);
/* Step-wise form of lsqr_solve (tests, timing). */
int lsqr_init(lsqr_t h, const lsqr_solve_params* p);
int lsqr_iterate(lsqr_t h, int64_t n_iter);
/* n_iter iterations without graph replay, with CUDA events around every kernel launch on the launching stream.
 * out[0] = total ms, out[1] = sum of aprod1 kernel ms (fused mode: the fused row kernel), out[2] = sum of aprod2
 * kernel ms (fused mode: the astro column pass), out[3] = kernels launched, out[4] = ms of the slowest single
 * iteration.  Synchronous. */
int lsqr_iterate_timed(lsqr_t h, int64_t n_iter, double* out);
int lsqr_finalize(lsqr_t h, lsqr_result* res, double* x_out, double* se_out);
/* State snapshot (host pointers, any may be NULL; synchronous): scalars [LSQR_NSCALARS]; u [n_local_rows+n_constr]
 * NORMALISED (u_k of Paige-Saunders); v, w, x, var [n_local_cols] in SCALED variables. */
int lsqr_get_state(lsqr_t h, double* scalars, double* u, double* v, double* w, double* x, double* var);
/* Teacher forcing: overwrite the iteration state (same layout as lsqr_get_state; NULL = keep). */
int lsqr_set_state(lsqr_t h, const double* scalars, const double* u, const double* v, const double* w,
                   const double* x, const double* var);
int lsqr_sync(lsqr_t h);

#ifdef __cplusplus
}
#endif
#endif /* LSQR_AVUGSR_H */

/*
 * proclus.h -- C ABI of the B200-native GPU-FAST-PROCLUS hot path.
 *
 * PROCLUS (Alg 1-6) as parallelised by GPU-FAST-PROCLUS
 * (P:221-362), re-designed for sm_100a.  Citations are to
 * /root/reference/PAPER.md line numbers (P:<n>); readings of garbled or
 * silent passages are listed in DESIGN.md section 3 and tagged [Rn].
 *
 * Problem statement (Alg 1 header P:107): given Data in R^{n x d}, the
 * number of clusters k, the average number of dimensions l, the sample
 * constants A, B, the bad-medoid threshold minDev and the patience itrPat,
 * return k disjoint clusters C, their subspaces D and medoids M.
 *
 * Conventions shared by every entry point:
 *  - Every function returns a proclus_status.  On a non-OK status the
 *    contents of output buffers are unspecified and proclus_last_error()
 *    returns a message describing the cause (thread-local, valid until the
 *    next call on the same thread).
 *  - Input data is row-major (point-major) n x d fp32.  Values must be finite.
 *  - A handle owns all device memory it allocates (data copy, the Dist cache
 *    of P:153, H of eq 5, labels, partial sums) and the CUDA graphs it
 *    instantiates for its runs (one per distinct run shape -- k, l, variant,
 *    output placement --, at most 256, least recently used evicted; a later
 *    run of the same shape, e.g. the next sweep over the same (k, l) grid,
 *    reuses them).  It is not thread-safe: one call at a time per handle.
 *    Distinct handles are independent.
 *  - Determinism: identical (data, parameters, seed, device type) give
 *    bit-identical outputs.
 *  - Randomness (P:241 leaves it unspecified) follows reading R2: SplitMix64
 *    streams keyed by (seed, k) for the sample / greedy start and by
 *    (seed, k, l) for MCur and the replacement draws.
 */
#ifndef PROCLUS_H
#define PROCLUS_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#if defined(__GNUC__)
#define PROCLUS_API __attribute__((visibility("default")))
#else
#define PROCLUS_API
#endif

#define PROCLUS_ABI_VERSION 1
#define PROCLUS_K_MAX 32   /* k <= 32: per-point medoid bitmasks are 32-bit */
#define PROCLUS_D_MAX 256  /* a 2-stage ring of 64-point chunks fits in SMEM */

typedef struct proclus_handle proclus_handle;
typedef struct proclus_group proclus_group;

typedef enum {
  PROCLUS_OK = 0,
  PROCLUS_EINVAL = -1,    /* argument outside the documented domain       */
  PROCLUS_ENOMEM = -2,    /* host or device allocation failed             */
  PROCLUS_ECUDA = -3,     /* a CUDA runtime call failed                   */
  PROCLUS_ENCCL = -4,     /* a NCCL call failed (world_size > 1)          */
  PROCLUS_EINTERNAL = -5  /* invariant violated inside the library        */
} proclus_status;

/* Full-space metric of Greedy (Alg 2 l.4) and ComputeL (Alg 3 l.3).
 * The paper uses Euclidean distance; north_star names
 * L1.  Reading R1: one option for both steps, L2 by default. */
typedef enum { PROCLUS_METRIC_L2 = 0, PROCLUS_METRIC_L1 = 1 } proclus_metric;

typedef struct {
  int32_t device;          /* CUDA device ordinal; -1 = current device      */
  int32_t metric;          /* proclus_metric                                */
  int32_t max_iter;        /* cap on iterative-phase iterations; <=0: 10000 */
  int32_t data_on_device;  /* 1: `data` passed to create/load is a device
                              pointer (row-major n x d fp32) on `device`    */
  void* stream;            /* cudaStream_t to run on; NULL: handle-owned    */
  int32_t trace;           /* 1: record a per-iteration trace (see below)   */
  /* Row-sharded multi-GPU (one process per GPU, P:235 data parallelism
   * extended across GPUs).  world_size 1 = single GPU.  With world_size > 1
   * this rank owns rows [row_offset, row_offset + n) of an n_global-row
   * dataset and every k x d partial sum is combined by ncclAllReduce. */
  int32_t world_size;
  int32_t rank;
  int64_t n_global;        /* 0: = n                                         */
  int64_t row_offset;
  const void* nccl_unique_id;  /* 128-byte ncclUniqueId (world_size > 1)    */
  int32_t stats;           /* 1: time every kernel launch with CUDA events on
                              the handle's stream (see proclus_get_stats)   */
  int32_t variant;         /* proclus_variant: which caches the iterative
                              phase keeps; every variant returns the same
                              clustering                     */
  proclus_group* group;    /* world_size > 1 without NCCL: the in-process
                              communicator from proclus_group_create (then
                              nccl_unique_id is ignored); NULL: NCCL        */
} proclus_options;

/* GPU-FAST-PROCLUS (default): the Dist row of every potential medoid is
 * computed once and cached (#M x n fp32), with incremental
 * locality bands and H (Theorems 3.1/3.2).
 * GPU-PROCLUS: no caches; every iteration recomputes the k distance rows,
 * the full L_i and X from scratch (the paper's ablation baseline).
 * GPU-FAST*-PROCLUS: Dist rows and H are kept only for the current slots from
 * the previous iteration (k x n fp32 instead of #M x n). */
typedef enum {
  PROCLUS_VARIANT_FAST = 0,
  PROCLUS_VARIANT_PLAIN = 1,
  PROCLUS_VARIANT_FAST_STAR = 2
} proclus_variant;

typedef struct {
  int32_t* labels;      /* [n] caller-allocated (host, or device if
                           labels_on_device): cluster id in [0,k), -1 for an
                           outlier (RemoveOutliers).  With
                           world_size > 1: this rank's n rows.               */
  int64_t* medoids;     /* [k] caller-allocated host: row index (global) of
                           the medoid of cluster i (MBest, P:134 [R16])      */
  uint8_t* dims;        /* [k*d] caller-allocated host: dims[i*d+j] = 1 iff
                           j is in D_i; k*l ones, >= 2 per row       */
  double cost;          /* costBest of the iterative phase (eq 8/9 [R4])    */
  int32_t iterations;   /* iterative-phase iterations executed              */
  int32_t labels_on_device;  /* 1: `labels` is a device pointer             */
} proclus_result;

/* Per-iteration trace of the last proclus_run (options.trace = 1).  Each
 * pointer may be NULL; arrays hold cap iterations (k or k*d per iteration).
 * mcur are positions into M (the B*k potential medoids). */
typedef struct {
  int32_t cap;
  int32_t count;        /* out: iterations recorded                         */
  int32_t* mcur;        /* [cap*k]   */
  double* delta;        /* [cap*k]   delta_i, Alg 3 l.4-7                  */
  int64_t* nL;          /* [cap*k]   |L_i|                                 */
  uint8_t* dims;        /* [cap*k*d] D                                     */
  int64_t* sizes;       /* [cap*k]   |C_i|                                 */
  double* cost;         /* [cap]                                           */
  uint8_t* improved;    /* [cap]                                           */
  uint8_t* bad;         /* [cap*k]   MBad                                  */
  double* X;            /* [cap*k*d] X_ij                                  */
} proclus_trace;

/* Per-kernel measurements of the last proclus_run (options.stats = 1).
 * kind order: pack, gather, greedy, prepare, locality, assign, cost,
 * refine_x, final, split_tail.  Only launches that did work are counted
 * (iterations enqueued speculatively after the device stopped return at
 * once and are excluded).  alg_bytes follows the byte model of DESIGN.md
 * section 6 (data bytes + Dist rows + labels; no padding, no partials). */
#define PROCLUS_STAT_KINDS 10
typedef struct {
  int64_t launches[PROCLUS_STAT_KINDS];
  double ms[PROCLUS_STAT_KINDS];         /* summed CUDA-event time          */
  double alg_bytes[PROCLUS_STAT_KINDS];  /* algorithmic bytes moved          */
  double run_ms;                         /* first to last event of the run  */
  int64_t total_launches;                /* every kernel launch of the run  */
  double tail_ms[4];      /* single-block tails (locality, assign, cost,
                             refine), device %globaltimer                  */
  int64_t fallbacks[4];   /* exact fp64 re-decisions (locality, assign,
                             final): points within the fp32 error bound    */
} proclus_stats;

/* In-process communicator for `world` row shards whose handles live in ONE
 * process (any devices, also several shards on one GPU: test layer F of
 * SURVEY 4.2).  Pass it as options.group with options.world_size = world and
 * a distinct options.rank per handle.  Each rank's proclus_create_ex /
 * proclus_run / proclus_run_multi must then be called from its own host
 * thread, the ranks with identical arguments except data and labels: the
 * calls rendezvous at every collective.  The partial sums (int64 fixed-point
 * cells, counts, per-dimension maxima, gathered sample rows) are combined
 * by a host-staged reduction in rank order, so the results are bit-identical
 * to the NCCL path and to world_size 1.
 * EINVAL: world < 1 or > 1024, out == NULL.  The caller destroys the group
 * after every handle that uses it (proclus_group_destroy is NULL-safe). */
PROCLUS_API proclus_status proclus_group_create(int32_t world, proclus_group** out);
PROCLUS_API void proclus_group_destroy(proclus_group* g);

/* Fill *opt with defaults (device -1, L2, max_iter 10000, host data, own
 * stream, no trace, world_size 1). */
PROCLUS_API proclus_status proclus_options_init(proclus_options* opt);

/* Copy `data` (row-major n x d fp32) to the device in the library's layout.
 * The caller keeps ownership of `data` and may free it on return.
 * EINVAL: n < 1, d < 2 (sigma divides by d-1), d > PROCLUS_D_MAX,
 * non-finite values, bad options. */
PROCLUS_API proclus_status proclus_create(const float* data, int64_t n, int32_t d,
                              proclus_handle** out);
PROCLUS_API proclus_status proclus_create_ex(const float* data, int64_t n, int32_t d,
                                 const proclus_options* opt,
                                 proclus_handle** out);

/* Replace the handle's data with new values of the same shape (host or
 * device pointer per the handle's options).  Drops all cached distances.
 * With world_size 1 the load is asynchronous on the handle's stream (copy,
 * pack and the fixed-point scales run on the device): the caller may reuse
 * a host buffer only after the next proclus_run returns, and a non-finite
 * value makes that proclus_run fail with EINVAL (proclus_create still
 * validates synchronously).  EINVAL: NULL arguments. */
PROCLUS_API proclus_status proclus_load(proclus_handle* h, const float* data);

/* Start copying the NEXT dataset `data` (host pointer, row-major n x d fp32
 * of the handle's shape; pinned memory makes the copy asynchronous) into the
 * handle's staging buffer on a separate copy stream and return at once, so
 * that the transfer overlaps the clustering a following proclus_run performs
 * on the current data.  A later proclus_load(h, data) with the same pointer
 * waits for that copy instead of copying again.  The caller keeps `data`
 * alive and unmodified until that proclus_load returns.  Nothing of the
 * current data or its results changes.
 * EINVAL: NULL arguments, a handle created with device-resident data. */
PROCLUS_API proclus_status proclus_prefetch(proclus_handle* h, const float* data);

/* One PROCLUS clustering (Alg 1): initialization (sample of A*k points,
 * Greedy to B*k potential medoids), iterative phase (Alg 1
 * l.5-14, with the FAST caches of section 3), refinement (Alg 1
 * l.16-19).  #S = min(A*k, n), #M = min(B*k, #S) (clamped, not an error).
 * EINVAL: k < 2, k > PROCLUS_K_MAX, l < 2, l > d, A < 1, B < 1, #M < k,
 * minDev <= 0 or not finite, itrPat < 1, out == NULL or missing arrays. */
PROCLUS_API proclus_status proclus_run(proclus_handle* h, int32_t k, int32_t l, int32_t A,
                           int32_t B, double minDev, int32_t itrPat,
                           uint64_t seed, proclus_result* out);

/* Multiple parameter settings over the grid ks x ls (k outer,
 * l inner; outs has nk*nl entries, each with its own arrays).
 * reuse_level 1: every setting equals an independent proclus_run(k, l, seed)
 *   ("multi-param 1": the Dist cache and H are reused between settings that
 *   share M, i.e. the same k).
 * reuse_level 2: S and M are drawn once for k_max (greedy once) and
 *   Dist, H, delta', |L| are reused across the whole grid ("multi-param 2").
 * reuse_level 3: level 2, and every setting after the first starts from a
 *   random subset of the previous setting's MBest ("multi-param 3";
 *   reading R21: partial Fisher-Yates over MBest_prev in slot order, topped
 *   up from the ascending positions of M \ MBest_prev when k grows; stream
 *   IT of the setting).  This heuristic changes the results: settings are
 *   sequential in caller order.
 * EINVAL: reuse_level not in {1,2,3}, empty grid, any invalid (k, l). */
PROCLUS_API proclus_status proclus_run_multi(proclus_handle* h, const int32_t* ks,
                                 int32_t nk, const int32_t* ls, int32_t nl,
                                 int32_t A, int32_t B, double minDev,
                                 int32_t itrPat, uint64_t seed,
                                 int32_t reuse_level, proclus_result* outs);

/* A list of independent settings (ks[s], ls[s]), s < nset, for
 * splitting a multi-parameter grid across GPUs or processes (settings
 * parallelism: every rank holds the whole dataset, no communication).
 * reuse_level 1: every setting equals proclus_run(ks[s], ls[s], seed).
 * reuse_level 2: S and M are drawn once for k_sample (>= every ks[s]) and
 *   the caches are shared, so outs[s] equals the result of that setting in
 *   proclus_run_multi(..., reuse_level 2) over any grid whose largest k is
 *   k_sample -- whichever rank runs it.
 * Level 3 (warm starts from the previous setting) is sequential and not
 * offered here.
 * EINVAL: nset < 1, reuse_level not in {1,2}, an invalid (k, l), k_sample
 * smaller than some ks[s] or outside [2, PROCLUS_K_MAX] (level 2). */
PROCLUS_API proclus_status proclus_run_list(proclus_handle* h, const int32_t* ks,
                                const int32_t* ls, int32_t nset, int32_t k_sample,
                                int32_t A, int32_t B, double minDev, int32_t itrPat,
                                uint64_t seed, int32_t reuse_level, proclus_result* outs);

/* Copy the trace of the last run (requires options.trace = 1). */
PROCLUS_API proclus_status proclus_get_trace(proclus_handle* h, proclus_trace* tr);

/* Copy the per-kernel measurements of the last run (options.stats = 1). */
PROCLUS_API proclus_status proclus_get_stats(proclus_handle* h, proclus_stats* st);

/* Number of kernel launches issued by the last run (for the bench's
 * gpu_launches). */
PROCLUS_API int64_t proclus_last_launches(proclus_handle* h);

/* NULL-safe; waits for outstanding work, frees everything the handle owns. */
PROCLUS_API void proclus_destroy(proclus_handle* h);

/* Thread-local description of the last failure on this thread. */
PROCLUS_API const char* proclus_last_error(void);

/* Library / ABI version and the sm architecture the kernels target (100). */
PROCLUS_API int32_t proclus_abi_version(void);
PROCLUS_API int32_t proclus_target_sm(void);

#ifdef __cplusplus
}
#endif
#endif /* PROCLUS_H */

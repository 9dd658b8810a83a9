/*
 * proclus_oracle.h -- TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, single-threaded fp64 CPU oracle of PROCLUS (Alg 1-6 of
 * GPU-FAST-PROCLUS, EDBT 2022; /root/reference/PAPER.md cited as P:<line>).
 * Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline /
 * --impl reference) may load this.  It shares no code, header, table or
 * constant generator with the CUDA library under
 * paper_conf_edbt_jorgensensape22_b200/ and it never includes ../include.
 *
 * Readings of garbled / silent passages follow SURVEY.md section 8(c) and
 * are listed in DESIGN.md section 3.
 *
 * Pins (tests/test_oracle.py, -m "not gpu"): every step below is checked
 * against something other than itself -- known-answer vectors (SplitMix64),
 * scipy / numpy (distances, Y / sigma / Z), brute force on tiny inputs
 * (greedy, delta / L, selection, assignment), the paper's closed forms
 * (sum Z = 0, sum Z^2 = d - 1; eq 2 = eq 9), worked examples in
 * tests/golden/, and the FAST-vs-plain equality of Theorems 3.1 / 3.2.
 * oracle_proclus / oracle_proclus_multi as a whole: parity unpinned by the
 * paper (it prints no clustering for any input); pinned only through those
 * steps, the run invariants (disjoint labels, k*l dimensions, >= 2 per
 * cluster, costBest non-increasing) and the recovery of planted subspaces.
 */
#ifndef PROCLUS_ORACLE_H
#define PROCLUS_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define ORC_OK 0
#define ORC_EINVAL (-1)
#define ORC_ENOMEM (-2)

#define ORC_METRIC_L2 0 /* Euclidean, P:89 P:95 P:153 (paper default) */
#define ORC_METRIC_L1 1 /* Manhattan, north_star option               */

/* ---- RNG: SplitMix64 (reading R2) ---- */
uint64_t oracle_splitmix_next(uint64_t* state);
uint64_t oracle_uniform(uint64_t* state, uint64_t m);
uint64_t oracle_stream_sm(uint64_t seed, int64_t k_sm);
uint64_t oracle_stream_it(uint64_t seed, int64_t k, int64_t l);

/* ---- O0 distances ---- */
double oracle_full(const float* p, const float* q, int32_t d, int32_t metric);
double oracle_seg(const float* p, const float* q, int32_t d, const uint8_t* dmask);

/* ---- individual steps (exported for pinning tests) ---- */
/* O3: partial Fisher-Yates over [0,n), nS draws. */
int oracle_sample(int64_t n, int64_t nS, uint64_t* state, int64_t* S);
/* O4: Greedy (Alg 2). Spos[nM] gets positions into S; pickdist[nM] (may be
 * NULL) gets the max-min distance at which each pick was made (pick 0: +inf). */
int oracle_greedy(const float* data, int32_t d, const int64_t* S, int64_t nS,
                  int64_t nM, int64_t q0, int32_t metric, int64_t* Spos,
                  double* pickdist);
/* Alg 3 l.4-7: delta_i = min_{j!=i} full(m_i, m_j). med = k rows of d. */
void oracle_delta(const float* med, int32_t k, int32_t d, int32_t metric,
                  double* delta);
/* Alg 3 l.8-12 + Alg 4 l.1-5: L_i membership and X_ij. inL may be NULL. */
void oracle_locality_X(const float* data, int64_t n, int32_t d,
                       const float* med, int32_t k, const double* delta,
                       int32_t metric, uint8_t* inL, int64_t* nL, double* X);
/* Alg 4 l.6-16: Y, sigma, Z and dimension selection. Z (k*d) may be NULL. */
int oracle_find_dimensions(const double* X, int32_t k, int32_t d, int32_t l,
                           uint8_t* dmask, double* Z, double* zgap);
/* Alg 5: labels[p] = argmin_i seg_{D_i}(x_p, m_i), ties -> smallest i. */
void oracle_assign(const float* data, int64_t n, int32_t d, const float* med,
                   int32_t k, const uint8_t* dmask, int32_t* labels,
                   double* min_rel_gap);
/* Alg 6 / eq 1, 2 (|Data| denominator of eq 8). sizes (k) may be NULL. */
double oracle_evaluate(const float* data, int64_t n, int32_t d,
                       const int32_t* labels, int32_t k, const uint8_t* dmask,
                       int64_t* sizes);
/* eq 9 form of the same cost, used only to pin eq 1-2 == eq 9. */
double oracle_evaluate_eq9(const float* data, int64_t n, int32_t d,
                           const int32_t* labels, int32_t k,
                           const uint8_t* dmask);
/* Alg 1 l.13: bad medoids from cluster sizes. */
void oracle_bad_medoids(const int64_t* sizes, int32_t k, int64_t n,
                        double minDev, uint8_t* bad);
/* Refinement X over clusters (Alg 1 l.16-17). */
void oracle_cluster_X(const float* data, int64_t n, int32_t d,
                      const int32_t* labels, const float* med, int32_t k,
                      double* X);
/* RemoveOutliers: labels[p] = -1 if outside every sphere. */
void oracle_remove_outliers(const float* data, int64_t n, int32_t d,
                            const float* med, int32_t k, const uint8_t* dmask,
                            int32_t* labels, double* Delta);

/* ---- whole algorithm ---- */
typedef struct {
  int32_t k, l, A, B;
  double minDev;
  int32_t itrPat;
  uint64_t seed;
  int32_t metric;
  int32_t max_iter;   /* <= 0 -> 10000 */
  int32_t fast;       /* 1: FAST-PROCLUS caches (Dist, H, delta', |L|) */
} oracle_params;

typedef struct {
  int32_t* labels;     /* [n]   */
  int64_t* medoids;    /* [k]   point ids (rows of data) of MBest */
  uint8_t* dims;       /* [k*d] D* mask of the refinement */
  double cost;         /* costBest */
  int32_t iterations;
  int64_t nS, nM;
} oracle_result;

/* Per-iteration trace; arrays sized cap*k (cap*k*d for dims). Any pointer
 * may be NULL. */
typedef struct {
  int32_t cap;
  int32_t count;
  int32_t* mcur;      /* positions into M */
  double* delta;
  int64_t* nL;
  uint8_t* dims;
  int64_t* sizes;
  double* cost;
  uint8_t* improved;
  uint8_t* bad;
  double* zgap;       /* smallest Z gap at the selection boundary        */
  double* costgap;    /* |cost-costBest|/max(cost,costBest), +inf first  */
  double* assign_gap; /* smallest relative gap best vs runner-up         */
  double* X;          /* cap*k*d */
} oracle_trace;

int oracle_validate(int64_t n, int32_t d, const float* data,
                    const oracle_params* p);
int oracle_proclus(const float* data, int64_t n, int32_t d,
                   const oracle_params* prm, oracle_result* out,
                   oracle_trace* trace);
/* Multi-parameter. reuse_level 1: every setting == an
 * independent oracle_proclus(k,l,seed). reuse_level 2: S and M drawn once
 * for k_max (stream SM keyed by k_max) and shared by every setting.
 * reuse_level 3 (reading R21): level 2, and every setting after the
 * first draws its initial MCur as a random subset of the previous setting's
 * MBest (topped up from M \ MBest_prev when k grows). outs is [nk*nl], k
 * outer, l inner; each outs[i] has its own arrays. */
int oracle_proclus_multi(const float* data, int64_t n, int32_t d,
                         const int32_t* ks, int32_t nk, const int32_t* ls,
                         int32_t nl, const oracle_params* base,
                         int32_t reuse_level, oracle_result* outs);

#ifdef __cplusplus
}
#endif
#endif

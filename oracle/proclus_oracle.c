/*
 * proclus_oracle.c -- TEST INFRASTRUCTURE ONLY (see proclus_oracle.h).
 *
 * Plain PROCLUS, written step by step in the order and notation of
 * /root/reference/PAPER.md (cited P:<line>, Alg <n> l.<m>), single thread,
 * fp64 on (double) casts of the fp32 inputs, compiled with
 * -O2 -ffp-contract=off (no FMA contraction, no fast-math).
 *
 * Sums over points run with p ascending; sums over dimensions with j
 * ascending.  Where the paper is silent or garbled the reading of
 * SURVEY.md 8(c) is used; each such place is tagged [Rn] and listed in
 * DESIGN.md section 3.
 */
#include "proclus_oracle.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>

/* ------------------------------------------------------------------ */
/* RNG [R2]: SplitMix64; uniform(m) = floor(next() * m / 2^64).        */
/* ------------------------------------------------------------------ */
uint64_t oracle_splitmix_next(uint64_t* state) {
  uint64_t z;
  *state += 0x9E3779B97F4A7C15ULL;
  z = *state;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}

uint64_t oracle_uniform(uint64_t* state, uint64_t m) {
  unsigned __int128 w = (unsigned __int128)oracle_splitmix_next(state) * m;
  return (uint64_t)(w >> 64);
}

static uint64_t F(uint64_t x) { return oracle_splitmix_next(&x); }

/* Stream SM (sample + greedy start) is keyed by (seed, k_sm). */
uint64_t oracle_stream_sm(uint64_t seed, int64_t k_sm) {
  return F(F(seed) + (uint64_t)k_sm);
}
/* Stream IT (initial MCur + replacement draws) is keyed by (seed, k, l). */
uint64_t oracle_stream_it(uint64_t seed, int64_t k, int64_t l) {
  return F(F(F(seed) + (uint64_t)k) + (uint64_t)l + 4294967296ULL);
}

/* ------------------------------------------------------------------ */
/* O0 distances.                                                       */
/* ------------------------------------------------------------------ */
/* ||p - q||_2 or ||p - q||_1 (metric option [R1]). */
double oracle_full(const float* p, const float* q, int32_t d, int32_t metric) {
  double s = 0.0;
  int32_t j;
  if (metric == ORC_METRIC_L1) {
    for (j = 0; j < d; ++j) s = s + fabs((double)p[j] - (double)q[j]);
    return s;
  }
  for (j = 0; j < d; ++j) {
    double t = (double)p[j] - (double)q[j];
    s = s + t * t;
  }
  return sqrt(s);
}

/* Manhattan segmental distance ||p - q||_1^{D} / |D| (Alg 5 l.4). */
double oracle_seg(const float* p, const float* q, int32_t d,
                  const uint8_t* dmask) {
  double s = 0.0;
  int32_t j, nd = 0;
  for (j = 0; j < d; ++j) {
    if (!dmask[j]) continue;
    s = s + fabs((double)p[j] - (double)q[j]);
    ++nd;
  }
  return s / (double)nd;
}

/* ------------------------------------------------------------------ */
/* Validation.                                           */
/* ------------------------------------------------------------------ */
int oracle_validate(int64_t n, int32_t d, const float* data,
                    const oracle_params* p) {
  int64_t nS, nM, i;
  if (n < 1 || d < 2 || !p) return ORC_EINVAL;
  if (p->k < 2 || p->l < 2 || p->l > d || p->A < 1 || p->B < 1) return ORC_EINVAL;
  if (!(p->minDev > 0.0) || !isfinite(p->minDev) || p->itrPat < 1) return ORC_EINVAL;
  if (p->metric != ORC_METRIC_L1 && p->metric != ORC_METRIC_L2) return ORC_EINVAL;
  nS = (int64_t)p->A * p->k;
  if (nS > n) nS = n;
  nM = (int64_t)p->B * p->k;
  if (nM > nS) nM = nS;
  if (nM < p->k) return ORC_EINVAL;
  if (data)
    for (i = 0; i < n * (int64_t)d; ++i)
      if (!isfinite(data[i])) return ORC_EINVAL;
  return ORC_OK;
}

/* ------------------------------------------------------------------ */
/* O3 Sample Data' (Alg 1 l.2) [R13]: partial Fisher-Yates.      */
/* ------------------------------------------------------------------ */
int oracle_sample(int64_t n, int64_t nS, uint64_t* state, int64_t* S) {
  int64_t t, *v = (int64_t*)malloc(sizeof(int64_t) * (size_t)n);
  if (!v) return ORC_ENOMEM;
  for (t = 0; t < n; ++t) v[t] = t;
  for (t = 0; t < nS; ++t) {
    int64_t r = t + (int64_t)oracle_uniform(state, (uint64_t)(n - t));
    int64_t tmp = v[t];
    v[t] = v[r];
    v[r] = tmp;
    S[t] = v[t];
  }
  free(v);
  return ORC_OK;
}

/* ------------------------------------------------------------------ */
/* O4 Greedy (Alg 2) [R7]: M_1 = S[q0]; then repeatedly the  */
/* unpicked point of S farthest from all picked points (max of the     */
/* min-distance), ties -> smallest position in S.                      */
/* ------------------------------------------------------------------ */
int oracle_greedy(const float* data, int32_t d, const int64_t* S, int64_t nS,
                  int64_t nM, int64_t q0, int32_t metric, int64_t* Spos,
                  double* pickdist) {
  double* dist = (double*)malloc(sizeof(double) * (size_t)nS);
  uint8_t* picked = (uint8_t*)calloc((size_t)nS, 1);
  int64_t i, q;
  if (!dist || !picked) {
    free(dist);
    free(picked);
    return ORC_ENOMEM;
  }
  /* Alg 2 l.1-4 */
  Spos[0] = q0;
  picked[q0] = 1;
  if (pickdist) pickdist[0] = INFINITY;
  for (q = 0; q < nS; ++q)
    dist[q] = oracle_full(data + S[q] * d, data + S[q0] * d, d, metric);
  /* Alg 2 l.6-13 */
  for (i = 1; i < nM; ++i) {
    int64_t best = -1;
    double bestd = -1.0;
    for (q = 0; q < nS; ++q) {
      if (picked[q]) continue;
      if (dist[q] > bestd) {
        bestd = dist[q];
        best = q;
      }
    }
    if (best < 0) break; /* cannot happen: nM <= nS */
    Spos[i] = best;
    picked[best] = 1;
    if (pickdist) pickdist[i] = bestd;
    for (q = 0; q < nS; ++q) {
      double t = oracle_full(data + S[q] * d, data + S[best] * d, d, metric);
      if (t < dist[q]) dist[q] = t;
    }
  }
  free(dist);
  free(picked);
  return ORC_OK;
}

/* ------------------------------------------------------------------ */
/* ComputeL (Alg 3) [R6, R9].                                    */
/* ------------------------------------------------------------------ */
void oracle_delta(const float* med, int32_t k, int32_t d, int32_t metric,
                  double* delta) {
  int32_t i, j;
  for (i = 0; i < k; ++i) {
    double m = INFINITY;
    for (j = 0; j < k; ++j) {
      double t;
      if (j == i) continue;
      t = oracle_full(med + (int64_t)i * d, med + (int64_t)j * d, d, metric);
      if (t < m) m = t;
    }
    delta[i] = m;
  }
}

/* L_i = {p : full(p, m_i) <= delta_i}; X_ij = sum_{p in L_i}
 * |p_j - m_ij| / |L_i| (Alg 4 l.1-5). */
void oracle_locality_X(const float* data, int64_t n, int32_t d,
                       const float* med, int32_t k, const double* delta,
                       int32_t metric, uint8_t* inL, int64_t* nL, double* X) {
  int32_t i, j;
  int64_t p;
  for (i = 0; i < k; ++i) {
    const float* m = med + (int64_t)i * d;
    int64_t cnt = 0;
    for (j = 0; j < d; ++j) X[(int64_t)i * d + j] = 0.0;
    for (p = 0; p < n; ++p) {
      const float* x = data + p * d;
      int in = oracle_full(x, m, d, metric) <= delta[i];
      if (inL) inL[p * k + i] = (uint8_t)in;
      if (!in) continue;
      ++cnt;
      for (j = 0; j < d; ++j)
        X[(int64_t)i * d + j] =
            X[(int64_t)i * d + j] + fabs((double)x[j] - (double)m[j]);
    }
    nL[i] = cnt;
    for (j = 0; j < d; ++j) X[(int64_t)i * d + j] = X[(int64_t)i * d + j] / (double)cnt;
  }
}

/* ------------------------------------------------------------------ */
/* FindDimensions (Alg 4 l.6-16) [R2, R3, R10].              */
/* ------------------------------------------------------------------ */
typedef struct {
  double z;
  int32_t i, j;
} zkey;

static int zkey_less(const zkey* a, const zkey* b) {
  if (a->z != b->z) return a->z < b->z;
  if (a->i != b->i) return a->i < b->i;
  return a->j < b->j;
}

/* Plain insertion sort: the key sets are at most k*d long. */
static void zkey_sort(zkey* v, int64_t m) {
  int64_t a, b;
  for (a = 1; a < m; ++a) {
    zkey t = v[a];
    b = a - 1;
    while (b >= 0 && zkey_less(&t, &v[b])) {
      v[b + 1] = v[b];
      --b;
    }
    v[b + 1] = t;
  }
}

int oracle_find_dimensions(const double* X, int32_t k, int32_t d, int32_t l,
                           uint8_t* dmask, double* Zout, double* zgap) {
  int32_t i, j;
  int64_t m = 0, need, t;
  double gap = INFINITY;
  double* Z = (double*)malloc(sizeof(double) * (size_t)k * d);
  zkey* row = (zkey*)malloc(sizeof(zkey) * (size_t)d);
  zkey* rest = (zkey*)malloc(sizeof(zkey) * (size_t)k * d);
  if (!Z || !row || !rest) {
    free(Z);
    free(row);
    free(rest);
    return ORC_ENOMEM;
  }
  memset(dmask, 0, (size_t)k * d);
  for (i = 0; i < k; ++i) {
    const double* x = X + (int64_t)i * d;
    double Y = 0.0, s2 = 0.0, sigma;
    for (j = 0; j < d; ++j) Y = Y + x[j];
    Y = Y / (double)d; /* Y_i = (sum_j X_ij)/d */
    for (j = 0; j < d; ++j) {
      double u = x[j] - Y;
      s2 = s2 + u * u;
    }
    sigma = sqrt(s2 / (double)(d - 1)); /* [R2] two-pass sample std */
    for (j = 0; j < d; ++j)
      Z[(int64_t)i * d + j] = (sigma == 0.0) ? 0.0 : (x[j] - Y) / sigma;
  }
  /* Alg 4 l.15: the two smallest Z_ij of every medoid, keys (Z, j). */
  for (i = 0; i < k; ++i) {
    for (j = 0; j < d; ++j) {
      row[j].z = Z[(int64_t)i * d + j];
      row[j].i = i;
      row[j].j = j;
    }
    zkey_sort(row, d);
    dmask[(int64_t)i * d + row[0].j] = 1;
    dmask[(int64_t)i * d + row[1].j] = 1;
    if (d > 2 && row[2].z - row[1].z < gap) gap = row[2].z - row[1].z;
  }
  /* Alg 4 l.16: the next k*l - 2k smallest overall, keys (Z, i, j). */
  for (i = 0; i < k; ++i)
    for (j = 0; j < d; ++j)
      if (!dmask[(int64_t)i * d + j]) {
        rest[m].z = Z[(int64_t)i * d + j];
        rest[m].i = i;
        rest[m].j = j;
        ++m;
      }
  zkey_sort(rest, m);
  need = (int64_t)k * l - 2 * (int64_t)k;
  for (t = 0; t < need; ++t) dmask[(int64_t)rest[t].i * d + rest[t].j] = 1;
  if (need > 0 && need < m && rest[need].z - rest[need - 1].z < gap)
    gap = rest[need].z - rest[need - 1].z;
  if (Zout) memcpy(Zout, Z, sizeof(double) * (size_t)k * d);
  if (zgap) *zgap = gap;
  free(Z);
  free(row);
  free(rest);
  return ORC_OK;
}

/* ------------------------------------------------------------------ */
/* AssignPoints (Alg 5) [R8]: ties -> smallest medoid index.    */
/* ------------------------------------------------------------------ */
void oracle_assign(const float* data, int64_t n, int32_t d, const float* med,
                   int32_t k, const uint8_t* dmask, int32_t* labels,
                   double* min_rel_gap) {
  int64_t p;
  int32_t i;
  double g = INFINITY;
  for (p = 0; p < n; ++p) {
    double best = INFINITY, second = INFINITY;
    int32_t bi = -1;
    for (i = 0; i < k; ++i) {
      double s = oracle_seg(data + p * d, med + (int64_t)i * d, d,
                            dmask + (int64_t)i * d);
      if (s < best) {
        second = best;
        best = s;
        bi = i;
      } else if (s < second) {
        second = s;
      }
    }
    labels[p] = bi;
    if (second < INFINITY) {
      double r = (second - best) / (best > 0.0 ? best : 1.0);
      if (r < g) g = r;
    }
  }
  if (min_rel_gap) *min_rel_gap = g;
}

/* ------------------------------------------------------------------ */
/* EvaluateCluster (eq 1-2 with the |Data| denominator of eq 8) */
/* [R4, R15].                                                          */
/* ------------------------------------------------------------------ */
double oracle_evaluate(const float* data, int64_t n, int32_t d,
                       const int32_t* labels, int32_t k, const uint8_t* dmask,
                       int64_t* sizes) {
  double cost = 0.0;
  int32_t i, j;
  int64_t p;
  for (i = 0; i < k; ++i) {
    int64_t c = 0;
    double w = 0.0;
    int32_t nd = 0;
    for (p = 0; p < n; ++p) c += (labels[p] == i);
    if (sizes) sizes[i] = c;
    if (c == 0) continue; /* [R15] empty cluster contributes 0 */
    for (j = 0; j < d; ++j) {
      double mu = 0.0, V = 0.0;
      if (!dmask[(int64_t)i * d + j]) continue;
      ++nd;
      for (p = 0; p < n; ++p)
        if (labels[p] == i) mu = mu + (double)data[p * d + j];
      mu = mu / (double)c; /* mu_ij */
      for (p = 0; p < n; ++p)
        if (labels[p] == i) V = V + fabs((double)data[p * d + j] - mu);
      V = V / (double)c; /* V_ij, eq 1 */
      w = w + V;
    }
    w = w / (double)nd;              /* w_i, eq 1 */
    cost = cost + (double)c * w;     /* eq 2 / eq 8 numerator */
  }
  return cost / (double)n;           /* eq 8: / |Data| */
}

/* eq 9: cost = sum_i sum_{j in D_i} sum_{p in C_i}
 * |p_j - mu_ij| / (|D_i| |Data|).  Used only as a pin of eq 1-2. */
double oracle_evaluate_eq9(const float* data, int64_t n, int32_t d,
                           const int32_t* labels, int32_t k,
                           const uint8_t* dmask) {
  double cost = 0.0;
  int32_t i, j;
  int64_t p;
  for (i = 0; i < k; ++i) {
    int64_t c = 0;
    int32_t nd = 0;
    for (p = 0; p < n; ++p) c += (labels[p] == i);
    for (j = 0; j < d; ++j) nd += dmask[(int64_t)i * d + j] ? 1 : 0;
    if (c == 0) continue;
    for (j = 0; j < d; ++j) {
      double mu = 0.0;
      if (!dmask[(int64_t)i * d + j]) continue;
      for (p = 0; p < n; ++p)
        if (labels[p] == i) mu = mu + (double)data[p * d + j];
      mu = mu / (double)c;
      for (p = 0; p < n; ++p)
        if (labels[p] == i)
          cost = cost + fabs((double)data[p * d + j] - mu) /
                            ((double)nd * (double)n);
    }
  }
  return cost;
}

/* ------------------------------------------------------------------ */
/* ComputeBadMedoids (Alg 1 l.13) [R11].                         */
/* ------------------------------------------------------------------ */
void oracle_bad_medoids(const int64_t* sizes, int32_t k, int64_t n,
                        double minDev, uint8_t* bad) {
  double thr = (double)n / (double)k * minDev;
  int32_t i, any = 0, smallest = 0;
  for (i = 0; i < k; ++i) {
    bad[i] = (double)sizes[i] < thr;
    any |= bad[i];
    if (sizes[i] < sizes[smallest]) smallest = i;
  }
  if (!any) bad[smallest] = 1;
}

/* ------------------------------------------------------------------ */
/* Refinement FindDimensions input (Alg 1 l.16-17): L <- CBest.        */
/* ------------------------------------------------------------------ */
void oracle_cluster_X(const float* data, int64_t n, int32_t d,
                      const int32_t* labels, const float* med, int32_t k,
                      double* X) {
  int32_t i, j;
  int64_t p;
  for (i = 0; i < k; ++i) {
    int64_t c = 0;
    for (j = 0; j < d; ++j) X[(int64_t)i * d + j] = 0.0;
    for (p = 0; p < n; ++p) {
      if (labels[p] != i) continue;
      ++c;
      for (j = 0; j < d; ++j)
        X[(int64_t)i * d + j] =
            X[(int64_t)i * d + j] +
            fabs((double)data[p * d + j] - (double)med[(int64_t)i * d + j]);
    }
    if (c == 0) continue; /* [R15] empty cluster -> row of 0 */
    for (j = 0; j < d; ++j) X[(int64_t)i * d + j] = X[(int64_t)i * d + j] / (double)c;
  }
}

/* RemoveOutliers [R5, R17]. */
void oracle_remove_outliers(const float* data, int64_t n, int32_t d,
                            const float* med, int32_t k, const uint8_t* dmask,
                            int32_t* labels, double* Delta) {
  int32_t i, j;
  int64_t p;
  double* D = Delta ? Delta : (double*)malloc(sizeof(double) * (size_t)k);
  for (i = 0; i < k; ++i) {
    double m = INFINITY;
    for (j = 0; j < k; ++j) {
      double t;
      if (j == i) continue;
      t = oracle_seg(med + (int64_t)i * d, med + (int64_t)j * d, d,
                     dmask + (int64_t)i * d);
      if (t < m) m = t;
    }
    D[i] = m;
  }
  for (p = 0; p < n; ++p) {
    int outside_all = 1;
    for (i = 0; i < k; ++i)
      if (!(oracle_seg(data + p * d, med + (int64_t)i * d, d,
                       dmask + (int64_t)i * d) > D[i])) {
        outside_all = 0;
        break;
      }
    if (outside_all) labels[p] = -1;
  }
  if (!Delta) free(D);
}

/* ------------------------------------------------------------------ */
/* FAST-PROCLUS caches: Dist rows, DistFound, delta',      */
/* |L| and H per potential medoid; Theorems 3.1 / 3.2.                 */
/* ------------------------------------------------------------------ */
typedef struct {
  int64_t nM, n;
  int32_t d;
  double* Dist;     /* nM * n, row allocated lazily */
  uint8_t* found;   /* DistFound */
  uint8_t* used;    /* delta' valid */
  double* dprev;    /* delta' */
  int64_t* nL;      /* |L| */
  double* H;        /* nM * d */
} fast_cache;

static int fast_init(fast_cache* c, int64_t nM, int64_t n, int32_t d) {
  c->nM = nM;
  c->n = n;
  c->d = d;
  c->Dist = (double*)malloc(sizeof(double) * (size_t)nM * (size_t)n);
  c->found = (uint8_t*)calloc((size_t)nM, 1);
  c->used = (uint8_t*)calloc((size_t)nM, 1);
  c->dprev = (double*)calloc((size_t)nM, sizeof(double));
  c->nL = (int64_t*)calloc((size_t)nM, sizeof(int64_t));
  c->H = (double*)calloc((size_t)nM * d, sizeof(double));
  return (c->Dist && c->found && c->used && c->dprev && c->nL && c->H)
             ? ORC_OK
             : ORC_ENOMEM;
}

static void fast_free(fast_cache* c) {
  free(c->Dist);
  free(c->found);
  free(c->used);
  free(c->dprev);
  free(c->nL);
  free(c->H);
}

/* One ComputeL + X for slot i using the cache (GPU-FAST-PROCLUS 4.2). */
static void fast_locality_X(fast_cache* c, const float* data, int64_t mpos,
                            const float* m, double delta, int32_t metric,
                            int64_t* nL, double* Xrow) {
  int64_t p, n = c->n, cnt = 0;
  int32_t j, d = c->d;
  double* row = c->Dist + mpos * n;
  double* H = c->H + mpos * d;
  double lam = 1.0;
  double lo, hi;
  int band_kind; /* 0: none, 1: first use (dist <= delta), 2: (lo, hi] */
  if (!c->found[mpos]) { /* compute distances only once */
    for (p = 0; p < n; ++p) row[p] = oracle_full(data + p * d, m, d, metric);
    c->found[mpos] = 1;
  }
  if (!c->used[mpos]) {
    band_kind = 1;
    lo = -INFINITY;
    hi = delta;
  } else if (delta > c->dprev[mpos]) { /* eq 3, increase: lambda = +1 */
    band_kind = 2;
    lo = c->dprev[mpos];
    hi = delta;
  } else if (delta < c->dprev[mpos]) { /* eq 3, decrease: lambda = -1 */
    band_kind = 2;
    lo = delta;
    hi = c->dprev[mpos];
    lam = -1.0;
  } else {
    band_kind = 0;
    lo = hi = 0.0;
  }
  if (band_kind) {
    double* s = (double*)calloc((size_t)d, sizeof(double));
    for (p = 0; p < n; ++p) {
      int in = (band_kind == 1) ? (row[p] <= hi) : (row[p] > lo && row[p] <= hi);
      if (!in) continue;
      ++cnt;
      for (j = 0; j < d; ++j)
        s[j] = s[j] + fabs((double)data[p * d + j] - (double)m[j]);
    }
    for (j = 0; j < d; ++j) H[j] = H[j] + lam * s[j]; /* eq 6 */
    c->nL[mpos] += (lam > 0 ? cnt : -cnt);
    free(s);
  }
  c->used[mpos] = 1;
  c->dprev[mpos] = delta;
  *nL = c->nL[mpos];
  for (j = 0; j < d; ++j) Xrow[j] = H[j] / (double)c->nL[mpos];
}

/* ------------------------------------------------------------------ */
/* Iterative + refinement phase on a given S and M (Alg 1 l.4-20).     */
/* ------------------------------------------------------------------ */
static void gather_rows(const float* data, int32_t d, const int64_t* ids,
                        int32_t k, float* out) {
  int32_t i;
  for (i = 0; i < k; ++i)
    memcpy(out + (int64_t)i * d, data + ids[i] * d, sizeof(float) * (size_t)d);
}

static int run_core(const float* data, int64_t n, int32_t d,
                    const int64_t* Mid /* point ids of M, nM */, int64_t nM,
                    const oracle_params* prm, uint64_t it_state,
                    oracle_result* out, oracle_trace* tr,
                    const int64_t* warm, int32_t nwarm, int64_t* mbest_out) {
  const int32_t k = prm->k, l = prm->l, metric = prm->metric;
  const int32_t max_iter = prm->max_iter > 0 ? prm->max_iter : 10000;
  int32_t i, j, itr = 0, iterations = 0;
  int rc = ORC_OK;
  double costBest = INFINITY;
  uint64_t st = it_state;
  int64_t *MCur = NULL, *MBest = NULL, *pool = NULL, *sizes = NULL,
          *sizesBest = NULL, *nL = NULL, *ids = NULL, t;
  int32_t *labels = NULL, *CBest = NULL, *tmpl;
  uint8_t *dmask = NULL, *bad = NULL, *inpool = NULL;
  double *delta = NULL, *X = NULL;
  float* med = NULL;
  fast_cache fc;
  memset(&fc, 0, sizeof(fc));

  MCur = (int64_t*)malloc(sizeof(int64_t) * k);
  MBest = (int64_t*)malloc(sizeof(int64_t) * k);
  ids = (int64_t*)malloc(sizeof(int64_t) * k);
  pool = (int64_t*)malloc(sizeof(int64_t) * (size_t)nM);
  inpool = (uint8_t*)malloc((size_t)nM);
  sizes = (int64_t*)malloc(sizeof(int64_t) * k);
  sizesBest = (int64_t*)calloc(k, sizeof(int64_t));
  nL = (int64_t*)malloc(sizeof(int64_t) * k);
  labels = (int32_t*)malloc(sizeof(int32_t) * (size_t)n);
  CBest = (int32_t*)malloc(sizeof(int32_t) * (size_t)n);
  dmask = (uint8_t*)malloc((size_t)k * d);
  bad = (uint8_t*)malloc((size_t)k);
  delta = (double*)malloc(sizeof(double) * k);
  X = (double*)malloc(sizeof(double) * (size_t)k * d);
  med = (float*)malloc(sizeof(float) * (size_t)k * d);
  if (!MCur || !MBest || !ids || !pool || !inpool || !sizes || !sizesBest ||
      !nL || !labels || !CBest || !dmask || !bad || !delta || !X || !med) {
    rc = ORC_ENOMEM;
    goto done;
  }
  if (prm->fast && fast_init(&fc, nM, n, d) != ORC_OK) {
    rc = ORC_ENOMEM;
    goto done;
  }

  if (warm && nwarm > 0) {
    /* Multi-param level 3 [R21]: MCur is a random subset of the
     * previous setting's MBest: partial Fisher-Yates over MBest_prev in slot
     * order for the first min(k, |MBest_prev|) slots; if k is larger, the
     * remaining slots by partial Fisher-Yates over the ascending positions of
     * M not in MBest_prev.  All draws from stream IT, in slot order. */
    const int32_t m = k < nwarm ? k : nwarm;
    int64_t np2 = 0;
    for (t = 0; t < nwarm; ++t) pool[t] = warm[t];
    for (i = 0; i < m; ++i) {
      int64_t r = i + (int64_t)oracle_uniform(&st, (uint64_t)(nwarm - i));
      int64_t tmp = pool[i];
      pool[i] = pool[r];
      pool[r] = tmp;
      MCur[i] = pool[i];
    }
    if (k > nwarm) {
      for (t = 0; t < nM; ++t) inpool[t] = 1;
      for (t = 0; t < nwarm; ++t) inpool[warm[t]] = 0;
      for (t = 0; t < nM; ++t)
        if (inpool[t]) pool[np2++] = t;
      for (i = nwarm; i < k; ++i) {
        const int64_t u = i - nwarm;
        int64_t r = u + (int64_t)oracle_uniform(&st, (uint64_t)(np2 - u));
        int64_t tmp = pool[u];
        pool[u] = pool[r];
        pool[r] = tmp;
        MCur[i] = pool[u];
      }
    }
  } else {
    /* O5 [R12]: MCur = k distinct positions of M (partial Fisher-Yates). */
    for (t = 0; t < nM; ++t) pool[t] = t;
    for (i = 0; i < k; ++i) {
      int64_t r = i + (int64_t)oracle_uniform(&st, (uint64_t)(nM - i));
      int64_t tmp = pool[i];
      pool[i] = pool[r];
      pool[r] = tmp;
      MCur[i] = pool[i];
    }
  }
  for (i = 0; i < k; ++i) MBest[i] = MCur[i];
  if (tr) tr->count = 0;

  /* Iterative phase, Alg 1 l.5-14 [R14]. */
  while (itr < prm->itrPat && iterations < max_iter) {
    double cost, zgap, agap;
    int improved;
    for (i = 0; i < k; ++i) ids[i] = Mid[MCur[i]];
    gather_rows(data, d, ids, k, med);
    /* l.6 ComputeL */
    oracle_delta(med, k, d, metric, delta);
    if (prm->fast) {
      for (i = 0; i < k; ++i)
        fast_locality_X(&fc, data, MCur[i], med + (int64_t)i * d, delta[i],
                        metric, &nL[i], X + (int64_t)i * d);
    } else {
      oracle_locality_X(data, n, d, med, k, delta, metric, NULL, nL, X);
    }
    /* l.7 FindDimensions */
    if (oracle_find_dimensions(X, k, d, l, dmask, NULL, &zgap) != ORC_OK) {
      rc = ORC_ENOMEM;
      goto done;
    }
    /* l.8 AssignPoints, l.9 EvaluateClusters */
    oracle_assign(data, n, d, med, k, dmask, labels, &agap);
    cost = oracle_evaluate(data, n, d, labels, k, dmask, sizes);
    /* l.10-12 */
    ++itr;
    ++iterations;
    improved = cost < costBest;
    if (tr && tr->count < tr->cap) {
      int32_t c = tr->count;
      if (tr->costgap)
        tr->costgap[c] = isinf(costBest) ? INFINITY
                                         : fabs(cost - costBest) /
                                               (cost > costBest ? cost : costBest);
    }
    if (improved) {
      itr = 0;
      costBest = cost;
      for (i = 0; i < k; ++i) {
        MBest[i] = MCur[i];
        sizesBest[i] = sizes[i];
      }
      tmpl = CBest;
      CBest = labels;
      labels = tmpl;
    }
    /* l.13 ComputeBadMedoids (from MBest / CBest) */
    oracle_bad_medoids(sizesBest, k, n, prm->minDev, bad);
    if (tr && tr->count < tr->cap) {
      int32_t c = tr->count;
      for (i = 0; i < k; ++i) {
        if (tr->mcur) tr->mcur[c * k + i] = (int32_t)MCur[i];
        if (tr->delta) tr->delta[c * k + i] = delta[i];
        if (tr->nL) tr->nL[c * k + i] = nL[i];
        if (tr->sizes) tr->sizes[c * k + i] = sizes[i];
        if (tr->bad) tr->bad[c * k + i] = bad[i];
      }
      if (tr->dims) memcpy(tr->dims + (int64_t)c * k * d, dmask, (size_t)k * d);
      if (tr->X) memcpy(tr->X + (int64_t)c * k * d, X, sizeof(double) * k * d);
      if (tr->cost) tr->cost[c] = cost;
      if (tr->improved) tr->improved[c] = (uint8_t)improved;
      if (tr->zgap) tr->zgap[c] = zgap;
      if (tr->assign_gap) tr->assign_gap[c] = agap;
      tr->count = c + 1;
    }
    /* l.14 replace bad medoids of MBest by random points of M \ MBest */
    {
      int64_t np = 0;
      memset(inpool, 1, (size_t)nM);
      for (i = 0; i < k; ++i) inpool[MBest[i]] = 0;
      for (t = 0; t < nM; ++t)
        if (inpool[t]) pool[np++] = t;
      for (i = 0; i < k; ++i) MCur[i] = MBest[i];
      for (i = 0; i < k; ++i) {
        int64_t r;
        if (!bad[i] || np == 0) continue;
        r = (int64_t)oracle_uniform(&st, (uint64_t)np);
        MCur[i] = pool[r];
        for (t = r; t + 1 < np; ++t) pool[t] = pool[t + 1];
        --np;
      }
    }
  }

  /* Refinement phase, Alg 1 l.16-19. */
  for (i = 0; i < k; ++i) ids[i] = Mid[MBest[i]];
  gather_rows(data, d, ids, k, med);
  oracle_cluster_X(data, n, d, CBest, med, k, X);
  if (oracle_find_dimensions(X, k, d, l, dmask, NULL, NULL) != ORC_OK) {
    rc = ORC_ENOMEM;
    goto done;
  }
  oracle_assign(data, n, d, med, k, dmask, out->labels, NULL);
  oracle_remove_outliers(data, n, d, med, k, dmask, out->labels, NULL);
  for (i = 0; i < k; ++i) out->medoids[i] = ids[i];
  memcpy(out->dims, dmask, (size_t)k * d);
  out->cost = costBest;
  out->iterations = iterations;
  if (mbest_out)
    for (i = 0; i < k; ++i) mbest_out[i] = MBest[i];
  (void)j;

done:
  if (prm->fast) fast_free(&fc);
  free(MCur);
  free(MBest);
  free(ids);
  free(pool);
  free(inpool);
  free(sizes);
  free(sizesBest);
  free(nL);
  free(labels);
  free(CBest);
  free(dmask);
  free(bad);
  free(delta);
  free(X);
  free(med);
  return rc;
}

/* Initialization phase (Alg 1 l.2-3) for a given k_sm, then run_core. */
static int init_phase(const float* data, int64_t n, int32_t d, int32_t k_sm,
                      const oracle_params* prm, int64_t* nS_out,
                      int64_t* nM_out, int64_t** Mid_out) {
  int64_t nS = (int64_t)prm->A * k_sm, nM, q0, t;
  uint64_t st = oracle_stream_sm(prm->seed, k_sm);
  int64_t *S, *Spos, *Mid;
  int rc;
  if (nS > n) nS = n;
  nM = (int64_t)prm->B * k_sm;
  if (nM > nS) nM = nS;
  S = (int64_t*)malloc(sizeof(int64_t) * (size_t)nS);
  Spos = (int64_t*)malloc(sizeof(int64_t) * (size_t)nM);
  Mid = (int64_t*)malloc(sizeof(int64_t) * (size_t)nM);
  if (!S || !Spos || !Mid) {
    free(S);
    free(Spos);
    free(Mid);
    return ORC_ENOMEM;
  }
  rc = oracle_sample(n, nS, &st, S);
  if (rc == ORC_OK) {
    q0 = (int64_t)oracle_uniform(&st, (uint64_t)nS);
    rc = oracle_greedy(data, d, S, nS, nM, q0, prm->metric, Spos, NULL);
  }
  if (rc == ORC_OK)
    for (t = 0; t < nM; ++t) Mid[t] = S[Spos[t]];
  free(S);
  free(Spos);
  if (rc != ORC_OK) {
    free(Mid);
    return rc;
  }
  *nS_out = nS;
  *nM_out = nM;
  *Mid_out = Mid;
  return ORC_OK;
}

int oracle_proclus(const float* data, int64_t n, int32_t d,
                   const oracle_params* prm, oracle_result* out,
                   oracle_trace* trace) {
  int64_t nS, nM, *Mid = NULL;
  int rc = oracle_validate(n, d, data, prm);
  if (rc != ORC_OK) return rc;
  rc = init_phase(data, n, d, prm->k, prm, &nS, &nM, &Mid);
  if (rc != ORC_OK) return rc;
  out->nS = nS;
  out->nM = nM;
  rc = run_core(data, n, d, Mid, nM, prm,
                oracle_stream_it(prm->seed, prm->k, prm->l), out, trace, NULL, 0, NULL);
  free(Mid);
  return rc;
}

int oracle_proclus_multi(const float* data, int64_t n, int32_t d,
                         const int32_t* ks, int32_t nk, const int32_t* ls,
                         int32_t nl, const oracle_params* base,
                         int32_t reuse_level, oracle_result* outs) {
  int32_t a, b, kmax = 0;
  int64_t nS = 0, nM = 0, *Mid = NULL;
  int rc = ORC_OK;
  oracle_params p = *base;
  if (nk < 1 || nl < 1 || reuse_level < 1 || reuse_level > 3) return ORC_EINVAL;
  for (a = 0; a < nk; ++a) {
    if (ks[a] > kmax) kmax = ks[a];
    for (b = 0; b < nl; ++b) {
      p.k = ks[a];
      p.l = ls[b];
      if ((rc = oracle_validate(n, d, a == 0 && b == 0 ? data : NULL, &p)) != ORC_OK)
        return rc;
    }
  }
  if (reuse_level == 1) {
    for (a = 0; a < nk; ++a)
      for (b = 0; b < nl; ++b) {
        p.k = ks[a];
        p.l = ls[b];
        rc = oracle_proclus(data, n, d, &p, &outs[a * nl + b], NULL);
        if (rc != ORC_OK) return rc;
      }
    return ORC_OK;
  }
  /* Level 2: greedy once for the largest k, shared M.  Level 3
   * [R21]: every setting after the first starts from a random subset
   * of the previous setting's MBest (grid in caller order). */
  p.k = kmax;
  rc = init_phase(data, n, d, kmax, &p, &nS, &nM, &Mid);
  if (rc != ORC_OK) return rc;
  {
    int64_t* warm = (int64_t*)malloc(sizeof(int64_t) * (size_t)kmax);
    int64_t* next = (int64_t*)malloc(sizeof(int64_t) * (size_t)kmax);
    int32_t nwarm = 0;
    if (!warm || !next) rc = ORC_ENOMEM;
    for (a = 0; a < nk && rc == ORC_OK; ++a)
      for (b = 0; b < nl && rc == ORC_OK; ++b) {
        p.k = ks[a];
        p.l = ls[b];
        outs[a * nl + b].nS = nS;
        outs[a * nl + b].nM = nM;
        rc = run_core(data, n, d, Mid, nM, &p, oracle_stream_it(p.seed, p.k, p.l),
                      &outs[a * nl + b], NULL, reuse_level == 3 ? warm : NULL,
                      reuse_level == 3 ? nwarm : 0, next);
        memcpy(warm, next, sizeof(int64_t) * (size_t)p.k);
        nwarm = p.k;
      }
    free(warm);
    free(next);
  }
  free(Mid);
  return rc;
}

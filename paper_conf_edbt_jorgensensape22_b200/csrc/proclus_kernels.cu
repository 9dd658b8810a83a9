// proclus_kernels.cu -- sm_100a kernels of the PROCLUS hot path
// (GPU-FAST-PROCLUS, section 4, re-designed for B200).
//
// Every per-iteration pass is a persistent, chunk-streaming kernel: the grid
// is a multiple of the SM count, block b owns the chunks b, b+G, b+2G, ...
// of P consecutive points (a static schedule, so every partial sum has a
// fixed reduction order and the whole run is deterministic).  A chunk is
// staged in shared memory as fp64 (one coalesced fp32 load per dimension and
// point, SoA layout), the per-point decisions are taken by one thread per
// point in exactly the oracle's fp64 arithmetic, and the per-(cluster,
// dimension) sums are computed by "cells": one thread per (i, j) walks the
// compacted member list of cluster / band i inside the chunk.  No floating
// point atomics anywhere.  The last block to finish reduces the per-block
// partials in block order and runs the small single-block step of the
// algorithm that follows (finalise H and select dimensions, centroids, cost
// and the Alg 1 l.10-14 control), so an iteration is three launches.
#include <math_constants.h>

#include "proclus_kernels.h"

namespace pc {

// ===================================================================== N0
__global__ void k_pack_soa(const float* __restrict__ in, long long n, int d,
                           long long n_pad, float* __restrict__ xs, int* bad) {
  __shared__ float tile[32][33];
  const long long p0 = (long long)blockIdx.x * 32;
  const int j0 = blockIdx.y * 32;
  const int tx = threadIdx.x, ty = threadIdx.y;
  int nonfinite = 0;
  for (int r = ty; r < 32; r += 8) {
    long long p = p0 + r;
    int j = j0 + tx;
    float v = 0.f;
    if (p < n && j < d) {
      v = in[p * d + j];
      if (!isfinite(v)) nonfinite = 1;
    }
    tile[r][tx] = v;
  }
  if (nonfinite) atomicOr(bad, 1);
  __syncthreads();
  for (int r = ty; r < 32; r += 8) {
    int j = j0 + r;
    long long p = p0 + tx;
    if (j < d && p < n_pad) xs[(long long)j * n_pad + p] = tile[tx][r];
  }
}

void launch_pack_soa(const float* in, long long n, int d, long long n_pad,
                     float* xs, int* bad, cudaStream_t s) {
  dim3 grid((unsigned)((n_pad + 31) / 32), (unsigned)((d + 31) / 32));
  k_pack_soa<<<grid, dim3(32, 8), 0, s>>>(in, n, d, n_pad, xs, bad);
}

__global__ void k_gather_rows(const float* __restrict__ xs, long long n_pad,
                              int d, const long long* __restrict__ ids,
                              long long row_offset, long long n_local, int cnt,
                              float* __restrict__ out) {
  const long long tot = (long long)cnt * d;
  for (long long e = blockIdx.x * (long long)blockDim.x + threadIdx.x; e < tot;
       e += (long long)gridDim.x * blockDim.x) {
    int t = (int)(e / d), j = (int)(e - (long long)t * d);
    long long r = ids[t] - row_offset;
    out[e] = (r >= 0 && r < n_local) ? xs[(long long)j * n_pad + r] : 0.f;
  }
}

void launch_gather_rows(const float* xs, long long n_pad, int d,
                        const long long* ids, long long row_offset,
                        long long n_local, int cnt, float* out, cudaStream_t s) {
  long long tot = (long long)cnt * d;
  int blocks = (int)((tot + 255) / 256);
  if (blocks < 1) blocks = 1;
  if (blocks > 1184) blocks = 1184;
  k_gather_rows<<<blocks, 256, 0, s>>>(xs, n_pad, d, ids, row_offset, n_local,
                                       cnt, out);
}

__global__ void k_gather_m(const float* __restrict__ srows,
                           const long long* __restrict__ sids,
                           const int* __restrict__ spos, int nM, int d,
                           float* __restrict__ mrows, long long* __restrict__ mids) {
  for (int e = blockIdx.x * blockDim.x + threadIdx.x; e < nM * d;
       e += gridDim.x * blockDim.x) {
    int i = e / d, j = e - i * d;
    mrows[e] = srows[(long long)spos[i] * d + j];
    if (j == 0) mids[i] = sids[spos[i]];
  }
}

void launch_gather_m(const float* srows, const long long* sids, const int* spos,
                     int nM, int d, float* mrows, long long* mids,
                     cudaStream_t s) {
  int blocks = (nM * d + 255) / 256;
  if (blocks < 1) blocks = 1;
  if (blocks > 592) blocks = 592;
  k_gather_m<<<blocks, 256, 0, s>>>(srows, sids, spos, nM, d, mrows, mids);
}

// ===================================================================== N1
// Greedy (Alg 2) in a single CTA: all #M-1 dependent picks in one
// launch instead of two launches per pick.  dist[q] is the min distance of
// S-position q to the picked set (-1 once picked, reading R7); the argmax
// prefers the larger value, then the smaller position.
__device__ __forceinline__ void argmax_merge(double& v, int& q, double v2, int q2) {
  if (v2 > v || (v2 == v && q2 < q)) {
    v = v2;
    q = q2;
  }
}

__global__ void __launch_bounds__(1024)
    k_greedy(const float* __restrict__ srows, int nS, int d, int nM, int q0,
             int metric, int rows_in_smem, int* __restrict__ spos,
             double* __restrict__ pickdist) {
  extern __shared__ double gsm[];
  double* dist = gsm;                               // [nS]
  double* prow = gsm + nS;                          // [d] picked row
  double* rows = prow + d;                          // [nS][d] if cached
  __shared__ double wv[32];
  __shared__ int wq[32];
  __shared__ int pick;
  const int tid = threadIdx.x, bd = blockDim.x;
  const int lane = tid & 31, w = tid >> 5, nw = (bd + 31) >> 5;

  if (rows_in_smem)
    for (int e = tid; e < nS * d; e += bd) rows[e] = (double)srows[e];
  for (int j = tid; j < d; j += bd) prow[j] = (double)srows[(long long)q0 * d + j];
  __syncthreads();

  auto dist_to_pick = [&](int q) -> double {
    if (rows_in_smem) return full_dist(rows + (long long)q * d, 1, prow, d, metric);
    const float* r = srows + (long long)q * d;
    double s = 0.0;
    if (metric == 1) {
      for (int j = 0; j < d; ++j) s = dadd(s, fabs(dsub((double)r[j], prow[j])));
      return s;
    }
    for (int j = 0; j < d; ++j) {
      double t = dsub((double)r[j], prow[j]);
      s = dadd(s, dmul(t, t));
    }
    return __dsqrt_rn(s);
  };

  for (int q = tid; q < nS; q += bd) dist[q] = (q == q0) ? -1.0 : dist_to_pick(q);
  if (tid == 0) {
    spos[0] = q0;
    if (pickdist) pickdist[0] = CUDART_INF;
  }
  for (int i = 1; i < nM; ++i) {
    __syncthreads();
    double v = -2.0;
    int q = 0x7fffffff;
    for (int t = tid; t < nS; t += bd) argmax_merge(v, q, dist[t], t);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      double v2 = __shfl_down_sync(0xffffffffu, v, o);
      int q2 = __shfl_down_sync(0xffffffffu, q, o);
      argmax_merge(v, q, v2, q2);
    }
    if (lane == 0) {
      wv[w] = v;
      wq[w] = q;
    }
    __syncthreads();
    if (w == 0) {
      v = lane < nw ? wv[lane] : -2.0;
      q = lane < nw ? wq[lane] : 0x7fffffff;
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) {
        double v2 = __shfl_down_sync(0xffffffffu, v, o);
        int q2 = __shfl_down_sync(0xffffffffu, q, o);
        argmax_merge(v, q, v2, q2);
      }
      if (lane == 0) {
        pick = q;
        spos[i] = q;
        if (pickdist) pickdist[i] = v;
      }
    }
    __syncthreads();
    const int qs = pick;
    for (int j = tid; j < d; j += bd)
      prow[j] = rows_in_smem ? rows[(long long)qs * d + j]
                             : (double)srows[(long long)qs * d + j];
    __syncthreads();
    for (int t = tid; t < nS; t += bd) {
      if (t == qs) {
        dist[t] = -1.0;
      } else if (dist[t] >= 0.0) {
        double u = dist_to_pick(t);
        if (u < dist[t]) dist[t] = u;
      }
    }
  }
}

cudaError_t launch_greedy(const float* srows, int nS, int d, int nM, int q0,
                          int metric, int* spos, double* pickdist,
                          cudaStream_t s) {
  size_t base = sizeof(double) * ((size_t)nS + d);
  size_t rows = sizeof(double) * (size_t)nS * d;
  int in_smem = base + rows <= 200 * 1024;
  size_t smem = base + (in_smem ? rows : 0);
  cudaError_t e = cudaFuncSetAttribute(k_greedy,
                                       cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       (int)smem);
  if (e != cudaSuccess) return e;
  k_greedy<<<1, 1024, smem, s>>>(srows, nS, d, nM, q0, metric, in_smem, spos,
                                 pickdist);
  return cudaGetLastError();
}

// ============================================================ block helpers
// Shared scratch for compacting per-point membership bitmasks into per-set
// member lists (ascending point order inside the chunk).
struct ListScratch {
  unsigned* ballot;   // [KMAX][WMAX]
  int* woff;          // [KMAX][WMAX]
  int* cnt;           // [KMAX]
  int* base;          // [KMAX]
  unsigned short* list;  // [sum of counts]
};

__device__ void build_lists(unsigned mask, int nsets, ListScratch ls) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const int W = blockDim.x >> 5;
  for (int a = 0; a < nsets; ++a) {
    unsigned b = __ballot_sync(0xffffffffu, (mask >> a) & 1u);
    if (lane == 0) ls.ballot[a * WMAX + w] = b;
  }
  __syncthreads();
  if (threadIdx.x < nsets) {
    const int a = threadIdx.x;
    int tot = 0;
    for (int v = 0; v < W; ++v) {
      ls.woff[a * WMAX + v] = tot;
      tot += __popc(ls.ballot[a * WMAX + v]);
    }
    ls.cnt[a] = tot;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    int s = 0;
    for (int a = 0; a < nsets; ++a) {
      ls.base[a] = s;
      s += ls.cnt[a];
    }
  }
  __syncthreads();
  const unsigned lt = (1u << lane) - 1u;
  unsigned m = mask;
  while (m) {
    const int a = __ffs(m) - 1;
    m &= m - 1u;
    int pos = ls.base[a] + ls.woff[a * WMAX + w] +
              __popc(ls.ballot[a * WMAX + w] & lt);
    ls.list[pos] = (unsigned short)threadIdx.x;
  }
  __syncthreads();
}

// sum_{t < cnt} f(x[L[t]]) with four interleaved partial sums combined in a
// fixed order (deterministic).  MODE 0: x, MODE 1: |x - c|.
template <int MODE>
__device__ __forceinline__ double list_sum(const double* __restrict__ xr,
                                           const unsigned short* __restrict__ L,
                                           int cnt, double c) {
  double s0 = 0.0, s1 = 0.0, s2 = 0.0, s3 = 0.0;
  int t = 0;
  for (; t + 4 <= cnt; t += 4) {
    double v0 = xr[L[t]], v1 = xr[L[t + 1]], v2 = xr[L[t + 2]], v3 = xr[L[t + 3]];
    if (MODE == 1) {
      v0 = fabs(dsub(v0, c));
      v1 = fabs(dsub(v1, c));
      v2 = fabs(dsub(v2, c));
      v3 = fabs(dsub(v3, c));
    }
    s0 = dadd(s0, v0);
    s1 = dadd(s1, v1);
    s2 = dadd(s2, v2);
    s3 = dadd(s3, v3);
  }
  for (; t < cnt; ++t) {
    double v = xr[L[t]];
    if (MODE == 1) v = fabs(dsub(v, c));
    s0 = dadd(s0, v);
  }
  return dadd(dadd(s0, s1), dadd(s2, s3));
}

// Stage one chunk (P points, all d dimensions) as fp64: x_s[j*(P+1) + p].
__device__ __forceinline__ void stage_chunk(const float* __restrict__ xs,
                                            long long n_pad, int d,
                                            long long base, int P,
                                            double* __restrict__ x_s) {
  const int p = threadIdx.x;
  const float* src = xs + base + p;
#pragma unroll 4
  for (int j = 0; j < d; ++j) x_s[j * (P + 1) + p] = (double)__ldg(src + (long long)j * n_pad);
}

// The last block to arrive (ticket) returns true; it then sees every other
// block's partials (threadfence before the ticket, reads with ld.cg).
__device__ bool last_block(unsigned int* ticket) {
  __shared__ int is_last;
  __threadfence();
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned t = atomicAdd(ticket, 1u);
    is_last = (t == gridDim.x - 1);
  }
  __syncthreads();
  if (is_last) {
    __threadfence();
    if (threadIdx.x == 0) *ticket = 0u;
  }
  return is_last;
}

// Sum the per-block partials in block order into red / redc.
__device__ void reduce_partials(const double* part, const long long* partc,
                                int G, int stride, int ncell, int ncnt,
                                double* red, long long* redc) {
  for (int c = threadIdx.x; c < ncell; c += blockDim.x) {
    double s = 0.0;
    for (int b = 0; b < G; ++b) s = dadd(s, __ldcg(part + (long long)b * stride + c));
    red[c] = s;
  }
  for (int c = threadIdx.x; c < ncnt; c += blockDim.x) {
    long long s = 0;
    for (int b = 0; b < G; ++b) s += __ldcg(partc + (long long)b * KMAX + c);
    redc[c] = s;
  }
  __syncthreads();
}

// ============================================================ FindDimensions
// Y_i, sigma_i, Z_ij (Alg 4 l.6-13, readings R2, R3) and the
// selection of Alg 4 l.15-16 (reading R10): per medoid the two smallest by
// (Z, j), then the k*l - 2k smallest of the rest by (Z, i, j), found with a
// block-wide radix select on order-preserving keys.  Whole block; X, Z,
// dmask, dlist in global memory; nD[k] gets |D_i|.
__device__ void zscore_select(const double* X, int k, int d, int l, double* Z,
                              unsigned char* dmask, int* dlist, int* nD) {
  __shared__ double Ys[KMAX], Ss[KMAX];
  __shared__ unsigned int hist[256];
  __shared__ unsigned long long prefix_s;
  __shared__ int need_s;
  __shared__ int tcount[1024];
  const int tid = threadIdx.x, bd = blockDim.x;
  const int kd = k * d;
  if (tid < k) {
    const double* x = X + (long long)tid * d;
    double Y = 0.0, s2 = 0.0;
    for (int j = 0; j < d; ++j) Y = dadd(Y, x[j]);
    Y = ddiv(Y, (double)d);
    for (int j = 0; j < d; ++j) {
      double u = dsub(x[j], Y);
      s2 = dadd(s2, dmul(u, u));
    }
    Ys[tid] = Y;
    Ss[tid] = __dsqrt_rn(ddiv(s2, (double)(d - 1)));
  }
  __syncthreads();
  for (int c = tid; c < kd; c += bd) {
    const int i = c / d;
    const double sg = Ss[i];
    Z[c] = (sg == 0.0) ? 0.0 : ddiv(dsub(X[c], Ys[i]), sg);
    dmask[c] = 0;
  }
  __syncthreads();
  if (tid < k) {  // two smallest per row, ties -> smaller j
    const double* z = Z + (long long)tid * d;
    int j1 = 0;
    for (int j = 1; j < d; ++j)
      if (z[j] < z[j1]) j1 = j;
    int j2 = (j1 == 0) ? 1 : 0;
    for (int j = 0; j < d; ++j)
      if (j != j1 && z[j] < z[j2]) j2 = j;
    dmask[(long long)tid * d + j1] = 1;
    dmask[(long long)tid * d + j2] = 1;
  }
  __syncthreads();
  const int R = k * l - 2 * k;
  if (R > 0) {
    // radix select of the R-th smallest key among the remaining cells
    if (tid == 0) {
      prefix_s = 0ull;
      need_s = R;
    }
    unsigned long long hmask = 0ull;
    for (int shift = 56; shift >= 0; shift -= 8) {
      for (int b = tid; b < 256; b += bd) hist[b] = 0u;
      __syncthreads();
      const unsigned long long pre = prefix_s;
      for (int c = tid; c < kd; c += bd) {
        if (dmask[c]) continue;
        unsigned long long key = sortable_key(Z[c]);
        if ((key & hmask) == pre) atomicAdd(&hist[(key >> shift) & 255ull], 1u);
      }
      __syncthreads();
      if (tid == 0) {
        int need = need_s, cum = 0, b = 0;
        for (b = 0; b < 256; ++b) {
          if (cum + (int)hist[b] >= need) break;
          cum += (int)hist[b];
        }
        need_s = need - cum;
        prefix_s = pre | ((unsigned long long)b << shift);
      }
      hmask |= 255ull << shift;
      __syncthreads();
    }
    const unsigned long long K = prefix_s;
    const int need = need_s;  // how many cells with key == K to take
    // cells with key < K are selected; of those equal to K the first `need`
    // in (i, j) order.  Contiguous index ranges per thread + a scan.
    const int per = (kd + bd - 1) / bd;
    const int c0 = tid * per, c1 = min(kd, c0 + per);
    int eq = 0;
    for (int c = c0; c < c1; ++c)
      if (!dmask[c] && sortable_key(Z[c]) == K) ++eq;
    tcount[tid] = eq;
    __syncthreads();
    if (tid == 0) {
      int s = 0;
      for (int t = 0; t < bd; ++t) {
        int v = tcount[t];
        tcount[t] = s;
        s += v;
      }
    }
    __syncthreads();
    int rank = tcount[tid];
    // each thread reads and writes only its own contiguous cell range here
    for (int c = c0; c < c1; ++c) {
      if (dmask[c]) continue;
      const unsigned long long key = sortable_key(Z[c]);
      if (key < K || (key == K && rank++ < need)) dmask[c] = 1;
    }
  }
  __syncthreads();
  if (tid < k) {
    int t = 0;
    for (int j = 0; j < d; ++j)
      if (dmask[(long long)tid * d + j]) dlist[(long long)tid * d + t++] = j;
    nD[tid] = t;
  }
  __syncthreads();
}

// ============================================================ iteration prologue
// Medoid rows of MCur (fp64), delta_i (Alg 3 l.4-7, reading R6), and the
// active slots of GPU-FAST-PROCLUS: new medoids get their Dist row computed,
// cached ones with a changed radius get the band of Theorem 3.1.
__device__ void prepare_iteration(const RunParams& p) {
  DevState* st = p.st;
  const int k = p.k, d = p.d;
  for (int e = threadIdx.x; e < k * d; e += blockDim.x) {
    const int i = e / d, j = e - i * d;
    p.med[e] = (double)p.mrows[(long long)st->mcur[i] * d + j];
  }
  __threadfence_block();
  __syncthreads();
  if (threadIdx.x < k) {
    const int i = threadIdx.x;
    double m = CUDART_INF;
    for (int j = 0; j < k; ++j) {
      if (j == i) continue;
      double t = full_dist(p.med + (long long)i * d, 1, p.med + (long long)j * d, d,
                           p.metric);
      if (t < m) m = t;
    }
    st->delta[i] = m;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    int na = 0;
    for (int i = 0; i < k; ++i) {
      const int mp = st->mcur[i];
      const double dl = st->delta[i];
      ActSlot a;
      a.slot = i;
      a.mpos = mp;
      a.compute = p.found[mp] ? 0 : 1;
      a.lam = 1;
      if (!p.used[mp]) {
        a.lo = -CUDART_INF;
        a.hi = dl;
      } else if (dl > p.dprev[mp]) {
        a.lo = p.dprev[mp];
        a.hi = dl;
      } else if (dl < p.dprev[mp]) {
        a.lo = dl;
        a.hi = p.dprev[mp];
        a.lam = -1;
      } else if (a.compute) {  // unreachable: used implies found
        a.lo = -CUDART_INF;
        a.hi = dl;
      } else {
        continue;  // delta unchanged: Delta L_i is empty (eq 3)
      }
      a.lo32 = __double2float_rn(a.lo);
      a.hi32 = __double2float_rn(a.hi);
      st->act[na++] = a;
    }
    st->n_act = na;
  }
  __syncthreads();
}

__global__ void k_prepare(RunParams p) { prepare_iteration(p); }

void launch_prepare(const RunParams& p, cudaStream_t s) {
  k_prepare<<<1, 256, 0, s>>>(p);
}

// ============================================================ smem carving
struct Carve {
  char* ptr;
  __device__ explicit Carve(void* base) : ptr((char*)base) {}
  template <class T>
  __device__ T* take(size_t count) {
    size_t a = alignof(T) < 8 ? 8 : alignof(T);
    ptr = (char*)(((size_t)ptr + a - 1) & ~(a - 1));
    T* r = (T*)ptr;
    ptr += sizeof(T) * count;
    return r;
  }
};

static size_t carve_size(std::initializer_list<size_t> parts) {
  size_t s = 0;
  for (size_t b : parts) s += (b + 15) & ~(size_t)15;
  return s + 64;
}

__device__ ListScratch carve_lists(Carve& cv, int list_len) {
  ListScratch ls;
  ls.ballot = cv.take<unsigned>(KMAX * WMAX);
  ls.woff = cv.take<int>(KMAX * WMAX);
  ls.cnt = cv.take<int>(KMAX);
  ls.base = cv.take<int>(KMAX);
  ls.list = cv.take<unsigned short>(list_len);
  return ls;
}

static size_t lists_bytes(int list_len) {
  return carve_size({sizeof(unsigned) * KMAX * WMAX, sizeof(int) * KMAX * WMAX,
                     sizeof(int) * KMAX, sizeof(int) * KMAX,
                     sizeof(unsigned short) * (size_t)list_len});
}

// ============================================================ tails
// Locality tail: H and |L| updates of Theorem 3.2 / eq 6 and P:203, the
// bookkeeping of DistFound / delta', X = H / |L|, FindDimensions.
__device__ void tail_locality(const RunParams& p) {
  DevState* st = p.st;
  const int d = p.d, na = st->n_act;
  for (int c = threadIdx.x; c < na * d; c += blockDim.x) {
    const int a = c / d, j = c - a * d;
    const ActSlot A = st->act[a];
    double* h = p.H + (long long)A.mpos * d + j;
    *h = dadd(*h, A.lam > 0 ? p.red[c] : -p.red[c]);
  }
  __syncthreads();
  if (threadIdx.x == 0 && na > 0)  // byte model: data once + one Dist row per slot
    st->bytes_loc += 4.0 * (double)p.n * (double)(d + na);
  if (threadIdx.x < na) {
    const ActSlot A = st->act[threadIdx.x];
    p.nL[A.mpos] += (A.lam > 0 ? p.redc[threadIdx.x] : -p.redc[threadIdx.x]);
    p.dprev[A.mpos] = st->delta[A.slot];
    p.used[A.mpos] = 1;
    p.found[A.mpos] = 1;
  }
  __threadfence_block();
  __syncthreads();
  for (int c = threadIdx.x; c < p.k * d; c += blockDim.x) {
    const int i = c / d, j = c - i * d;
    const int mp = st->mcur[i];
    p.X[c] = ddiv(p.H[(long long)mp * d + j], (double)p.nL[mp]);
  }
  __threadfence_block();
  __syncthreads();
  zscore_select(p.X, p.k, d, p.l, p.Z, p.dmask, p.dlist, st->nD);
  // trace
  const int it = st->iterations;
  if (p.tr.cap > 0 && it < p.tr.cap) {
    for (int c = threadIdx.x; c < p.k * d; c += blockDim.x) {
      if (p.tr.X) p.tr.X[(long long)it * p.k * d + c] = p.X[c];
      if (p.tr.dims) p.tr.dims[(long long)it * p.k * d + c] = p.dmask[c];
    }
    if (threadIdx.x < p.k) {
      const int i = threadIdx.x;
      if (p.tr.mcur) p.tr.mcur[it * p.k + i] = st->mcur[i];
      if (p.tr.delta) p.tr.delta[it * p.k + i] = st->delta[i];
      if (p.tr.nL) p.tr.nL[it * p.k + i] = p.nL[st->mcur[i]];
    }
  }
  __syncthreads();
}

// Assign tail: |C_i| and the centroid mu_ij = sum / |C_i| on j in D_i.
__device__ void tail_assign(const RunParams& p) {
  DevState* st = p.st;
  const int d = p.d;
  for (int c = threadIdx.x; c < p.k * d; c += blockDim.x) {
    const int i = c / d, t = c - i * d;
    const long long sz = p.redc[i];
    p.mu[c] = (t < st->nD[i] && sz > 0) ? ddiv(p.red[c], (double)sz) : 0.0;
  }
  if (threadIdx.x < p.k) st->sizes[threadIdx.x] = p.redc[threadIdx.x];
  __syncthreads();
}

// Cost tail: eq 1-2 with the |Data| denominator (eq 8, reading R4), then
// Alg 1 l.10-14: keep the best, ComputeBadMedoids (reading R11),
// replace bad medoids from M \ MBest (reading R12), stop after itrPat
// iterations without improvement, and prepare the next iteration.
__device__ void tail_cost(const RunParams& p) {
  DevState* st = p.st;
  const int k = p.k, d = p.d;
  __shared__ int done_s;
  if (threadIdx.x == 0) {
    double cost = 0.0;
    for (int i = 0; i < k; ++i) {
      const long long c = st->sizes[i];
      if (c == 0) continue;
      double w = 0.0;
      const int nd = st->nD[i];
      for (int t = 0; t < nd; ++t) w = dadd(w, ddiv(p.red[i * d + t], (double)c));
      w = ddiv(w, (double)nd);
      cost = dadd(cost, dmul((double)c, w));
    }
    cost = ddiv(cost, (double)p.n_total);
    st->cost = cost;
    st->itr += 1;
    const int it = st->iterations;
    st->iterations = it + 1;
    const int improved = cost < st->cost_best;
    st->improved = improved;
    if (improved) {
      st->itr = 0;
      st->cost_best = cost;
      for (int i = 0; i < k; ++i) {
        st->mbest[i] = st->mcur[i];
        st->sizes_best[i] = st->sizes[i];
      }
      st->best_buf = st->cur_buf;
      st->cur_buf ^= 1;
    }
    // ComputeBadMedoids from MBest
    unsigned bad = 0u;
    const double thr = dmul(ddiv((double)p.n_total, (double)k), p.minDev);
    int smallest = 0;
    for (int i = 0; i < k; ++i) {
      if ((double)st->sizes_best[i] < thr) bad |= 1u << i;
      if (st->sizes_best[i] < st->sizes_best[smallest]) smallest = i;
    }
    if (!bad) bad = 1u << smallest;
    if (p.tr.cap > 0 && it < p.tr.cap) {
      if (p.tr.cost) p.tr.cost[it] = cost;
      if (p.tr.improved) p.tr.improved[it] = (unsigned char)improved;
      for (int i = 0; i < k; ++i) {
        if (p.tr.sizes) p.tr.sizes[it * k + i] = st->sizes[i];
        if (p.tr.bad) p.tr.bad[it * k + i] = (bad >> i) & 1u;
      }
    }
    // replacement: MCur = MBest with bad slots drawn from M \ MBest
    int np = 0;
    for (int t = 0; t < p.nM; ++t) {
      bool inb = false;
      for (int i = 0; i < k; ++i) inb |= (st->mbest[i] == t);
      if (!inb) p.pool[np++] = t;
    }
    for (int i = 0; i < k; ++i) st->mcur[i] = st->mbest[i];
    unsigned long long rng = st->rng;
    for (int i = 0; i < k; ++i) {
      if (!((bad >> i) & 1u) || np == 0) continue;
      int r = (int)sm64_uniform(&rng, (unsigned long long)np);
      st->mcur[i] = p.pool[r];
      for (int t = r; t + 1 < np; ++t) p.pool[t] = p.pool[t + 1];
      --np;
    }
    st->rng = rng;
    st->done = (st->itr >= p.itrPat || st->iterations >= p.max_iter) ? 1 : 0;
    done_s = st->done;
  }
  __threadfence_block();
  __syncthreads();
  if (!done_s) prepare_iteration(p);
}

// Refinement tail (Alg 1 l.16-17): X over CBest (empty cluster -> 0 row,
// reading R15), FindDimensions -> D*, and the outlier radii
// Delta_i = min_{j != i} seg_{D*_i}(m_i, m_j) (reading R5).
__device__ void tail_refine(const RunParams& p) {
  DevState* st = p.st;
  const int k = p.k, d = p.d;
  for (int c = threadIdx.x; c < k * d; c += blockDim.x) {
    const int i = c / d;
    const long long sz = p.redc[i];
    p.X[c] = sz > 0 ? ddiv(p.red[c], (double)sz) : 0.0;
  }
  __threadfence_block();
  __syncthreads();
  zscore_select(p.X, k, d, p.l, p.Z, p.dmask, p.dlist, st->nD);
  if (threadIdx.x < k) {
    const int i = threadIdx.x, nd = st->nD[i];
    const int* dl = p.dlist + (long long)i * d;
    double m = CUDART_INF;
    for (int j = 0; j < k; ++j) {
      if (j == i) continue;
      double s = 0.0;
      for (int t = 0; t < nd; ++t)
        s = dadd(s, fabs(dsub(p.med[(long long)i * d + dl[t]], p.med[(long long)j * d + dl[t]])));
      double q = ddiv(s, (double)nd);
      if (q < m) m = q;
    }
    p.Delta[i] = m;
  }
  __syncthreads();
}

// ============================================================ pass kernels
// Per-point segmental distances to every medoid over D_i (Alg 5 l.4) and the
// argmin with ties to the smallest i (reading R8), in the oracle's exact
// fp64 expression.  The fast path compares s_i * (1/|D_i|); only when the
// runner-up is within 1e-14 relative are the correctly rounded quotients
// s_i / |D_i| formed and compared.
__device__ __forceinline__ int assign_point(const double* __restrict__ x, int xs_stride,
                                            const double* __restrict__ med,
                                            const int* __restrict__ dl,
                                            const int* __restrict__ nD,
                                            const double* __restrict__ rcp, int k,
                                            int d) {
  double best = CUDART_INF, second = CUDART_INF;
  int bi = 0;
  for (int i = 0; i < k; ++i) {
    const int nd = nD[i];
    const int* L = dl + i * d;
    const double* m = med + i * d;
    double s = 0.0;
    for (int t = 0; t < nd; ++t) {
      const int j = L[t];
      s = dadd(s, fabs(dsub(x[j * xs_stride], m[j])));
    }
    const double q = dmul(s, rcp[i]);
    if (q < best) {
      second = best;
      best = q;
      bi = i;
    } else if (q < second) {
      second = q;
    }
  }
  if (second > dmul(best, 1.0 + 1e-14)) return bi;
  // near tie: exact quotients
  best = CUDART_INF;
  bi = 0;
  for (int i = 0; i < k; ++i) {
    const int nd = nD[i];
    const int* L = dl + i * d;
    const double* m = med + i * d;
    double s = 0.0;
    for (int t = 0; t < nd; ++t) {
      const int j = L[t];
      s = dadd(s, fabs(dsub(x[j * xs_stride], m[j])));
    }
    const double q = ddiv(s, (double)nd);
    if (q < best) {
      best = q;
      bi = i;
    }
  }
  return bi;
}

// --- ComputeL + FindDimensions X (Alg 3, Alg 4 l.1-5) with the FAST caches.
__global__ void __launch_bounds__(256) k_locality(RunParams p) {
  DevState* st = p.st;
  if (st->done) return;
  extern __shared__ __align__(16) unsigned char smraw[];
  const int P = p.P, d = p.d, k = p.k;
  const int na = st->n_act;
  Carve cv(smraw);
  double* x_s = cv.take<double>((size_t)d * (P + 1));
  double* med_s = cv.take<double>((size_t)k * d);
  double* acc_s = cv.take<double>((size_t)k * d);
  long long* cacc_s = cv.take<long long>(KMAX);
  ActSlot* act_s = cv.take<ActSlot>(KMAX);
  ListScratch ls = carve_lists(cv, KMAX * P);
  const int tid = threadIdx.x;

  for (int a = tid; a < na; a += blockDim.x) act_s[a] = st->act[a];
  __syncthreads();
  for (int e = tid; e < na * d; e += blockDim.x) {
    const int a = e / d, j = e - a * d;
    med_s[e] = p.med[(long long)act_s[a].slot * d + j];
    acc_s[e] = 0.0;
  }
  for (int a = tid; a < KMAX; a += blockDim.x) cacc_s[a] = 0;
  __syncthreads();

  if (na > 0) {
    for (long long ch = blockIdx.x; ch < p.nchunks; ch += gridDim.x) {
      const long long base = ch * P;
      stage_chunk(p.xs, p.n_pad, d, base, P, x_s);
      __syncthreads();
      const long long gp = base + tid;
      unsigned mask = 0u;
      if (gp < p.n) {
        const double* xp = x_s + tid;
        for (int a = 0; a < na; ++a) {
          const ActSlot A = act_s[a];
          float* drow = p.dist + (long long)A.mpos * p.n_pad + gp;
          bool in;
          if (A.compute) {  // compute distances only once
            const double dv = full_dist(xp, P + 1, med_s + a * d, d, p.metric);
            *drow = __double2float_rn(dv);
            in = (dv > A.lo) && (dv <= A.hi);
          } else {  // cached fp32 row: certified decision, exact fallback
            const float f = __ldg(drow);
            const int rhi = (f < A.hi32) ? 1 : ((f > A.hi32) ? 0 : -1);
            const int rlo = (A.lo == -CUDART_INF) ? 1
                            : (f > A.lo32)        ? 1
                            : (f < A.lo32)        ? 0
                                                  : -1;
            if (rhi == 0 || rlo == 0) {
              in = false;
            } else if (rhi == 1 && rlo == 1) {
              in = true;
            } else {
              const double dv = full_dist(xp, P + 1, med_s + a * d, d, p.metric);
              in = (dv > A.lo) && (dv <= A.hi);
            }
          }
          if (in) mask |= 1u << a;
        }
      }
      build_lists(mask, na, ls);
      // cells (a, j): sum over the band of |x_j - m_aj| (eq 6)
      for (int c = tid; c < na * d; c += blockDim.x) {
        const int a = c / d, j = c - a * d;
        const int cnt = ls.cnt[a];
        if (cnt == 0) continue;
        acc_s[c] = dadd(acc_s[c], list_sum<1>(x_s + j * (P + 1), ls.list + ls.base[a],
                                              cnt, med_s[c]));
      }
      if (tid < na) cacc_s[tid] += ls.cnt[tid];
      __syncthreads();
    }
  }
  // per-block partials
  const int stride = k * d;
  for (int c = tid; c < na * d; c += blockDim.x)
    p.part[(long long)blockIdx.x * stride + c] = acc_s[c];
  for (int a = tid; a < KMAX; a += blockDim.x)
    p.partc[(long long)blockIdx.x * KMAX + a] = cacc_s[a];
  if (!p.fuse_tail) return;
  if (!last_block(&st->ticket[0])) return;
  reduce_partials(p.part, p.partc, gridDim.x, stride, na * d, na, p.red, p.redc);
  tail_locality(p);
}

// --- AssignPoints (Alg 5) + centroid sums of EvaluateCluster (Alg 6 l.1-8).
__global__ void __launch_bounds__(256) k_assign(RunParams p) {
  DevState* st = p.st;
  if (st->done) return;
  extern __shared__ __align__(16) unsigned char smraw[];
  const int P = p.P, d = p.d, k = p.k;
  Carve cv(smraw);
  double* x_s = cv.take<double>((size_t)d * (P + 1));
  double* med_s = cv.take<double>((size_t)k * d);
  double* acc_s = cv.take<double>((size_t)k * d);
  long long* cacc_s = cv.take<long long>(KMAX);
  int* dl_s = cv.take<int>((size_t)k * d);
  int* nD_s = cv.take<int>(KMAX);
  double* rcp_s = cv.take<double>(KMAX);
  ListScratch ls = carve_lists(cv, P);
  const int tid = threadIdx.x;
  unsigned char* lab = st->cur_buf ? p.lab1 : p.lab0;

  for (int e = tid; e < k * d; e += blockDim.x) {
    med_s[e] = p.med[e];
    dl_s[e] = p.dlist[e];
    acc_s[e] = 0.0;
  }
  for (int i = tid; i < KMAX; i += blockDim.x) {
    cacc_s[i] = 0;
    if (i < k) {
      nD_s[i] = st->nD[i];
      rcp_s[i] = ddiv(1.0, (double)st->nD[i]);
    }
  }
  __syncthreads();
  for (long long ch = blockIdx.x; ch < p.nchunks; ch += gridDim.x) {
    const long long base = ch * P;
    stage_chunk(p.xs, p.n_pad, d, base, P, x_s);
    __syncthreads();
    const long long gp = base + tid;
    unsigned mask = 0u;
    if (gp < p.n) {
      const int bi = assign_point(x_s + tid, P + 1, med_s, dl_s, nD_s, rcp_s, k, d);
      lab[gp] = (unsigned char)bi;
      mask = 1u << bi;
    }
    build_lists(mask, k, ls);
    for (int c = tid; c < k * d; c += blockDim.x) {
      const int i = c / d, t = c - i * d;
      const int cnt = ls.cnt[i];
      if (t >= nD_s[i] || cnt == 0) continue;
      const int j = dl_s[c];
      acc_s[c] = dadd(acc_s[c], list_sum<0>(x_s + j * (P + 1), ls.list + ls.base[i], cnt, 0.0));
    }
    if (tid < k) cacc_s[tid] += ls.cnt[tid];
    __syncthreads();
  }
  const int stride = k * d;
  for (int c = tid; c < stride; c += blockDim.x)
    p.part[(long long)blockIdx.x * stride + c] = acc_s[c];
  for (int a = tid; a < KMAX; a += blockDim.x)
    p.partc[(long long)blockIdx.x * KMAX + a] = cacc_s[a];
  if (!p.fuse_tail) return;
  if (!last_block(&st->ticket[1])) return;
  reduce_partials(p.part, p.partc, gridDim.x, stride, stride, k, p.red, p.redc);
  tail_assign(p);
}

// --- EvaluateCluster deviations (Alg 6 l.9-13, eq 9) + control tail.
__global__ void __launch_bounds__(256) k_cost(RunParams p) {
  DevState* st = p.st;
  if (st->done) return;
  extern __shared__ __align__(16) unsigned char smraw[];
  const int P = p.P, d = p.d, k = p.k;
  Carve cv(smraw);
  double* x_s = cv.take<double>((size_t)d * (P + 1));
  double* mu_s = cv.take<double>((size_t)k * d);
  double* acc_s = cv.take<double>((size_t)k * d);
  int* dl_s = cv.take<int>((size_t)k * d);
  int* nD_s = cv.take<int>(KMAX);
  ListScratch ls = carve_lists(cv, P);
  const int tid = threadIdx.x;
  const unsigned char* lab = st->cur_buf ? p.lab1 : p.lab0;

  for (int e = tid; e < k * d; e += blockDim.x) {
    mu_s[e] = p.mu[e];
    dl_s[e] = p.dlist[e];
    acc_s[e] = 0.0;
  }
  for (int i = tid; i < k; i += blockDim.x) nD_s[i] = st->nD[i];
  __syncthreads();
  for (long long ch = blockIdx.x; ch < p.nchunks; ch += gridDim.x) {
    const long long base = ch * P;
    stage_chunk(p.xs, p.n_pad, d, base, P, x_s);
    const long long gp = base + tid;
    const unsigned mask = (gp < p.n) ? (1u << lab[gp]) : 0u;
    __syncthreads();
    build_lists(mask, k, ls);
    for (int c = tid; c < k * d; c += blockDim.x) {
      const int i = c / d, t = c - i * d;
      const int cnt = ls.cnt[i];
      if (t >= nD_s[i] || cnt == 0) continue;
      const int j = dl_s[c];
      acc_s[c] = dadd(acc_s[c], list_sum<1>(x_s + j * (P + 1), ls.list + ls.base[i], cnt,
                                            mu_s[c]));
    }
    __syncthreads();
  }
  const int stride = k * d;
  for (int c = tid; c < stride; c += blockDim.x)
    p.part[(long long)blockIdx.x * stride + c] = acc_s[c];
  if (!p.fuse_tail) return;
  if (!last_block(&st->ticket[2])) return;
  reduce_partials(p.part, p.partc, gridDim.x, stride, stride, 0, p.red, p.redc);
  tail_cost(p);
}

// --- Refinement X over CBest (Alg 1 l.16-17): sums of |x_j - mbest_ij| for
// every dimension over each best cluster.  p.med holds the MBest rows.
__global__ void __launch_bounds__(256) k_refine_x(RunParams p) {
  DevState* st = p.st;
  extern __shared__ __align__(16) unsigned char smraw[];
  const int P = p.P, d = p.d, k = p.k;
  Carve cv(smraw);
  double* x_s = cv.take<double>((size_t)d * (P + 1));
  double* med_s = cv.take<double>((size_t)k * d);
  double* acc_s = cv.take<double>((size_t)k * d);
  long long* cacc_s = cv.take<long long>(KMAX);
  ListScratch ls = carve_lists(cv, P);
  const int tid = threadIdx.x;
  const unsigned char* lab = st->best_buf ? p.lab1 : p.lab0;
  for (int e = tid; e < k * d; e += blockDim.x) {
    const int i = e / d, j = e - i * d;
    med_s[e] = (double)p.mrows[(long long)st->mbest[i] * d + j];
    acc_s[e] = 0.0;
  }
  for (int a = tid; a < KMAX; a += blockDim.x) cacc_s[a] = 0;
  __syncthreads();
  for (long long ch = blockIdx.x; ch < p.nchunks; ch += gridDim.x) {
    const long long base = ch * P;
    stage_chunk(p.xs, p.n_pad, d, base, P, x_s);
    const long long gp = base + tid;
    const unsigned mask = (gp < p.n) ? (1u << lab[gp]) : 0u;
    __syncthreads();
    build_lists(mask, k, ls);
    for (int c = tid; c < k * d; c += blockDim.x) {
      const int i = c / d, j = c - i * d;
      const int cnt = ls.cnt[i];
      if (cnt == 0) continue;
      acc_s[c] = dadd(acc_s[c], list_sum<1>(x_s + j * (P + 1), ls.list + ls.base[i], cnt,
                                            med_s[c]));
    }
    if (tid < k) cacc_s[tid] += ls.cnt[tid];
    __syncthreads();
  }
  const int stride = k * d;
  for (int c = tid; c < stride; c += blockDim.x)
    p.part[(long long)blockIdx.x * stride + c] = acc_s[c];
  for (int a = tid; a < KMAX; a += blockDim.x)
    p.partc[(long long)blockIdx.x * KMAX + a] = cacc_s[a];
  if (!p.fuse_tail) return;
  if (!last_block(&st->ticket[3])) return;
  // MBest rows (fp64) for Delta
  for (int e = threadIdx.x; e < k * d; e += blockDim.x) p.med[e] = med_s[e];
  reduce_partials(p.part, p.partc, gridDim.x, stride, stride, k, p.red, p.redc);
  tail_refine(p);
}

// --- Final AssignPoints with D* (Alg 1 l.18) and RemoveOutliers (l.19):
// outlier iff seg_{D*_i}(x, m_i) > Delta_i for every i (reading R17).
__global__ void __launch_bounds__(256) k_final(RunParams p) {
  DevState* st = p.st;
  extern __shared__ __align__(16) unsigned char smraw[];
  const int P = p.P, d = p.d, k = p.k;
  Carve cv(smraw);
  double* x_s = cv.take<double>((size_t)d * (P + 1));
  double* med_s = cv.take<double>((size_t)k * d);
  int* dl_s = cv.take<int>((size_t)k * d);
  int* nD_s = cv.take<int>(KMAX);
  double* rcp_s = cv.take<double>(KMAX);
  double* Dl_s = cv.take<double>(KMAX);
  const int tid = threadIdx.x;
  for (int e = tid; e < k * d; e += blockDim.x) {
    med_s[e] = p.med[e];
    dl_s[e] = p.dlist[e];
  }
  for (int i = tid; i < k; i += blockDim.x) {
    nD_s[i] = st->nD[i];
    rcp_s[i] = ddiv(1.0, (double)st->nD[i]);
    Dl_s[i] = p.Delta[i];
  }
  __syncthreads();
  for (long long ch = blockIdx.x; ch < p.nchunks; ch += gridDim.x) {
    const long long base = ch * P;
    stage_chunk(p.xs, p.n_pad, d, base, P, x_s);
    __syncthreads();
    const long long gp = base + tid;
    if (gp < p.n) {
      const double* xp = x_s + tid;
      const int bi = assign_point(xp, P + 1, med_s, dl_s, nD_s, rcp_s, k, d);
      bool outside_all = true;
      for (int i = 0; i < k && outside_all; ++i) {
        const int nd = nD_s[i];
        double s = 0.0;
        for (int t = 0; t < nd; ++t) {
          const int j = dl_s[i * d + t];
          s = dadd(s, fabs(dsub(xp[j * (P + 1)], med_s[i * d + j])));
        }
        const double q = dmul(s, rcp_s[i]);
        const double D = Dl_s[i];
        bool gt;
        if (q > dmul(D, 1.0 + 1e-14))
          gt = true;
        else if (q < dmul(D, 1.0 - 1e-14))
          gt = false;
        else
          gt = ddiv(s, (double)nd) > D;
        outside_all = gt;
      }
      p.out_labels[gp] = outside_all ? -1 : bi;
    }
    __syncthreads();
  }
}

// ============================================================ multi-GPU tails
__global__ void k_reduce(RunParams p, int tail, int G) {
  DevState* st = p.st;
  if (tail != TAIL_REF && st->done) return;
  const int kd = p.k * p.d;
  int ncell = kd, ncnt = p.k;
  if (tail == TAIL_LOC) {
    ncell = st->n_act * p.d;
    ncnt = st->n_act;
  } else if (tail == TAIL_COST) {
    ncnt = 0;
  }
  // unused entries are zeroed so a full-length allreduce is exact
  for (int c = threadIdx.x; c < kd; c += blockDim.x) p.red[c] = 0.0;
  for (int c = threadIdx.x; c < KMAX; c += blockDim.x) p.redc[c] = 0;
  __syncthreads();
  reduce_partials(p.part, p.partc, G, kd, ncell, ncnt, p.red, p.redc);
}

__global__ void k_tail(RunParams p, int tail) {
  DevState* st = p.st;
  if (tail == TAIL_LOC) {
    if (st->done) return;
    tail_locality(p);
  } else if (tail == TAIL_ASG) {
    if (st->done) return;
    tail_assign(p);
  } else if (tail == TAIL_COST) {
    if (st->done) return;
    tail_cost(p);
  } else {
    for (int e = threadIdx.x; e < p.k * p.d; e += blockDim.x) {
      const int i = e / p.d, j = e - i * p.d;
      p.med[e] = (double)p.mrows[(long long)st->mbest[i] * p.d + j];
    }
    __syncthreads();
    tail_refine(p);
  }
}

void launch_reduce(const RunParams& p, const PassShape& ps, int tail,
                   cudaStream_t s) {
  k_reduce<<<1, 256, 0, s>>>(p, tail, ps.grid);
}

void launch_tail(const RunParams& p, int tail, cudaStream_t s) {
  k_tail<<<1, 256, 0, s>>>(p, tail);
}

// ============================================================ shapes
static size_t smem_loc(int P, int d, int k) {
  return carve_size({sizeof(double) * (size_t)d * (P + 1), sizeof(double) * (size_t)k * d,
                     sizeof(double) * (size_t)k * d, sizeof(long long) * KMAX,
                     sizeof(ActSlot) * KMAX}) +
         lists_bytes(KMAX * P);
}
static size_t smem_asg(int P, int d, int k) {
  return carve_size({sizeof(double) * (size_t)d * (P + 1), sizeof(double) * (size_t)k * d,
                     sizeof(double) * (size_t)k * d, sizeof(long long) * KMAX,
                     sizeof(int) * (size_t)k * d, sizeof(int) * KMAX,
                     sizeof(double) * KMAX}) +
         lists_bytes(P);
}
static size_t smem_cost(int P, int d, int k) {
  return carve_size({sizeof(double) * (size_t)d * (P + 1), sizeof(double) * (size_t)k * d,
                     sizeof(double) * (size_t)k * d, sizeof(int) * (size_t)k * d,
                     sizeof(int) * KMAX}) +
         lists_bytes(P);
}
static size_t smem_ref(int P, int d, int k) {
  return carve_size({sizeof(double) * (size_t)d * (P + 1), sizeof(double) * (size_t)k * d,
                     sizeof(double) * (size_t)k * d, sizeof(long long) * KMAX}) +
         lists_bytes(P);
}
static size_t smem_fin(int P, int d, int k) {
  return carve_size({sizeof(double) * (size_t)d * (P + 1), sizeof(double) * (size_t)k * d,
                     sizeof(int) * (size_t)k * d, sizeof(int) * KMAX,
                     sizeof(double) * KMAX, sizeof(double) * KMAX});
}

PassShape pass_shape(int d, int k, int num_sms) {
  PassShape ps;
  int P = PMAX;
  const size_t budget = 100 * 1024;
  while (P > 32 && (smem_loc(P, d, k) > budget || smem_asg(P, d, k) > budget)) P >>= 1;
  ps.P = P;
  ps.smem_loc = smem_loc(P, d, k);
  ps.smem_asg = smem_asg(P, d, k);
  ps.smem_cost = smem_cost(P, d, k);
  ps.smem_ref = smem_ref(P, d, k);
  ps.smem_fin = smem_fin(P, d, k);
  size_t mx = ps.smem_loc;
  if (ps.smem_asg > mx) mx = ps.smem_asg;
  // resident blocks per SM limited by shared memory (228 KB per SM) and by
  // 2048 threads per SM
  int by_smem = (int)((228 * 1024) / (mx + 1024));
  int by_thr = 2048 / P;
  int per_sm = by_smem < by_thr ? by_smem : by_thr;
  if (per_sm < 1) per_sm = 1;
  if (per_sm > 8) per_sm = 8;
  ps.grid = num_sms * per_sm;
  return ps;
}

cudaError_t configure_kernels(const PassShape& ps) {
  cudaError_t e;
  const void* fns[] = {(const void*)k_locality, (const void*)k_assign, (const void*)k_cost,
                       (const void*)k_refine_x, (const void*)k_final};
  size_t sm[] = {ps.smem_loc, ps.smem_asg, ps.smem_cost, ps.smem_ref, ps.smem_fin};
  for (int i = 0; i < 5; ++i) {
    e = cudaFuncSetAttribute(fns[i], cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm[i]);
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

void launch_locality(const RunParams& p, const PassShape& ps, cudaStream_t s) {
  k_locality<<<ps.grid, ps.P, ps.smem_loc, s>>>(p);
}
void launch_assign(const RunParams& p, const PassShape& ps, cudaStream_t s) {
  k_assign<<<ps.grid, ps.P, ps.smem_asg, s>>>(p);
}
void launch_cost(const RunParams& p, const PassShape& ps, cudaStream_t s) {
  k_cost<<<ps.grid, ps.P, ps.smem_cost, s>>>(p);
}
void launch_refine_x(const RunParams& p, const PassShape& ps, cudaStream_t s) {
  k_refine_x<<<ps.grid, ps.P, ps.smem_ref, s>>>(p);
}
void launch_final(const RunParams& p, const PassShape& ps, cudaStream_t s) {
  k_final<<<ps.grid, ps.P, ps.smem_fin, s>>>(p);
}

}  // namespace pc

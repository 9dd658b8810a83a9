// proclus_kernels.cu -- sm_100a kernels of the PROCLUS hot path
// (GPU-FAST-PROCLUS, section 4, re-designed for B200).
//
// Every per-iteration pass is a persistent kernel that streams the data in
// chunks of P points (SoA fp32, one 1-D bulk copy per dimension row) through
// a 2-3 stage shared-memory ring filled by cp.async.bulk (TMA) and tracked by
// mbarriers, so HBM traffic overlaps the compute of the previous chunks.
// Chunks are small (P = 128 points for d <= 64) so that 4-8 blocks share an
// SM and one block's barriers are hidden by the others.  Block b owns chunks
// b, b+G, ...; inside a chunk
//  (A) one thread per point takes the per-point decision (ComputeL band
//      membership, AssignPoints argmin) in fp32 with a certified error bound
//      and falls back to the oracle's exact fp64 expression only when the
//      fp32 value is within that bound of the threshold / runner-up;
//  (B) the per-point decisions are compacted into per-set member lists;
//  (C) "cells" (S threads per (set, dimension)) sum over their list in fp64
//      and quantise the chunk's sum to int64 fixed point (scale 2^e_j per
//      dimension), accumulated exactly in shared memory and finally with one
//      int64 atomicAdd per cell per block into one of NCOPY global copies.
//      Integer addition is associative, so the totals do not depend on block
//      scheduling, grid size or the number of GPUs: runs are bit-reproducible.
// The last block to finish (ticket) runs the small single-block step that
// follows (finalise H and select dimensions / centroids / cost and the
// Alg 1 l.10-14 control), so an iteration is three launches; inside a CUDA
// graph while-node the cost tail also sets the loop condition.
#include <math_constants.h>

#include <algorithm>
#include <map>
#include <mutex>
#include <cstdio>
#include <cstdlib>

#include "proclus_kernels.h"

namespace pc {

// ===================================================================== PTX
__device__ __forceinline__ unsigned smem_u32(const void* p) {
  return static_cast<unsigned>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(unsigned long long* bar, unsigned count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count)
               : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(unsigned long long* bar, unsigned bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
               "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_wait(unsigned long long* bar, unsigned phase) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1, 0x989680;\n"
      "@!p bra WAIT_%=;\n"
      "}\n" ::"r"(smem_u32(bar)),
      "r"(phase)
      : "memory");
}
#ifndef MBAR_HINT_NS
#define MBAR_HINT_NS 10000000  // suspend-time hint (ns) of the ring waits; 0: none
#endif
#define PC_STR_(x) #x
#define PC_STR(x) PC_STR_(x)
#if MBAR_HINT_NS > 0
#define MBAR_HINT ", " PC_STR(MBAR_HINT_NS)
#else
#define MBAR_HINT ""
#endif
// the same with the barrier's 32-bit shared address computed once per kernel
// (a generic-to-shared conversion per spin iteration costs an S2UR chain)
__device__ __forceinline__ void mbar_wait(unsigned bar, unsigned phase) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "WAITA_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1" MBAR_HINT ";\n"
      "@!p bra WAITA_%=;\n"
      "}\n" ::"r"(bar),
      "r"(phase)
      : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(unsigned bar, unsigned bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, unsigned bytes,
                                         unsigned bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(bar)
      : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, unsigned bytes,
                                         unsigned long long* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}
// L2 eviction priorities for the streamed rows: evict-last for the data
// (re-read by every pass of an iteration; 60 MB at C3 fits the 126 MB L2),
// evict-first for the cached Dist rows (read once per locality pass).
__device__ __forceinline__ unsigned long long l2_policy(int last) {
  unsigned long long pol;
  if (last)
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
  else
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  return pol;
}
__device__ __forceinline__ void bulk_g2s_h(void* dst, const void* src, unsigned bytes, unsigned bar,
                                           unsigned long long pol) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], "
      "%2, [%3], %4;" ::"r"(smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(bar), "l"(pol)
      : "memory");
}
__device__ __forceinline__ void fence_proxy_async() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}

// ===================================================================== N0
// row-major [n][d] -> SoA [d][n_pad] (zero padding), non-finite flag and the
// per-dimension max |x| (as float bits; non-negative floats order as uints).
// A block packs pp consecutive points (<= 512, a multiple of 32, <= 48 KB of
// shared memory): their pp x d floats are one
// contiguous range of the input, read with coalesced 16-byte loads into
// shared memory (point q's row at stride ds = d | 1: odd, so the column reads
// below are conflict-free), then written as d coalesced rows of PK_P floats;
// max |x_j| is reduced per warp (a warp's 32 consecutive outputs share j),
// then per block, one atomicMax per column and block.
constexpr int PK_T = 256;
__global__ void __launch_bounds__(PK_T) k_pack_soa(const float* __restrict__ in, long long n, int d,
                                                   long long n_pad, float* __restrict__ xs, int* bad,
                                                   unsigned* colmax, int PK_P) {
  extern __shared__ __align__(16) float pk[];  // [pp][ds]
  const int ds = d | 1;
  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  const long long p0 = (long long)blockIdx.x * PK_P;
  const int np = (int)(p0 < n ? (n - p0 < PK_P ? n - p0 : PK_P) : 0);
  const int nf = np * d;
  const float* src = in + p0 * d;
  const bool vec = ((reinterpret_cast<unsigned long long>(src) & 15ull) == 0);
  int e0 = 0;
  if (vec) {
    const float4* s4 = reinterpret_cast<const float4*>(src);
    const int n4 = nf >> 2;
    if (ds == d) {  // odd d: the shared rows are the input's flat layout: one bulk copy
      __shared__ __align__(8) unsigned long long pbar;
      const unsigned bytes = (unsigned)nf * 4u & ~15u;
      if (tid == 0) {
        mbar_init(&pbar, 1);
        fence_mbar_init();
        if (bytes) {
          mbar_expect_tx(&pbar, bytes);
          bulk_g2s(pk, src, bytes, &pbar);
        }
      }
      for (int f = (int)(bytes >> 2) + tid; f < nf; f += PK_T) pk[f] = src[f];
      __syncthreads();  // the barrier's init is visible
      if (bytes) mbar_wait(&pbar, 0u);
      e0 = nf;
    } else {  // (q, j) of element 4 e, advanced without division
      const int step = 4 * PK_T, dq = step / d, dj = step - dq * d;
      int q = (4 * tid) / d, j = 4 * tid - q * d;
      for (int e = tid; e < n4; e += PK_T) {
        const float4 v = __ldcs(s4 + e);
        const float vv[4] = {v.x, v.y, v.z, v.w};
        int qq = q, jj = j;
#pragma unroll
        for (int c = 0; c < 4; ++c) {
          pk[qq * ds + jj] = vv[c];
          if (++jj == d) {
            jj = 0;
            ++qq;
          }
        }
        q += dq;
        j += dj;
        if (j >= d) {
          j -= d;
          ++q;
        }
      }
    }
    if (ds != d) e0 = n4 << 2;
  }
  for (int f = e0 + tid; f < nf; f += PK_T) {
    const int q = f / d, j = f - q * d;
    pk[q * ds + j] = __ldcs(src + f);
  }
  __syncthreads();
  // one warp per output row j: consecutive lanes take consecutive points
  // (coalesced stores; column reads at the odd stride ds are conflict-free)
  int nonfinite = 0;
  const int nstore = (int)(n_pad - p0 < PK_P ? n_pad - p0 : PK_P);  // multiple of 32
  for (int j = w; j < d; j += PK_T / 32) {
    float amax = 0.f;
    float* dst = xs + (size_t)j * n_pad + p0;
    for (int q0 = 0; q0 < nstore; q0 += 128) {
      float v[4];
#pragma unroll
      for (int c = 0; c < 4; ++c) {
        const int q = q0 + 32 * c + lane;
        v[c] = q < np ? pk[q * ds + j] : 0.f;
        const float a = fabsf(v[c]);
        nonfinite |= !(a <= 3.402823466e38f);
        amax = fmaxf(amax, a);  // a NaN operand is ignored
      }
#pragma unroll
      for (int c = 0; c < 4; ++c)
        if (q0 + 32 * c < nstore) dst[q0 + 32 * c + lane] = v[c];
    }
    const unsigned m = __reduce_max_sync(0xffffffffu, __float_as_uint(amax));
    // one of PACK_COPIES partial maxima per column (same-address atomics
    // from every block serialised in L2), folded by k_fold_colmax
    if (lane == 0 && m) atomicMax(colmax + (size_t)(blockIdx.x % PACK_COPIES) * d + j, m);
  }
  if (nonfinite) atomicOr(bad, 1);
}

__global__ void k_fold_colmax(unsigned* colmax, int d) {
  for (int j = threadIdx.x; j < d; j += blockDim.x) {
    unsigned m = colmax[j];
    for (int c = 1; c < PACK_COPIES; ++c) m = max(m, colmax[(size_t)c * d + j]);
    colmax[j] = m;
  }
}

void launch_pack_soa(const float* in, long long n, int d, long long n_pad, float* xs, int* bad,
                     unsigned* colmax, cudaStream_t s) {
  const int ds = d | 1;
  int pp = (int)((48 * 1024 / 4) / ds) / 32 * 32;
  if (pp > 512) pp = 512;
  if (pp < 32) pp = 32;  // d <= 256 (binding cap): 32 x 257 floats fit
  const size_t smem = sizeof(float) * (size_t)pp * ds;
  const unsigned grid = (unsigned)((n_pad + pp - 1) / pp);
  k_pack_soa<<<grid, PK_T, smem, s>>>(in, n, d, n_pad, xs, bad, colmax, pp);
  k_fold_colmax<<<1, 256, 0, s>>>(colmax, d);
}

// Per-dimension fixed-point scales 2^e_j from max |x_j| (colmax, float bits):
// e_j = 61 - ceil(log2(2 n_total max|x_j|)), at most 50 - ceil(log2(2
// max|x_j|)), clamped to [-1000, 1000]; ceil(log2 x) is taken exactly from the
// binary exponent (frexp), so the host path (scales_of in proclus_api.cu)
// computes the same values.  qflag = 0 if some band sum of <= 256 terms can
// reach 2^51 at its scale (quant_sum then converts instead of the fma).
__device__ __forceinline__ int ceil_log2_dev(double x) {
  int ex;
  const double f = frexp(x, &ex);
  return f == 0.5 ? ex - 1 : ex;
}
__global__ void k_scales(const unsigned* __restrict__ colmax, int d, long long n_total,
                         double* __restrict__ scale, double* __restrict__ iscale, int* qflag) {
  __shared__ int ok;
  if (threadIdx.x == 0) ok = 1;
  __syncthreads();
  for (int j = threadIdx.x; j < d; j += blockDim.x) {
    const float m = __uint_as_float(colmax[j]);
    int e = 0;
    if (m > 0.f) {
      e = 61 - ceil_log2_dev(2.0 * (double)n_total * (double)m);
      e = min(e, 50 - ceil_log2_dev(2.0 * (double)m));
      e = max(-1000, min(1000, e));
      if (ldexp(512.0 * (double)m, e) >= 2251799813685248.0) atomicAnd(&ok, 0);  // 2^51
    }
    scale[j] = ldexp(1.0, e);
    iscale[j] = ldexp(1.0, -e);
  }
  __syncthreads();
  if (threadIdx.x == 0) *qflag = ok;
}
void launch_scales(const unsigned* colmax, int d, long long n_total, double* scale,
                   double* iscale, int* qflag, cudaStream_t s) {
  k_scales<<<1, 256, 0, s>>>(colmax, d, n_total, scale, iscale, qflag);
}

// Small host -> device uploads as kernel parameters (no copy-engine work, so
// they never queue behind a proclus_prefetch transfer of the next dataset).
struct Blob {
  unsigned char b[BLOB_BYTES];
};
__global__ void k_put(unsigned char* __restrict__ dst, Blob src, int bytes) {
  for (int i = threadIdx.x; i < bytes; i += blockDim.x) dst[i] = src.b[i];
}
void launch_put(void* dst, const void* src, size_t bytes, cudaStream_t s) {
  for (size_t off = 0; off < bytes; off += BLOB_BYTES) {
    Blob b;
    const size_t n = bytes - off < (size_t)BLOB_BYTES ? bytes - off : (size_t)BLOB_BYTES;
    memcpy(b.b, (const unsigned char*)src + off, n);
    k_put<<<1, 256, 0, s>>>((unsigned char*)dst + off, b, (int)n);
  }
}

__global__ void k_gather_rows(const float* __restrict__ xs, long long n_pad, int d,
                              const long long* __restrict__ ids, long long row_offset,
                              long long n_local, int cnt, float* __restrict__ out) {
  const long long tot = (long long)cnt * d;
  for (long long e = blockIdx.x * (long long)blockDim.x + threadIdx.x; e < tot;
       e += (long long)gridDim.x * blockDim.x) {
    int t = (int)(e / d), j = (int)(e - (long long)t * d);
    long long r = ids[t] - row_offset;
    out[e] = (r >= 0 && r < n_local) ? xs[(long long)j * n_pad + r] : 0.f;
  }
}

void launch_gather_rows(const float* xs, long long n_pad, int d, const long long* ids,
                        long long row_offset, long long n_local, int cnt, float* out,
                        cudaStream_t s) {
  long long tot = (long long)cnt * d;
  int blocks = (int)((tot + 255) / 256);
  if (blocks < 1) blocks = 1;
  if (blocks > 1184) blocks = 1184;
  k_gather_rows<<<blocks, 256, 0, s>>>(xs, n_pad, d, ids, row_offset, n_local, cnt, out);
}

__global__ void k_gather_m(const float* __restrict__ srows, const long long* __restrict__ sids,
                           const int* __restrict__ spos, int nM, int d,
                           float* __restrict__ mrows, long long* __restrict__ mids) {
  for (int e = blockIdx.x * blockDim.x + threadIdx.x; e < nM * d;
       e += gridDim.x * blockDim.x) {
    int i = e / d, j = e - i * d;
    mrows[e] = srows[(long long)spos[i] * d + j];
    if (j == 0) mids[i] = sids[spos[i]];
  }
}

void launch_gather_m(const float* srows, const long long* sids, const int* spos, int nM, int d,
                     float* mrows, long long* mids, cudaStream_t s) {
  int blocks = (nM * d + 255) / 256;
  if (blocks < 1) blocks = 1;
  if (blocks > 592) blocks = 592;
  k_gather_m<<<blocks, 256, 0, s>>>(srows, sids, spos, nM, d, mrows, mids);
}

// ===================================================================== N1
// Greedy (Alg 2).  Step 1 (whole GPU): the exact fp64 distance
// matrix Ds[a][q] = full(S_q, S_a) of the sample, in the oracle's expression
// (all #M picks read rows of it).  Step 2 (one CTA, all #M-1 dependent picks
// in one launch; the paper uses two launches per pick): dist[q] =
// min(dist[q], Ds[pick][q]) and a block argmax (larger distance, then smaller
// position, reading R7) with redux.sync on a 64-bit order key: 0 for picked
// points, bits(dist) + 1 otherwise.
constexpr int GR_TPB = 1024;

struct KeyIdx {
  unsigned hi, lo, idx;
};
__device__ __forceinline__ KeyIdx warp_argmax(unsigned hi, unsigned lo, unsigned idx);
__device__ __forceinline__ unsigned long long dkey(double v);

// Cluster variant: the same picks spread over a thread-block cluster of CS
// CTAs (one per SM), so the fp64 distance work of a pick runs on CS SMs.
// Every CTA holds the whole sample in shared memory and owns positions
// g, g + CS*GC_TPB, ... (g = rank*GC_TPB + tid).  Per pick each CTA reduces
// each warp reduces its candidate and pushes it (16 bytes) into its slot of
// every CTA of the cluster with st.async, completing 16 bytes of tx on the
// receiver's mbarrier; a CTA proceeds when all CS*GC_W = 32 candidates landed
// and reduces them with one warp argmax (slots parity double buffered: pick
// i uses slot i&1).
#ifndef GC_CS
#define GC_CS 8  // CTAs per greedy cluster (32 warps in all; 8 x 128 threads: 58 vs 60 us at C3)
#endif
constexpr int GC_TPB = 1024 / GC_CS;  // threads per CTA
constexpr int GC_W = GC_TPB / 32;

__device__ __forceinline__ unsigned cluster_rank() {
  unsigned r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ void cluster_sync_all() {
  asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::
                   : "memory");
}
__device__ __forceinline__ unsigned mapa_u32(unsigned laddr, unsigned rank) {
  unsigned r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(laddr), "r"(rank));
  return r;
}
__device__ __forceinline__ void st_async_v4(unsigned raddr, unsigned a, unsigned b, unsigned c,
                                            unsigned d, unsigned rbar) {
  asm volatile(
      "st.async.shared::cluster.mbarrier::complete_tx::bytes.v4.b32 [%0], {%1, %2, %3, %4}, "
      "[%5];" ::"r"(raddr),
      "r"(a), "r"(b), "r"(c), "r"(d), "r"(rbar)
      : "memory");
}

// Distances of the owned positions to pick qs: DP > 0 is d rounded up to a
// multiple of 8 (zero-padded dimensions add exact zeros to the oracle-order
// sum, so the result is unchanged) and fully unrolled; DP = 0 loops over d.
template <int NP, int METRIC, int CS, int DP>
__device__ __forceinline__ void greedy_update_c(const double* __restrict__ gT, int nSp, int nS,
                                                int d, int g, int qs, bool first,
                                                double (&dreg)[NP]) {
  constexpr int STRIDE = CS * GC_TPB;
  double acc[NP];
#pragma unroll
  for (int t = 0; t < NP; ++t) acc[t] = 0.0;
  if (DP > 0) {
#pragma unroll
    for (int j = 0; j < DP; ++j) {
      const double pj = gT[j * nSp + qs];
#pragma unroll
      for (int t = 0; t < NP; ++t) {
        const double df = dsub(gT[j * nSp + g + t * STRIDE], pj);
        acc[t] = dadd(acc[t], METRIC == 1 ? fabs(df) : dmul(df, df));
      }
    }
  } else {
    for (int j = 0; j < d; ++j) {
      const double pj = gT[j * nSp + qs];
#pragma unroll
      for (int t = 0; t < NP; ++t) {
        const double df = dsub(gT[j * nSp + g + t * STRIDE], pj);
        acc[t] = dadd(acc[t], METRIC == 1 ? fabs(df) : dmul(df, df));
      }
    }
  }
#pragma unroll
  for (int t = 0; t < NP; ++t) {
    const int q = g + t * STRIDE;
    const double u = METRIC == 1 ? acc[t] : __dsqrt_rn(acc[t]);
    if (first) {
      dreg[t] = (q < nS && q != qs) ? u : -1.0;
    } else if (q == qs) {
      dreg[t] = -1.0;
    } else if (dreg[t] >= 0.0 && u < dreg[t]) {
      dreg[t] = u;
    }
  }
}

// Sample rows [nS][d] fp32 -> [dp][nSp] fp64 (zero padded), the layout the
// cluster greedy copies into each CTA's shared memory with bulk copies.
__global__ void k_sample_soa(const float* __restrict__ srows, int nS, int d, int dp, int nSp,
                             double* __restrict__ out) {
  const int tot = dp * nSp;
  for (int e = blockIdx.x * blockDim.x + threadIdx.x; e < tot; e += gridDim.x * blockDim.x) {
    const int j = e / nSp, q = e - j * nSp;
    out[e] = (q < nS && j < d) ? (double)srows[(long long)q * d + j] : 0.0;
  }
}

template <int NP, int METRIC, int CS, int DP>
__global__ void __launch_bounds__(GC_TPB)
    k_greedy_cluster(const double* __restrict__ sT, int nS, int d, int dp, int nM, int q0,
                     int* __restrict__ spos, double* __restrict__ pickdist) {
  extern __shared__ __align__(16) double gT[];  // [dp][nSp], nSp = NP * CS * GC_TPB
  static_assert(CS * GC_W == 32, "one candidate slot per lane");
  __shared__ __align__(16) unsigned cand[2][CS * GC_W][4];
  __shared__ __align__(8) unsigned long long bar[3];
  constexpr int nSp = NP * CS * GC_TPB;
  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  const unsigned rank = cluster_rank();
  const int g = (int)rank * GC_TPB + tid;
  if (tid == 0) {
    mbar_init(&bar[0], 1);
    mbar_init(&bar[1], 1);
    mbar_init(&bar[2], 1);
    fence_mbar_init();
  }
  __syncthreads();
  if (tid == 0) {  // the whole sample: bulk copies of <= 32 KB on bar[2]
    const unsigned bytes = (unsigned)(sizeof(double) * (size_t)dp * nSp);
    mbar_expect_tx(&bar[2], bytes);
    for (unsigned off = 0; off < bytes; off += 32768u) {
      const unsigned len = bytes - off < 32768u ? bytes - off : 32768u;
      bulk_g2s((char*)gT + off, (const char*)sT + off, len, &bar[2]);
    }
  }
  cluster_sync_all();  // every CTA's barriers are initialised before any push
  mbar_wait(&bar[2], 0u);
  double dreg[NP];
  greedy_update_c<NP, METRIC, CS, DP>(gT, nSp, nS, d, g, q0, true, dreg);
  if (rank == 0 && tid == 0) {
    spos[0] = q0;
    if (pickdist) pickdist[0] = CUDART_INF;
  }
  for (int i = 1; i < nM; ++i) {
    const int par = i & 1;
    const unsigned ph = (unsigned)(((i - 1) >> 1) & 1);  // use count of slot par
    if (tid == 0) mbar_expect_tx(&bar[par], CS * GC_W * 16u);
    unsigned long long bk = 0ull;
    unsigned bq = 0xffffffffu;
#pragma unroll
    for (int t = 0; t < NP; ++t) {
      const unsigned long long key = dkey(dreg[t]);
      if (key > bk) {
        bk = key;
        bq = g + t * CS * GC_TPB;
      }
    }
    // every warp pushes its candidate into slot (rank, w) of every CTA
    KeyIdx r = warp_argmax((unsigned)(bk >> 32), (unsigned)bk, bq);
    if (lane < CS)
      st_async_v4(mapa_u32(smem_u32(&cand[par][rank * GC_W + w][0]), (unsigned)lane), r.hi, r.lo,
                  r.idx, 0u, mapa_u32(smem_u32(&bar[par]), (unsigned)lane));
    mbar_wait(&bar[par], ph);
    KeyIdx s = warp_argmax(cand[par][lane][0], cand[par][lane][1], cand[par][lane][2]);
    const int qs = (int)s.idx;
    if (rank == 0 && tid == 0) {
      spos[i] = qs;
      if (pickdist) {
        unsigned long long kk = ((unsigned long long)s.hi << 32) | s.lo;
        pickdist[i] = __longlong_as_double((long long)(kk - 1ull));
      }
    }
    if (i + 1 < nM) greedy_update_c<NP, METRIC, CS, DP>(gT, nSp, nS, d, g, qs, false, dreg);
  }
  cluster_sync_all();  // no CTA leaves while a peer may still push into it
}


// Greedy with the sample resident in shared memory, transposed to [j][q]
// (fp64, zero padded to NP*256 positions): every pick recomputes the
// distances of the NP owned positions to the new medoid in registers.  The d
// per-dimension terms are formed four at a time ahead of the oracle-order
// chain of additions (j ascending), so only the dadd chain is serial.  One
// barrier per pick and a redundant 8-way argmax.
template <int NP, int METRIC>
__device__ __forceinline__ void greedy_update(const double* __restrict__ gT, int nSp, int nS,
                                              int d, int qs, bool first, double (&dreg)[NP]) {
  const int tid = threadIdx.x;
  double acc[NP];
#pragma unroll
  for (int t = 0; t < NP; ++t) acc[t] = 0.0;
  int j = 0;
  for (; j + 4 <= d; j += 4) {
    double pj[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) pj[u] = gT[(j + u) * nSp + qs];
    double tm[NP][4];
#pragma unroll
    for (int t = 0; t < NP; ++t)
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const double df = dsub(gT[(j + u) * nSp + tid + t * 256], pj[u]);
        tm[t][u] = METRIC == 1 ? fabs(df) : dmul(df, df);
      }
#pragma unroll
    for (int t = 0; t < NP; ++t)
      acc[t] = dadd(dadd(dadd(dadd(acc[t], tm[t][0]), tm[t][1]), tm[t][2]), tm[t][3]);
  }
  for (; j < d; ++j) {
    const double pj = gT[j * nSp + qs];
#pragma unroll
    for (int t = 0; t < NP; ++t) {
      const double df = dsub(gT[j * nSp + tid + t * 256], pj);
      acc[t] = dadd(acc[t], METRIC == 1 ? fabs(df) : dmul(df, df));
    }
  }
#pragma unroll
  for (int t = 0; t < NP; ++t) {
    const int q = tid + t * 256;
    const double u = METRIC == 1 ? acc[t] : __dsqrt_rn(acc[t]);
    if (first) {
      dreg[t] = (q < nS && q != qs) ? u : -1.0;
    } else if (q == qs) {
      dreg[t] = -1.0;
    } else if (dreg[t] >= 0.0 && u < dreg[t]) {
      dreg[t] = u;
    }
  }
}

template <int NP, int METRIC>
__global__ void __launch_bounds__(256)
    k_greedy_smem(const float* __restrict__ srows, int nS, int d, int nM, int q0,
                  int* __restrict__ spos, double* __restrict__ pickdist) {
  extern __shared__ double gT[];  // [d][NP*256]
  __shared__ unsigned whi[2][8], wlo[2][8], widx[2][8];
  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  constexpr int nSp = NP * 256;
  for (int e = tid; e < nSp * d; e += 256) {
    const int j = e / nSp, q = e - j * nSp;
    gT[e] = q < nS ? (double)srows[(long long)q * d + j] : 0.0;
  }
  __syncthreads();
  double dreg[NP];
  greedy_update<NP, METRIC>(gT, nSp, nS, d, q0, true, dreg);
  if (tid == 0) {
    spos[0] = q0;
    if (pickdist) pickdist[0] = CUDART_INF;
  }
  for (int i = 1; i < nM; ++i) {
    // pick i: argmax over unpicked (larger distance, then smaller position)
    unsigned long long bk = 0ull;
    unsigned bq = 0xffffffffu;
#pragma unroll
    for (int t = 0; t < NP; ++t) {
      const unsigned long long key = dkey(dreg[t]);
      if (key > bk) {
        bk = key;
        bq = tid + t * 256;
      }
    }
    KeyIdx r = warp_argmax((unsigned)(bk >> 32), (unsigned)bk, bq);
    const int par = i & 1;
    if (lane == 0) {
      whi[par][w] = r.hi;
      wlo[par][w] = r.lo;
      widx[par][w] = r.idx;
    }
    __syncthreads();
    KeyIdx s = warp_argmax(lane < 8 ? whi[par][lane] : 0u, lane < 8 ? wlo[par][lane] : 0u,
                           lane < 8 ? widx[par][lane] : 0xffffffffu);
    const int qs = (int)s.idx;
    if (tid == 0) {
      spos[i] = qs;
      if (pickdist) {
        unsigned long long kk = ((unsigned long long)s.hi << 32) | s.lo;
        pickdist[i] = __longlong_as_double((long long)(kk - 1ull));
      }
    }
    if (i + 1 < nM) greedy_update<NP, METRIC>(gT, nSp, nS, d, qs, false, dreg);
  }
}

__device__ __forceinline__ KeyIdx warp_argmax(unsigned hi, unsigned lo, unsigned idx);
__device__ __forceinline__ unsigned long long dkey(double v);

// Greedy with the sample rows resident in shared memory (fp64): every pick
// recomputes the distances of the owned positions to the new medoid in
// registers (NP positions per thread, the j loop outside so the NP oracle-
// order chains interleave), then one barrier and a redundant 8-way argmax.
template <int NP>
__global__ void __launch_bounds__(256)
    k_greedy_smem(const float* __restrict__ srows, int nS, int d, int nM, int q0, int metric,
                  int* __restrict__ spos, double* __restrict__ pickdist) {
  extern __shared__ double grows[];  // [nS][d]
  __shared__ unsigned whi[2][8], wlo[2][8], widx[2][8];
  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  for (int e = tid; e < nS * d; e += 256) grows[e] = (double)srows[e];
  __syncthreads();
  double dreg[NP];
  // distances of the owned positions to pick qs (oracle order, j ascending)
  auto update = [&](int qs, bool first) {
    double acc[NP];
#pragma unroll
    for (int t = 0; t < NP; ++t) acc[t] = 0.0;
    const double* pr = grows + (long long)qs * d;
    for (int j = 0; j < d; ++j) {
      const double pj = pr[j];
#pragma unroll
      for (int t = 0; t < NP; ++t) {
        const int q = tid + t * 256;
        const double x = q < nS ? grows[(long long)q * d + j] : 0.0;
        const double df = dsub(x, pj);
        acc[t] = metric == 1 ? dadd(acc[t], fabs(df)) : dadd(acc[t], dmul(df, df));
      }
    }
#pragma unroll
    for (int t = 0; t < NP; ++t) {
      const int q = tid + t * 256;
      const double u = metric == 1 ? acc[t] : __dsqrt_rn(acc[t]);
      if (first) {
        dreg[t] = (q < nS && q != qs) ? u : -1.0;
      } else if (q == qs) {
        dreg[t] = -1.0;
      } else if (dreg[t] >= 0.0 && u < dreg[t]) {
        dreg[t] = u;
      }
    }
  };
  update(q0, true);
  if (tid == 0) {
    spos[0] = q0;
    if (pickdist) pickdist[0] = CUDART_INF;
  }
  for (int i = 1; i < nM; ++i) {
    // pick i: argmax over unpicked (larger distance, then smaller position)
    unsigned long long bk = 0ull;
    unsigned bq = 0xffffffffu;
#pragma unroll
    for (int t = 0; t < NP; ++t) {
      const unsigned long long key = dkey(dreg[t]);
      if (key > bk) {
        bk = key;
        bq = tid + t * 256;
      }
    }
    KeyIdx r = warp_argmax((unsigned)(bk >> 32), (unsigned)bk, bq);
    const int par = i & 1;
    if (lane == 0) {
      whi[par][w] = r.hi;
      wlo[par][w] = r.lo;
      widx[par][w] = r.idx;
    }
    __syncthreads();
    KeyIdx s = warp_argmax(lane < 8 ? whi[par][lane] : 0u, lane < 8 ? wlo[par][lane] : 0u,
                           lane < 8 ? widx[par][lane] : 0xffffffffu);
    const int qs = (int)s.idx;
    if (tid == 0) {
      spos[i] = qs;
      if (pickdist) {
        unsigned long long kk = ((unsigned long long)s.hi << 32) | s.lo;
        pickdist[i] = __longlong_as_double((long long)(kk - 1ull));
      }
    }
    if (i + 1 < nM) update(qs, false);
  }
}

__device__ __forceinline__ KeyIdx warp_argmax(unsigned hi, unsigned lo, unsigned idx) {
  const unsigned full = 0xffffffffu;
  unsigned mhi = __reduce_max_sync(full, hi);
  unsigned mlo = __reduce_max_sync(full, hi == mhi ? lo : 0u);
  unsigned midx = __reduce_min_sync(full, (hi == mhi && lo == mlo) ? idx : 0xffffffffu);
  return {mhi, mlo, midx};
}

__device__ __forceinline__ unsigned long long dkey(double v) {
  return v >= 0.0 ? (unsigned long long)__double_as_longlong(v) + 1ull : 0ull;
}

// gate of the exact-matrix greedy path: #S <= GM_TPB * GM_PPT = 4096
constexpr int GM_TPB = 256;
constexpr int GM_PPT = 16;

__global__ void __launch_bounds__(GR_TPB)
    k_greedy_big(const float* __restrict__ srows, int nS, int d, int nM, int q0, int metric,
                 double* __restrict__ dist, int* __restrict__ spos, double* __restrict__ pickdist) {
  extern __shared__ double prow[];
  __shared__ unsigned whi[32], wlo[32], widx[32];
  __shared__ int pick_s;
  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  const int nw = GR_TPB / 32;
  for (int j = tid; j < d; j += GR_TPB) prow[j] = (double)srows[(long long)q0 * d + j];
  __syncthreads();
  for (int q = tid; q < nS; q += GR_TPB)
    dist[q] = (q == q0) ? -1.0 : full_dist(srows + (long long)q * d, 1, prow, d, metric);
  if (tid == 0) {
    spos[0] = q0;
    if (pickdist) pickdist[0] = CUDART_INF;
  }
  for (int i = 1; i < nM; ++i) {
    unsigned long long bk = 0ull;
    unsigned bq = 0xffffffffu;
    for (int q = tid; q < nS; q += GR_TPB) {
      const unsigned long long key = dkey(dist[q]);
      if (key > bk) {
        bk = key;
        bq = q;
      }
    }
    KeyIdx r = warp_argmax((unsigned)(bk >> 32), (unsigned)bk, bq);
    if (lane == 0) {
      whi[w] = r.hi;
      wlo[w] = r.lo;
      widx[w] = r.idx;
    }
    __syncthreads();
    if (w == 0) {
      KeyIdx s = warp_argmax(lane < nw ? whi[lane] : 0u, lane < nw ? wlo[lane] : 0u,
                             lane < nw ? widx[lane] : 0xffffffffu);
      if (lane == 0) {
        pick_s = (int)s.idx;
        spos[i] = (int)s.idx;
        if (pickdist) {
          unsigned long long kk = ((unsigned long long)s.hi << 32) | s.lo;
          pickdist[i] = __longlong_as_double((long long)(kk - 1ull));
        }
      }
    }
    __syncthreads();
    const int qs = pick_s;
    for (int j = tid; j < d; j += GR_TPB) prow[j] = (double)srows[(long long)qs * d + j];
    __syncthreads();
    for (int q = tid; q < nS; q += GR_TPB) {
      if (q == qs) {
        dist[q] = -1.0;
      } else if (dist[q] >= 0.0) {
        const double u = full_dist(srows + (long long)q * d, 1, prow, d, metric);
        if (u < dist[q]) dist[q] = u;
      }
    }
    __syncthreads();
  }
}

size_t greedy_scratch_doubles(int nS) {
  // distance matrix (k_greedy), or the fp64 SoA sample of the cluster greedy
  const size_t m = nS <= GM_PPT * GM_TPB ? (size_t)nS * nS : (size_t)nS;
  const size_t soa = (size_t)32 * 4 * 16 * 64;
  return m > soa ? m : soa;
}

template <int NP>
static cudaError_t greedy_smem_launch(const float* srows, int nS, int d, int nM, int q0,
                                      int metric, int* spos, double* pickdist, cudaStream_t s) {
  const size_t bytes = sizeof(double) * (size_t)NP * 256 * d;
  cudaError_t e;
  if (metric == 1) {
    e = cudaFuncSetAttribute(k_greedy_smem<NP, 1>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)bytes);
    if (e == cudaSuccess)
      k_greedy_smem<NP, 1><<<1, 256, bytes, s>>>(srows, nS, d, nM, q0, spos, pickdist);
  } else {
    e = cudaFuncSetAttribute(k_greedy_smem<NP, 0>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)bytes);
    if (e == cudaSuccess)
      k_greedy_smem<NP, 0><<<1, 256, bytes, s>>>(srows, nS, d, nM, q0, spos, pickdist);
  }
  if (e != cudaSuccess) return e;
  return cudaGetLastError();
}

template <int NP, int METRIC, int DP>
static cudaError_t greedy_cluster_launch(const double* sT, int nS, int d, int dp, int nM, int q0,
                                         int* spos, double* pickdist, cudaStream_t s) {
  constexpr int CS = GC_CS;
  const size_t bytes = sizeof(double) * (size_t)NP * CS * GC_TPB * dp;
  auto fn = k_greedy_cluster<NP, METRIC, CS, DP>;
  cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(fn, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
  if (e != cudaSuccess) return e;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(CS, 1, 1);
  cfg.blockDim = dim3(GC_TPB, 1, 1);
  cfg.dynamicSmemBytes = bytes;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = CS;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, fn, sT, nS, d, dp, nM, q0, spos, pickdist);
}

template <int NP, int DP>
static cudaError_t greedy_cluster_m(const double* sT, int nS, int d, int dp, int nM, int q0,
                                    int metric, int* spos, double* pickdist, cudaStream_t s) {
  return metric == 1
             ? greedy_cluster_launch<NP, 1, DP>(sT, nS, d, dp, nM, q0, spos, pickdist, s)
             : greedy_cluster_launch<NP, 0, DP>(sT, nS, d, dp, nM, q0, spos, pickdist, s);
}

template <int NP>
static cudaError_t greedy_cluster_np(const double* sT, int nS, int d, int dp, int nM, int q0,
                                     int metric, int* spos, double* pickdist, cudaStream_t s) {
  switch (dp) {
    case 8: return greedy_cluster_m<NP, 8>(sT, nS, d, dp, nM, q0, metric, spos, pickdist, s);
    case 16: return greedy_cluster_m<NP, 16>(sT, nS, d, dp, nM, q0, metric, spos, pickdist, s);
    case 32: return greedy_cluster_m<NP, 32>(sT, nS, d, dp, nM, q0, metric, spos, pickdist, s);
    default: return greedy_cluster_m<NP, 0>(sT, nS, d, dp, nM, q0, metric, spos, pickdist, s);
  }
}

// Exact #S x #S sample distances (O0's expression: j ascending, no FMA) by
// 64 x 64 tiles of the upper triangle, written to both halves (full(p, q)
// and full(q, p) are bit-identical: the terms are squares / absolute values
// of negated differences).  A thread keeps 4 x 4 independent accumulation
// chains, so the 100-step dependent DADD chain of a d = 100 distance is
// overlapped 16 ways; rows are staged once in shared memory as fp64.
constexpr int SD_T = 64, SD_J = 32;
__global__ void __launch_bounds__(256) k_sdist_tiled(const float* __restrict__ srows, int nS,
                                                     int d, int metric,
                                                     double* __restrict__ Ds) {
  __shared__ double sa[SD_J][SD_T], sq[SD_J][SD_T];
  // upper-triangle tile (ta <= tq) of linear index blockIdx.x
  const int nt = (nS + SD_T - 1) / SD_T;
  int t = blockIdx.x, ta = 0;
  while (t >= nt - ta) {
    t -= nt - ta;
    ++ta;
  }
  const int tq = ta + t;
  const int a0 = ta * SD_T, q0 = tq * SD_T;
  const int tx = threadIdx.x & 15, ty = threadIdx.x >> 4;
  double acc[4][4];
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int k2 = 0; k2 < 4; ++k2) acc[i][k2] = 0.0;
  for (int j0 = 0; j0 < d; j0 += SD_J) {
    __syncthreads();
    for (int e = threadIdx.x; e < SD_J * SD_T; e += 256) {
      const int jj = e / SD_T, r = e - jj * SD_T, j = j0 + jj;
      const int a = a0 + r, q = q0 + r;
      sa[jj][r] = (j < d && a < nS) ? (double)srows[(long long)a * d + j] : 0.0;
      sq[jj][r] = (j < d && q < nS) ? (double)srows[(long long)q * d + j] : 0.0;
    }
    __syncthreads();
    const int jn = min(SD_J, d - j0);
    for (int jj = 0; jj < jn; ++jj) {
      double va[4], vq[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        va[i] = sa[jj][ty + 16 * i];
        vq[i] = sq[jj][tx + 16 * i];
      }
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int k2 = 0; k2 < 4; ++k2) {
          const double u = dsub(vq[k2], va[i]);  // p = S[q], q = S[a] as in O4
          acc[i][k2] = metric == 1 ? dadd(acc[i][k2], fabs(u)) : dadd(acc[i][k2], dmul(u, u));
        }
    }
  }
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int k2 = 0; k2 < 4; ++k2) {
      const int a = a0 + ty + 16 * i, q = q0 + tx + 16 * k2;
      if (a < nS && q < nS) {
        const double v = metric == 1 ? acc[i][k2] : __dsqrt_rn(acc[i][k2]);
        Ds[(long long)a * nS + q] = v;
        Ds[(long long)q * nS + a] = v;
      }
    }
}

// Greedy over the precomputed exact distance matrix (k_sdist_tiled) with the
// candidates spread over a cluster of 16 CTAs (NP per thread): every pick
// each SM reads only its slice of row qs (the single-CTA k_greedy pulls the
// whole 8 nS-byte row through one SM), and the argmax is exchanged through
// distributed shared memory exactly as in k_greedy_cluster.  Same keys, same
// ascending-position tie rule, so the same picks.
template <int NP>
__global__ void __launch_bounds__(GC_TPB)
    k_greedy_mat(const double* __restrict__ Ds, int nS, int nM, int q0, int* __restrict__ spos,
                 double* __restrict__ pickdist) {
  constexpr int CS = GC_CS;
  static_assert(CS * GC_W == 32, "one candidate slot per lane");
  __shared__ __align__(16) unsigned cand[2][CS * GC_W][4];
  __shared__ __align__(8) unsigned long long bar[2];
  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  const unsigned rank = cluster_rank();
  const int g = (int)rank * GC_TPB + tid;
  if (tid == 0) {
    mbar_init(&bar[0], 1);
    mbar_init(&bar[1], 1);
    fence_mbar_init();
  }
  __syncthreads();
  double dreg[NP];
#pragma unroll
  for (int t = 0; t < NP; ++t) {
    const int q = g + t * CS * GC_TPB;
    dreg[t] = (q < nS && q != q0) ? __ldg(Ds + (long long)q0 * nS + q) : -1.0;
  }
  cluster_sync_all();  // every CTA's barriers are initialised before any push
  if (rank == 0 && tid == 0) {
    spos[0] = q0;
    if (pickdist) pickdist[0] = CUDART_INF;
  }
  for (int i = 1; i < nM; ++i) {
    const int par = i & 1;
    const unsigned ph = (unsigned)(((i - 1) >> 1) & 1);  // use count of slot par
    if (tid == 0) mbar_expect_tx(&bar[par], CS * GC_W * 16u);
    unsigned long long bk = 0ull;
    unsigned bq = 0xffffffffu;
#pragma unroll
    for (int t = 0; t < NP; ++t) {
      const unsigned long long key = dkey(dreg[t]);
      if (key > bk) {  // ascending position: strict > keeps the smaller one
        bk = key;
        bq = g + t * CS * GC_TPB;
      }
    }
    KeyIdx r = warp_argmax((unsigned)(bk >> 32), (unsigned)bk, bq);
    if (lane < CS)
      st_async_v4(mapa_u32(smem_u32(&cand[par][rank * GC_W + w][0]), (unsigned)lane), r.hi, r.lo,
                  r.idx, 0u, mapa_u32(smem_u32(&bar[par]), (unsigned)lane));
    mbar_wait(&bar[par], ph);
    KeyIdx sb = warp_argmax(cand[par][lane][0], cand[par][lane][1], cand[par][lane][2]);
    const int qs = (int)sb.idx;
    if (rank == 0 && tid == 0) {
      spos[i] = qs;
      if (pickdist) {
        unsigned long long kk = ((unsigned long long)sb.hi << 32) | sb.lo;
        pickdist[i] = __longlong_as_double((long long)(kk - 1ull));
      }
    }
    if (i + 1 < nM) {
      const double* row = Ds + (long long)qs * nS;
#pragma unroll
      for (int t = 0; t < NP; ++t) {
        const int q = g + t * CS * GC_TPB;
        if (q == qs) {
          dreg[t] = -1.0;
        } else if (dreg[t] >= 0.0) {
          const double u = __ldg(row + q);
          if (u < dreg[t]) dreg[t] = u;
        }
      }
    }
  }
  cluster_sync_all();  // no CTA leaves while a peer may still push into it
}

template <int NP>
static cudaError_t greedy_mat_launch(const double* Ds, int nS, int nM, int q0, int* spos,
                                     double* pickdist, cudaStream_t s) {
  constexpr int CS = GC_CS;
  auto fn = k_greedy_mat<NP>;
  cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
  if (e != cudaSuccess) return e;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(CS, 1, 1);
  cfg.blockDim = dim3(GC_TPB, 1, 1);
  cfg.dynamicSmemBytes = 0;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = CS;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, fn, Ds, nS, nM, q0, spos, pickdist);
}

cudaError_t launch_greedy(const float* srows, int nS, int d, int nM, int q0, int metric,
                          double* scratch, int* spos, double* pickdist, cudaStream_t s) {
  {  // cluster of 16 CTAs x 64 threads: NP positions per thread
    const int per = GC_CS * GC_TPB;
    const int npc = nS <= per ? 1 : nS <= 2 * per ? 2 : nS <= 4 * per ? 4 : 0;
    const int dp = d <= 8 ? 8 : d <= 16 ? 16 : d <= 32 ? 32 : ((d + 1) / 2) * 2;
    const size_t soa = (size_t)dp * npc * per;  // doubles
    if (npc && sizeof(double) * soa <= 200 * 1024 && soa <= greedy_scratch_doubles(nS)) {
      k_sample_soa<<<(int)((soa + 255) / 256), 256, 0, s>>>(srows, nS, d, dp, npc * per, scratch);
      return npc == 1 ? greedy_cluster_np<1>(scratch, nS, d, dp, nM, q0, metric, spos, pickdist, s)
             : npc == 2 ? greedy_cluster_np<2>(scratch, nS, d, dp, nM, q0, metric, spos, pickdist, s)
                        : greedy_cluster_np<4>(scratch, nS, d, dp, nM, q0, metric, spos, pickdist, s);
    }
  }
  const int np = nS <= 256 ? 1 : nS <= 512 ? 2 : nS <= 1024 ? 4 : nS <= 2048 ? 8 : 16;
  if (nS <= 16 * 256 && sizeof(double) * (size_t)np * 256 * d <= 200 * 1024) {
    switch (np) {
      case 1: return greedy_smem_launch<1>(srows, nS, d, nM, q0, metric, spos, pickdist, s);
      case 2: return greedy_smem_launch<2>(srows, nS, d, nM, q0, metric, spos, pickdist, s);
      case 4: return greedy_smem_launch<4>(srows, nS, d, nM, q0, metric, spos, pickdist, s);
      case 8: return greedy_smem_launch<8>(srows, nS, d, nM, q0, metric, spos, pickdist, s);
      default: return greedy_smem_launch<16>(srows, nS, d, nM, q0, metric, spos, pickdist, s);
    }
  }
  if (nS <= GM_PPT * GM_TPB) {  // <= 4096: exact matrix, picks in a 16-CTA cluster
    const int nt = (nS + SD_T - 1) / SD_T;
    k_sdist_tiled<<<nt * (nt + 1) / 2, 256, 0, s>>>(srows, nS, d, metric, scratch);
    const int per = GC_CS * GC_TPB;
    return nS <= 2 * per ? greedy_mat_launch<2>(scratch, nS, nM, q0, spos, pickdist, s)
                         : greedy_mat_launch<4>(scratch, nS, nM, q0, spos, pickdist, s);
  }
  k_greedy_big<<<1, GR_TPB, sizeof(double) * d, s>>>(srows, nS, d, nM, q0, metric, scratch,
                                                     spos, pickdist);
  return cudaGetLastError();
}

// ============================================================ pipeline
// Warp-specialised chunk pipeline: the last warp of a block is the TMA
// producer, the other NW warps consume.  full[s] completes when the bulk
// copies of a chunk landed (expect_tx); empty[s] completes when all NW
// consumer warps released the stage (one arrive each), after which the
// producer refills it.  No block-wide barrier inside the chunk loop.
__device__ __forceinline__ void mbar_arrive(unsigned long long* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_arrive(unsigned bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}

__device__ __forceinline__ void named_bar_sync(int id, int nthreads) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}


__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

struct ExtraRows {
  int n;
  int row0;                // ring row of the first extra row
  const float* src[KMAX];  // global row bases (indexed by point)
  float* drow[KMAX];       // k_locality: Dist row of active slot a (new rows are stored there)
};

struct Pipe {
  float* buf;                 // [stages][rows][P]
  unsigned char* lab;         // [stages][P] (label passes) or nullptr
  unsigned long long* full;   // [SMAX]
  unsigned long long* empty;  // [SMAX]
  int rows;
  int ldr;                    // row stride in floats (>= P)
  unsigned full_a, empty_a;   // 32-bit shared addresses of full[0] / empty[0]
};

__device__ __forceinline__ void pipe_init(const RunParams& p, const Pipe& R, int nw) {
  if (threadIdx.x == 0) {
    for (int s = 0; s < p.stages; ++s) {
      mbar_init(&R.full[s], 1);
      mbar_init(&R.empty[s], (unsigned)nw);
    }
    fence_mbar_init();
  }
}

// Producer warp: stream this block's chunks b, b+G, ... through the ring.
__device__ void pipe_produce(const RunParams& p, const Pipe& R, long long nmy,
                             const unsigned char* labsrc, const ExtraRows* ex) {
  const int lane = threadIdx.x & 31;
  const unsigned row = (unsigned)p.P * 4u;
  const int nex = ex ? ex->n : 0;
  const unsigned bytes = row * (unsigned)(p.d + nex) + (labsrc ? (unsigned)p.P : 0u);
  const unsigned long long pol_last = l2_policy(1), pol_first = l2_policy(0);
  int stg = 0, round = 0;
  for (long long i = 0; i < nmy; ++i) {
    if (round > 0) {  // the consumers of chunk i - stages released this stage
      mbar_wait(R.empty_a + 8u * stg, (unsigned)((round - 1) & 1));
      fence_proxy_async();
    }
    const long long base = (blockIdx.x + i * gridDim.x) * (long long)p.P;
    if (lane == 0) mbar_expect_tx(R.full_a + 8u * stg, bytes);
    __syncwarp();
    float* dst = R.buf + (size_t)stg * R.rows * R.ldr;
    for (int j = lane; j < p.d + nex; j += 32) {
      const float* src = j < p.d ? p.xs + (size_t)j * p.n_pad + base : ex->src[j - p.d] + base;
      const int jr = j < p.d ? j : ex->row0 + (j - p.d);
      bulk_g2s_h(dst + (size_t)jr * R.ldr, src, row, R.full_a + 8u * stg,
                 j < p.d ? pol_last : pol_first);
    }
    if (labsrc && lane == 0)
      bulk_g2s(R.lab + (size_t)stg * p.P, labsrc + base, (unsigned)p.P, R.full_a + 8u * stg);
    if (++stg == p.stages) {
      stg = 0;
      ++round;
    }
  }
}

// Consumer-side ring position: stage index and the parity of its full
// barrier, advanced without integer division.
struct RingPos {
  int stg = 0;
  unsigned ph = 0;
  __device__ __forceinline__ void next(int stages) {
    if (++stg == stages) {
      stg = 0;
      ph ^= 1u;
    }
  }
};

__device__ __forceinline__ void pipe_release(const Pipe& R, int stg) {
  __syncwarp();
  if ((threadIdx.x & 31) == 0) mbar_arrive(R.empty_a + 8u * stg);
}

// The last block to arrive (ticket) returns true; it then sees every other
// block's atomics (acquire-release ticket, ld.cg reads after).
// One acquire-release atomic at gpu scope instead of two sequentially
// consistent fences: the barrier orders the block's flush atomics before
// thread 0's release (cumulativity), and the last block's acquire plus the
// barrier order its later L2 (ld.cg) reads after every other block's release.
__device__ bool last_block(unsigned int* ticket) {
  __shared__ int is_last;
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned t;
    asm volatile("atom.add.acq_rel.gpu.u32 %0, [%1], 1;" : "=r"(t) : "l"(ticket) : "memory");
    is_last = (t == gridDim.x - 1);
    if (is_last) *ticket = 0u;
  }
  __syncthreads();
  return is_last;
}


// Combine the per-warp accumulators (exact int64) and add them to one of the
// NCOPY global copies with one atomic per non-zero cell.  Whole block.
__device__ void flush_warps(const RunParams& p, const long long* acc_s, int nw, int ncap,
                            int ncell, const long long* cnt_s, int ncnt, int nacc = -1) {
  if (nacc < 0) nacc = nw;
  const int cp = blockIdx.x % NCOPY;
  long long* acc = p.accg + (size_t)cp * p.k * p.d;
  long long* cnt = p.cntg + (size_t)cp * KMAX;
  for (int c = threadIdx.x; c < ncell; c += blockDim.x) {
    long long s = 0;
    for (int w = 0; w < nacc; ++w) s += acc_s[w * ncap + c];
    if (s) atomicAdd((unsigned long long*)&acc[c], (unsigned long long)s);
  }
  for (int c = threadIdx.x; c < ncnt; c += blockDim.x) {
    long long s = 0;
    for (int w = 0; w < nw; ++w) s += cnt_s[w * KMAX + c];
    if (s) atomicAdd((unsigned long long*)&cnt[c], (unsigned long long)s);
  }
}

// Exact total of accumulator c over the NCOPY copies; zeroes them.  All
// loads are issued before any store (one memory round trip).
__device__ __forceinline__ long long take_acc(const RunParams& p, int c) {
  const size_t stride = (size_t)p.k * p.d;
  long long v[NCOPY];
#pragma unroll
  for (int q = 0; q < NCOPY; ++q) v[q] = __ldcg(p.accg + q * stride + c);
  long long s = 0;
#pragma unroll
  for (int q = 0; q < NCOPY; ++q) {
    s += v[q];
    __stcg(p.accg + q * stride + c, 0ll);
  }
  return s;
}
__device__ __forceinline__ long long take_cnt(const RunParams& p, int c) {
  long long v[NCOPY];
#pragma unroll
  for (int q = 0; q < NCOPY; ++q) v[q] = __ldcg(p.cntg + q * KMAX + c);
  long long s = 0;
#pragma unroll
  for (int q = 0; q < NCOPY; ++q) {
    s += v[q];
    __stcg(p.cntg + q * KMAX + c, 0ll);
  }
  return s;
}

// One summation cell: set a (cluster / band slot), dimension j, centre c,
// index of its accumulator.
struct Cell {
  int a, j, acc;
  double c;
};

// Cells of one warp's sub-chunk (32*PPT points starting at q0): lane l owns
// cells l, l+32, ...; the member set of a is the ballot bitmask bal[a*PPT+u]
// of the warp's points.  fp64 sum (two interleaved accumulators, ascending
// point order), quantised to int64 at scale 2^e_j and added to the lane's
// own accumulator.  MODE 0: x, MODE 1: |x - c|.
template <int MODE, int PPT, bool IL = false, bool ATOM = false>
__device__ __forceinline__ void warp_cells(const float* __restrict__ xs, int P, int q0,
                                           const Cell* __restrict__ cells, int ncell,
                                           const unsigned* __restrict__ bal,
                                           long long* __restrict__ acc,
                                           const double* __restrict__ scale_s) {
  const int lane = threadIdx.x & 31;
  for (int ci = lane; ci < ncell; ci += 32) {
    const Cell C = cells[ci];
    const float* xr = xs + (size_t)C.j * P + q0;
    double s0 = 0.0, s1 = 0.0;
#pragma unroll
    for (int u = 0; u < PPT; ++u) {
      unsigned m = bal[C.a * PPT + u];
      // IL: bit b of ballot u is the point 2 b + u (paired points per lane)
      const float* xu = IL ? xr + u : xr + u * 32;
      while (m) {
        const int b0 = __ffs(m) - 1;
        m &= m - 1u;
        double v0 = (double)xu[IL ? 2 * b0 : b0];
        if (MODE == 1) v0 = fabs(dsub(v0, C.c));
        if (m) {
          const int b1 = __ffs(m) - 1;
          m &= m - 1u;
          double v1 = (double)xu[IL ? 2 * b1 : b1];
          if (MODE == 1) v1 = fabs(dsub(v1, C.c));
          s1 = dadd(s1, v1);
        }
        s0 = dadd(s0, v0);
      }
    }
    const double s = dadd(s0, s1);
    if (s != 0.0) {
      const long long v = __double2ll_rn(dmul(s, scale_s[C.j]));
      // ATOM: one block-wide copy shared by the warps (integer sums: the
      // order of the additions does not change the total)
      if (ATOM)
        atomicAdd((unsigned long long*)&acc[C.acc], (unsigned long long)v);
      else
        acc[C.acc] += v;
    }
  }
}

// ============================================================ smem carving
struct Carve {
  char* ptr;
  __device__ explicit Carve(void* base) : ptr((char*)base) {}
  template <class T>
  __device__ T* take(size_t count) {
    ptr = (char*)(((size_t)ptr + 15) & ~(size_t)15);
    T* r = (T*)ptr;
    ptr += sizeof(T) * count;
    return r;
  }
};

struct CarveSize {
  size_t s = 0;
  template <class T>
  CarveSize& add(size_t count) {
    s = ((s + 15) & ~(size_t)15) + sizeof(T) * count;
    return *this;
  }
};

__device__ Pipe carve_pipe(Carve& cv, const RunParams& p, int rows, bool with_lab) {
  Pipe R;
  R.rows = rows;
  R.ldr = p.P;
  R.full = cv.take<unsigned long long>(SMAX);
  R.empty = cv.take<unsigned long long>(SMAX);
  R.buf = cv.take<float>((size_t)p.stages * rows * p.P);
  R.lab = with_lab ? cv.take<unsigned char>((size_t)p.stages * p.P) : nullptr;
  R.full_a = smem_u32(R.full);
  R.empty_a = smem_u32(R.empty);
  return R;
}

// ============================================================ certified tests
// The fp32 value f approximates the oracle's fp64 value v with
// |f - v| <= G * v (G from the error analysis of the fp32 evaluation,
// DESIGN.md section 5).  Returns 1 if v <= T for sure, 0 if v > T for sure,
// -1 if undecided (tiny or huge values are always undecided).
__device__ __forceinline__ int cert_le(float f, double T, double G) {
  const double fd = (double)f;
  if (!(fd >= 1e-30) || !(T >= 1e-30) || !(fd < 1e30)) return -1;
  if (fd < T * (1.0 - G)) return 1;
  if (fd > T * (1.0 + G)) return 0;
  return -1;
}

// Exact (oracle) argmin of seg_{D_i}(x, m_i) = (sum_{j in D_i} |x_j - m_ij|)/|D_i|
// with ties to the smallest i (Alg 5, reading R8), fp64 from fp32 inputs.
// sq (may be null) receives every quotient.
__device__ __noinline__ int exact_argmin(const float* __restrict__ x, int P,
                                         const float* __restrict__ med32,
                                         const int* __restrict__ dl, const int* __restrict__ nD,
                                         int k, int d, const double* __restrict__ Dl,
                                         int* outside) {
  double best = CUDART_INF;
  int bi = 0, out = 1;
  for (int i = 0; i < k; ++i) {
    const int nd = nD[i];
    double s = 0.0;
    for (int t = 0; t < nd; ++t) {
      const int j = dl[i * d + t];
      s = dadd(s, fabs(dsub((double)x[j * P], (double)med32[i * d + j])));
    }
    const double q = ddiv(s, (double)nd);
    if (Dl && !(q > Dl[i])) out = 0;
    if (q < best) {
      best = q;
      bi = i;
    }
  }
  if (outside) *outside = out;
  return bi;
}

// ============================================================ tails
// The single-block steps between passes run on a shared-memory copy of the
// device state (DevState) and of every small array they touch.  They are
// latency-bound (a few hundred values), so each tail is organised in as few
// global-memory round trips as possible: the independent loads (state words,
// accumulators, small tables) are all issued before the first one is used,
// and the serial logic runs on warps with ballots / redux instead of single
// threads walking shared memory.
#ifdef PROCLUS_TAIL_PROFILE
__shared__ unsigned long long g_tst_last;
#define TST_START()                                        \
  do {                                                     \
    if (threadIdx.x == 0) g_tst_last = clock64();          \
  } while (0)
#define TST(T, idx)                                        \
  do {                                                     \
    __syncthreads();                                       \
    if (threadIdx.x == 0) {                                \
      const unsigned long long t_ = clock64();             \
      (T).S->dbg_cyc[idx] += t_ - g_tst_last;              \
      g_tst_last = t_;                                     \
    }                                                      \
  } while (0)
#define TSTW_DECL() unsigned long long tw_last_ = clock64()
#define TSTW(T, idx)                                                  \
  do {                                                                \
    __syncwarp();                                                     \
    const unsigned long long t_ = clock64();                          \
    if ((threadIdx.x & 31) == 0) (T).S->dbg_cyc[idx] += t_ - tw_last_; \
    tw_last_ = t_;                                                    \
  } while (0)
#else
#define TSTW_DECL() do {} while (0)
#define TSTW(T, idx) do {} while (0)
#define TST_START() \
  do {              \
  } while (0)
#define TST(T, idx) \
  do {              \
  } while (0)
#endif

struct TailMem {
  DevState* S;
  double* X;          // [k*d]
  double* Z;          // [k*d] (also raw accumulator values before Z exists)
  double* med;        // [k*d] medoid rows, fp64
  double* dev;        // [k*d] (also H rows / selection keys)
  unsigned char* dm;  // [k*d]
  int* pool;          // [nM]
  double* fnd;        // [3*KMAX]: found / used / delta' of the current slots
  double* isc;        // [d] 2^-e_j
  int* dl;            // [k*d] dimension lists
  double* dd;         // [k*k] medoid distances
  float* mrow;        // [nM*d] rows of M, or nullptr (not cached)
  unsigned char* fall;  // [nM] DistFound of M (with mrow)
  unsigned char* uall;  // [nM] delta' valid
  double* pall;         // [nM] delta'
};

__device__ __forceinline__ TailMem tail_mem(const RunParams& p, unsigned char* base) {
  const TailLayout& t = p.tl;
  TailMem T;
  T.S = (DevState*)(base + t.S);
  T.X = (double*)(base + t.X);
  T.Z = (double*)(base + t.Z);
  T.med = (double*)(base + t.med);
  T.dev = (double*)(base + t.dev);
  T.dm = base + t.dm;
  T.pool = (int*)(base + t.pool);
  T.fnd = (double*)(base + t.fnd);
  T.isc = (double*)(base + t.isc);
  T.dl = (int*)(base + t.dl);
  T.dd = (double*)(base + t.dd);
  T.mrow = t.mrow >= 0 ? (float*)(base + t.mrow) : nullptr;
  T.fall = t.mrow >= 0 ? base + t.fall : nullptr;
  T.uall = t.mrow >= 0 ? base + t.uall : nullptr;
  T.pall = t.mrow >= 0 ? (double*)(base + t.pall) : nullptr;
  return T;
}

// DevState words in registers: issue() starts the loads, commit() stores them
// into the shared copy, so their latency overlaps the loads in between.
constexpr int STATE_WORDS = (int)(sizeof(DevState) / 4);
constexpr int STATE_REGS = 8;  // words in flight per thread; the rest is copied in commit()
struct StateRegs {
  unsigned v[STATE_REGS];
};
__device__ __forceinline__ void state_issue(const RunParams& p, StateRegs& r) {
  const unsigned* src = (const unsigned*)p.st;
#pragma unroll
  for (int q = 0; q < STATE_REGS; ++q) {
    const int i = threadIdx.x + q * blockDim.x;
    r.v[q] = i < STATE_WORDS ? __ldcg(src + i) : 0u;
  }
}
__device__ __forceinline__ void state_commit(const RunParams& p, const StateRegs& r, DevState* S) {
  unsigned* dst = (unsigned*)S;
#pragma unroll
  for (int q = 0; q < STATE_REGS; ++q) {
    const int i = threadIdx.x + q * blockDim.x;
    if (i < STATE_WORDS) dst[i] = r.v[q];
  }
  const unsigned* src = (const unsigned*)p.st;  // small blocks: the remainder
  for (int i = threadIdx.x + STATE_REGS * blockDim.x; i < STATE_WORDS; i += blockDim.x)
    dst[i] = __ldcg(src + i);
}
__device__ void state_load(const RunParams& p, DevState* S) {
  StateRegs r;
  state_issue(p, r);
  state_commit(p, r, S);
  __syncthreads();
}
__device__ void state_store(const RunParams& p, const DevState* S) {
  __syncthreads();
  const unsigned* src = (const unsigned*)S;
  unsigned* dst = (unsigned*)p.st;
  for (int i = threadIdx.x; i < STATE_WORDS; i += blockDim.x) dst[i] = src[i];
}

// Position of the (r+1)-th set bit of w (r 0-based, r < popc(w)): a binary
// search on population counts (the __fns intrinsic is a long sequence).
__device__ __forceinline__ int nth_set_bit(unsigned w, int r) {
  int base = 0;
#pragma unroll
  for (int sh = 16; sh >= 1; sh >>= 1) {
    const unsigned low = w & ((1u << sh) - 1u);
    const int c = __popc(low);
    const bool up = r >= c;
    r = up ? r - c : r;
    w = up ? (w >> sh) : low;
    base += up ? sh : 0;
  }
  return base;
}

// Warp argmin of (key, j) over keys[0..d) skipping j == excl: smallest key,
// then smaller j.  Every lane returns the winning j.
__device__ __forceinline__ int warp_argmin_row(const unsigned long long* keys, int d, int excl) {
  const int lane = threadIdx.x & 31;
  unsigned long long bk = ~0ull;
  unsigned bj = 0xffffffffu;
  for (int j = lane; j < d; j += 32) {
    const unsigned long long kj = keys[j];
    if (j != excl && kj < bk) {  // ascending j per lane: strict < keeps the smaller j
      bk = kj;
      bj = (unsigned)j;
    }
  }
  const unsigned full = 0xffffffffu;
  const unsigned hi = (unsigned)(bk >> 32), lo = (unsigned)bk;
  const unsigned mhi = __reduce_min_sync(full, hi);
  const unsigned mlo = __reduce_min_sync(full, hi == mhi ? lo : 0xffffffffu);
  return (int)__reduce_min_sync(full, (hi == mhi && lo == mlo) ? bj : 0xffffffffu);
}

// ------------------------------------------------------------ FindDimensions
// Y_i, sigma_i, Z_ij (Alg 4 l.6-13, readings R2, R3) and the
// selection of Alg 4 l.15-16 (reading R10): per medoid the two smallest by
// (Z, j), then the k*l - 2k smallest of the rest by (Z, i, j).  The order is
// taken on order-preserving 64-bit keys of Z (T.dev); the rest is selected by
// rank scan (k*d <= 512), else a block-wide radix select (8 passes of
// 8-bit histograms).  Writes D as a mask (T.dm), |D_i|
// (S->nD) and, in global memory, the mask and the ascending dimension lists
// used by the passes.  Needs X in T.X; clobbers T.Z and T.dev.
__device__ void zscore_select_s(const RunParams& p, TailMem& T, int tq = -1) {
  __shared__ double Ys[KMAX], Ss[KMAX];
  const int tid = threadIdx.x, bd = blockDim.x, lane = tid & 31, w = tid >> 5, nw = bd >> 5;
  const int k = p.k, d = p.d, l = p.l, kd = k * d;
  const double* X = T.X;
  double* Z = T.Z;
  unsigned char* dm = T.dm;
  unsigned long long* key = (unsigned long long*)T.dev;
  if (tid < k) {  // oracle order: j ascending, four loads in flight
    const double* x = X + tid * d;
    double Y = 0.0, s2 = 0.0;
    int j = 0;
    for (; j + 4 <= d; j += 4) {
      const double a = x[j], b = x[j + 1], c = x[j + 2], e = x[j + 3];
      Y = dadd(dadd(dadd(dadd(Y, a), b), c), e);
    }
    for (; j < d; ++j) Y = dadd(Y, x[j]);
    Y = ddiv(Y, (double)d);
    for (j = 0; j + 4 <= d; j += 4) {
      const double a = dsub(x[j], Y), b = dsub(x[j + 1], Y), c = dsub(x[j + 2], Y),
                   e = dsub(x[j + 3], Y);
      s2 = dadd(dadd(dadd(dadd(s2, dmul(a, a)), dmul(b, b)), dmul(c, c)), dmul(e, e));
    }
    for (; j < d; ++j) {
      const double u = dsub(x[j], Y);
      s2 = dadd(s2, dmul(u, u));
    }
    Ys[tid] = Y;
    Ss[tid] = __dsqrt_rn(ddiv(s2, (double)(d - 1)));
  }
  __syncthreads();
  TST(T, tq < 0 ? 2 : tq);
  for (int c = tid; c < kd; c += bd) {
    const int i = c / d;
    const double sg = Ss[i];
    const double z = (sg == 0.0) ? 0.0 : ddiv(dsub(X[c], Ys[i]), sg);
    Z[c] = z;
    key[c] = sortable_key(z);
    dm[c] = 0;
  }
  __syncthreads();
  TST(T, tq < 0 ? 3 : tq);
  const int R = k * l - 2 * k;
  if (d <= 64) {
    // two smallest per row by (key, j), one thread per row: a sequential
    // scan of d shared keys beats two warp reductions per row here
    // two smallest per row by (key, j): every cell counts the cells of its
    // row that precede it (d <= 64 compares, all cells in parallel)
    bool top2 = false;
    const int c = tid;
    if (c < kd) {
      const int i = c / d, j = c - i * d;
      const unsigned long long* kr = key + i * d;
      const unsigned long long kc = kr[j];
      int r = 0;
      for (int o = 0; o < d; ++o) {
        const unsigned long long v = kr[o];
        r += (v < kc) | ((v == kc) & (o < j));
      }
      top2 = r < 2;
      if (top2) dm[c] = 1;
    }
    for (int e = tid + bd; e < kd; e += bd) {  // k d > blockDim: the rest
      const int i = e / d, j = e - i * d;
      const unsigned long long* kr = key + i * d;
      const unsigned long long kc = kr[j];
      int r = 0;
      for (int o = 0; o < d; ++o) {
        const unsigned long long v = kr[o];
        r += (v < kc) | ((v == kc) & (o < j));
      }
      if (r < 2) dm[e] = 1;
    }
    __syncthreads();  // every row's ranks were taken on the original keys
    if (R > 0)        // taken cells never rank before a free one
      for (int e = tid; e < kd; e += bd)
        if (dm[e]) key[e] = ~0ull;
  } else {
    for (int i = w; i < k; i += nw) {  // two smallest per row, ties -> smaller j
      const int j1 = warp_argmin_row(key + i * d, d, -1);
      const int j2 = warp_argmin_row(key + i * d, d, j1);
      if (lane == 0) {
        dm[i * d + j1] = 1;
        dm[i * d + j2] = 1;
      }
    }
    __syncthreads();
    if (R > 0 && kd <= 512)
      for (int c = tid; c < kd; c += bd)
        if (dm[c]) key[c] = ~0ull;  // taken: never before a free cell
  }
  __syncthreads();
  TST(T, tq < 0 ? 4 : tq);
  if (R > 0 && kd <= 512) {
    // rank of every free cell among the free cells by (key, i, j) = (key,
    // cell index): O(kd^2 / threads) broadcast reads, two keys per load
    const ulonglong2* key2 = reinterpret_cast<const ulonglong2*>(key);
    const int kd2 = kd >> 1;
    for (int c = tid; c < kd; c += bd) {
      const unsigned long long kc = key[c];
      if (kc == ~0ull) continue;
      int r0 = 0, r1 = 0;
#pragma unroll 4
      for (int o2 = 0; o2 < kd2; ++o2) {
        const ulonglong2 v = key2[o2];
        const int o = 2 * o2;
        r0 += (v.x < kc) | ((v.x == kc) & (o < c));
        r1 += (v.y < kc) | ((v.y == kc) & (o + 1 < c));
      }
      if (kd & 1) {
        const unsigned long long v = key[kd - 1];
        r0 += (v < kc) | ((v == kc) & (kd - 1 < c));
      }
      if (r0 + r1 < R) dm[c] = 1;
    }
  } else if (R > 0) {
    // k d > 512: most-significant-digit radix select (8-bit digits) of the R
    // smallest free keys; as soon as the bucket that holds the R-th key has
    // at most bd members it is finished by an exact (key, cell) rank among
    // its members.  Cells below the bucket's prefix are selected.
    __shared__ unsigned int hist[256];
    __shared__ unsigned long long prefix_s;
    __shared__ int need_s, bsize_s, bcnt_s;
    int* blist = reinterpret_cast<int*>(T.Z);  // [<= bd] bucket members (Z is dead here)
    if (tid == 0) {
      prefix_s = 0ull;
      need_s = R;
      bsize_s = kd;
    }
    unsigned long long hmask = 0ull;
    for (int shift = 56; shift >= 0; shift -= 8) {
      for (int bb = tid; bb < 256; bb += bd) hist[bb] = 0u;
      __syncthreads();
      if (bsize_s <= bd) break;  // small bucket: exact rank below
      const unsigned long long pre = prefix_s;
      for (int c = tid; c < kd; c += bd) {
        if (dm[c]) continue;
        const unsigned long long kc = key[c];
        if ((kc & hmask) == pre) atomicAdd(&hist[(kc >> shift) & 255ull], 1u);
      }
      __syncthreads();
      if (tid < 32) {  // warp scan over 256 bins, 8 per lane
        unsigned loc[8], tot = 0;
#pragma unroll
        for (int q = 0; q < 8; ++q) {
          loc[q] = hist[tid * 8 + q];
          tot += loc[q];
        }
        unsigned x = tot;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const unsigned y = __shfl_up_sync(0xffffffffu, x, o);
          if (tid >= o) x += y;
        }
        const unsigned before = x - tot;
        const int need = need_s;
        __syncwarp();  // every lane has read need_s before one lane rewrites it
        const bool here = (int)before < need && need <= (int)x;
        const unsigned who = __ballot_sync(0xffffffffu, here);
        if (here && tid == __ffs(who) - 1) {
          unsigned cum = before;
          int q = 0;
          for (; q < 8; ++q) {
            if ((int)(cum + loc[q]) >= need) break;
            cum += loc[q];
          }
          need_s = need - (int)cum;
          bsize_s = (int)loc[q];
          prefix_s = pre | ((unsigned long long)(tid * 8 + q) << shift);
        }
      }
      hmask |= 255ull << shift;
      __syncthreads();
    }
    // bucket = free cells whose decided digits equal the prefix; below it: selected
    const unsigned long long pre = prefix_s;
    if (tid == 0) bcnt_s = 0;
    __syncthreads();
    for (int c = tid; c < kd; c += bd) {
      if (dm[c]) continue;
      const unsigned long long kp = key[c] & hmask;
      if (kp < pre) {
        dm[c] = 2;  // selected (marked 2 until the bucket is ranked: still "free" there)
      } else if (kp == pre) {
        blist[atomicAdd(&bcnt_s, 1)] = c;
      }
    }
    __syncthreads();
    const int nb = bcnt_s, need = need_s;
    for (int t = tid; t < nb; t += bd) {  // exact rank inside the bucket by (key, cell)
      const int c = blist[t];
      const unsigned long long kc = key[c];
      int r = 0;
      for (int o = 0; o < nb; ++o) {
        const int co = blist[o];
        const unsigned long long ko = key[co];
        r += (ko < kc) | ((ko == kc) & (co < c));
      }
      if (r < need) dm[c] = 2;
    }
    __syncthreads();
    for (int c = tid; c < kd; c += bd)
      if (dm[c] == 2) dm[c] = 1;
  }
  __syncthreads();
  TST(T, tq < 0 ? 6 : tq);
  for (int i = w; i < k; i += nw) {  // |D_i| and the ascending lists, one warp per row
    int base = 0;
    for (int j0 = 0; j0 < d; j0 += 32) {
      const int j = j0 + lane;
      const bool on = j < d && dm[i * d + j];
      const unsigned b = __ballot_sync(0xffffffffu, on);
      if (on) p.dlist[i * d + base + __popc(b & ((1u << lane) - 1u))] = j;
      base += __popc(b);
    }
    if (lane == 0) T.S->nD[i] = base;
  }
  for (int c = tid; c < kd; c += bd) p.dmask[c] = dm[c];
  __syncthreads();
  TST(T, tq < 0 ? 7 : tq);
}

// ------------------------------------------------------------ iteration prologue
// Medoid rows of MCur (fp64), delta_i (Alg 3 l.4-7, reading R6), and the
// active slots of GPU-FAST-PROCLUS: new medoids get their Dist row computed,
// cached ones with a changed radius get the band of Theorem 3.1.  With
// T.mrow the rows of M and the DistFound / delta' tables are read from the
// shared-memory copies the cost tail loaded up front.
__device__ void prepare_s(const RunParams& p, TailMem& T) {
  DevState* S = T.S;
  const int k = p.k, d = p.d, tid = threadIdx.x, bd = blockDim.x;
  const bool cached = T.mrow != nullptr;
  for (int e = tid; e < k * d; e += bd) {
    const int i = e / d, j = e - i * d;
    const long long r = (long long)S->mcur[i] * d + j;
    T.med[e] = (double)(cached ? T.mrow[r] : p.mrows[r]);
  }
  for (int i = tid; i < k; i += bd) {
    // cache row of slot i: the M position (FAST), the slot if it still holds
    // the same medoid as in the previous iteration (FAST*), none (plain)
    const int mp = S->mcur[i];
    const int key = p.variant == 2 ? i : mp;
    const bool valid = p.variant == 0 || (p.variant == 2 && S->cown[i] == mp);
    T.fnd[i] = valid ? (double)(cached ? T.fall[key] : p.found[key]) : 0.0;
    T.fnd[KMAX + i] = valid ? (double)(cached ? T.uall[key] : p.used[key]) : 0.0;
    T.fnd[2 * KMAX + i] = valid ? (cached ? T.pall[key] : p.dprev[key]) : 0.0;
  }
  __syncthreads();
  TST(T, 15);
  for (int e = tid; e < k * k; e += bd) {  // one thread per ordered pair (i, j)
    const int i = e / k, j = e - i * k;
    T.dd[e] = (i == j) ? CUDART_INF : full_dist(T.med + i * d, 1, T.med + j * d, d, p.metric);
  }
  __syncthreads();
  if (tid < k) {
    double m = CUDART_INF;
    for (int j = 0; j < k; ++j) {
      const double t = T.dd[tid * k + j];
      if (t < m) m = t;
    }
    S->delta[tid] = m;
  }
  __syncthreads();
  TST(T, 16);
  if (tid < 32) {  // active slots in slot order, one lane per slot
    const int i = tid;
    ActSlot a;
    bool on = false;
    if (i < k) {
      const double dl = S->delta[i];
      const double dp = T.fnd[2 * KMAX + i];
      a.slot = i;
      a.mpos = S->mcur[i];
      a.key = p.variant == 2 ? i : a.mpos;
      a.compute = T.fnd[i] != 0.0 ? 0 : 1;
      a.lam = 1;
      on = true;
      if (T.fnd[KMAX + i] == 0.0) {
        a.lo = -CUDART_INF;
        a.hi = dl;
      } else if (dl > dp) {
        a.lo = dp;
        a.hi = dl;
      } else if (dl < dp) {
        a.lo = dl;
        a.hi = dp;
        a.lam = -1;
      } else {
        on = false;  // delta unchanged: Delta L_i is empty (eq 3)
      }
    }
    const unsigned b = __ballot_sync(0xffffffffu, on);
    if (on) S->act[__popc(b & ((1u << i) - 1u))] = a;
    if (i == 0) S->n_act = __popc(b);
  }
  __syncthreads();
  TST(T, 17);
}

__global__ void __launch_bounds__(1024, 1) k_prepare(RunParams p) {
  extern __shared__ __align__(16) unsigned char smraw[];
  TailMem T = tail_mem(p, smraw);
  T.mrow = nullptr;  // first iteration: read M and the tables from global memory
  TST_START();
  state_load(p, T.S);
  if (*p.badflag) {  // the last (asynchronous) load found a non-finite value
    if (threadIdx.x == 0) {
      T.S->err = ERR_NONFINITE;
      T.S->done = 1;
      if (p.use_cond) cudaGraphSetConditional((cudaGraphConditionalHandle)p.cond, 0u);
    }
    state_store(p, T.S);
    return;
  }
  prepare_s(p, T);
  state_store(p, T.S);
}

void launch_prepare(const RunParams& p, cudaStream_t s) {
  k_prepare<<<1, 1024, p.tail_smem, s>>>(p);
}

// ------------------------------------------------------------ per-pass tails
// Locality tail: H and |L| updates of Theorem 3.2 / eq 6 and P:203 (in fixed
// point, so the incremental H is exact integer arithmetic), DistFound /
// delta' bookkeeping, X = H / |L| and FindDimensions.  Round trip 1:
// the state; round trip 2: band sums and counts of every slot (unused ones
// are zero), the H rows and |L| of MCur, and 2^-e_j.
__device__ void tail_locality(const RunParams& p, TailMem& T) {
  DevState* S = T.S;
  const int d = p.d, k = p.k, kd = k * d, tid = threadIdx.x, bd = blockDim.x;
  __shared__ long long cnt_s[KMAX], nL_s[KMAX];
  long long* Hs = (long long*)T.dev;  // [k][d] H rows of MCur by slot
  long long* va = (long long*)T.Z;    // [na][d] band sums by active slot
  state_load(p, S);
  TST(T, 5);
  const int na = S->n_act;
  for (int c = tid; c < kd; c += bd) {
    const int i = c / d, j = c - i * d;
    const int key = p.variant == 2 ? i : S->mcur[i];
    const long long h = __ldcg(p.Hq + (long long)key * d + j);
    const long long v = c < na * d ? take_acc(p, c) : 0ll;
    Hs[c] = h;
    va[c] = v;
  }
  if (tid < k) {
    const long long nl = __ldcg(p.nL + (p.variant == 2 ? tid : S->mcur[tid]));
    const long long v = tid < na ? take_cnt(p, tid) : 0ll;
    nL_s[tid] = nl;
    cnt_s[tid] = v;
  }
  TST(T, 8);
  for (int j = tid; j < d; j += bd) T.isc[j] = p.iscale[j];
  if (tid == 0 && na > 0)  // byte model: data once + one Dist row per slot
    S->bytes_loc += 4.0 * (double)p.n * (double)(d + (p.variant == 1 ? 0 : na));
  __syncthreads();
  TST(T, 0);
  for (int c = tid; c < na * d; c += bd) {
    const int a = c / d, j = c - a * d;
    const ActSlot& A = S->act[a];
    const int e = A.slot * d + j;
    // first use of the cache row (lo = -inf): H = the sum over L_i itself
    const long long h =
        A.lo == -CUDART_INF ? va[c] : Hs[e] + (A.lam > 0 ? va[c] : -va[c]);
    Hs[e] = h;
    p.Hq[(long long)A.key * d + j] = h;
  }
  if (tid < na) {
    const ActSlot& A = S->act[tid];
    const long long nl = A.lo == -CUDART_INF
                             ? cnt_s[tid]
                             : nL_s[A.slot] + (A.lam > 0 ? cnt_s[tid] : -cnt_s[tid]);
    nL_s[A.slot] = nl;
    p.nL[A.key] = nl;
    p.dprev[A.key] = S->delta[A.slot];
    p.used[A.key] = 1;
    p.found[A.key] = p.variant == 1 ? 0 : 1;
    if (p.variant == 2) S->cown[A.slot] = A.mpos;
  }
  __syncthreads();
  for (int c = tid; c < kd; c += bd) {
    const int i = c / d, j = c - i * d;
    T.X[c] = ddiv(dmul((double)Hs[c], T.isc[j]), (double)nL_s[i]);
  }
  __syncthreads();
  TST(T, 1);
  zscore_select_s(p, T);
  const int it = S->iterations;
  if (p.tr.cap > 0 && it < p.tr.cap) {
    for (int c = tid; c < kd; c += bd) {
      if (p.tr.X) p.tr.X[(long long)it * kd + c] = T.X[c];
      if (p.tr.dims) p.tr.dims[(long long)it * kd + c] = T.dm[c];
    }
    if (tid < k) {
      if (p.tr.mcur) p.tr.mcur[it * k + tid] = S->mcur[tid];
      if (p.tr.delta) p.tr.delta[it * k + tid] = S->delta[tid];
      if (p.tr.nL) p.tr.nL[it * k + tid] = nL_s[tid];
    }
  }
}

// Assign tail: |C_i| and the centroid mu_ij = sum / |C_i| on j in D_i.
// One round trip: state, sums, counts, dimension lists and 2^-e_j together.
__device__ void tail_assign(const RunParams& p, TailMem& T) {
  DevState* S = T.S;
  const int d = p.d, k = p.k, kd = k * d, tid = threadIdx.x, bd = blockDim.x;
  __shared__ long long sz_s[KMAX];
  long long* raw = (long long*)T.Z;
  StateRegs sr;
  state_issue(p, sr);
  for (int c = tid; c < kd; c += bd) {
    const int dl = p.dlist[c];
    const long long v = take_acc(p, c);
    T.dl[c] = dl;
    raw[c] = v;
  }
  if (tid < k) sz_s[tid] = take_cnt(p, tid);
  for (int j = tid; j < d; j += bd) T.isc[j] = p.iscale[j];
  state_commit(p, sr, S);
  __syncthreads();
  TST(T, 20);
  if (tid < k) S->sizes[tid] = sz_s[tid];
  for (int c = tid; c < kd; c += bd) {
    const int i = c / d, t = c - i * d;
    const long long sz = sz_s[i];
    double m = 0.0;
    if (t < S->nD[i] && sz > 0) m = ddiv(dmul((double)raw[c], T.isc[T.dl[c]]), (double)sz);
    p.mu[c] = m;
  }
  TST(T, 21);
}

// Cost tail: eq 1-2 with the |Data| denominator (eq 8, reading R4), then
// Alg 1 l.10-14: keep the best, ComputeBadMedoids (reading R11),
// replace bad medoids from M \ MBest (reading R12), stop after itrPat
// iterations without improvement, and prepare the next iteration.  One round
// trip brings the state, the deviation sums, the dimension lists, 2^-e_j and
// (when cached) the rows of M with their DistFound / delta' entries, so the
// prologue of the next iteration needs no further global loads.
__device__ int cost_qexp(const double* sc, int sgn, const int* dl, const int* nD, int k, int d);
__device__ void tail_cost(const RunParams& p, TailMem& T) {
  DevState* S = T.S;
  const int k = p.k, d = p.d, kd = k * d, nM = p.nM;
  const int tid = threadIdx.x, bd = blockDim.x, lane = tid & 31;
  __shared__ double cw_s[KMAX];
  long long* raw = (long long*)T.Z;
  StateRegs sr;
  state_issue(p, sr);
  for (int c = tid; c < kd; c += bd) {
    const int dl = p.dlist[c];
    const long long v = (!p.cost1 || c < k) ? take_acc(p, c) : 0ll;
    T.dl[c] = dl;
    raw[c] = v;
  }
  for (int j = tid; j < d; j += bd) T.isc[j] = p.iscale[j];
  if (T.mrow) {
    // every load of a thread is issued before its first shared-memory store
    // (the compiler cannot reorder them across a possibly aliasing store)
    constexpr int MR = 8;
    const int nmd = nM * d;
    float mv[MR];
#pragma unroll
    for (int q = 0; q < MR; ++q) {
      const int e = tid + q * bd;
      mv[q] = e < nmd ? __ldcg(p.mrows + e) : 0.f;
    }
    unsigned char fv = 0, uv = 0;
    double pv = 0.0;
    if (tid < nM) {
      fv = __ldcg(p.found + tid);
      uv = __ldcg(p.used + tid);
      pv = __ldcg(p.dprev + tid);
    }
#pragma unroll
    for (int q = 0; q < MR; ++q) {
      const int e = tid + q * bd;
      if (e < nmd) T.mrow[e] = mv[q];
    }
    for (int e = tid + MR * bd; e < nmd; e += bd) T.mrow[e] = p.mrows[e];
    if (tid < nM) {
      T.fall[tid] = fv;
      T.uall[tid] = uv;
      T.pall[tid] = pv;
    }
    for (int m = tid + bd; m < nM; m += bd) {
      T.fall[m] = p.found[m];
      T.uall[m] = p.used[m];
      T.pall[m] = p.dprev[m];
    }
  }
  state_commit(p, sr, S);
  __syncthreads();
  TST(T, 10);
  if (p.cost1) {  // |C_i| w_i = (sum_t dev_it) / |D_i| (eq 1 with eq 2's weight)
    const int ec = cost_qexp(T.isc, -1, T.dl, S->nD, k, d);
    if (tid < k) {
      const int i = tid;
      const long long c = S->sizes[i];
      cw_s[i] = c != 0 ? ddiv(scalbn((double)raw[i], -ec), (double)S->nD[i]) : 0.0;
    }
  } else {
    for (int c = tid; c < kd; c += bd) {  // dev_it and the per-term quotients of eq 1
      const int i = c / d, t = c - i * d;
      const long long ci = S->sizes[i];
      const bool on = t < S->nD[i];
      const double dv = on ? dmul((double)raw[c], T.isc[T.dl[c]]) : 0.0;
      T.dev[c] = dv;
      T.Z[c] = (on && ci != 0) ? ddiv(dv, (double)ci) : 0.0;
    }
    __syncthreads();
    if (tid < k) {  // |C_i| * w_i of eq 1, terms added in t order
      const int i = tid;
      const long long c = S->sizes[i];
      double cw = 0.0;
      if (c != 0) {
        double wv = 0.0;
        const int nd = S->nD[i];
        for (int t = 0; t < nd; ++t) wv = dadd(wv, T.Z[i * d + t]);
        wv = ddiv(wv, (double)nd);
        cw = dmul((double)c, wv);
      }
      cw_s[i] = cw;
    }
  }
  __syncthreads();
  TST(T, 11);
  if (tid < 32) {  // control, one warp
    TSTW_DECL();
    const unsigned full = 0xffffffffu;
    double cost = 0.0;
    if (lane == 0) {
      for (int i = 0; i < k; ++i)  // eq 2 / eq 8, i ascending; empty clusters add 0
        if (S->sizes[i] != 0) cost = dadd(cost, cw_s[i]);
      cost = ddiv(cost, (double)p.n_total);
    }
    cost = __shfl_sync(full, cost, 0);
    const int it = S->iterations;
    const int improved = cost < S->cost_best;
    __syncwarp();
    if (improved && lane < k) {
      S->mbest[lane] = S->mcur[lane];
      S->sizes_best[lane] = S->sizes[lane];
    }
    if (lane == 0) {
      S->cost = cost;
      S->itr = improved ? 0 : S->itr + 1;
      S->iterations = it + 1;
      S->improved = improved;
      if (improved) {
        S->cost_best = cost;
        S->best_buf = S->cur_buf;
        S->cur_buf ^= 1;
      }
    }
    __syncwarp();
    TSTW(T, 12);
    // bad medoids (R11): |C_i| < n/k * minDev in CBest, else the smallest
    const double thr = dmul(ddiv((double)p.n_total, (double)k), p.minDev);
    const long long sb = lane < k ? S->sizes_best[lane] : 0ll;
    unsigned bad = __ballot_sync(full, lane < k && (double)sb < thr);
    if (!bad) {  // first smallest |C_i| (sizes are < 2^63, non-negative)
      const unsigned long long u = lane < k ? (unsigned long long)sb : ~0ull;
      const unsigned hi = (unsigned)(u >> 32), lo = (unsigned)u;
      const unsigned mhi = __reduce_min_sync(full, hi);
      const unsigned mlo = __reduce_min_sync(full, hi == mhi ? lo : 0xffffffffu);
      const unsigned at = __reduce_min_sync(full, (hi == mhi && lo == mlo) ? (unsigned)lane : 32u);
      bad = 1u << at;
    }
    if (lane == 0 && p.tr.cap > 0 && it < p.tr.cap) {
      if (p.tr.cost) p.tr.cost[it] = cost;
      if (p.tr.improved) p.tr.improved[it] = (unsigned char)improved;
      for (int i = 0; i < k; ++i) {
        if (p.tr.sizes) p.tr.sizes[it * k + i] = S->sizes[i];
        if (p.tr.bad) p.tr.bad[it * k + i] = (bad >> i) & 1u;
      }
    }
    if (lane < k) S->mcur[lane] = S->mbest[lane];
    __syncwarp();
    TSTW(T, 13);
    // pool = ascending positions of M not in MBest, as a bitmap in shared
    // memory (word w holds positions 32 w .. 32 w + 31); the r-th remaining
    // pool entry is found by a warp prefix count of the words' populations
    // and a find-n-th-set-bit, and removed by clearing its bit -- the same
    // draws as erasing it from the ascending list (reading R12)
    unsigned* avail = reinterpret_cast<unsigned*>(T.pool);
    const int nwrd = (nM + 31) >> 5;
    for (int w0 = lane; w0 < nwrd; w0 += 32) {
      const int rem = nM - 32 * w0;
      avail[w0] = rem >= 32 ? 0xffffffffu : ((1u << rem) - 1u);
    }
    __syncwarp();
    if (lane < k) atomicAnd(&avail[S->mbest[lane] >> 5], ~(1u << (S->mbest[lane] & 31)));
    __syncwarp();
    int np = nM - k;  // MBest holds k distinct positions of M
    TSTW(T, 18);
    // replacement draws (stream IT): the r-th remaining pool entry, in order;
    // every lane runs the same generator
    unsigned long long rng = S->rng;
    __syncwarp();  // every lane has read S->rng before lane 0 stores it back
    for (int i = 0; i < k; ++i) {
      if (!((bad >> i) & 1u) || np == 0) continue;
      int r = (int)sm64_uniform(&rng, (unsigned long long)np);
      int pos = -1;
      for (int w0 = 0; w0 < nwrd && pos < 0; w0 += 32) {
        const unsigned wv = w0 + lane < nwrd ? avail[w0 + lane] : 0u;
        const int c = __popc(wv);
        int x = c;  // inclusive prefix count over the lanes of this group
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const int y = __shfl_up_sync(full, x, o);
          if (lane >= o) x += y;
        }
        const unsigned hit = __ballot_sync(full, r < x && r >= x - c);
        if (hit) {
          const int src = __ffs(hit) - 1;
          const int before = __shfl_sync(full, x - c, src);
          const unsigned sw = __shfl_sync(full, wv, src);
          const int bit = nth_set_bit(sw, r - before);
          pos = 32 * (w0 + src) + bit;
        } else {
          r -= __shfl_sync(full, x, 31);
        }
      }
      if (lane == 0) {
        S->mcur[i] = pos;
        avail[pos >> 5] &= ~(1u << (pos & 31));
      }
      __syncwarp();
      --np;
    }
    TSTW(T, 19);
    if (lane == 0) {
      S->rng = rng;
      S->done = (S->itr >= p.itrPat || S->iterations >= p.max_iter) ? 1 : 0;
      if (p.use_cond)
        cudaGraphSetConditional((cudaGraphConditionalHandle)p.cond, S->done ? 0u : 1u);
    }
    TSTW(T, 22);
  }
  __syncthreads();
  TST(T, 14);
  if (!S->done) prepare_s(p, T);
}

// Refinement tail (Alg 1 l.16-17): X over CBest (empty cluster -> 0 row,
// reading R15), FindDimensions -> D*, and the outlier radii
// Delta_i = min_{j != i} seg_{D*_i}(m_i, m_j) (reading R5).
__device__ void tail_refine(const RunParams& p, TailMem& T) {
  DevState* S = T.S;
  const int k = p.k, d = p.d, kd = k * d, tid = threadIdx.x, bd = blockDim.x;
  __shared__ long long sz_s[KMAX];
  long long* raw = (long long*)T.Z;
  StateRegs sr;
  state_issue(p, sr);
  for (int c = tid; c < kd; c += bd) raw[c] = take_acc(p, c);
  if (tid < k) sz_s[tid] = take_cnt(p, tid);
  for (int j = tid; j < d; j += bd) T.isc[j] = p.iscale[j];
  state_commit(p, sr, S);
  __syncthreads();
  for (int e = tid; e < kd; e += bd) {
    const int i = e / d, j = e - i * d;
    T.med[e] = (double)p.mrows[(long long)S->mbest[i] * d + j];
    const long long sz = sz_s[i];
    T.X[e] = sz > 0 ? ddiv(dmul((double)raw[e], T.isc[j]), (double)sz) : 0.0;
  }
  __syncthreads();
  zscore_select_s(p, T);
  if (tid < k) {
    const int i = tid;
    double m = CUDART_INF;
    for (int j = 0; j < k; ++j) {
      if (j == i) continue;
      double s = 0.0;
      int nd = 0;
      for (int t = 0; t < d; ++t) {
        if (!T.dm[i * d + t]) continue;
        s = dadd(s, fabs(dsub(T.med[i * d + t], T.med[j * d + t])));
        ++nd;
      }
      const double q = ddiv(s, (double)nd);
      if (q < m) m = q;
    }
    p.Delta[i] = m;
  }
}

// Run a tail (each tail loads the state itself), store the state back.  The
// tickets are stored as 0: the copy may predate last_block()'s reset.
#define RUN_TAIL(FN, KIND)                                          \
  do {                                                              \
    const unsigned long long t0_ = gtimer();                        \
    TailMem T_ = tail_mem(p, smraw + p.lay[LAYK].tail);             \
    TST_START();                                                    \
    FN(p, T_);                                                      \
    __syncthreads();                                                \
    if (threadIdx.x < 4) T_.S->ticket[threadIdx.x] = 0u;            \
    if (threadIdx.x == 0) T_.S->tail_ns[KIND] += gtimer() - t0_;    \
    state_store(p, T_.S);                                           \
  } while (0)

// ============================================================ pass kernels
// Block = NW consumer warps + 1 producer warp.  Consumer warp w owns the
// sub-chunk of 32*PPT points starting at q0 = w*32*PPT of every chunk.
// Shared-memory arrays live at host-computed offsets (p.lay[kind]).
#define SMP(T, field) reinterpret_cast<T*>(smraw + L.field)

__device__ __forceinline__ long long chunks_of_block(const RunParams& p) {
  return (p.nchunks > blockIdx.x) ? (p.nchunks - blockIdx.x + gridDim.x - 1) / gridDim.x : 0;
}

__device__ __forceinline__ Pipe pipe_of(const SmemLayout& L, unsigned char* smraw, int rows) {
  Pipe R;
  R.full = SMP(unsigned long long, full);
  R.empty = SMP(unsigned long long, empty);
  R.buf = SMP(float, buf);
  R.lab = L.lab >= 0 ? SMP(unsigned char, lab) : nullptr;
  R.rows = rows;
  R.ldr = L.ldr > 0 ? L.ldr : L.P;
  R.full_a = smem_u32(R.full);
  R.empty_a = smem_u32(R.empty);
  return R;
}

// Cells (i, t < |D_i|) in cluster order: exclusive scan of |D_i| by warp 0,
// then a parallel fill.  dl_s[i*d+t] is the dimension, ctr_s[i*d+t] the
// centre (null: 0).  Returns the number of cells (after a block barrier).
__device__ int build_cells(Cell* cells, const int* nD_s, int k, int d, int* off_s,
                           const int* dl_s, const double* ctr_s) {
  if (threadIdx.x < 32) {
    const int v = (int)threadIdx.x < k ? nD_s[threadIdx.x] : 0;
    int x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int y = __shfl_up_sync(0xffffffffu, x, o);
      if ((int)threadIdx.x >= o) x += y;
    }
    if ((int)threadIdx.x < k) off_s[threadIdx.x] = x - v;
    if (threadIdx.x == 31) off_s[KMAX] = x;
  }
  __syncthreads();
  for (int e = threadIdx.x; e < k * d; e += blockDim.x) {
    const int i = e / d, t = e - i * d;
    if (t < nD_s[i]) cells[off_s[i] + t] = Cell{i, dl_s[e], e, ctr_s ? ctr_s[e] : 0.0};
  }
  __syncthreads();
  return off_s[KMAX];
}

// fp32 certified thresholds of one band (lo, hi]: a fp32 value f with
// |f - v| <= G v decides v <= T when f < T(1-G) (then "<=") or f > T(1+G)
// (then ">"); the bounds are rounded outwards to fp32 once per launch.
struct __align__(16) Thr {
  float in_hi, out_hi;  // f < in_hi: v <= hi;  f > out_hi: v > hi
  float in_lo, out_lo;  // f > out_lo: v > lo;  f < in_lo: v <= lo
};
__device__ __forceinline__ Thr make_thr(double lo, double hi, double G) {
  Thr t;
  const bool hok = hi >= 1e-30 && hi < 1e30;
  t.in_hi = hok ? __double2float_rd(hi * (1.0 - G)) : -1.0f;
  t.out_hi = hok ? __double2float_ru(hi * (1.0 + G)) : CUDART_INF_F;
  if (lo == -CUDART_INF) {
    t.out_lo = -1.0f;  // every f >= 0 is above
    t.in_lo = -2.0f;
  } else {
    const bool lok = lo >= 1e-30 && lo < 1e30;
    t.in_lo = lok ? __double2float_rd(lo * (1.0 - G)) : -1.0f;
    t.out_lo = lok ? __double2float_ru(lo * (1.0 + G)) : CUDART_INF_F;
  }
  return t;
}

// Fixed-point quantisation round(s * 2^e_j) of a band / cell sum.  With
// |s 2^e_j| < 2^51 (*p.qflag, set with the scales for every dimension) one
// fma with 1.5 * 2^52 rounds to the integer grid exactly as __double2ll_rn
// (the scale is a power of two, so s * 2^e_j itself is exact), on the fp64
// pipe instead of the 16/clk/SM conversion pipe.
__device__ __forceinline__ long long quant_sum(double s, double sc, int magic) {
  if (magic) {
    const double v = __fma_rn(s, sc, 6755399441055744.0);  // 1.5 * 2^52
    return __double_as_longlong(v) - 0x4338000000000000LL;
  }
  return __double2ll_rn(dmul(s, sc));
}

// --- k_locality<16> consumer (d <= 16).  Warp w owns the LOC16_PPT * 32
// points of columns [w * 32 PPT, (w + 1) * 32 PPT) of every chunk, lane l
// the points l, l + 32, ...; the active slots are handled one at a time (the
// loop body is not unrolled over slots: instruction-cache footprint), so the
// per-slot constants are loaded once per 32 PPT points.  Lane = point for the
// band decision: the certified fp32 distance (computed for a slot whose Dist
// row is new, else read from the cached row in the ring), a ballot per point
// group, and the member's rank, which compacts the members into a per-warp
// byte list in ascending column order (no bit walks).  Lane = (half h,
// dimension j) for the band sum of eq 6: half h adds the exact fp64 terms
// |x_j - m_aj| of the members at ranks h, h + 2, ... (two interleaved
// accumulators), the halves are added, and the sum is quantised per (slot,
// dimension, 32 PPT-point group) into the warp's accumulator.  Groups are
// aligned to 32 PPT points, so the totals do not depend on the grid or on
// 1024-aligned shard boundaries.
constexpr int LOC16_PPT = 1;  // 2 measured slower (fewer warps per SM)

// The exact fp64 band decision of a point whose fp32 distance is within the
// error bound (rare): out of line, so that its registers do not count
// against the consumer loop.
__device__ __noinline__ bool exact_band(const float* __restrict__ x, int LD,
                                        const float* __restrict__ m, int d, int metric,
                                        double lo, double hi) {
  const double dv = full_dist(x, LD, m, d, metric);
  return (dv > lo) && (dv <= hi);
}

// Shared memory is addressed through 32-bit offsets from the dynamic
// shared-memory base (generic 64-bit pointers cost an IMAD + LEA per access).
// explicit 32-bit shared-window addressing from a base computed once per
// kernel (the compiler otherwise re-derives the window base per access)
__device__ __forceinline__ float lds_f32(unsigned a) {
  float v;
  asm volatile("ld.shared.f32 %0, [%1];" : "=f"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ unsigned lds_u8(unsigned a) {
  unsigned v;
  asm volatile("ld.shared.u8 %0, [%1];" : "=r"(v) : "r"(a));
  return v;
}
#define SMF(off) lds_f32(sbase + 4u * (unsigned)(off))
#define SMB(off) lds_u8(sbase + (unsigned)(off))

template <int METRIC>
__device__ __forceinline__ float loc16_dist(const float (&x)[16], const float* __restrict__ m) {
  // padded coordinates (j >= d) are 0 in m and in x
  float s0 = 0.f, s1 = 0.f;
#pragma unroll
  for (int j4 = 0; j4 < 4; ++j4) {
    const float4 v = reinterpret_cast<const float4*>(m)[j4];
    const float t0 = x[4 * j4] - v.x, t1 = x[4 * j4 + 1] - v.y;
    const float t2 = x[4 * j4 + 2] - v.z, t3 = x[4 * j4 + 3] - v.w;
    if (METRIC == 1) {
      s0 = s0 + fabsf(t0);
      s1 = s1 + fabsf(t1);
      s0 = s0 + fabsf(t2);
      s1 = s1 + fabsf(t3);
    } else {
      s0 = __fmaf_rn(t0, t0, s0);
      s1 = __fmaf_rn(t1, t1, s1);
      s0 = __fmaf_rn(t2, t2, s0);
      s1 = __fmaf_rn(t3, t3, s1);
    }
  }
  return METRIC == 1 ? s0 + s1 : sqrtf(s0 + s1);
}

// buf_f: float offset of the ring; lst_b: byte offset of this warp's list
template <int METRIC>
__device__ __forceinline__ void loc16_consume(const RunParams& p, const Pipe& R, int buf_f,
                                              long long nmy, int na, int ncomp,
                                              const float* __restrict__ med_s,
                                              const double* __restrict__ medd_s,
                                              const int* __restrict__ row_s,
                                              const Thr* __restrict__ thr_s,
                                              const ActSlot* __restrict__ act_s,
                                              const ExtraRows* __restrict__ ex, int lst_b,
                                              long long* __restrict__ acc,
                                              long long* __restrict__ cnt,
                                              const double* __restrict__ scale_s, long long& nfb) {
  extern __shared__ __align__(16) unsigned char smraw[];
  const unsigned sbase = smem_u32(smraw);
  constexpr int PPT = LOC16_PPT;
  static_assert(PPT == 1, "x[] holds the coordinates of one point per lane");
  const int lane = threadIdx.x & 31, c0 = (threadIdx.x >> 5) * 32 * PPT, d = p.d;
  const int LD = R.ldr, P = p.P, sstride = R.rows * LD;
  const int h = lane >> 4, j = lane & 15;
  const unsigned lt = (1u << lane) - 1u;
  const double sc = scale_s[j < d ? j : 0];
  const int magic = *p.qflag;
  const int variant = p.variant;
  const long long n = p.n;
  long long gp = (long long)blockIdx.x * P + c0 + lane;
  const long long gstep = (long long)gridDim.x * P;
  RingPos rp;
  for (long long i = 0; i < nmy; ++i, gp += gstep, rp.next(p.stages)) {
    const int stg = rp.stg;
    mbar_wait(R.full_a + 8u * stg, rp.ph);
    const int xs = buf_f + stg * sstride;  // stage base (floats)
    const int xq = xs + c0 + lane;         // lane's first point, row 0
    const int xr = xs + j * LD + c0;       // (h, j) view; j >= d: unused rows
    float x[16];
    if (ncomp > 0) {  // coordinates in registers when a Dist row is computed; rows >= d are 0
#pragma unroll
      for (int jj = 0; jj < 16; ++jj) x[jj] = SMF(xq + jj * LD);
    }
#ifdef LOC_NOP
    if (na > 0) { pipe_release(R, stg); continue; }  // timing experiment only
#endif
    for (int a = 0; a < na; ++a) {
      const int rs = row_s[a];
      const Thr t = thr_s[a];
      int m = 0;
#pragma unroll
      for (int u = 0; u < PPT; ++u) {
        const bool valid = gp + 32 * u < n;
        float f;
        if (rs < 0) {  // a new Dist row
          f = loc16_dist<METRIC>(x, med_s + a * 16);
          if (variant != 1 && valid) ex->drow[a][gp + 32 * u] = f;
        } else {
          f = SMF(xq + rs + 32 * u);
        }
        bool in = f < t.in_hi && f > t.out_lo;
        if (valid && !in && !(f > t.out_hi || f < t.in_lo)) {
          // within the fp32 error bound: the oracle's fp64 value decides
          in = exact_band(reinterpret_cast<const float*>(smraw) + xq + 32 * u, LD,
                          med_s + a * 16, d, METRIC, act_s[a].lo, act_s[a].hi);
          ++nfb;
        }
        in = in && valid;
        const unsigned bl = __ballot_sync(0xffffffffu, in);
        if (in) smraw[lst_b + m + __popc(bl & lt)] = (unsigned char)(32 * u + lane);
        m += __popc(bl);
      }
      if (m == 0) continue;
      if (lane == 0) cnt[a] += m;
      const double c = medd_s[a * 16 + j];
      __syncwarp();
      double s0 = 0.0, s1 = 0.0;
      int v = h;
#pragma unroll 1
      for (; v + 2 < m; v += 4) {
        const double t0 = fabs(dsub((double)SMF(xr + SMB(lst_b + v)), c));
        const double t1 = fabs(dsub((double)SMF(xr + SMB(lst_b + v + 2)), c));
        s0 = dadd(s0, t0);
        s1 = dadd(s1, t1);
      }
      if (v < m) s0 = dadd(s0, fabs(dsub((double)SMF(xr + SMB(lst_b + v)), c)));
      double s = dadd(s0, s1);
      s = dadd(s, __shfl_xor_sync(0xffffffffu, s, 16));
      if (h == 0 && j < d && s != 0.0) acc[a * d + j] += quant_sum(s, sc, magic);
      __syncwarp();  // the list is rewritten by the next slot
    }
    pipe_release(R, stg);
  }
}
#undef SMF
#undef SMB

// --- k_locality consumer for d > 16 (wide rows; C4: d = 100).  The LOCW_NW
// consumer warps share every chunk of P points instead of owning 32 points
// each (at long rows a chunk is short, P = 64, and per-warp point ownership
// left 2 consumer warps per block).  Phase A, items (slot a, point block pb
// of 32 points): lane = point; the certified fp32 distance (computed from
// the ring for a new Dist row, else read from the cached row), a ballot, and
// the member's rank compact the members of (a, pb) into a byte list of the
// ring stage.  Consumer barrier.  Phase B, items (slot a, dimension block jb
// of 32): lane = dimension j = 32 jb + lane; fp64 sum of the exact terms
// |x_j - m_aj| over the members of slot a in ascending point order (two
// interleaved accumulators), quantised per (slot, dimension, chunk) into the
// block's single accumulator copy: the item -> warp map is fixed within a
// launch, so every cell has one writer.  A chunk (P | 1024 points, aligned)
// is one quantisation group, so the totals do not depend on the grid or on
// 1024-aligned shard boundaries.
constexpr int LOCW_NW = 8;

template <int METRIC>
__device__ __forceinline__ void locw_consume(const RunParams& p, const Pipe& R, long long nmy,
                                             int na, const float* __restrict__ med_s, int MS,
                                             const int* __restrict__ row_s,
                                             const Thr* __restrict__ thr_s,
                                             const ActSlot* __restrict__ act_s,
                                             unsigned char* __restrict__ lst_s,
                                             int* __restrict__ lcnt_s,
                                             long long* __restrict__ acc,
                                             long long* __restrict__ cnt,
                                             const double* __restrict__ scale_s, long long& nfb) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, d = p.d, P = p.P, LD = R.ldr;
  const int npb = P >> 5, nb = (d + 31) >> 5;
  const int nA = na * npb, nB = na * nb;
  const int magic = *p.qflag, variant = p.variant;
  const unsigned lt = (1u << lane) - 1u;
  const long long n = p.n, n_pad = p.n_pad;
  long long base = (long long)blockIdx.x * P;
  const long long gstep = (long long)gridDim.x * P;
  RingPos rp;
  for (long long i = 0; i < nmy; ++i, base += gstep, rp.next(p.stages)) {
    const int stg = rp.stg;
    mbar_wait(R.full_a + 8u * stg, rp.ph);
    const float* xs = R.buf + (size_t)stg * R.rows * LD;
    unsigned char* lst = lst_s + (size_t)stg * KMAX * P;
    int* lcnt = lcnt_s + stg * KMAX * 8;
    for (int it = w; it < nA; it += LOCW_NW) {  // phase A: band decisions
      const int a = it / npb, pb = it - a * npb;
      const int q = pb * 32 + lane;
      const long long gp = base + q;
      const bool valid = gp < n;
      const int rs = row_s[a];
      float f;
      if (rs < 0) {  // a new Dist row, two fp32 chains
        const float* m = med_s + a * MS;
        const float* xq = xs + q;
        float s0 = 0.f, s1 = 0.f;
        int j = 0;
        for (; j + 2 <= d; j += 2) {
          const float t0 = xq[j * LD] - m[j], t1 = xq[(j + 1) * LD] - m[j + 1];
          if (METRIC == 1) {
            s0 = s0 + fabsf(t0);
            s1 = s1 + fabsf(t1);
          } else {
            s0 = __fmaf_rn(t0, t0, s0);
            s1 = __fmaf_rn(t1, t1, s1);
          }
        }
        if (j < d) {
          const float t0 = xq[j * LD] - m[j];
          s0 = METRIC == 1 ? s0 + fabsf(t0) : __fmaf_rn(t0, t0, s0);
        }
        f = METRIC == 1 ? s0 + s1 : sqrtf(s0 + s1);
        if (variant != 1 && valid) p.dist[(long long)act_s[a].key * n_pad + gp] = f;
      } else {
        f = xs[rs + q];
      }
      const Thr t = thr_s[a];
      bool in = f < t.in_hi && f > t.out_lo;
      if (valid && !in && !(f > t.out_hi || f < t.in_lo)) {
        // within the fp32 error bound: the oracle's fp64 value decides
        const ActSlot A = act_s[a];
        const double dv = full_dist(xs + q, LD, med_s + a * MS, d, METRIC);
        in = (dv > A.lo) && (dv <= A.hi);
        ++nfb;
      }
      in = in && valid;
      const unsigned b = __ballot_sync(0xffffffffu, in);
      if (in) lst[a * P + pb * 32 + __popc(b & lt)] = (unsigned char)lane;
      if (lane == 0) {
        lcnt[a * 8 + pb] = __popc(b);
        cnt[w * KMAX + a] += __popc(b);
      }
    }
    named_bar_sync(1, LOCW_NW * 32);  // every (slot, point block) list of the chunk is written
    for (int it = w; it < nB; it += LOCW_NW) {  // phase B: band sums of eq 6
      const int a = it / nb, jb = it - a * nb;
      const int j = jb * 32 + lane;
      const bool jv = j < d;
      const float* xr = xs + (size_t)(jv ? j : 0) * LD;
      const double c = (double)med_s[a * MS + (jv ? j : 0)];
      double s0 = 0.0, s1 = 0.0;
      for (int pb = 0; pb < npb; ++pb) {
        const int m = lcnt[a * 8 + pb];
        const unsigned char* la = lst + a * P + pb * 32;
        const float* xb = xr + pb * 32;
        int v = 0;
        for (; v + 2 <= m; v += 2) {
          const double t0 = fabs(dsub((double)xb[la[v]], c));
          const double t1 = fabs(dsub((double)xb[la[v + 1]], c));
          s0 = dadd(s0, t0);
          s1 = dadd(s1, t1);
        }
        if (v < m) s0 = dadd(s0, fabs(dsub((double)xb[la[v]], c)));
      }
      const double s = dadd(s0, s1);
      if (jv && s != 0.0) acc[a * d + j] += quant_sum(s, scale_s[j], magic);
    }
    pipe_release(R, stg);
  }
}

// --- ComputeL + FindDimensions X (Alg 3, Alg 4 l.1-5) with the FAST caches.
// One point per lane; the cached Dist rows of the active slots arrive through
// the same TMA ring as the data (rows d..).  DR: coordinates in registers.
template <int DR>
#ifndef LOC_MINB
#define LOC_MINB 3
#endif
__global__ void __launch_bounds__(288, LOC_MINB) k_locality(RunParams p) {
  DevState* st = p.st;
#ifdef PROCLUS_TAIL_PROFILE
  if (threadIdx.x == 0) atomicMin(&st->dbg_t[0], gtimer());
#define LOC_T(idx) \
  do {             \
    if (threadIdx.x == 0) atomicMax(&st->dbg_t[idx], gtimer()); \
  } while (0)
#else
#define LOC_T(idx) do {} while (0)
#endif
  extern __shared__ __align__(16) unsigned char smraw[];
  const SmemLayout& L = p.lay[KK_LOC];
#define LAYK KK_LOC
  const int d = p.d, k = p.k;
  const int nw = L.nw, w = threadIdx.x >> 5;
  // one round trip for the control words: stop flag, |active|, every slot of
  // the active list (whatever |active| is), 2^e_j
  __shared__ int ctl_s[2];
  if (threadIdx.x == 0) {
    ctl_s[0] = st->done;
    ctl_s[1] = st->n_act;
  }
  const int ncap = k * d;
  // d <= 16: the extra (cached Dist) rows start at ring row 16 and rows d..15
  // stay zero, so that a lane loads all 16 coordinate rows unconditionally
  const int row0 = DR == 16 ? 16 : d;
  const Pipe R = pipe_of(L, smraw, row0 + k);
  float* med_s = SMP(float, med);
  ActSlot* act_s = SMP(ActSlot, act);
  int* row_s = SMP(int, row);
  double* scale_s = SMP(double, scale);
  long long* acc_s = SMP(long long, acc);
  long long* cnt_s = SMP(long long, cnt);
  ExtraRows* ex = SMP(ExtraRows, ex);
  Thr* thr_s = SMP(Thr, thr);
  double* medd_s = DR == 16 ? SMP(double, ctr) : nullptr;          // [na][16] fp64 medoid rows
#ifdef LOC_EMPTY
  const long long nmy = 0;  // timing experiment only: prologue, epilogue and tail
#else
  const long long nmy = chunks_of_block(p);
#endif
  const double G = (double)(d + 8) * 5.9604644775390625e-08;  // (d+8) 2^-24

  for (int a = threadIdx.x; a < KMAX; a += blockDim.x) {
    const ActSlot A = st->act[a];  // slots >= |active| are stale and unused
    act_s[a] = A;
    thr_s[a] = make_thr(A.lo, A.hi, G);
  }
  for (int j = threadIdx.x; j < d; j += blockDim.x) scale_s[j] = p.scale[j];
  for (int e = threadIdx.x; e < (DR == 16 ? nw : 1) * ncap; e += blockDim.x) acc_s[e] = 0;
  for (int e = threadIdx.x; e < nw * KMAX; e += blockDim.x) cnt_s[e] = 0;
  if (DR == 16 && d < 16)  // zero padding rows d..15 of every stage (never copied into)
    for (int e = threadIdx.x; e < p.stages * (16 - d) * R.ldr; e += blockDim.x) {
      const int sg = e / ((16 - d) * R.ldr), r = e - sg * (16 - d) * R.ldr;
      R.buf[(size_t)sg * R.rows * R.ldr + (size_t)d * R.ldr + r] = 0.f;
    }
  pipe_init(p, R, nw);
  __syncthreads();
  if (ctl_s[0]) return;
  const int na = ctl_s[1];
  if (threadIdx.x < 32 || w == nw) {  // rows of the cached slots (warp ballot scan);
    // the producer warp derives the same list for its own TMA, so that the
    // ring starts filling while the consumers load the medoid rows
    const int a = threadIdx.x & 31;
    const bool cached = a < na && !act_s[a].compute;
    const unsigned b = __ballot_sync(0xffffffffu, cached);
    const int r = __popc(b & ((1u << a) - 1u));
    if (w == 0) {
      if (a < na) {
        row_s[a] = cached ? (row0 + r) * R.ldr : -1;
        ex->drow[a] = p.dist + (size_t)act_s[a].key * p.n_pad;
      }
    } else {
      if (cached) ex->src[r] = p.dist + (size_t)act_s[a].key * p.n_pad;
      if (a == 0) {
        ex->n = __popc(b);
        ex->row0 = row0;
      }
      __syncwarp();
    }
  }
  // medoid rows at stride MS (zero padded to DR for float4 loads)
  constexpr int MSD = DR > 0 ? DR : 0;
  const int MS = MSD > 0 ? MSD : d;
  if (w < nw) {
    for (int e = threadIdx.x; e < na * MS; e += nw * 32) {
      const int a = e / MS, j = e - a * MS;
      const float m = j < d ? p.mrows[(long long)act_s[a].mpos * d + j] : 0.f;
      med_s[e] = m;
      if (DR == 16) medd_s[e] = (double)m;
    }
    named_bar_sync(2, nw * 32);  // consumers only: the producer is already streaming
  }
  LOC_T(1);  // prologue done
  long long nfb = 0;
  int ncomp = 0;  // active slots whose Dist row is computed in this pass (consumers)
  if (w < nw)
    for (int a = 0; a < na; ++a) ncomp += row_s[a] < 0;
  if (na > 0) {
    if (w == nw) {
      pipe_produce(p, R, nmy, nullptr, ex);
    } else if constexpr (DR == 16) {
      if (p.metric == 1)
        loc16_consume<1>(p, R, L.buf / 4, nmy, na, ncomp, med_s, medd_s, row_s, thr_s, act_s, ex,
                         L.tab + w * 32 * LOC16_PPT, acc_s + (size_t)w * ncap, cnt_s + w * KMAX, scale_s,
                         nfb);
      else
        loc16_consume<0>(p, R, L.buf / 4, nmy, na, ncomp, med_s, medd_s, row_s, thr_s, act_s, ex,
                         L.tab + w * 32 * LOC16_PPT, acc_s + (size_t)w * ncap, cnt_s + w * KMAX, scale_s,
                         nfb);
    } else {
      unsigned char* lst_s = SMP(unsigned char, tab);  // [stages][KMAX][P] member lists
      int* lcnt_s = SMP(int, dl);                      // [stages][KMAX][8] list lengths
      if (p.metric == 1)
        locw_consume<1>(p, R, nmy, na, med_s, MS, row_s, thr_s, act_s, lst_s, lcnt_s, acc_s,
                        cnt_s, scale_s, nfb);
      else
        locw_consume<0>(p, R, nmy, na, med_s, MS, row_s, thr_s, act_s, lst_s, lcnt_s, acc_s,
                        cnt_s, scale_s, nfb);
    }
  }
  LOC_T(2);  // this block's chunks done
  __syncthreads();
  flush_warps(p, acc_s, nw, ncap, na * d, cnt_s, na, DR == 16 ? nw : 1);
  if (nfb) atomicAdd((unsigned long long*)&st->fallback[0], (unsigned long long)nfb);
  LOC_T(3);  // flushed
  if (!p.fuse_tail) return;
  if (!last_block(&st->ticket[0])) return;
#ifdef PROCLUS_TAIL_PROFILE
  if (threadIdx.x == 0) {
    const unsigned long long t0 = __ldcg(&st->dbg_t[0]);
    st->dbg_ts[1] += __ldcg(&st->dbg_t[1]) - t0;
    st->dbg_ts[2] += __ldcg(&st->dbg_t[2]) - t0;
    st->dbg_ts[3] += __ldcg(&st->dbg_t[3]) - t0;
    st->dbg_ts[4] += gtimer() - t0;  // tail start (after the ticket)
    st->dbg_ts[0] += 1;
    st->dbg_t[0] = ~0ull;
    st->dbg_t[1] = st->dbg_t[2] = st->dbg_t[3] = 0ull;
  }
  __syncthreads();  // before the tail's state_load reads these words
#endif
  RUN_TAIL(tail_locality, 0);
#undef LOC_T
#undef LAYK
}

// --- AssignPoints (Alg 5) + centroid sums of EvaluateCluster (Alg 6 l.1-8).
// PPT points per lane so every term-table entry loaded serves PPT points.
struct __align__(16) Term {
  float m, m2;  // m_ij twice: one 64-bit operand of the packed subtraction
  int joff;     // byte offset of row j in a ring stage: j * P * 4
  int pad;
};
#define LDX(base, boff) (*reinterpret_cast<const float*>(reinterpret_cast<const char*>(base) + (boff)))

// Packed fp32 subtraction (FADD2, sm_100): (x0 - m, x1 - m) for a lane's two
// adjacent points, each half rounded exactly as the scalar fsub_rn.
__device__ __forceinline__ unsigned long long fsub2(unsigned long long x, unsigned long long m) {
  unsigned long long r;
  asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(x), "l"(m));
  return r;
}
__device__ __forceinline__ float lo_f(unsigned long long v) { return __uint_as_float((unsigned)v); }
__device__ __forceinline__ float hi_f(unsigned long long v) {
  return __uint_as_float((unsigned)(v >> 32));
}
#define LDX2(base, boff) \
  (*reinterpret_cast<const unsigned long long*>(reinterpret_cast<const char*>(base) + (boff)))
#define TMM(e) (*reinterpret_cast<const unsigned long long*>(&(e).m))

// Paired-point terms (assign, 2 points per lane at xp, xp + 1): one 64-bit
// shared load and one packed subtraction per term serve both points; the
// two sums are formed in two chains (even / odd terms).
template <int ND>
__device__ __forceinline__ void dist_terms2(const float* __restrict__ xp,
                                            const Term* __restrict__ tb, float (&s)[2]) {
  float a0 = 0.f, a1 = 0.f, b0 = 0.f, b1 = 0.f;
#pragma unroll
  for (int t = 0; t < ND; t += 2) {
    const Term e0 = tb[t];
    const unsigned long long r0 = fsub2(LDX2(xp, e0.joff), TMM(e0));
    a0 += fabsf(lo_f(r0));
    a1 += fabsf(hi_f(r0));
    if (t + 1 < ND) {
      const Term e1 = tb[t + 1];
      const unsigned long long r1 = fsub2(LDX2(xp, e1.joff), TMM(e1));
      b0 += fabsf(lo_f(r1));
      b1 += fabsf(hi_f(r1));
    }
  }
  s[0] = ND > 1 ? a0 + b0 : a0;
  s[1] = ND > 1 ? a1 + b1 : a1;
}
// The same with 32-bit shared-window addresses (xa: the lane's first point
// in a ring stage, ta: the cluster's first table entry), so that no 64-bit
// generic pointers stay live across the cluster loop.
__device__ __forceinline__ void lds_term(unsigned a, unsigned long long& m2, int& joff) {
  unsigned lo, hi, jo;
  asm volatile("{\n.reg .b32 pad;\nld.shared.v4.b32 {%0, %1, %2, pad}, [%3];\n}"
               : "=r"(lo), "=r"(hi), "=r"(jo)
               : "r"(a));
  m2 = ((unsigned long long)hi << 32) | lo;
  joff = (int)jo;
}
__device__ __forceinline__ unsigned long long lds_u64(unsigned a) {
  unsigned long long v;
  asm volatile("ld.shared.u64 %0, [%1];" : "=l"(v) : "r"(a));
  return v;
}
template <int ND>
__device__ __forceinline__ void dist_terms2s(unsigned xa, unsigned ta, float (&s)[2]) {
  float a0 = 0.f, a1 = 0.f, b0 = 0.f, b1 = 0.f;
#pragma unroll
  for (int t = 0; t < ND; t += 2) {
    unsigned long long m0;
    int j0;
    lds_term(ta + 16u * t, m0, j0);
    const unsigned long long r0 = fsub2(lds_u64(xa + (unsigned)j0), m0);
    a0 += fabsf(lo_f(r0));
    a1 += fabsf(hi_f(r0));
    if (t + 1 < ND) {
      unsigned long long m1;
      int j1;
      lds_term(ta + 16u * (t + 1), m1, j1);
      const unsigned long long r1 = fsub2(lds_u64(xa + (unsigned)j1), m1);
      b0 += fabsf(lo_f(r1));
      b1 += fabsf(hi_f(r1));
    }
  }
  s[0] = ND > 1 ? a0 + b0 : a0;
  s[1] = ND > 1 ? a1 + b1 : a1;
}
__device__ __noinline__ void dist_terms2s_n(unsigned xa, unsigned ta, int nd, float (&s)[2]) {
  float a0 = 0.f, a1 = 0.f, b0 = 0.f, b1 = 0.f;
  int t = 0;
  for (; t + 2 <= nd; t += 2) {
    unsigned long long m0, m1;
    int j0, j1;
    lds_term(ta + 16u * t, m0, j0);
    lds_term(ta + 16u * (t + 1), m1, j1);
    const unsigned long long r0 = fsub2(lds_u64(xa + (unsigned)j0), m0);
    const unsigned long long r1 = fsub2(lds_u64(xa + (unsigned)j1), m1);
    a0 += fabsf(lo_f(r0));
    a1 += fabsf(hi_f(r0));
    b0 += fabsf(lo_f(r1));
    b1 += fabsf(hi_f(r1));
  }
  if (t < nd) {
    unsigned long long m;
    int j;
    lds_term(ta + 16u * t, m, j);
    const unsigned long long r = fsub2(lds_u64(xa + (unsigned)j), m);
    a0 += fabsf(lo_f(r));
    a1 += fabsf(hi_f(r));
  }
  s[0] = a0 + b0;
  s[1] = a1 + b1;
}
__device__ __noinline__ void dist_terms2_n(const float* __restrict__ xp,
                                           const Term* __restrict__ tb, int nd, float (&s)[2]) {
  float a0 = 0.f, a1 = 0.f, b0 = 0.f, b1 = 0.f;
  int t = 0;
  for (; t + 2 <= nd; t += 2) {
    const Term e0 = tb[t], e1 = tb[t + 1];
    const unsigned long long r0 = fsub2(LDX2(xp, e0.joff), TMM(e0));
    const unsigned long long r1 = fsub2(LDX2(xp, e1.joff), TMM(e1));
    a0 += fabsf(lo_f(r0));
    a1 += fabsf(hi_f(r0));
    b0 += fabsf(lo_f(r1));
    b1 += fabsf(hi_f(r1));
  }
  if (t < nd) {
    const Term e = tb[t];
    const unsigned long long r = fsub2(LDX2(xp, e.joff), TMM(e));
    a0 += fabsf(lo_f(r));
    a1 += fabsf(hi_f(r));
  }
  s[0] = a0 + b0;
  s[1] = a1 + b1;
}


// --- AssignPoints (Alg 5) + centroid sums for long rows (chunks of P <= 64
// points): the ASW_NW consumer warps share every chunk instead of owning 32
// points each (round 1 ran C4 with 4 consumer warps per SM).
// Phase A, items (32-point block pb, cluster range q): lane = point; the
//   certified fp32 segmental distances of the clusters of range q (two fp32
//   chains; the certified bound only needs the number of terms) reduced to
//   (best, second, argmin) in shared memory.
// Phase B, one warp per point block: merge the ranges in cluster order
//   (ties -> the smaller cluster, reading R8), certify against the runner-up
//   or take the exact fp64 argmin, store the u8 label; per-cluster ballots
//   give the chunk's member masks.
// Phase C, cells (cluster c, t < |D_c|) over all consumer threads: fp64 sum
//   of x_j over the chunk's members of c, quantised per (cell, chunk) into
//   the block's single accumulator copy (one writer per cell), |C_c| counts.
constexpr int ASW_NW = 8;
struct __align__(16) Part {
  float best, second;
  int bi, pad;
};
__global__ void __launch_bounds__(288) k_assign_w(RunParams p) {
  DevState* st = p.st;
  extern __shared__ __align__(16) unsigned char smraw[];
  const SmemLayout& L = p.lay[KK_ASG];
#define LAYK KK_ASG
  const int P = p.P, d = p.d, k = p.k;
  const int nw = ASW_NW, w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int ncap = k * d;
  const Pipe R = pipe_of(L, smraw, d);
  const int LD = R.ldr;
  float* med_s = SMP(float, med);     // [k][d] medoid rows (exact fallback)
  Term* tab_s = SMP(Term, tab);       // [k*l] terms, cluster c from off_s[c]
  int* dl_s = SMP(int, dl);           // [k][d] dimension lists
  int* nD_s = SMP(int, nD);
  int* off_s = SMP(int, off);
  float* rcp_s = SMP(float, rcp);
  double* scale_s = SMP(double, scale);
  Cell* cells = SMP(Cell, cells);     // [k*l]
  unsigned* msk_s = SMP(unsigned, bal);   // [KMAX][npb] member masks of the chunk
  long long* acc_s = SMP(long long, acc);  // [k*d] one copy
  long long* cnt_s = SMP(long long, cnt);  // [nw][KMAX], row 0 used
  Part* part = SMP(Part, row);             // [nq][P]
  const long long nmy = chunks_of_block(p);
  for (int j = threadIdx.x; j < d; j += blockDim.x) scale_s[j] = p.scale[j];
  for (int e = threadIdx.x; e < ncap; e += blockDim.x) acc_s[e] = 0;
  for (int e = threadIdx.x; e < nw * KMAX; e += blockDim.x) cnt_s[e] = 0;
  pipe_init(p, R, nw);
  __syncthreads();
  if (st->done) return;
  unsigned char* lab = st->cur_buf ? p.lab1 : p.lab0;
  for (int i = threadIdx.x; i < k; i += blockDim.x) {
    nD_s[i] = st->nD[i];
    rcp_s[i] = 1.0f / (float)st->nD[i];
  }
  for (int e = threadIdx.x; e < k * d; e += blockDim.x) {
    const int i = e / d;
    med_s[e] = p.mrows[(long long)st->mcur[i] * d + (e - i * d)];
    dl_s[e] = p.dlist[e];
  }
  __syncthreads();
  const int ncell = build_cells(cells, nD_s, k, d, off_s, dl_s, nullptr);  // also off_s
  for (int e = threadIdx.x; e < ncell; e += blockDim.x) {
    const Cell C = cells[e];
    Term t;
    t.m = med_s[C.a * d + C.j];
    t.m2 = t.m;
    t.joff = C.j * LD;  // float offset of row j in a ring stage
    t.pad = 0;
    tab_s[e] = t;
  }
  int ndmax = 0;
  for (int i = 0; i < k; ++i) ndmax = max(ndmax, nD_s[i]);
  const double G = (double)(ndmax + 6) * 5.9604644775390625e-08;
  __syncthreads();
  long long nfb = 0;
  if (w == nw) {
    pipe_produce(p, R, nmy, nullptr, nullptr);
  } else {
    const int npb = P >> 5, nq = nw / npb;
    const int magic = *p.qflag;
    long long base = (long long)blockIdx.x * P;
    const long long gstep = (long long)gridDim.x * P;
    RingPos rp;
    for (long long i = 0; i < nmy; ++i, base += gstep, rp.next(p.stages)) {
      const int stg = rp.stg;
      mbar_wait(R.full_a + 8u * stg, rp.ph);
      const float* xs = R.buf + (size_t)stg * R.rows * LD;
      {  // phase A: item (pb, q) = warp w
        const int pb = w % npb, q = w / npb;
        const int c0 = q * k / nq, c1 = (q + 1) * k / nq;
        const float* xq = xs + pb * 32 + lane;
        float best = CUDART_INF_F, second = CUDART_INF_F;
        int bi = c0;
        for (int c = c0; c < c1; ++c) {
          const Term* tb = tab_s + off_s[c];
          const int nd = nD_s[c];
          float a0 = 0.f, a1 = 0.f;
          int t = 0;
          for (; t + 2 <= nd; t += 2) {
            const Term e0 = tb[t], e1 = tb[t + 1];
            a0 += fabsf(xq[e0.joff] - e0.m);
            a1 += fabsf(xq[e1.joff] - e1.m);
          }
          if (t < nd) a0 += fabsf(xq[tb[t].joff] - tb[t].m);
          const float qv = (a0 + a1) * rcp_s[c];
          second = qv < best ? best : fminf(second, qv);
          bi = qv < best ? c : bi;
          best = fminf(best, qv);
        }
        Part pr;
        pr.best = best;
        pr.second = second;
        pr.bi = bi;
        pr.pad = 0;
        part[q * P + pb * 32 + lane] = pr;
      }
      named_bar_sync(1, nw * 32);
      if (w < npb) {  // phase B: point block w
        const int qp = w * 32 + lane;
        const long long gp = base + qp;
        float best = CUDART_INF_F, second = CUDART_INF_F;
        int bi = 0;
        for (int q = 0; q < nq; ++q) {  // cluster order: the earlier range wins ties
          const Part pr = part[q * P + qp];
          if (pr.best < best) {
            second = fminf(best, fminf(second, pr.second));
            best = pr.best;
            bi = pr.bi;
          } else {
            second = fminf(second, pr.best);
          }
        }
        int lbl = -1;
        if (gp < p.n) {
          const bool certain = (best >= 1e-30f) && (second < 1e30f) &&
                               ((double)second * (1.0 - G) > (double)best * (1.0 + G));
          lbl = bi;
          if (!certain) {
            lbl = exact_argmin(xs + qp, LD, med_s, dl_s, nD_s, k, d, nullptr, nullptr);
            ++nfb;
          }
          lab[gp] = (unsigned char)lbl;
        }
        unsigned mine = 0u;
        for (int c = 0; c < k; ++c) {
          const unsigned b = __ballot_sync(0xffffffffu, lbl == c);
          if (lane == c) mine = b;
        }
        if (lane < k) msk_s[lane * npb + w] = mine;
      }
      named_bar_sync(1, nw * 32);
      {  // phase C: centroid cells and counts
        const int tid = threadIdx.x;
        for (int ci = tid; ci < ncell; ci += nw * 32) {
          const Cell C = cells[ci];
          const float* xr = xs + (size_t)C.j * LD;
          double s0 = 0.0, s1 = 0.0;
          for (int pb = 0; pb < npb; ++pb) {
            unsigned m = msk_s[C.a * npb + pb];
            const float* xb = xr + pb * 32;
            while (m) {
              const int b0 = __ffs(m) - 1;
              m &= m - 1u;
              s0 = dadd(s0, (double)xb[b0]);
              if (m) {
                const int b1 = __ffs(m) - 1;
                m &= m - 1u;
                s1 = dadd(s1, (double)xb[b1]);
              }
            }
          }
          const double sm = dadd(s0, s1);
          if (sm != 0.0) acc_s[C.acc] += quant_sum(sm, scale_s[C.j], magic);
        }
        if (tid < k) {
          int cn = 0;
          for (int pb = 0; pb < npb; ++pb) cn += __popc(msk_s[tid * npb + pb]);
          cnt_s[tid] += cn;
        }
      }
      pipe_release(R, stg);
      named_bar_sync(1, nw * 32);  // masks and parts are rewritten by the next chunk
    }
  }
  __syncthreads();
  flush_warps(p, acc_s, nw, ncap, k * d, cnt_s, k, 1);
  if (nfb) atomicAdd((unsigned long long*)&st->fallback[1], (unsigned long long)nfb);
  if (!p.fuse_tail) return;
  if (!last_block(&st->ticket[1])) return;
  RUN_TAIL(tail_assign, 1);
#undef LAYK
}

// --- EvaluateCluster deviations (Alg 6 l.9-13, eq 9) + control tail, and the
// refinement X over CBest (Alg 1 l.16-17) which has the same shape.
// REF = 0: cells (i, t) over D_i of |x - mu_i|, labels of the current buffer.
// REF = 1: cells (i, j) over all d of |x - mbest_ij|, labels of CBest.
template <int REF>
__global__ void __launch_bounds__(288) k_labelsum(RunParams p) {
  DevState* st = p.st;
  if (!REF && st->done) return;
  extern __shared__ __align__(16) unsigned char smraw[];
  const SmemLayout& L = p.lay[KK_LSUM];
#define LAYK KK_LSUM
  const int P = p.P, d = p.d, k = p.k;
  const int nw = L.nw, w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int ncap = k * d;
  const Pipe R = pipe_of(L, smraw, d);
  double* ctr_s = SMP(double, ctr);
  int* dl_s = SMP(int, dl);
  int* nD_s = SMP(int, nD);
  int* off_s = SMP(int, off);
  double* scale_s = SMP(double, scale);
  Cell* cells = SMP(Cell, cells);
  unsigned* bal_s = SMP(unsigned, bal);
  long long* acc_s = SMP(long long, acc);
  long long* cnt_s = SMP(long long, cnt);
  const unsigned char* lab =
      REF ? (st->best_buf ? p.lab1 : p.lab0) : (st->cur_buf ? p.lab1 : p.lab0);
  const long long nmy = chunks_of_block(p);
  for (int e = threadIdx.x; e < k * d; e += blockDim.x) {
    const int i = e / d;
    ctr_s[e] = REF ? (double)p.mrows[(long long)st->mbest[i] * d + (e - i * d)] : p.mu[e];
    dl_s[e] = REF ? e - i * d : p.dlist[e];
  }
  for (int i = threadIdx.x; i < k; i += blockDim.x) nD_s[i] = REF ? d : st->nD[i];
  for (int j = threadIdx.x; j < d; j += blockDim.x) scale_s[j] = p.scale[j];
  for (int e = threadIdx.x; e < nw * ncap; e += blockDim.x) acc_s[e] = 0;
  for (int e = threadIdx.x; e < nw * KMAX; e += blockDim.x) cnt_s[e] = 0;
  pipe_init(p, R, nw);
  __syncthreads();
  const int ncell = build_cells(cells, nD_s, k, d, off_s, dl_s, ctr_s);
  if (w == nw) {
    pipe_produce(p, R, nmy, lab, nullptr);
  } else {
    unsigned* bal = bal_s + w * KMAX;
    long long* acc = acc_s + (size_t)w * ncap;
    const int q = w * 32 + lane;
    long long gp = (long long)blockIdx.x * P + q;
    const long long gstep = (long long)gridDim.x * P;
    RingPos rp;
    for (long long i = 0; i < nmy; ++i, gp += gstep, rp.next(p.stages)) {
      const int stg = rp.stg;
      mbar_wait(R.full_a + 8u * stg, rp.ph);
      const float* xs = R.buf + (size_t)stg * R.rows * P;
      const int lb = gp < p.n ? (int)R.lab[(size_t)stg * P + q] : -1;
      // one ballot per cluster: lane c of the warp keeps cluster c's mask
      unsigned mine = 0u;
      for (int c = 0; c < k; ++c) {
        const unsigned b = __ballot_sync(0xffffffffu, lb == c);
        if (lane == c) mine = b;
      }
      if (lane < k) {
        bal[lane] = mine;
        if (REF) cnt_s[w * KMAX + lane] += __popc(mine);
      }
      __syncwarp();
      warp_cells<1, 1>(xs, P, w * 32, cells, ncell, bal, acc, scale_s);
      pipe_release(R, stg);
    }
  }
  __syncthreads();
  flush_warps(p, acc_s, nw, ncap, k * d, cnt_s, REF ? k : 0);
  if (!p.fuse_tail) return;
  if (!last_block(&st->ticket[REF ? 3 : 2])) return;
  if (REF)
    RUN_TAIL(tail_refine, 3);
  else
    RUN_TAIL(tail_cost, 2);
#undef LAYK
}

// ============================================================ lane-private sums
// Per-term fixed point: the term t (|x - c| or x) of dimension j becomes
// round(t * 2^e_j) as an int64 via the 1.5 * 2^52 "magic" addend -- one DFMA
// forms x*2^e_j - c*2^e_j (c*2^e_j exact: a power-of-two scale) with one
// rounding, one DADD rounds it to an integer held in the low mantissa bits
// (|t| 2^e_j < 2^51 by the choice of e_j, proclus_api.cu).  The int64 values
// are added exactly, so the totals do not depend on the order, the grid or the
// number of GPUs; the error per term is <= 2^-(e_j+1).
constexpr double QMAGIC_D = 6755399441055744.0;  // 1.5 * 2^52
constexpr long long QMAGIC_BITS = 0x4338000000000000ll;
__device__ __forceinline__ long long q_abs(float x, double sc, double cq) {
  const double r = __fma_rn((double)x, sc, -cq);
  return __double_as_longlong(__dadd_rn(fabs(r), QMAGIC_D)) - QMAGIC_BITS;
}
__device__ __forceinline__ long long q_val(float x, double sc) {
  return __double_as_longlong(__fma_rn((double)x, sc, QMAGIC_D)) - QMAGIC_BITS;
}

// Producer of the kernels with their own chunk geometry (SmemLayout P, ldr,
// stages): chunk c covers points [c P, c P + P) clipped to n_pad (a multiple of
// 32, so every copy stays a multiple of 16 bytes); dimension row j of stage s
// lands at buf + (s d + j) ldr floats, the labels (if any) at lab + s P.
__device__ void pipe_produce_k(const RunParams& p, const Pipe& R, const SmemLayout& L,
                               long long nmy, const unsigned char* labsrc) {
  const int lane = threadIdx.x & 31;
  const int P = L.P, d = p.d;
  const unsigned long long pol_last = l2_policy(1);
  int stg = 0, round = 0;
  for (long long i = 0; i < nmy; ++i) {
    if (round > 0) {
      mbar_wait(R.empty_a + 8u * stg, (unsigned)((round - 1) & 1));
      fence_proxy_async();
    }
    const long long base = (blockIdx.x + i * gridDim.x) * (long long)P;
    const long long left = p.n_pad - base;
    const unsigned cnt = (unsigned)(left < P ? left : P);
    const unsigned bytes = cnt * 4u * (unsigned)d + (labsrc ? cnt : 0u);
    if (lane == 0) mbar_expect_tx(R.full_a + 8u * stg, bytes);
    __syncwarp();
    float* dst = R.buf + (size_t)stg * d * L.ldr;
    for (int j = lane; j < d; j += 32)
      bulk_g2s_h(dst + (size_t)j * L.ldr, p.xs + (size_t)j * p.n_pad + base, cnt * 4u, R.full_a + 8u * stg,
                 pol_last);
    if (labsrc && lane == 0) bulk_g2s(R.lab + (size_t)stg * P, labsrc + base, cnt, R.full_a + 8u * stg);
    if (++stg == L.stages) {
      stg = 0;
      ++round;
    }
  }
}
__device__ __forceinline__ long long chunks_of_block_k(const RunParams& p, int P) {
  const long long nch = (p.n + P - 1) / P;
  return (nch > blockIdx.x) ? (nch - blockIdx.x + gridDim.x - 1) / gridDim.x : 0;
}

// One work item of a sorted-member pass: cell (i, t) of dimension j (row
// offset joff in a ring stage), the residue r of the members it takes
// (members r, r + R, r + 2R, ... of cluster i in each chunk), 2^e_j and
// centre * 2^e_j.  Items live in registers-free shared tables; their int64
// partial sums in an item-private shared array (no two threads share one).
struct __align__(16) Item {
  int joff, c, r, R;
  double sc, cq;
};

// Counting sort of one chunk's points by cluster (labels in the ring) among
// the consumer threads: list[base_c + pos] = q for the points of cluster c,
// hist[c] = |members|, base_s[c] = base_c.  Two named barriers; hist, base
// and list are double-buffered by chunk parity (hist_next, the other
// buffer's histogram, is cleared between the two barriers).  The order
// inside a cluster depends on atomics, which is harmless: every sum over the
// members is an exact integer sum.
__device__ __forceinline__ void sort_chunk(const unsigned char* lab_s, long long nvalid, int q,
                                           int nct, int k, int* hist, int* hist_next, int* base_s,
                                           int* list) {
  const int lane = threadIdx.x & 31;
  const bool valid = q < nvalid;
  const int c = valid ? (int)lab_s[q] : 0;
  int pos = 0;
  if (valid) pos = atomicAdd(&hist[c], 1);
  named_bar_sync(1, nct);
  const int h = lane < k ? hist[lane] : 0;
  int x = h;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const int y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  const int base = __shfl_sync(0xffffffffu, x - h, c);
  if (valid) list[base + pos] = q;
  if (threadIdx.x < 32 && lane < k) base_s[lane] = x - h;
  if (threadIdx.x < KMAX) hist_next[threadIdx.x] = 0;  // read last in the previous chunk
  named_bar_sync(1, nct);
}

// The same with PPTS points per thread, given as (q[r], c[r]) in registers
// (c < 0: no point).
template <int PPTS>
__device__ __forceinline__ void sort_chunk_m(const int (&q)[PPTS], const int (&c)[PPTS], int nct,
                                             int k, int* hist, int* hist_next, int* base_s,
                                             int* list) {
  const int lane = threadIdx.x & 31;
  int pos[PPTS];
#pragma unroll
  for (int r = 0; r < PPTS; ++r) pos[r] = c[r] >= 0 ? atomicAdd(&hist[c[r]], 1) : 0;
  named_bar_sync(1, nct);
  const int h = lane < k ? hist[lane] : 0;
  int x = h;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const int y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
#pragma unroll
  for (int r = 0; r < PPTS; ++r) {
    const int base = __shfl_sync(0xffffffffu, x - h, c[r] < 0 ? 0 : c[r]);
    if (c[r] >= 0) list[base + pos[r]] = q[r];
  }
  if (threadIdx.x < 32 && lane < k) base_s[lane] = x - h;
  if (threadIdx.x < KMAX) hist_next[threadIdx.x] = 0;
  named_bar_sync(1, nct);
}

// packed fp32x2 arithmetic (sm_100 FADD2): two points per instruction
__device__ __forceinline__ float2 f2_sub_abs_add(float2 acc, float2 x, float m) {
  // acc + |x - m| on both halves (FADD2 with a broadcast operand and |.|)
  unsigned long long r, a = *reinterpret_cast<unsigned long long*>(&acc),
                        xv = *reinterpret_cast<unsigned long long*>(&x);
  unsigned long long mm = ((unsigned long long)__float_as_uint(m) << 32) | __float_as_uint(m);
  unsigned long long t;
  asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(t) : "l"(xv), "l"(mm));
  const float2 tf = *reinterpret_cast<float2*>(&t);
  const float2 ab = make_float2(fabsf(tf.x), fabsf(tf.y));
  const unsigned long long abv = *reinterpret_cast<const unsigned long long*>(&ab);
  asm("add.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(a), "l"(abv));
  return *reinterpret_cast<float2*>(&r);
}

// Per-block state of the sorted-member item machinery (shared memory).
struct ItemCtx {
  Item* items;       // [nitem]
  long long* iacc;   // [nitem] item-private int64 sums
  int* gix;          // [cells] global cell index i * d + t
  int* hist0;        // [2][KMAX] histograms + [2][KMAX] bases (double buffer)
  int* list0;        // [2][P] sorted chunk points
  long long* ccnt;   // [KMAX] |members| per cluster (MODE 1, 2)
  int* off_s;        // [KMAX] first cell of cluster i
  int* nd_s;         // [KMAX] cells of cluster i
  int* rr_s;         // [KMAX] R_i
  int* ib_s;         // [KMAX + 1] first item of cluster i
  int nitem, nct;
};

// MODE 0: cells (i, t < |D_i|) of |x_j - mu_ij| (cost, Alg 6 l.9-13);
// MODE 1: cells (i, j < d) of |x_j - mbest_ij| (refinement X, Alg 1 l.16);
// MODE 2: cells (i, t < |D_i|) of x_j (centroid sums, Alg 6 l.1-8).
// R_i (threads per cell of cluster i) is proportional to the expected
// |C_i| (sizes of the current / best / previous clustering).  Block-wide.
template <int MODE>
__device__ void items_build(const RunParams& p, const SmemLayout& L, ItemCtx& X) {
  const DevState* st = p.st;
  const int d = p.d, k = p.k, lane = threadIdx.x & 31;
  if (threadIdx.x < 32) {
    const int i = lane;
    const int nd = i < k ? (MODE == 1 ? d : st->nD[i]) : 0;
    const long long sz = i < k ? (MODE == 1 ? st->sizes_best[i] : st->sizes[i]) : 0;
    int x = nd;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int y = __shfl_up_sync(0xffffffffu, x, o);
      if (lane >= o) x += y;
    }
    double wsum = (double)nd * (double)sz;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) wsum += __shfl_xor_sync(0xffffffffu, wsum, o);
    const int tot = __shfl_sync(0xffffffffu, x, 31);  // number of cells
    int Ri = 1;
    if (wsum > 0.0 && i < k) {
      const double f = floor((double)X.nct * (double)sz / wsum);
      Ri = f < 1.0 ? 1 : (f > 4096.0 ? 4096 : (int)f);
    } else if (i < k) {  // no estimate: spread evenly
      Ri = tot > 0 ? max(1, X.nct / tot) : 1;
    }
    const int ni = i < k ? nd * Ri : 0;
    int y2 = ni;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int y = __shfl_up_sync(0xffffffffu, y2, o);
      if (lane >= o) y2 += y;
    }
    if (i < k) {
      X.off_s[i] = x - nd;
      X.nd_s[i] = nd;
      X.rr_s[i] = Ri;
      X.ib_s[i] = y2 - ni;
    }
    if (lane == 31) X.ib_s[KMAX] = y2;
    X.hist0[lane] = 0;
    X.hist0[KMAX + lane] = 0;
    if (MODE != 0) X.ccnt[lane] = 0;
  }
  __syncthreads();
  X.nitem = X.ib_s[KMAX];
  for (int it = threadIdx.x; it < X.nitem; it += blockDim.x) {
    int i = 0;
    while (i + 1 < k && X.ib_s[i + 1] <= it) ++i;
    const int loc = it - X.ib_s[i], nd = X.nd_s[i];
    const int r = loc / nd, t = loc - r * nd;
    const int e = i * d + t;
    const int j = MODE == 1 ? t : p.dlist[e];
    const double sc = p.scale[j];
    double c = 0.0;
    if (MODE == 0) c = p.mu[e];
    if (MODE == 1) c = (double)p.mrows[(long long)st->mbest[i] * d + j];
    X.items[it] = Item{j * L.ldr * 4, i, r, X.rr_s[i], sc, c * sc};
    X.iacc[it] = 0;
    if (r == 0) X.gix[X.off_s[i] + t] = e;
  }
}

// The items of one sorted chunk (after sort_chunk): thread q adds its items'
// members in registers, then once into its item-private accumulators.
template <int MODE>
__device__ __forceinline__ void items_chunk(const ItemCtx& X, const char* xs, const int* hist,
                                            const int* base_s, const int* list, int q, int k) {
  for (int it = q; it < X.nitem; it += X.nct) {
    const Item I = X.items[it];
    const int cnt = hist[I.c];
    const int* lm = list + base_s[I.c];
    const char* xj = xs + I.joff;
    long long a = 0, b = 0;
    int m = I.r;
    // 4 members in flight: their list entries and coordinates are loaded
    // before any of them is converted
    for (; m + 3 * I.R < cnt; m += 4 * I.R) {
      const int q0 = lm[m], q1 = lm[m + I.R], q2 = lm[m + 2 * I.R], q3 = lm[m + 3 * I.R];
      const float x0 = *reinterpret_cast<const float*>(xj + q0 * 4);
      const float x1 = *reinterpret_cast<const float*>(xj + q1 * 4);
      const float x2 = *reinterpret_cast<const float*>(xj + q2 * 4);
      const float x3 = *reinterpret_cast<const float*>(xj + q3 * 4);
      if (MODE == 2) {
        a += q_val(x0, I.sc) + q_val(x1, I.sc);
        b += q_val(x2, I.sc) + q_val(x3, I.sc);
      } else {
        a += q_abs(x0, I.sc, I.cq) + q_abs(x1, I.sc, I.cq);
        b += q_abs(x2, I.sc, I.cq) + q_abs(x3, I.sc, I.cq);
      }
    }
    for (; m < cnt; m += I.R) {
      const float x = *reinterpret_cast<const float*>(xj + lm[m] * 4);
      a += MODE == 2 ? q_val(x, I.sc) : q_abs(x, I.sc, I.cq);
    }
    X.iacc[it] += a + b;
  }
  if (MODE != 0 && q < k) X.ccnt[q] += hist[q];
}

// Per cell: the sum of its R_i items; one int64 atomic per cell (and count)
// per block into one of the NCOPY global copies.  Block-wide.
template <int MODE>
__device__ void items_flush(const RunParams& p, const ItemCtx& X) {
  const int k = p.k;
  const int cp = blockIdx.x % NCOPY;
  long long* acc = p.accg + (size_t)cp * p.k * p.d;
  const int ncell = X.off_s[k - 1] + X.nd_s[k - 1];
  for (int cell = threadIdx.x; cell < ncell; cell += blockDim.x) {
    int i = 0;
    while (i + 1 < k && X.off_s[i + 1] <= cell) ++i;
    const int t = cell - X.off_s[i], nd = X.nd_s[i];
    long long s = 0;
    for (int r = 0; r < X.rr_s[i]; ++r) s += X.iacc[X.ib_s[i] + r * nd + t];
    if (s) atomicAdd((unsigned long long*)&acc[X.gix[cell]], (unsigned long long)s);
  }
  if (MODE != 0) {
    long long* cnt = p.cntg + (size_t)cp * KMAX;
    if (threadIdx.x < k && X.ccnt[threadIdx.x])
      atomicAdd((unsigned long long*)&cnt[threadIdx.x], (unsigned long long)X.ccnt[threadIdx.x]);
  }
}

__device__ __forceinline__ ItemCtx item_ctx(const SmemLayout& L, unsigned char* smraw, int* off_s,
                                            int* nd_s, int* rr_s, int* ib_s) {
  ItemCtx X;
  X.items = SMP(Item, tab);
  X.iacc = SMP(long long, acc);
  X.gix = SMP(int, nD);
  X.hist0 = SMP(int, bal);
  X.list0 = SMP(int, row);
  X.ccnt = SMP(long long, cnt);
  X.off_s = off_s;
  X.nd_s = nd_s;
  X.rr_s = rr_s;
  X.ib_s = ib_s;
  X.nct = L.nw * 32;
  X.nitem = 0;
  return X;
}

__device__ __forceinline__ void pipe_init_k(const SmemLayout& L, const Pipe& R) {
  if (threadIdx.x == 0) {
    for (int s2 = 0; s2 < L.stages; ++s2) {
      mbar_init(&R.full[s2], 1);
      mbar_init(&R.empty[s2], (unsigned)L.nw);
    }
    fence_mbar_init();
  }
}

// --- AssignPoints (Alg 5) + centroid sums of EvaluateCluster (Alg 6 l.1-8),
// chunks of >= 128 points.  A lane owns the adjacent points q0 + 2 lane + u
// (u = 0, 1) of its warp's 64 columns: certified fp32 argmin over the
// clusters (packed terms; clusters visited in groups of equal |D_c|, one
// switch per group selects the unrolled term code),
// fp64 fallback near a tie (reading R8), u8 label.  Then the chunk is
// counting-sorted by the new labels among the consumer threads and the item
// threads (cell (c, t), residue r, stride R_c ~ |C_c|) add round(x_j 2^e_j)
// of the members in registers: exact int64 centroid sums, independent of the
// order, the grid and the GPU count, with no per-cluster ballots or bit walks.
#define ASG_UPD(c, s)                                                       \
  do {                                                                      \
    const float r_ = rcp_s[c];                                              \
    _Pragma("unroll") for (int u = 0; u < 2; ++u) {                         \
      const float qv = (s)[u] * r_;                                         \
      second[u] = qv < best[u] ? best[u] : fminf(second[u], qv);            \
      bi[u] = qv < best[u] ? (c) : bi[u];                                   \
      best[u] = fminf(best[u], qv);                                         \
    }                                                                       \
  } while (0)
template <int PPT>
__global__ void __launch_bounds__(160) k_assign(RunParams p) {
  static_assert(PPT == 2, "two adjacent points per lane");
  DevState* st = p.st;
  extern __shared__ __align__(16) unsigned char smraw[];
  const SmemLayout& L = p.lay[KK_ASG];
#define LAYK KK_ASG
  const int P = p.P, d = p.d, k = p.k;
  const int nw = L.nw, w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int nct = nw * 32;
  const Pipe R = pipe_of(L, smraw, d);
  float* med_s = SMP(float, med);
  Term* tab_s = SMP(Term, tab);
  int* dl_s = SMP(int, dl);
  int* nD_s = SMP(int, nD);
  float* rcp_s = SMP(float, rcp);
  __shared__ int off_s[KMAX], ndi_s[KMAX], rr_s[KMAX], ib_s[KMAX + 1];
  __shared__ int ord_s[KMAX], gst_s[KMAX + 1], gnd_s[KMAX], ngrp_s;
  ItemCtx X;
  X.items = SMP(Item, cells);
  X.iacc = SMP(long long, acc);
  X.gix = SMP(int, ctr);
  X.hist0 = SMP(int, bal);
  X.list0 = SMP(int, row);
  X.ccnt = SMP(long long, cnt);
  X.off_s = off_s;
  X.nd_s = ndi_s;
  X.rr_s = rr_s;
  X.ib_s = ib_s;
  X.nct = nct;
  X.nitem = 0;
  const long long nmy = chunks_of_block(p);
  pipe_init(p, R, nw);
  __syncthreads();
  if (st->done) return;
  unsigned char* lab = st->cur_buf ? p.lab1 : p.lab0;
  for (int i = threadIdx.x; i < k; i += blockDim.x) {
    nD_s[i] = st->nD[i];
    rcp_s[i] = 1.0f / (float)st->nD[i];
  }
  for (int e = threadIdx.x; e < k * d; e += blockDim.x) {
    const int i = e / d;
    med_s[e] = p.mrows[(long long)st->mcur[i] * d + (e - i * d)];
    dl_s[e] = p.dlist[e];
  }
  items_build<2>(p, L, X);  // block-wide (barrier inside)
  __syncthreads();
  for (int e = threadIdx.x; e < k * d; e += blockDim.x) {
    const int i = e / d, t = e - i * d;
    if (t < nD_s[i]) {
      const int j = dl_s[e];
      tab_s[e].joff = j * P * 4;
      tab_s[e].m = med_s[i * d + j];
      tab_s[e].m2 = med_s[i * d + j];
    }
  }
  __syncthreads();
  if (threadIdx.x < 32) {  // clusters ordered by (|D_c|, c), groups of equal |D_c|
    const int c = lane;
    const int nd = c < k ? nD_s[c] : 1 << 30;
    int rank = 0;
    for (int o = 0; o < k; ++o) {
      const int no = nD_s[o];
      rank += (no < nd) | ((no == nd) & (o < c));
    }
    if (c < k) ord_s[rank] = c;
    __syncwarp();
    const int r = lane;
    const int ndr = r < k ? nD_s[ord_s[r]] : -1;
    const int ndp = __shfl_up_sync(0xffffffffu, ndr, 1);
    const bool head = r < k && (r == 0 || ndp != ndr);
    const unsigned hb = __ballot_sync(0xffffffffu, head);
    if (head) {
      const int g = __popc(hb & ((1u << lane) - 1u));
      gst_s[g] = r;
      gnd_s[g] = ndr;
    }
    if (lane == 0) {
      ngrp_s = __popc(hb);
      gst_s[__popc(hb)] = k;
    }
  }
  __syncthreads();
  const int ngrp = ngrp_s;
  int ndmax = 0;
  for (int i = 0; i < k; ++i) ndmax = max(ndmax, nD_s[i]);
  const double G = (double)(ndmax + 6) * 5.9604644775390625e-08;
  long long nfb = 0;
  if (w == nw) {
    pipe_produce(p, R, nmy, nullptr, nullptr);
  } else {
    const int q0 = w * 64, tq = threadIdx.x;
    long long base = (long long)blockIdx.x * P;
    const long long gstep = (long long)gridDim.x * P;
    RingPos rp;
    for (long long i = 0; i < nmy; ++i, base += gstep, rp.next(p.stages)) {
      const int stg = rp.stg;
      const int hb = (int)(i & 1);
      mbar_wait(R.full_a + 8u * stg, rp.ph);
      const float* xs = R.buf + (size_t)stg * R.rows * P;
      const float* xq = xs + q0 + 2 * lane;
      const unsigned xqa = smem_u32(xq), taa = smem_u32(tab_s);
      float best[2], second[2];
      int bi[2];
#pragma unroll
      for (int u = 0; u < 2; ++u) {
        best[u] = CUDART_INF_F;
        second[u] = CUDART_INF_F;
        bi[u] = 0;
      }
      // clusters grouped by |D_c| (one switch per group; the argmin does not
      // depend on the visiting order: an exact fp32 tie is never certified)
      for (int g = 0; g < ngrp; ++g) {
        const int r0 = gst_s[g], r1 = gst_s[g + 1];
        switch (gnd_s[g]) {
#define DT(N)                                              \
  case N:                                                  \
    for (int r = r0; r < r1; ++r) {                        \
      const int c = ord_s[r];                              \
      float s[2];                                          \
      dist_terms2s<N>(xqa, taa + 16u * (unsigned)(c * d), s); \
      ASG_UPD(c, s);                                       \
    }                                                      \
    break;
          DT(1) DT(2) DT(3) DT(4) DT(5) DT(6) DT(7) DT(8)
          DT(9) DT(10) DT(11) DT(12) DT(13) DT(14) DT(15) DT(16)
#undef DT
          default:
            for (int r = r0; r < r1; ++r) {
              const int c = ord_s[r];
              float s[2];
              dist_terms2s_n(xqa, taa + 16u * (unsigned)(c * d), gnd_s[g], s);
              ASG_UPD(c, s);
            }
        }
      }
      int qq[2], cc[2];
#pragma unroll
      for (int u = 0; u < 2; ++u) {
        const int q = q0 + 2 * lane + u;
        const long long gp = base + q;
        qq[u] = q;
        cc[u] = -1;
        if (gp >= p.n) continue;
        const bool certain = (best[u] >= 1e-30f) && (second[u] < 1e30f) &&
                             ((double)second[u] * (1.0 - G) > (double)best[u] * (1.0 + G));
        int lbl = bi[u];
        if (!certain) {
          lbl = exact_argmin(xs + q, P, med_s, dl_s, nD_s, k, d, nullptr, nullptr);
          ++nfb;
        }
        lab[gp] = (unsigned char)lbl;
        cc[u] = lbl;
      }
      sort_chunk_m<2>(qq, cc, nct, k, X.hist0 + hb * KMAX, X.hist0 + (hb ^ 1) * KMAX,
                      X.hist0 + 2 * KMAX + hb * KMAX, X.list0 + hb * P);
      items_chunk<2>(X, reinterpret_cast<const char*>(xs), X.hist0 + hb * KMAX,
                     X.hist0 + 2 * KMAX + hb * KMAX, X.list0 + hb * P, tq, k);
      pipe_release(R, stg);
    }
  }
  __syncthreads();
  items_flush<2>(p, X);
  if (nfb) atomicAdd((unsigned long long*)&st->fallback[1], (unsigned long long)nfb);
  if (!p.fuse_tail) return;
  if (!last_block(&st->ticket[1])) return;
  RUN_TAIL(tail_assign, 1);
#undef LAYK
}

// --- EvaluateCluster deviations (Alg 6 l.9-13, eq 9) / refinement X over
// CBest (Alg 1 l.16-17).  Each chunk is counting-sorted by cluster; every
// consumer thread owns a fixed set of work items (cell, residue r, stride
// R_i) for the whole launch, with R_i proportional to the cluster's size, so
// the members of cluster i are spread evenly over the R_i * |D_i| threads of
// its cells and each thread adds ~|members| / R_i exact int64 terms per chunk
// in a register (no shared-memory read-modify-write per term, no walk over
// ballot masks, no divergence from unequal |D_i|).
// REF = 0: cells (i, t < |D_i|) of |x_j - mu_ij|; REF = 1: cells (i, j < d)
// of |x_j - mbest_ij| plus |C_i|.
template <int REF>
__global__ void __launch_bounds__(416) k_lsum2(RunParams p) {
  DevState* st = p.st;
  if (!REF && st->done) return;
  extern __shared__ __align__(16) unsigned char smraw[];
  const SmemLayout& L = p.lay[REF ? KK_REF2 : KK_LS2];
  const int P = L.P, d = p.d, k = p.k;
  const int nw = L.nw, w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int nct = nw * 32;
  Pipe R = pipe_of(L, smraw, d);
  __shared__ int off_s[KMAX], nd_s[KMAX], rr_s[KMAX], ib_s[KMAX + 1];
  ItemCtx X = item_ctx(L, smraw, off_s, nd_s, rr_s, ib_s);
  const unsigned char* lab =
      REF ? (st->best_buf ? p.lab1 : p.lab0) : (st->cur_buf ? p.lab1 : p.lab0);
  const long long nmy = chunks_of_block_k(p, P);
  pipe_init_k(L, R);
  items_build<REF ? 1 : 0>(p, L, X);
  __syncthreads();
  if (w == nw) {
    pipe_produce_k(p, R, L, nmy, lab);
  } else {
    const int q = w * 32 + lane;
    long long g0 = (long long)blockIdx.x * P;
    const long long gstep = (long long)gridDim.x * P;
    RingPos rp;
    for (long long ch = 0; ch < nmy; ++ch, g0 += gstep, rp.next(L.stages)) {
      const int stg = rp.stg;
      const int hb = (int)(ch & 1);
      int* hist = X.hist0 + hb * KMAX;
      int* base_s = X.hist0 + 2 * KMAX + hb * KMAX;
      int* list = X.list0 + hb * P;
      mbar_wait(R.full_a + 8u * stg, rp.ph);
      sort_chunk(R.lab + (size_t)stg * P, p.n - g0, q, nct, k, hist, X.hist0 + (hb ^ 1) * KMAX,
                 base_s, list);
      items_chunk<REF ? 1 : 0>(X, reinterpret_cast<const char*>(R.buf + (size_t)stg * d * L.ldr),
                               hist, base_s, list, q, k);
      pipe_release(R, stg);
    }
  }
  __syncthreads();
  items_flush<REF ? 1 : 0>(p, X);
  if (!p.fuse_tail) return;
  if (!last_block(&st->ticket[REF ? 3 : 2])) return;
  if (REF) {
#define LAYK KK_REF2
    RUN_TAIL(tail_refine, 3);
#undef LAYK
  } else {
#define LAYK KK_LS2
    RUN_TAIL(tail_cost, 2);
#undef LAYK
  }
}


// --- EvaluateCluster (Alg 6, eq 9) with per-cluster sums.  The cost only
// needs, per cluster i, sum_{t < |D_i|} sum_{p in C_i} |x_pj - mu_ij| (the
// division by |C_i| of eq 1 cancels against the weight |C_i| of eq 2), so
// every term is quantised on its own at ONE scale 2^e_c (cost_qexp) and a
// point's |D_c| terms go into a lane-private int64 accumulator of its
// cluster (a shared-memory column per lane): no sort, no ballot, no barrier
// in the chunk loop, one table entry + one ring read + 4 DP ops per term.
// The integer totals do not depend on the order, the grid or the GPU count.
struct __align__(16) CItem {
  int joff;   // byte offset of dimension row j in a ring stage
  int pad;
  double cq;  // mu_ij * 2^e_c (exact: power-of-two scale)
};

// e_c = min e_j over the dimensions of D minus hb, 2^hb >= max |D_i|: one
// dimension's total stays < 2^(61 - hb) (proclus_api.cu), a cluster's sum
// over its <= 2^hb dimensions < 2^61, and one term < 2^51 (q_abs).  Block-
// wide (one cell per thread, shared-memory min / max); sc[j] = 2^(sgn e_j).
__device__ int cost_qexp(const double* sc, int sgn, const int* dl, const int* nD, int k, int d) {
  __shared__ int emin_s, ndmax_s;
  if (threadIdx.x == 0) {
    emin_s = 1 << 20;
    ndmax_s = 1;
  }
  __syncthreads();
  for (int e = threadIdx.x; e < k * d; e += blockDim.x) {
    const int i = e / d, t = e - i * d;
    if (t < nD[i]) atomicMin(&emin_s, sgn * ilogb(sc[dl[e]]));
    if (t == 0) atomicMax(&ndmax_s, nD[i]);
  }
  __syncthreads();
  const int r = emin_s - (32 - __clz(ndmax_s));
  __syncthreads();
  return r;
}

__global__ void __launch_bounds__(288) k_cost1(RunParams p) {
  DevState* st = p.st;
  extern __shared__ __align__(16) unsigned char smraw[];
  const SmemLayout& L = p.lay[KK_COST1];
#define LAYK KK_COST1
  const int P = p.P, d = p.d, k = p.k;
  const int nw = L.nw, w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const Pipe R = pipe_of(L, smraw, d);
  CItem* tab = SMP(CItem, tab);            // [k*l]: cluster c's items from off_s[c]
  int* nD_s = SMP(int, nD);
  int* off_s = SMP(int, off);
  long long* acc_s = SMP(long long, acc);  // [nw][k][32] lane-private columns
  const long long nmy = chunks_of_block(p);
  for (int e = threadIdx.x; e < nw * k * 32; e += blockDim.x) acc_s[e] = 0;
  pipe_init(p, R, nw);
  __syncthreads();
  if (st->done) return;
  const unsigned char* lab = st->cur_buf ? p.lab1 : p.lab0;
  for (int i = threadIdx.x; i < k; i += blockDim.x) nD_s[i] = st->nD[i];
  __syncthreads();
  if (k * d > 512) {  // compact item table (sum |D_i| = k l entries): frees shared memory
    if (threadIdx.x == 0) {
      int o = 0;
      for (int i = 0; i < k; ++i) {
        off_s[i] = o;
        o += nD_s[i];
      }
    }
  } else {
    for (int i = threadIdx.x; i < k; i += blockDim.x) off_s[i] = i * d;
  }
  const double sc = scalbn(1.0, cost_qexp(p.scale, 1, p.dlist, nD_s, k, d));
  for (int e = threadIdx.x; e < k * d; e += blockDim.x) {
    const int i = e / d, t = e - i * d;
    if (t < nD_s[i]) tab[off_s[i] + t] = CItem{p.dlist[e] * R.ldr * 4, 0, dmul(p.mu[e], sc)};
  }
  __syncthreads();
  if (w == nw) {
    pipe_produce(p, R, nmy, lab, nullptr);
  } else {
    long long* acc = acc_s + (size_t)w * k * 32 + lane;
    const int q = w * 32 + lane;
    long long gp = (long long)blockIdx.x * P + q;
    const long long gstep = (long long)gridDim.x * P;
    RingPos rp;
    for (long long i = 0; i < nmy; ++i, gp += gstep, rp.next(p.stages)) {
      const int stg = rp.stg;
      mbar_wait(R.full_a + 8u * stg, rp.ph);
      if (gp < p.n) {
        const int c = R.lab[(size_t)stg * P + q];
        const char* xq = reinterpret_cast<const char*>(R.buf + (size_t)stg * R.rows * R.ldr + q);
        const CItem* tb = tab + off_s[c];
        const int nd = nD_s[c];
        long long a0 = 0, a1 = 0;
        int t = 0;
        for (; t + 2 <= nd; t += 2) {
          const CItem e0 = tb[t], e1 = tb[t + 1];
          const float x0 = *reinterpret_cast<const float*>(xq + e0.joff);
          const float x1 = *reinterpret_cast<const float*>(xq + e1.joff);
          a0 += q_abs(x0, sc, e0.cq);
          a1 += q_abs(x1, sc, e1.cq);
        }
        if (t < nd) {
          const CItem e0 = tb[t];
          a0 += q_abs(*reinterpret_cast<const float*>(xq + e0.joff), sc, e0.cq);
        }
        acc[c * 32] += a0 + a1;
      }
      pipe_release(R, stg);
    }
  }
  __syncthreads();
  {  // per cluster: warps, then lanes; one atomic per block and cluster
    const int cp = blockIdx.x % NCOPY;
    for (int c = w; c < k; c += nw + 1) {
      long long s = 0;
      for (int ww = 0; ww < nw; ++ww) s += acc_s[((size_t)ww * k + c) * 32 + lane];
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
      if (lane == 0 && s)
        atomicAdd((unsigned long long*)&p.accg[(size_t)cp * k * d + c], (unsigned long long)s);
    }
  }
  if (!p.fuse_tail) return;
  if (!last_block(&st->ticket[2])) return;
  RUN_TAIL(tail_cost, 2);
#undef LAYK
}

// --- Final AssignPoints with D* (Alg 1 l.18) and RemoveOutliers (l.19):
// outlier iff seg_{D*_i}(x, m_i) > Delta_i for every i (reading R17).
template <int PPT>
__global__ void __launch_bounds__(160, 4) k_final(RunParams p) {
  DevState* st = p.st;
  extern __shared__ __align__(16) unsigned char smraw[];
  const SmemLayout& L = p.lay[KK_FIN];
  const int P = p.P, d = p.d, k = p.k;
  const int nw = L.nw, w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const Pipe R = pipe_of(L, smraw, d);
  float* med_s = SMP(float, med);
  Term* tab_s = SMP(Term, tab);
  int* dl_s = SMP(int, dl);
  int* nD_s = SMP(int, nD);
  float* rcp_s = SMP(float, rcp);
  double* Dl_s = SMP(double, Dl);
  const long long nmy = chunks_of_block(p);
  for (int i = threadIdx.x; i < k; i += blockDim.x) {
    nD_s[i] = st->nD[i];
    rcp_s[i] = 1.0f / (float)st->nD[i];
    Dl_s[i] = p.Delta[i];
  }
  for (int e = threadIdx.x; e < k * d; e += blockDim.x) {
    const int i = e / d;
    med_s[e] = p.mrows[(long long)st->mbest[i] * d + (e - i * d)];
    dl_s[e] = p.dlist[e];
  }
  pipe_init(p, R, nw);
  __syncthreads();
  for (int e = threadIdx.x; e < k * d; e += blockDim.x) {
    const int i = e / d, t = e - i * d;
    if (t < nD_s[i]) {
      const int j = dl_s[e];
      tab_s[e].joff = j * P * 4;
      tab_s[e].m = med_s[i * d + j];
      tab_s[e].m2 = med_s[i * d + j];
    }
  }
  __syncthreads();
  int ndmax = 0;
  for (int i = 0; i < k; ++i) ndmax = max(ndmax, nD_s[i]);
  const double G = (double)(ndmax + 6) * 5.9604644775390625e-08;
  // PPT == 2: clusters in groups of equal |D_c| (as k_assign) and fp32
  // certified thresholds of the outlier test seg <= Delta_c, rounded outwards
  __shared__ int ord_s[KMAX], gst_s[KMAX + 1], gnd_s[KMAX], ngrp_s;
  __shared__ float din_s[KMAX], dout_s[KMAX];
  if (PPT == 2 && threadIdx.x < 32) {
    const int c = lane;
    const int nd = c < k ? nD_s[c] : 1 << 30;
    int rank = 0;
    for (int o = 0; o < k; ++o) {
      const int no = nD_s[o];
      rank += (no < nd) | ((no == nd) & (o < c));
    }
    if (c < k) {
      ord_s[rank] = c;
      const double D = Dl_s[c];
      const bool ok = D >= 1e-30 && D < 1e30;
      din_s[c] = ok ? __double2float_rd(D * (1.0 - G)) : -1.0f;
      dout_s[c] = ok ? __double2float_ru(D * (1.0 + G)) : CUDART_INF_F;
    }
    __syncwarp();
    const int r = lane;
    const int ndr = r < k ? nD_s[ord_s[r]] : -1;
    const int ndp = __shfl_up_sync(0xffffffffu, ndr, 1);
    const bool head = r < k && (r == 0 || ndp != ndr);
    const unsigned hb = __ballot_sync(0xffffffffu, head);
    if (head) {
      const int g = __popc(hb & ((1u << lane) - 1u));
      gst_s[g] = r;
      gnd_s[g] = ndr;
    }
    if (lane == 0) {
      ngrp_s = __popc(hb);
      gst_s[__popc(hb)] = k;
    }
  }
  __syncthreads();
  long long nfb = 0;
  if (w == nw) {
    pipe_produce(p, R, nmy, nullptr, nullptr);
  } else if constexpr (PPT == 2) {
    // a lane owns the adjacent points q0 + 2 lane + u (packed terms)
    const int q0 = w * 64, ngrp = ngrp_s;
    RingPos rp;
    for (long long i = 0; i < nmy; ++i, rp.next(p.stages)) {
      const int stg = rp.stg;
      const long long base = (blockIdx.x + i * gridDim.x) * (long long)P;
      mbar_wait(R.full_a + 8u * stg, rp.ph);
      const float* xs = R.buf + (size_t)stg * R.rows * P;
      const float* xq = xs + q0 + 2 * lane;
      float best[2], second[2];
      int bi[2], out[2], und[2];
#pragma unroll
      for (int u = 0; u < 2; ++u) {
        best[u] = CUDART_INF_F;
        second[u] = CUDART_INF_F;
        bi[u] = 0;
        out[u] = 1;  // outside every sphere so far (certainly)
        und[u] = 0;  // some sphere test needs the exact value
      }
#define FIN_UPD(c, s)                                                      \
  do {                                                                     \
    const float r_ = rcp_s[c], in_ = din_s[c], ou_ = dout_s[c];            \
    _Pragma("unroll") for (int u = 0; u < 2; ++u) {                        \
      const float qv = (s)[u] * r_;                                        \
      second[u] = qv < best[u] ? best[u] : fminf(second[u], qv);           \
      bi[u] = qv < best[u] ? (c) : bi[u];                                  \
      best[u] = fminf(best[u], qv);                                        \
      const bool rng = qv >= 1e-30f && qv < 1e30f;                         \
      if (rng && qv < in_) out[u] = 0;                                     \
      else if (!(rng && qv > ou_)) und[u] = 1;                             \
    }                                                                      \
  } while (0)
      for (int g = 0; g < ngrp; ++g) {
        const int r0 = gst_s[g], r1 = gst_s[g + 1];
        switch (gnd_s[g]) {
#define DT(N)                                              \
  case N:                                                  \
    for (int r = r0; r < r1; ++r) {                        \
      const int c = ord_s[r];                              \
      float s[2];                                          \
      dist_terms2<N>(xq, tab_s + c * d, s);                \
      FIN_UPD(c, s);                                       \
    }                                                      \
    break;
          DT(1) DT(2) DT(3) DT(4) DT(5) DT(6) DT(7) DT(8)
          DT(9) DT(10) DT(11) DT(12) DT(13) DT(14) DT(15) DT(16)
#undef DT
          default:
            for (int r = r0; r < r1; ++r) {
              const int c = ord_s[r];
              float s[2];
              dist_terms2_n(xq, tab_s + c * d, gnd_s[g], s);
              FIN_UPD(c, s);
            }
        }
      }
#undef FIN_UPD
#pragma unroll
      for (int u = 0; u < 2; ++u) {
        const int q = q0 + 2 * lane + u;
        const long long gp = base + q;
        if (gp >= p.n) continue;
        const double b = (double)best[u], s2v = (double)second[u];
        const bool certain = (b >= 1e-30) && (s2v < 1e30) && (s2v * (1.0 - G) > b * (1.0 + G));
        int lbl = bi[u], o = out[u];
        if (!certain || (o && und[u])) {
          int outx = 0;
          lbl = exact_argmin(xs + q, P, med_s, dl_s, nD_s, k, d, Dl_s, &outx);
          if (o && und[u]) o = outx;
          ++nfb;
        }
        p.out_labels[gp] = o ? -1 : lbl;
      }
      pipe_release(R, stg);
    }
  } else {
    const int q0 = w * 32 * PPT;
    RingPos rp;
    for (long long i = 0; i < nmy; ++i, rp.next(p.stages)) {
      const int stg = rp.stg;
      const long long base = (blockIdx.x + i * gridDim.x) * (long long)P;
      mbar_wait(R.full_a + 8u * stg, rp.ph);
      const float* xs = R.buf + (size_t)stg * R.rows * P;
#pragma unroll
      for (int u = 0; u < PPT; ++u) {
        const int q = q0 + u * 32 + lane;
        const long long gp = base + q;
        if (gp >= p.n) continue;
        float best = CUDART_INF_F, second = CUDART_INF_F;
        int bi = 0;
        int out = 1;        // outside every sphere so far (certainly)
        int undecided = 0;  // some sphere test needs the exact value
        for (int c = 0; c < k; ++c) {
          const int nd = nD_s[c];
          const Term* tb = tab_s + c * d;
          float s = 0.f, s2 = 0.f;
          int t = 0;
          for (; t + 2 <= nd; t += 2) {
            s += fabsf(LDX(xs + q, tb[t].joff) - tb[t].m);
            s2 += fabsf(LDX(xs + q, tb[t + 1].joff) - tb[t + 1].m);
          }
          if (t < nd) s += fabsf(LDX(xs + q, tb[t].joff) - tb[t].m);
          const float qv = (s + s2) * rcp_s[c];
          if (qv < best) {
            second = best;
            best = qv;
            bi = c;
          } else if (qv < second) {
            second = qv;
          }
          const int le = cert_le(qv, Dl_s[c], G);  // seg <= Delta_c ?
          if (le == 1) out = 0;
          if (le < 0) undecided = 1;
        }
        const double b = (double)best, s2v = (double)second;
        const bool certain =
            (b >= 1e-30) && (s2v < 1e30) && (s2v * (1.0 - G) > b * (1.0 + G));
        int lbl = bi;
        if (!certain || (out && undecided)) {
          int outx = 0;
          lbl = exact_argmin(xs + q, P, med_s, dl_s, nD_s, k, d, Dl_s, &outx);
          if (out && undecided) out = outx;
          ++nfb;
        }
        p.out_labels[gp] = out ? -1 : lbl;
      }
      pipe_release(R, stg);
    }
  }
  if (nfb) atomicAdd((unsigned long long*)&st->fallback[2], (unsigned long long)nfb);
}

// ============================================================ multi-GPU tail
__global__ void __launch_bounds__(1024, 1) k_tail(RunParams p, int tail) {
  extern __shared__ __align__(16) unsigned char smraw[];
  DevState* st = p.st;
  if (tail != TAIL_REF && st->done) return;
  TailMem T = tail_mem(p, smraw);
  TST_START();
  if (tail == TAIL_LOC)
    tail_locality(p, T);
  else if (tail == TAIL_ASG)
    tail_assign(p, T);
  else if (tail == TAIL_COST)
    tail_cost(p, T);
  else
    tail_refine(p, T);
  state_store(p, T.S);
}

void launch_tail(const RunParams& p, int tail, cudaStream_t s) {
  k_tail<<<1, 1024, p.tail_smem, s>>>(p, tail);
}

// ============================================================ shapes
// Chunk P = 32 * PPT * NW points.  d <= 32: P = 256 (locality / labelsum 8
// consumer warps x 1 point per lane, assign / final 4 warps x 2 points);
// larger d: P = 128 or 64 so that the ring of (d + k) rows stays small.
struct LB {
  size_t off = 0;
  int take(size_t bytes) {
    off = (off + 15) & ~(size_t)15;
    const int r = (int)off;
    off += bytes;
    return r;
  }
};

static SmemLayout blank_layout() {
  SmemLayout L;
  int* q = reinterpret_cast<int*>(&L);
  for (size_t i = 0; i < sizeof(L) / sizeof(int); ++i) q[i] = -1;  // -1 = unused
  return L;
}

static TailLayout tail_layout(int d, int k, int nM) {
  TailLayout t;
  LB b;
  const size_t kd = (size_t)k * d;
  t.S = b.take(sizeof(DevState));
  t.X = b.take(8 * kd);
  t.Z = b.take(8 * kd);
  t.med = b.take(8 * kd);
  t.dev = b.take(8 * kd);
  t.dm = b.take(kd);
  t.pool = b.take(4 * (size_t)(nM > 0 ? nM : 1));
  t.fnd = b.take(8 * 3 * KMAX);
  t.isc = b.take(8 * (size_t)d);
  t.dl = b.take(4 * kd);
  t.dd = b.take(8 * (size_t)k * k);
  // the cost tail caches M (fp32 rows + DistFound / delta' tables) when small
  const size_t m = (size_t)(nM > 0 ? nM : 1);
  LB c = b;
  const int mrow = c.take(4 * m * d), fall = c.take(m), uall = c.take(m), pall = c.take(8 * m);
  if (c.off <= 40 * 1024) {
    b = c;
    t.mrow = mrow;
    t.fall = fall;
    t.uall = uall;
    t.pall = pall;
  } else {
    t.mrow = t.fall = t.uall = t.pall = -1;
  }
  t.bytes = (int)((b.off + 15) & ~(size_t)15);
  return t;
}

static thread_local bool g_split_tails = false;  // set by pass_shape (per thread) before the layouts are built
static void finish(SmemLayout& L, LB& b, const TailLayout& tl) {
  L.tail = L.buf;
  size_t end = b.off;
  if (!g_split_tails && (size_t)L.tail + tl.bytes > end) end = (size_t)L.tail + tl.bytes;
  L.bytes = (int)((end + 64 + 15) & ~(size_t)15);
}

PassShape pass_shape(int d, int k, int l, int nM, int num_sms) {
  PassShape ps;
  memset(&ps, 0, sizeof(ps));  // padding too: the graph cache compares it bytewise
  int P = 256, stages = 3;
  const int cfg[6][2] = {{256, 3}, {256, 2}, {128, 3}, {128, 2}, {64, 3}, {64, 2}};
  for (int c = 0; c < 6; ++c) {
    P = cfg[c][0];
    stages = cfg[c][1];
    if ((size_t)stages * (d + k) * P * 4 <= 60 * 1024) break;
  }
  ps.P = P;
  ps.stages = stages;
  // consumer warps at 1 point per lane (locality, cost, refinement) and at
  // PPT2 points per lane (assign, final): 2, or 1 when the chunk is short
  // (large d) so that a block keeps at least two consumer warps
  const int ppt2 = P >= 128 ? 2 : 1;
  const int nw1 = P / 32, nw2 = P / (32 * ppt2);
  ps.ppt2 = ppt2;
  ps.tpb_loc = 32 * ((d <= 16 ? nw1 / LOC16_PPT : LOCW_NW) + 1);
  ps.tpb_asg = 32 * (nw2 + 1);  // updated below when assign takes 2 P
  ps.tpb_lsum = 32 * (nw1 + 1);
  ps.tpb_fin = 32 * (nw2 + 1);
  const size_t kd = (size_t)k * d;
  ps.tl = tail_layout(d, k, nM);
  ps.tail_smem = ps.tl.bytes;
  // large k d: the single-block tails (radix selection over k d
  // cells, k^2 medoid distances) run as 1024-thread kernels of their own, and
  // the pass kernels do not reserve shared memory for them
  ps.split_tails = kd > 512 ? 1 : 0;
  g_split_tails = ps.split_tails != 0;
  {  // locality
    SmemLayout L = blank_layout();
    LB b;
    // d <= 16: LOC16_PPT points per lane (k_locality<16>); d > 16: LOCW_NW
    // consumer warps share each chunk (locw_consume)
    const int nwl = d <= 16 ? nw1 / LOC16_PPT : LOCW_NW;
    L.nw = nwl;
    L.P = P;
    // rows padded by 4 floats so that the lane-per-dimension band sums of
    // k_locality read a point's coordinates with at most 2- (d <= 16) or
    // 4-way bank conflicts
    L.ldr = P + 4;
    L.full = b.take(8 * SMAX);
    L.empty = b.take(8 * SMAX);
    // >= 16 rows: k_locality<16> loads rows 0..15 of every stage unconditionally
    L.buf = b.take((size_t)stages * ((d <= 16 ? 16 : d) + k) * L.ldr * 4);
    L.med = b.take(4 * (size_t)k * (d < 32 ? 32 : d));  // rows padded to 16 / 32
    L.act = b.take(sizeof(ActSlot) * KMAX);
    L.row = b.take(4 * KMAX);
    L.scale = b.take(8 * (size_t)d);
    L.bal = b.take(4 * (size_t)nwl * KMAX);
    L.acc = b.take(8 * (size_t)(d <= 16 ? nwl : 1) * kd);  // wide: one shared copy
    L.cnt = b.take(8 * (size_t)nwl * KMAX);
    L.ex = b.take(sizeof(ExtraRows));
    L.thr = b.take(sizeof(Thr) * KMAX);
    if (d <= 16) {
      L.ctr = b.take(8 * (size_t)k * 16);        // fp64 medoid rows of the d <= 16 consumer
      L.tab = b.take((size_t)nw1 * 32);          // per-warp member lists (32 PPT points)
    } else {
      L.tab = b.take((size_t)stages * KMAX * P);  // per-stage member lists of (slot, block)
      L.dl = b.take(4 * (size_t)stages * KMAX * 8);  // their lengths (P <= 256: 8 blocks)
    }
    finish(L, b, ps.tl);
    ps.lay[KK_LOC] = L;
  }
  // assign: short chunks (ppt2 == 1, long rows) run chunks of 2 P points with
  // 4 consumer warps sharing one accumulator copy, when that fits (the
  // per-block cluster tables dominate the shared memory at large k d)
  auto asg_layout = [&](int Pa) {
    const int nwa = Pa / (32 * ppt2);
    const int imax = 32 * nwa + (int)kd;  // items: sum_i |D_i| R_i <= threads + cells
    SmemLayout L = blank_layout();
    LB b;
    L.nw = nwa;
    L.P = Pa;
    L.ldr = Pa;
    L.full = b.take(8 * SMAX);
    L.empty = b.take(8 * SMAX);
    L.buf = b.take((size_t)stages * d * Pa * 4);
    L.med = b.take(4 * kd);
    L.tab = b.take(sizeof(Term) * kd);
    L.dl = b.take(4 * kd);
    L.nD = b.take(4 * KMAX);
    L.rcp = b.take(4 * KMAX);
    L.cells = b.take(sizeof(Item) * (size_t)imax);  // centroid items
    L.acc = b.take(8 * (size_t)imax);               // their int64 sums
    L.ctr = b.take(4 * kd);                         // cell -> accumulator index
    L.bal = b.take(4 * 4 * KMAX);                   // histograms + bases (double buffer)
    L.row = b.take(4 * 2 * (size_t)Pa);             // sorted chunk points (double buffer)
    L.cnt = b.take(8 * KMAX);                       // |C_i| of the block
    finish(L, b, ps.tl);
    return L;
  };
  ps.P_asg = P;
  ps.lay[KK_ASG] = asg_layout(P);
  ps.asg_w = 0;
  if (ppt2 == 1) {  // long rows: k_assign_w, ASW_NW consumer warps share a chunk
    SmemLayout L = blank_layout();
    LB b;
    const int kl = k * l;
    L.nw = ASW_NW;
    L.P = P;
    L.ldr = P + 4;  // phase C lanes read different rows of one column: <= 4-way conflicts
    L.full = b.take(8 * SMAX);
    L.empty = b.take(8 * SMAX);
    L.buf = b.take((size_t)stages * d * L.ldr * 4);
    L.med = b.take(4 * kd);
    L.tab = b.take(sizeof(Term) * (size_t)kl);
    L.dl = b.take(4 * kd);
    L.nD = b.take(4 * KMAX);
    L.off = b.take(4 * (KMAX + 1));
    L.rcp = b.take(4 * KMAX);
    L.scale = b.take(8 * (size_t)d);
    L.cells = b.take(sizeof(Cell) * (size_t)kl);
    L.bal = b.take(4 * (size_t)KMAX * (P / 32));
    L.acc = b.take(8 * kd);
    L.cnt = b.take(8 * (size_t)ASW_NW * KMAX);
    L.row = b.take(sizeof(Part) * (size_t)(ASW_NW / (P / 32)) * P);
    finish(L, b, ps.tl);
    ps.lay[KK_ASG] = L;
    ps.asg_w = 1;
  }
  {  // labelsum (cost / refinement X)
    SmemLayout L = blank_layout();
    LB b;
    L.nw = nw1;
    L.P = P;
    L.ldr = P;
    L.full = b.take(8 * SMAX);
    L.empty = b.take(8 * SMAX);
    L.buf = b.take((size_t)stages * d * P * 4);
    L.lab = b.take((size_t)stages * P);
    L.ctr = b.take(8 * kd);
    L.dl = b.take(4 * kd);
    L.nD = b.take(4 * KMAX);
    L.off = b.take(4 * (KMAX + 1));
    L.scale = b.take(8 * (size_t)d);
    L.cells = b.take(sizeof(Cell) * kd);
    L.bal = b.take(4 * (size_t)nw1 * KMAX);
    L.acc = b.take(8 * (size_t)nw1 * kd);
    L.cnt = b.take(8 * (size_t)nw1 * KMAX);
    finish(L, b, ps.tl);
    ps.lay[KK_LSUM] = L;
  }
  {  // final
    SmemLayout L = blank_layout();
    LB b;
    L.nw = nw2;
    L.P = P;
    L.ldr = P;
    L.full = b.take(8 * SMAX);
    L.empty = b.take(8 * SMAX);
    L.buf = b.take((size_t)stages * d * P * 4);
    L.med = b.take(4 * kd);
    L.tab = b.take(sizeof(Term) * kd);
    L.dl = b.take(4 * kd);
    L.nD = b.take(4 * KMAX);
    L.rcp = b.take(4 * KMAX);
    L.Dl = b.take(8 * KMAX);
    finish(L, b, ps.tl);
    ps.lay[KK_FIN] = L;
  }
  // lane-private accumulator passes (k_lsum2): the most consumer warps whose
  // accumulators [nw][cells][32] int64 fit next to the ring
  // sorted-member passes (k_lsum2): 12 consumer warps, chunks of 384 points,
  // ring rows padded by 4 floats (conflict-free row gathers)
  auto ls2_layout = [&](int ncell, int& nw_out, size_t cap) -> SmemLayout {
    SmemLayout best = blank_layout();
    nw_out = 0;
    for (int nw = 12; nw >= 4; nw -= 4) {
      for (int stg = 3; stg >= 2; --stg) {
        const int Pk = 32 * nw;
        const int imax = 32 * nw + ncell;  // sum_i |D_i| R_i <= lanes + cells
        SmemLayout L = blank_layout();
        LB b;
        L.nw = nw;
        L.P = Pk;
        L.ldr = Pk + 4;
        L.stages = stg;
        L.full = b.take(8 * SMAX);
        L.empty = b.take(8 * SMAX);
        L.buf = b.take((size_t)stg * d * (Pk + 4) * 4);
        L.lab = b.take((size_t)stg * Pk);
        L.tab = b.take(sizeof(Item) * (size_t)imax);
        L.acc = b.take(8 * (size_t)imax);
        L.nD = b.take(4 * kd);
        L.bal = b.take(4 * 4 * KMAX);
        L.row = b.take(4 * 2 * (size_t)Pk);
        L.cnt = b.take(8 * KMAX);
        finish(L, b, ps.tl);
        if ((size_t)L.bytes <= cap) {
          nw_out = nw;
          return L;
        }
      }
    }
    return best;
  };
  {
    int nw = 0;
    ps.lay[KK_LS2] = ls2_layout(k * l, nw, 110 * 1024);  // the cost cells: sum |D_i| = k*l
    ps.lsum2 = nw >= 4;
    ps.tpb_ls2 = 32 * (nw + 1);
    ps.smem_ls2 = ps.lsum2 ? ps.lay[KK_LS2].bytes : 0;
    // refinement: two blocks per SM when they fit, else one block with the
    // largest layout under the opt-in limit (long rows, many cells: C4)
    ps.lay[KK_REF2] = ls2_layout((int)kd, nw, 110 * 1024);
    if (nw < 4) ps.lay[KK_REF2] = ls2_layout((int)kd, nw, 220 * 1024);
    ps.ref2 = nw >= 4;
    ps.tpb_ref2 = 32 * (nw + 1);
    ps.smem_ref2 = ps.ref2 ? ps.lay[KK_REF2].bytes : 0;
  }
  {  // per-cluster cost pass (k_cost1): lane-private columns [nw][k][32]
    SmemLayout L = blank_layout();
    LB b;
    L.nw = nw1;
    L.P = P;
    L.ldr = P;  // a lane reads its own point: conflict-free whatever the row
    L.full = b.take(8 * SMAX);
    L.empty = b.take(8 * SMAX);
    L.buf = b.take((size_t)stages * d * P * 4);
    L.lab = b.take((size_t)stages * P);
    L.tab = b.take(sizeof(CItem) * (kd > 512 ? (size_t)k * l : kd));  // compact at large k d
    L.nD = b.take(4 * KMAX);
    L.off = b.take(4 * (KMAX + 1));
    L.acc = b.take(8 * (size_t)L.nw * k * 32);
    finish(L, b, ps.tl);
    ps.lay[KK_COST1] = L;
    ps.cost1 = L.bytes <= 200 * 1024;
    ps.tpb_cost1 = 32 * (L.nw + 1);
    ps.smem_cost1 = ps.cost1 ? L.bytes : 0;
  }
  ps.smem_loc = ps.lay[KK_LOC].bytes;
  ps.smem_asg = ps.lay[KK_ASG].bytes;
  ps.tpb_asg = 32 * (ps.lay[KK_ASG].nw + 1);
  ps.smem_cost = ps.lay[KK_LSUM].bytes;
  ps.smem_ref = ps.smem_cost;
  ps.smem_fin = ps.lay[KK_FIN].bytes;
  // persistent grids: as many resident blocks per SM as shared memory and
  // the 2048-thread limit and the register file allow (<= 8), per kernel, so
  // that the whole grid is one resident wave
  auto grid_of = [&](const void* fn, size_t smem, int tpb) {
    cudaFuncAttributes fa;
    size_t stat = 0;
    int regs = 0;
    if (cudaFuncGetAttributes(&fa, fn) == cudaSuccess) {
      stat = fa.sharedSizeBytes;
      regs = fa.numRegs;
    } else {
      cudaGetLastError();
    }
    int per_sm = (int)((227 * 1024) / (smem + stat + 1024));
    if (per_sm > 2048 / tpb) per_sm = 2048 / tpb;
    if (regs > 0) {
      const int warp_regs = ((regs * 32 + 255) / 256) * 256;
      const int by_regs = 65536 / (warp_regs * ((tpb + 31) / 32));
      if (per_sm > by_regs) per_sm = by_regs;
    }
    if (per_sm > 8) per_sm = 8;
    if (per_sm < 1) per_sm = 1;
    return num_sms * per_sm;
  };
  const void* loc_fn = d <= 16 ? (const void*)k_locality<16>
                       : d <= 32 ? (const void*)k_locality<32>
                                 : (const void*)k_locality<0>;
  ps.grid_loc = grid_of(loc_fn, ps.smem_loc, ps.tpb_loc);
  ps.grid_asg = grid_of(ppt2 == 2 ? (const void*)k_assign<2> : (const void*)k_assign_w,
                        ps.smem_asg, ps.tpb_asg);
  ps.grid_lsum = grid_of((const void*)k_labelsum<0>, ps.smem_cost, ps.tpb_lsum);
  ps.grid_fin = grid_of(ppt2 == 2 ? (const void*)k_final<2> : (const void*)k_final<1>,
                        ps.smem_fin, ps.tpb_fin);
  ps.grid_ls2 = ps.lsum2 ? grid_of((const void*)k_lsum2<0>, ps.smem_ls2, ps.tpb_ls2) : 0;
  ps.grid_ref2 = ps.ref2 ? grid_of((const void*)k_lsum2<1>, ps.smem_ref2, ps.tpb_ref2) : 0;
  ps.grid_cost1 = ps.cost1 ? grid_of((const void*)k_cost1, ps.smem_cost1, ps.tpb_cost1) : 0;
  ps.grid = ps.grid_loc;
  ps.per_sm = ps.grid_loc / num_sms;
  return ps;
}

// The dynamic shared-memory opt-in is a process-wide attribute of a kernel
// (per device).  Handles of different shapes may run concurrently from
// different threads, so the attribute only ever grows: each (device, kernel)
// is raised to the largest size any handle has needed, under a mutex.
static std::mutex g_attr_mu;
static std::map<std::pair<int, const void*>, int> g_attr_max;

static cudaError_t raise_smem(int dev, const void* fn, size_t bytes) {
  const int want = (int)bytes;
  auto& cur = g_attr_max[{dev, fn}];
  if (cur == 0) {
#ifdef SMEM_CARVEOUT
    // one L1 / shared-memory split for every pass kernel: no carve-out
    // reconfiguration between consecutive kernels of an iteration
    const cudaError_t ec = cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout,
                                                cudaSharedmemCarveoutMaxShared);
    if (ec != cudaSuccess) return ec;
#endif
    cur = -1;
  }
  if (want <= cur) return cudaSuccess;
  const cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, want);
  if (e == cudaSuccess) cur = want;
  return e;
}

cudaError_t configure_kernels(const PassShape& ps) {
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  std::lock_guard<std::mutex> lk(g_attr_mu);
  const void* fns[] = {(const void*)k_locality<16>, (const void*)k_locality<32>,
                       (const void*)k_locality<0>,  (const void*)k_assign<2>,
                       (const void*)k_labelsum<0>,  (const void*)k_labelsum<1>,
                       (const void*)k_final<2>,     (const void*)k_prepare,
                       (const void*)k_tail,         (const void*)k_assign_w,
                       (const void*)k_final<1>};
  const size_t sm[] = {ps.smem_loc,  ps.smem_loc, ps.smem_loc,   ps.smem_asg, ps.smem_cost,
                       ps.smem_ref,  ps.smem_fin, (size_t)ps.tail_smem, (size_t)ps.tail_smem,
                       ps.smem_asg,  ps.smem_fin};
  for (int i = 0; i < 11; ++i)
    if ((e = raise_smem(dev, fns[i], sm[i])) != cudaSuccess) return e;
  if (ps.lsum2 && (e = raise_smem(dev, (const void*)k_lsum2<0>, ps.smem_ls2)) != cudaSuccess)
    return e;
  if (ps.ref2 && (e = raise_smem(dev, (const void*)k_lsum2<1>, ps.smem_ref2)) != cudaSuccess)
    return e;
  if (ps.cost1 && (e = raise_smem(dev, (const void*)k_cost1, ps.smem_cost1)) != cudaSuccess)
    return e;
  return cudaSuccess;
}

void launch_locality(const RunParams& p, const PassShape& ps, cudaStream_t s) {
  if (p.d <= 16)
    k_locality<16><<<ps.grid_loc, ps.tpb_loc, ps.smem_loc, s>>>(p);
  else if (p.d <= 32)
    k_locality<32><<<ps.grid_loc, ps.tpb_loc, ps.smem_loc, s>>>(p);
  else
    k_locality<0><<<ps.grid_loc, ps.tpb_loc, ps.smem_loc, s>>>(p);
}
void launch_assign(const RunParams& p, const PassShape& ps, cudaStream_t s) {
  if (ps.ppt2 == 2)
    k_assign<2><<<ps.grid_asg, ps.tpb_asg, ps.smem_asg, s>>>(p);
  else
    k_assign_w<<<ps.grid_asg, ps.tpb_asg, ps.smem_asg, s>>>(p);
}
void launch_cost(const RunParams& p, const PassShape& ps, cudaStream_t s) {
  if (ps.cost1)
    k_cost1<<<ps.grid_cost1, ps.tpb_cost1, ps.smem_cost1, s>>>(p);
  else if (ps.lsum2)
    k_lsum2<0><<<ps.grid_ls2, ps.tpb_ls2, ps.smem_ls2, s>>>(p);
  else
    k_labelsum<0><<<ps.grid_lsum, ps.tpb_lsum, ps.smem_cost, s>>>(p);
}
void launch_refine_x(const RunParams& p, const PassShape& ps, cudaStream_t s) {
  if (ps.ref2)
    k_lsum2<1><<<ps.grid_ref2, ps.tpb_ref2, ps.smem_ref2, s>>>(p);
  else
    k_labelsum<1><<<ps.grid_lsum, ps.tpb_lsum, ps.smem_ref, s>>>(p);
}
void launch_final(const RunParams& p, const PassShape& ps, cudaStream_t s) {
  if (ps.ppt2 == 2)
    k_final<2><<<ps.grid_fin, ps.tpb_fin, ps.smem_fin, s>>>(p);
  else
    k_final<1><<<ps.grid_fin, ps.tpb_fin, ps.smem_fin, s>>>(p);
}

}  // namespace pc

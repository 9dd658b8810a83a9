// proclus_device.cuh -- device-side state, parameters and exact-arithmetic
// helpers of the B200 PROCLUS hot path.  Citations: /root/reference/PAPER.md
// line numbers (P:<n>); readings [Rn] are listed in DESIGN.md section 3.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

namespace pc {

constexpr int KMAX = 32;    // k <= 32: per-point medoid membership is a u32
constexpr int TPB_MAX = 1024;  // threads of the standalone tail kernels
constexpr int WMAX = 8;     // warps per pass block
constexpr int UMAX = 4;     // points per thread in a chunk
constexpr int SMAX = 3;     // max bulk-copy ring depth
#ifndef PROCLUS_NCOPY
#define PROCLUS_NCOPY 2
#endif
constexpr int NCOPY = PROCLUS_NCOPY;  // copies of the global accumulators (atomic spread; 2: the
                                      // tails load fewer copies, 1 serialises the cost flush)
constexpr int PAD_ALIGN = 1024;  // n_pad multiple; shard boundaries for invariance

// One medoid slot whose locality set changes in this iteration
// (GPU-FAST-PROCLUS).  The band is (lo, hi]: Theorem 3.1 / eq 3.
constexpr int ERR_NONFINITE = 7;  // DevState::err: non-finite data (asynchronous load)

struct ActSlot {
  int slot;      // cluster slot i in MCur
  int mpos;      // MIdx_i: position in M: the medoid's row of M
  int key;       // cache row of Dist / H / |L| / delta': mpos (FAST) or slot (FAST*)
  int compute;   // 1: DistFound is false -> compute and store the Dist row
  int lam;       // lambda_i (eq 6): +1 grow, -1 shrink
  double lo, hi; // band (lo, hi]; lo = -inf on first use (L_i itself)
};

// Mutable control state of one run, resident in device memory so that the
// whole iterative phase (Alg 1 l.5-14) is decided on the GPU.
struct DevState {
  unsigned long long rng;       // stream IT (reading R2), device copy
  int mcur[KMAX];               // MCur as positions into M
  int mbest[KMAX];              // MBest
  long long sizes[KMAX];        // |C_i| of the current clustering
  long long sizes_best[KMAX];   // |C_i| of CBest
  double delta[KMAX];           // delta_i
  double cost, cost_best;
  int itr, iterations, done, cur_buf, best_buf, improved;
  int n_act;
  ActSlot act[KMAX];
  int nD[KMAX];                 // |D_i|
  int cown[KMAX];               // FAST*: M position cached in slot i's rows (-1: none)
  unsigned int ticket[4];       // last-block tickets of the pass kernels
  int err;
  double bytes_loc;             // algorithmic bytes of the locality passes
  long long fallback[4];        // exact fp64 re-decisions (loc, asg, fin, -)
  unsigned long long tail_ns[4];  // %globaltimer time in the single-block tails
  unsigned long long dbg_cyc[24];  // per-phase SM cycles of the tails (PROCLUS_TAIL_PROFILE builds)
  unsigned long long dbg_t[8];     // k_locality phase times of the current launch (profile builds)
  unsigned long long dbg_ts[8];    // their sums over the run, ns after the first block's entry
};

struct TraceBufs {
  int cap;
  int* mcur;
  double* delta;
  long long* nL;
  unsigned char* dims;
  long long* sizes;
  double* cost;
  unsigned char* improved;
  unsigned char* bad;
  double* X;
};

// Byte offsets into a pass kernel's dynamic shared memory, computed on the
// host (fixed offsets: no pointer arithmetic re-done inside the hot loops).
struct SmemLayout {
  int full, empty, buf, lab;                    // TMA ring and its mbarriers
  int med, act, row, scale, cells, bal, acc, cnt, ex;
  int tab, dl, nD, off, rcp, ctr, Dl, thr;
  int P, ldr, stages;  // chunk points, ring row stride (floats), ring depth (k_lsum2 etc.)
  int tail;      // start of the tail scratch (reuses the ring region)
  int bytes;     // total dynamic shared memory of the kernel
  int nw;        // consumer warps
};
// Offsets (relative to SmemLayout::tail) of the single-block tail's scratch.
struct TailLayout {
  int S, X, Z, med, dev, dm, pool, fnd, isc, dl, dd;
  int mrow, fall, uall, pall;  // rows of M and their tables, or mrow = -1
  int bytes;
};
enum KernelKind { KK_LOC = 0, KK_ASG = 1, KK_LSUM = 2, KK_FIN = 3, KK_LS2 = 4, KK_REF2 = 5, KK_COST1 = 6 };
constexpr int NLAY = 7;

struct RunParams {
  long long n;        // rows on this device
  long long n_pad;    // padded row count of the SoA layout (multiple of PAD_ALIGN)
  long long n_total;  // |Data| (all ranks): threshold of P:91 and eq 8
  int d, k, l, nM, itrPat, max_iter, metric;
  double minDev;
  const float* xs;         // data, SoA [d][n_pad] fp32
  const float* mrows;      // rows of M [nM][d] fp32
  float* dist;             // Dist cache [nM][n_pad] fp32, certified values
  unsigned char* lab0;     // label buffers (current / best, swapped by index)
  unsigned char* lab1;
  long long* Hq;           // [nM][d] H of eq 5 in fixed point (scale 2^e_j)
  double* dprev;           // [nM] delta' of the previous use
  long long* nL;           // [nM] |L|
  unsigned char* found;    // [nM] DistFound
  unsigned char* used;     // [nM] delta' valid
  double* med;             // [k][d] current (or best) medoid rows, fp64
  int* dlist;              // [k][d] D_i as ascending dimension lists
  unsigned char* dmask;    // [k][d]
  double* X;               // [k][d]
  double* Z;               // [k][d] scratch
  double* mu;              // [k][d] centroid on D_i, index (i, t)
  long long* accg;         // [NCOPY][k*d] global fixed-point cell sums (atomics)
  long long* cntg;         // [NCOPY][KMAX] global counts
  const double* scale;     // [d] 2^e_j   (fixed-point scale of dimension j)
  const double* iscale;    // [d] 2^-e_j
  int* pool;               // [nM] scratch of the replacement step
  DevState* st;
  int P;                   // points per chunk (threads per block = P / PPT)
  int stages;              // ring depth (2 or 3)
  long long nchunks;
  int fuse_tail;           // 1: last block finalises (single GPU)
  int cost1;               // 1: the cost pass sums per cluster (k_cost1), cells 0..k-1
  const int* qflag;        // device: 1 = band sums of <= 256 terms stay below 2^51 at 2^e_j
  const int* badflag;      // device: 1 = the loaded data has a non-finite value
  int variant;             // proclus_variant: 0 FAST, 1 plain (no caches), 2 FAST*
  int use_cond;            // 1: running inside a graph while-node
  unsigned long long cond; // cudaGraphConditionalHandle
  TraceBufs tr;
  int* out_labels;         // final labels [n] int32 (refinement)
  double* Delta;           // [k] outlier radii
  SmemLayout lay[NLAY];    // per KernelKind
  TailLayout tl;
  int tail_smem;           // dynamic smem of the standalone tail kernels
};

// ---- exact fp64 arithmetic: explicit round-to-nearest intrinsics so that
// nvcc never contracts into FMA; every expression below repeats the
// oracle's evaluation order (ascending j, left-to-right).
__device__ __forceinline__ double dadd(double a, double b) { return __dadd_rn(a, b); }
__device__ __forceinline__ double dsub(double a, double b) { return __dsub_rn(a, b); }
__device__ __forceinline__ double dmul(double a, double b) { return __dmul_rn(a, b); }
__device__ __forceinline__ double ddiv(double a, double b) { return __ddiv_rn(a, b); }

// Full-space distance ||p - q||: L2 = sqrt(sum_j (p_j - q_j)^2), L1
// = sum_j |p_j - q_j|, j ascending.  p has stride ps, q stride 1.
template <class TP, class TQ>
__device__ __forceinline__ double full_dist(const TP* p, int ps, const TQ* q, int d,
                                            int metric) {
  double s = 0.0;
  if (metric == 1) {
    for (int j = 0; j < d; ++j) s = dadd(s, fabs(dsub((double)p[j * ps], (double)q[j])));
    return s;
  }
  for (int j = 0; j < d; ++j) {
    double t = dsub((double)p[j * ps], (double)q[j]);
    s = dadd(s, dmul(t, t));
  }
  return __dsqrt_rn(s);
}

// SplitMix64 (reading R2), the library's own device implementation.
__device__ __forceinline__ unsigned long long sm64_next(unsigned long long* s) {
  unsigned long long z = (*s += 0x9E3779B97F4A7C15ULL);
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}
__device__ __forceinline__ unsigned long long sm64_uniform(unsigned long long* s,
                                                           unsigned long long m) {
  return __umul64hi(sm64_next(s), m);
}

// Order-preserving u64 key of a double (non-NaN); -0 is folded to +0 first.
__device__ __forceinline__ unsigned long long sortable_key(double z) {
  z = dadd(z, 0.0);
  unsigned long long u = (unsigned long long)__double_as_longlong(z);
  return (u >> 63) ? ~u : (u | 0x8000000000000000ULL);
}

}  // namespace pc

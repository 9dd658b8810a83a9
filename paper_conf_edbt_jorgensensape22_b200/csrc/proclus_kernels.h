// proclus_kernels.h -- host-side launchers of the sm_100a kernels
// (implemented in proclus_kernels.cu, called by the C ABI in proclus_api.cu).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include "proclus_device.cuh"

namespace pc {

struct PassShape {
  int P;          // points per chunk
  int stages;     // bulk-copy ring depth
  int tpb_loc, tpb_asg, tpb_lsum, tpb_fin;  // threads per block of each pass
  int ppt2;       // points per lane of assign / final (2, or 1 for short chunks)
  int P_asg;      // points per chunk of assign (2 P when ppt2 == 1 and it fits)
  int per_sm;     // resident blocks per SM (locality)
  int grid;       // persistent blocks (SM count x per_sm)
  int grid_loc, grid_asg, grid_lsum, grid_fin;  // per kernel
  size_t smem_loc, smem_asg, smem_cost, smem_ref, smem_fin;
  SmemLayout lay[NLAY];  // per KernelKind
  int lsum2, ref2;       // 1: lane-private accumulator passes (k_lsum2) fit in shared memory
  int cost1;             // 1: per-cluster cost pass (k_cost1)
  int grid_cost1, tpb_cost1;
  size_t smem_cost1;
  int grid_ls2, grid_ref2, tpb_ls2, tpb_ref2;
  size_t smem_ls2, smem_ref2;
  TailLayout tl;
  int tail_smem;
  int split_tails;       // 1: the single-block tails run as kernels of their own (k d > 512)
  int asg_w;             // 1: long rows, k_assign_w (ASW_NW warps share a chunk)
};

// N0: row-major [n][d] -> SoA [d][n_pad]; *bad |= 1 on a non-finite value;
// colmax[j] = max(colmax[j], bits of max |x_j|).  colmax holds PACK_COPIES x d
// words, all zero on entry; copies 1.. are scratch (partial maxima).
constexpr int PACK_COPIES = 32;
void launch_pack_soa(const float* in, long long n, int d, long long n_pad, float* xs, int* bad,
                     unsigned* colmax, cudaStream_t s);
// 2^e_j, 2^-e_j and the quant_sum fma flag from max |x_j| on the device
// (the asynchronous load path: no host round trip).
void launch_scales(const unsigned* colmax, int d, long long n_total, double* scale,
                   double* iscale, int* qflag, cudaStream_t s);
// rows of the given (global) ids; rows outside [row_offset, row_offset+n)
// are zero (they are filled by another rank and summed by the allreduce).
void launch_gather_rows(const float* xs, long long n_pad, int d, const long long* ids,
                        long long row_offset, long long n_local, int cnt, float* out,
                        cudaStream_t s);
// Greedy (Alg 2): spos[nM] positions into S.  scratch holds
// greedy_scratch_doubles(nS) doubles (the #S x #S distance matrix).
size_t greedy_scratch_doubles(int nS);
cudaError_t launch_greedy(const float* srows, int nS, int d, int nM, int q0, int metric,
                          double* scratch, int* spos, double* pickdist, cudaStream_t s);
// M rows and ids from S rows and positions.
void launch_gather_m(const float* srows, const long long* sids, const int* spos, int nM, int d,
                     float* mrows, long long* mids, cudaStream_t s);

// Small H2D upload through kernel parameters (chunks of BLOB_BYTES).
constexpr int BLOB_BYTES = 30000;  // < the 32764-byte kernel parameter limit (CUDA >= 12.1)
void launch_put(void* dst, const void* src, size_t bytes, cudaStream_t s);

PassShape pass_shape(int d, int k, int l, int nM, int num_sms);
cudaError_t configure_kernels(const PassShape& ps);

// iteration prologue (delta, active slots) for the state's MCur
void launch_prepare(const RunParams& p, cudaStream_t s);
// the three passes of one iteration (Alg 3+4, Alg 5, Alg 6 + Alg 1 l.10-14)
void launch_locality(const RunParams& p, const PassShape& ps, cudaStream_t s);
void launch_assign(const RunParams& p, const PassShape& ps, cudaStream_t s);
void launch_cost(const RunParams& p, const PassShape& ps, cudaStream_t s);
// refinement (Alg 1 l.16-19)
void launch_refine_x(const RunParams& p, const PassShape& ps, cudaStream_t s);
void launch_final(const RunParams& p, const PassShape& ps, cudaStream_t s);

// multi-GPU: single-block finalisation after the NCCL allreduce of the
// fixed-point cell sums (accg) and counts (cntg).
enum Tail { TAIL_LOC = 0, TAIL_ASG = 1, TAIL_COST = 2, TAIL_REF = 3 };
void launch_tail(const RunParams& p, int tail, cudaStream_t s);

}  // namespace pc

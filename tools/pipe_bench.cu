// Streaming-pipeline microbenchmark (B200, sm_100a): how fast can a block
// ring of cp.async.bulk copies stream 60 MB (1M points x 15 dims fp32) when
// the consumers do (almost) nothing?  Compares
//   rows: a chunk = d separate row copies of P*4 bytes (SoA [d][n_pad])
//   blk : a chunk = one contiguous copy of d*P*4 bytes (blocked [chunk][d][P])
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/pipe_bench tools/pipe_bench.cu
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ unsigned smem_u32(const void* p) {
  return static_cast<unsigned>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(unsigned long long* bar, unsigned count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(unsigned long long* bar, unsigned bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(unsigned long long* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(unsigned long long* bar, unsigned phase) {
  asm volatile("{\n.reg .pred p;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra W_%=;\n}\n" ::"r"(smem_u32(bar)), "r"(phase) : "memory");
}
__device__ __forceinline__ void bulk(void* dst, const void* src, unsigned bytes, unsigned long long* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}

__global__ void k_stream(const float* __restrict__ x, long long n_pad, int d, int P, int stages,
                         long long nchunks, int blocked, float* out) {
  extern __shared__ __align__(16) unsigned char sm[];
  unsigned long long* full = (unsigned long long*)sm;
  unsigned long long* empty = full + 4;
  float* buf = (float*)(sm + 64);
  const int nw = blockDim.x / 32 - 1, w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int s = 0; s < stages; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], nw); }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  const long long nmy = nchunks > blockIdx.x ? (nchunks - blockIdx.x + gridDim.x - 1) / gridDim.x : 0;
  const unsigned bytes = (unsigned)(P * d * 4);
  float acc = 0.f;
  if (w == nw) {
    for (long long i = 0; i < nmy; ++i) {
      const int st = (int)(i % stages);
      if (i >= stages) { mbar_wait(&empty[st], (unsigned)(((i / stages) - 1) & 1)); asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
      const long long c = blockIdx.x + i * gridDim.x;
      if (lane == 0) mbar_expect_tx(&full[st], bytes);
      __syncwarp();
      float* dst = buf + (size_t)st * d * P;
      if (blocked) {
        if (lane == 0) bulk(dst, x + c * (long long)d * P, bytes, &full[st]);
      } else {
        for (int j = lane; j < d; j += 32) bulk(dst + j * P, x + j * n_pad + c * P, P * 4, &full[st]);
      }
    }
  } else {
    for (long long i = 0; i < nmy; ++i) {
      const int st = (int)(i % stages);
      mbar_wait(&full[st], (unsigned)((i / stages) & 1));
      const float* b = buf + (size_t)st * d * P;
      for (int j = 0; j < d; ++j) acc += b[j * P + w * 32 + lane];
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty[st]);
    }
  }
  if (acc == 12345.f) out[0] = acc;
}

__global__ void k_ldg(const float4* __restrict__ x, long long n4, float* out) {
  float acc = 0.f;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n4;
       i += (long long)gridDim.x * blockDim.x) {
    float4 v = __ldg(x + i);
    acc += v.x + v.w;
  }
  if (acc == 12345.f) out[0] = acc;
}

static void plain(float* flush, float* out, int sms) {
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  for (long long mb : {60LL, 240LL, 1024LL}) {
    float* x;
    cudaMalloc(&x, mb << 20);
    cudaMemset(x, 0, mb << 20);
    for (int per_sm : {4, 8, 16}) {
      float best = 1e30f;
      for (int rep = 0; rep < 5; ++rep) {
        cudaMemsetAsync(flush, rep, 256 << 20);
        cudaEventRecord(a);
        k_ldg<<<sms * per_sm, 256>>>((const float4*)x, (mb << 20) / 16, out);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        if (rep > 0 && ms < best) best = ms;
      }
      printf("ldg %5lld MB  blk/SM %2d  %8.1f us  %6.0f GB/s\n", mb, per_sm, best * 1e3,
             (double)(mb << 20) / (best * 1e-3) / 1e9);
    }
    cudaFree(x);
  }
}

int main() {
  const long long n = 1000000, n_pad = 1000448;
  const int d = 15;
  float *x, *out;
  cudaMalloc(&x, sizeof(float) * d * n_pad);
  cudaMemset(x, 0, sizeof(float) * d * n_pad);
  cudaMalloc(&out, 4);
  float* flush;
  cudaMalloc(&flush, 256 << 20);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  cudaFuncSetAttribute(k_stream, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
  plain(flush, out, sms);
  const double bytes = 4.0 * d * n;
  printf("%6s %4s %6s %6s %8s %8s\n", "layout", "P", "stages", "blk/SM", "us", "GB/s");
  for (int blocked = 0; blocked < 2; ++blocked)
    for (int P : {128, 256, 512, 1024})
      for (int stages : {2, 3, 4})
        for (int per_sm : {1, 2, 4, 8}) {
          const size_t smem = 64 + (size_t)stages * d * P * 4;
          if (smem * per_sm > 220 * 1024) continue;
          const int threads = P + 32;  // P/32 consumer warps + producer
          if (threads > 1024 || threads * per_sm > 2048) continue;
          const long long nchunks = (n + P - 1) / P;
          const int grid = sms * per_sm;
          float best = 1e30f;
          for (int rep = 0; rep < 5; ++rep) {
            cudaMemsetAsync(flush, rep, 256 << 20);
            cudaEventRecord(a);
            k_stream<<<grid, threads, smem>>>(x, n_pad, d, P, stages, nchunks, blocked, out);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            float ms;
            cudaEventElapsedTime(&ms, a, b);
            if (rep > 0 && ms < best) best = ms;
          }
          cudaError_t e = cudaGetLastError();
          if (e != cudaSuccess) { printf("error %s\n", cudaGetErrorString(e)); return 1; }
          printf("%6s %4d %6d %6d %8.1f %8.0f\n", blocked ? "blk" : "rows", P, stages, per_sm,
                 best * 1e3, bytes / (best * 1e-3) / 1e9);
        }
  return 0;
}

// Microbenchmark of the per-SM instruction throughputs that bound the PROCLUS
// passes on B200 (sm_100a): fp32 FADD (register form), fp64 DADD, F2F.F64.F32
// conversion, LDS.32 / LDS.128.  Build: nvcc -gencode arch=compute_100a,code=sm_100a
// -O3 -o /tmp/mb tools/microbench.cu ; run: /tmp/mb
#include <cstdio>
#include <cuda_runtime.h>

#define ITERS 4096

__global__ void k_fadd(float* out, float a) {
  float x0 = threadIdx.x, x1 = x0 + 1, x2 = x0 + 2, x3 = x0 + 3, x4 = x0 + 4, x5 = x0 + 5,
        x6 = x0 + 6, x7 = x0 + 7;
  float b = a * 0.5f;
  for (int i = 0; i < ITERS; ++i) {
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      x0 = __fadd_rn(x0, b); x1 = __fadd_rn(x1, b); x2 = __fadd_rn(x2, b); x3 = __fadd_rn(x3, b);
      x4 = __fadd_rn(x4, b); x5 = __fadd_rn(x5, b); x6 = __fadd_rn(x6, b); x7 = __fadd_rn(x7, b);
      b = __fadd_rn(b, x0);
    }
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = x0 + x1 + x2 + x3 + x4 + x5 + x6 + x7;
}

__global__ void k_dadd(double* out, double a) {
  double x0 = threadIdx.x, x1 = x0 + 1, x2 = x0 + 2, x3 = x0 + 3, x4 = x0 + 4, x5 = x0 + 5,
         x6 = x0 + 6, x7 = x0 + 7;
  double b = a * 0.5;
  for (int i = 0; i < ITERS; ++i) {
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      x0 = __dadd_rn(x0, b); x1 = __dadd_rn(x1, b); x2 = __dadd_rn(x2, b); x3 = __dadd_rn(x3, b);
      x4 = __dadd_rn(x4, b); x5 = __dadd_rn(x5, b); x6 = __dadd_rn(x6, b); x7 = __dadd_rn(x7, b);
      b = __dadd_rn(b, x0);
    }
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = x0 + x1 + x2 + x3 + x4 + x5 + x6 + x7;
}

__global__ void k_f2f(double* out, float a) {
  float f0 = threadIdx.x * a, f1 = f0 + 1, f2 = f0 + 2, f3 = f0 + 3;
  double s0 = 0, s1 = 0, s2 = 0, s3 = 0;
  for (int i = 0; i < ITERS; ++i) {
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      s0 = __dadd_rn(s0, (double)f0); s1 = __dadd_rn(s1, (double)f1);
      s2 = __dadd_rn(s2, (double)f2); s3 = __dadd_rn(s3, (double)f3);
      f0 = __fadd_rn(f0, 1.0f); f1 = __fadd_rn(f1, 1.0f); f2 = __fadd_rn(f2, 1.0f); f3 = __fadd_rn(f3, 1.0f);
    }
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = s0 + s1 + s2 + s3;
}

__global__ void k_lds32(float* out, int stride) {
  __shared__ float sm[8192];
  for (int i = threadIdx.x; i < 8192; i += blockDim.x) sm[i] = i;
  __syncthreads();
  float acc = 0;
  int idx = threadIdx.x;
  for (int i = 0; i < ITERS; ++i) {
#pragma unroll
    for (int u = 0; u < 8; ++u) acc += sm[(idx + u * stride) & 8191];
    idx += 32;
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}

__global__ void k_lds128(float* out, int stride) {
  __shared__ float4 sm[2048];
  for (int i = threadIdx.x; i < 2048; i += blockDim.x) sm[i] = make_float4(i, i, i, i);
  __syncthreads();
  float acc = 0;
  int idx = threadIdx.x;
  for (int i = 0; i < ITERS; ++i) {
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      float4 v = sm[(idx + u * stride) & 2047];
      acc += v.x + v.w;
    }
    idx += 32;
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}

__global__ void k_d2ll(long long* out, double a) {
  double x0 = threadIdx.x * a, x1 = x0 + 1, x2 = x0 + 2, x3 = x0 + 3;
  long long s0 = 0, s1 = 0, s2 = 0, s3 = 0;
  for (int i = 0; i < ITERS; ++i) {
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      s0 += __double2ll_rn(x0); s1 += __double2ll_rn(x1);
      s2 += __double2ll_rn(x2); s3 += __double2ll_rn(x3);
      x0 += 1.0; x1 += 1.0; x2 += 1.0; x3 += 1.0;
    }
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = s0 + s1 + s2 + s3;
}

__global__ void k_f2i(int* out, float a) {
  float x0 = threadIdx.x * a, x1 = x0 + 1, x2 = x0 + 2, x3 = x0 + 3;
  int s0 = 0, s1 = 0, s2 = 0, s3 = 0;
  for (int i = 0; i < ITERS; ++i) {
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      s0 += __float2int_rn(x0); s1 += __float2int_rn(x1);
      s2 += __float2int_rn(x2); s3 += __float2int_rn(x3);
      x0 += 1.0f; x1 += 1.0f; x2 += 1.0f; x3 += 1.0f;
    }
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = s0 + s1 + s2 + s3;
}

__global__ void k_i64(long long* out, long long a) {
  long long x0 = threadIdx.x, x1 = x0 + 1, x2 = x0 + 2, x3 = x0 + 3, x4 = x0 + 4, x5 = x0 + 5,
            x6 = x0 + 6, x7 = x0 + 7;
  for (int i = 0; i < ITERS; ++i) {
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      x0 += a; x1 += x0; x2 += a; x3 += x2; x4 += a; x5 += x4; x6 += a; x7 += x6;
      a ^= x7;
    }
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = x0 + x1 + x2 + x3 + x4 + x5 + x6 + x7;
}

int main() {
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  int clk = 0;
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  const int blocks = sms * 4, threads = 512;
  float* fo;
  double* dout;
  cudaMalloc(&fo, sizeof(float) * blocks * threads);
  cudaMalloc(&dout, sizeof(double) * blocks * threads);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  auto report = [&](const char* name, double ops_per_thread, auto launch) {
    launch();
    cudaDeviceSynchronize();
    cudaEventRecord(a);
    launch();
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    double ops = ops_per_thread * blocks * threads;
    double per_clk_sm = ops / (ms * 1e-3) / (sms * (clk * 1e3));
    printf("%-10s %8.3f ms  %8.1f Gop/s  %6.1f /clk/SM (at %d MHz nominal)\n", name, ms,
           ops / ms / 1e6, per_clk_sm, clk / 1000);
  };
  report("FADD", ITERS * 4.0 * 9, [&] { k_fadd<<<blocks, threads>>>(fo, 1.0f); });
  report("DADD", ITERS * 4.0 * 9, [&] { k_dadd<<<blocks, threads>>>(dout, 1.0); });
  report("F2F+DADD", ITERS * 4.0 * 4, [&] { k_f2f<<<blocks, threads>>>(dout, 1.0f); });
  report("D2LL", ITERS * 4.0 * 4, [&] { k_d2ll<<<blocks, threads>>>((long long*)dout, 1.0); });
  report("F2I", ITERS * 4.0 * 4, [&] { k_f2i<<<blocks, threads>>>((int*)fo, 1.0f); });
  report("I64ADD", ITERS * 4.0 * 9, [&] { k_i64<<<blocks, threads>>>((long long*)dout, 3); });
  report("LDS.32", ITERS * 8.0, [&] { k_lds32<<<blocks, threads>>>(fo, 33); });
  report("LDS.128", ITERS * 8.0, [&] { k_lds128<<<blocks, threads>>>(fo, 9); });
  printf("(LDS rows: loads per thread per s; x4 bytes for .32, x16 for .128)\n");
  return 0;
}

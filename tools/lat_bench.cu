// Dependent-chain latency of a few fp64 / conversion / shared-memory ops on
// one warp (cycles per op).  nvcc -gencode arch=compute_100a,code=sm_100a -O3 tools/lat_bench.cu
#include <cstdio>
#include <cuda_runtime.h>

__global__ void k(double* out, long long* cyc, float* fo, int n) {
  __shared__ double sm[64];
  __shared__ float sf[64];
  if (threadIdx.x < 64) { sm[threadIdx.x] = 1.0 + threadIdx.x * 1e-9; sf[threadIdx.x] = 1.0f; }
  __syncthreads();
  double a = out[0], b = out[1];
  float f = fo[0];
  long long t0, t1;
  // DADD chain
  t0 = clock64();
  for (int i = 0; i < n; ++i) { a = __dadd_rn(a, b); a = __dadd_rn(a, b); a = __dadd_rn(a, b); a = __dadd_rn(a, b); }
  t1 = clock64(); cyc[0] = (t1 - t0); out[2] = a;
  // DMUL chain
  t0 = clock64();
  for (int i = 0; i < n; ++i) { a = __dmul_rn(a, b); a = __dmul_rn(a, b); a = __dmul_rn(a, b); a = __dmul_rn(a, b); }
  t1 = clock64(); cyc[1] = (t1 - t0); out[3] = a;
  // FADD chain
  t0 = clock64();
  for (int i = 0; i < n; ++i) { f = __fadd_rn(f, 1.0f); f = __fadd_rn(f, 1.0f); f = __fadd_rn(f, 1.0f); f = __fadd_rn(f, 1.0f); }
  t1 = clock64(); cyc[2] = (t1 - t0); fo[1] = f;
  // F2F chain: float -> double -> float
  t0 = clock64();
  for (int i = 0; i < n; ++i) { double x = (double)f; f = (float)(x * 1.0000001); double y = (double)f; f = (float)y; }
  t1 = clock64(); cyc[3] = (t1 - t0); fo[2] = f;
  // dsqrt chain
  t0 = clock64();
  for (int i = 0; i < n; ++i) { a = __dsqrt_rn(a); a = __dsqrt_rn(a); a = __dsqrt_rn(a); a = __dsqrt_rn(a); }
  t1 = clock64(); cyc[4] = (t1 - t0); out[4] = a;
  // ddiv chain
  t0 = clock64();
  for (int i = 0; i < n; ++i) { a = __ddiv_rn(a, b); a = __ddiv_rn(a, b); a = __ddiv_rn(a, b); a = __ddiv_rn(a, b); }
  t1 = clock64(); cyc[5] = (t1 - t0); out[5] = a;
  // LDS.64 pointer chase-ish: index from value
  int idx = threadIdx.x & 31;
  t0 = clock64();
  for (int i = 0; i < n; ++i) {
    double v = sm[idx]; idx = ((int)v + idx) & 31; v = sm[idx]; idx = ((int)v + idx) & 31;
    v = sm[idx]; idx = ((int)v + idx) & 31; v = sm[idx]; idx = ((int)v + idx) & 31;
  }
  t1 = clock64(); cyc[6] = (t1 - t0); out[6] = idx;
  // redux.sync chain
  unsigned u = threadIdx.x;
  t0 = clock64();
  for (int i = 0; i < n; ++i) { u = __reduce_max_sync(0xffffffffu, u) + threadIdx.x; u = __reduce_max_sync(0xffffffffu, u) + threadIdx.x; u = __reduce_max_sync(0xffffffffu, u) + threadIdx.x; u = __reduce_max_sync(0xffffffffu, u) + threadIdx.x; }
  t1 = clock64(); cyc[7] = (t1 - t0); out[7] = u;
  // DADD chain again (warm)
  t0 = clock64();
  for (int i = 0; i < n; ++i) { a = __dadd_rn(a, b); a = __dadd_rn(a, b); a = __dadd_rn(a, b); a = __dadd_rn(a, b); }
  t1 = clock64(); cyc[9] = (t1 - t0); out[8] = a;
  // DFMA chain
  t0 = clock64();
  for (int i = 0; i < n; ++i) { a = __fma_rn(a, b, b); a = __fma_rn(a, b, b); a = __fma_rn(a, b, b); a = __fma_rn(a, b, b); }
  t1 = clock64(); cyc[10] = (t1 - t0); out[9] = a;
  // DADD as fma(a, 1, b)
  t0 = clock64();
  for (int i = 0; i < n; ++i) { a = __fma_rn(a, 1.0, b); a = __fma_rn(a, 1.0, b); a = __fma_rn(a, 1.0, b); a = __fma_rn(a, 1.0, b); }
  t1 = clock64(); cyc[11] = (t1 - t0); out[10] = a;
  // __syncthreads (1 warp)
  t0 = clock64();
  for (int i = 0; i < n; ++i) { __syncthreads(); __syncthreads(); __syncthreads(); __syncthreads(); }
  t1 = clock64(); cyc[8] = (t1 - t0);
}

int main() {
  double* out; long long* cyc; float* fo;
  cudaMallocManaged(&out, 64 * 8); cudaMallocManaged(&cyc, 64 * 8); cudaMallocManaged(&fo, 64 * 4);
  out[0] = 1.0; out[1] = 1.0000001; fo[0] = 1.0f;
  const int n = 1000;
  const char* names[] = {"DADD", "DMUL", "FADD", "F2F(d<-f, f<-d x2 + dmul)", "DSQRT", "DDIV", "LDS.64+IADD", "REDUX+IADD", "BAR(1 warp)", "DADD (again)", "DFMA", "DFMA(a,1,b)"};
  for (int tpb : {32, 256}) {
    k<<<1, tpb>>>(out, cyc, fo, n);
    cudaDeviceSynchronize();
    printf("tpb=%d\n", tpb);
    for (int i = 0; i < 12; ++i) printf("  %-28s %.1f cyc/op\n", names[i], (double)cyc[i] / (4.0 * n));
  }
  return 0;
}

// Throughput probe: MUFU.EX2 vs SHFL vs a mix on one B200 (is SHFL competing
// with MUFU for the MIO queue?).  nvcc -gencode arch=compute_100a,code=sm_100a -O3
#include <cstdio>
#include <cuda_runtime.h>
__device__ __forceinline__ float ex2(float x) { float y; asm volatile("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x)); return y; }
template <int NM, int NS>
__global__ void k(float *out, int iters, float seed) {
  float a[8], b[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) { a[i] = seed * (threadIdx.x + i); b[i] = a[i] + 1.f; }
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      if (i < NM) a[i] = ex2(a[i]) - 0.5f;
      if (i < NS) b[i] = __shfl_down_sync(0xffffffffu, b[i], 1) + 0.25f;
    }
  }
  float s = 0; for (int i = 0; i < 8; ++i) s += a[i] + b[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
template <int NM, int NS> void run(float *d, const char *name) {
  int blocks = 148 * 8, threads = 256, iters = 4096;
  k<NM, NS><<<blocks, threads>>>(d, 16, 0.001f);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  cudaEventRecord(e0);
  k<NM, NS><<<blocks, threads>>>(d, iters, 0.001f);
  cudaEventRecord(e1); cudaEventSynchronize(e1);
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  double lanes = (double)blocks * threads * iters;
  printf("%-22s %8.3f ms  mufu %.3e/s  shfl %.3e/s  (per SM per ns: mufu %.2f shfl %.2f)\n", name, ms,
         lanes * NM / (ms * 1e-3), lanes * NS / (ms * 1e-3), lanes * NM / (ms * 1e6) / 148, lanes * NS / (ms * 1e6) / 148);
}
int main() {
  float *d; cudaMalloc(&d, 148 * 8 * 256 * 4);
  run<8, 0>(d, "mufu only");
  run<0, 8>(d, "shfl only");
  run<8, 4>(d, "mufu 8 : shfl 4");
  run<8, 6>(d, "mufu 8 : shfl 6");
  run<8, 8>(d, "mufu 8 : shfl 8");
  run<4, 8>(d, "mufu 4 : shfl 8");
  return 0;
}

// peaks.cu -- micro-benchmarks for the roofline denominators of DESIGN.md:
// MUFU.EX2 and FFMA issue rates per SM per clock, and the SM clock under
// that load.  Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/peaks tools/peaks.cu
#include <cstdio>
#include <cuda_runtime.h>

constexpr int CHAINS = 8;
constexpr int ITERS = 4096;

__global__ void ex2_kernel(float *out, float seed, long long *clk)
{
    float v[CHAINS];
#pragma unroll
    for (int c = 0; c < CHAINS; ++c) v[c] = seed * (threadIdx.x + c) * 1e-9f;
    long long t0 = clock64();
    for (int i = 0; i < ITERS; ++i) {
#pragma unroll
        for (int c = 0; c < CHAINS; ++c) asm volatile("ex2.approx.ftz.f32 %0, %0;" : "+f"(v[c]));
    }
    long long t1 = clock64();
    float s = 0;
#pragma unroll
    for (int c = 0; c < CHAINS; ++c) s += v[c];
    if (s == 1234.5f) out[0] = s;
    if (threadIdx.x == 0 && blockIdx.x == 0) *clk = t1 - t0;
}

__global__ void ffma_kernel(float *out, float seed, long long *clk)
{
    float v[CHAINS];
    float a = seed, b = seed * 0.5f;
#pragma unroll
    for (int c = 0; c < CHAINS; ++c) v[c] = seed * (threadIdx.x + c);
    long long t0 = clock64();
    for (int i = 0; i < ITERS; ++i) {
#pragma unroll
        for (int c = 0; c < CHAINS; ++c) v[c] = fmaf(v[c], a, b);
    }
    long long t1 = clock64();
    float s = 0;
#pragma unroll
    for (int c = 0; c < CHAINS; ++c) s += v[c];
    if (s == 1234.5f) out[0] = s;
    if (threadIdx.x == 0 && blockIdx.x == 0) *clk = t1 - t0;
}

template <typename K>
void run(const char *name, K kernel, int sms)
{
    float *out;
    long long *clk;
    cudaMalloc(&out, 4);
    cudaMalloc(&clk, 8);
    const int blocks = sms * 8, threads = 256;
    kernel<<<blocks, threads>>>(out, 1.0f, clk);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    cudaEventRecord(a);
    kernel<<<blocks, threads>>>(out, 1.0f, clk);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    long long c;
    cudaMemcpy(&c, clk, 8, cudaMemcpyDeviceToHost);
    const double ops = (double)blocks * threads * ITERS * CHAINS;
    const double per_s = ops / (ms * 1e-3);
    const double mhz = (double)c / (ms * 1e-3) / 1e6;   // approx: one CTA's clock span
    printf("{\"op\": \"%s\", \"ops_per_s\": %.4e, \"ms\": %.4f, \"sm_mhz_est\": %.0f, "
           "\"ops_per_clk_per_sm\": %.2f}\n",
           name, per_s, ms, mhz, per_s / (mhz * 1e6) / sms);
    cudaFree(out);
    cudaFree(clk);
}

int main()
{
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    int clk_khz = 0;
    cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, 0);
    printf("{\"sms\": %d, \"clock_rate_khz_attr\": %d}\n", sms, clk_khz);
    run("ex2.approx.ftz.f32", ex2_kernel, sms);
    run("ffma.f32", ffma_kernel, sms);
    return 0;
}

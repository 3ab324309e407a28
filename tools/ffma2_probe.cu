// Does sm_100 FFMA2 / FMUL2 / FADD2 round exactly like scalar FFMA / FMUL / FADD?
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
__global__ void k(const float *a, const float *b, const float *c, int n, unsigned *bad)
{
    int i = 2 * (blockIdx.x * blockDim.x + threadIdx.x);
    if (i + 1 >= n) return;
    float2 A = make_float2(a[i], a[i + 1]), B = make_float2(b[i], b[i + 1]), C = make_float2(c[i], c[i + 1]);
    float2 f2 = __ffma2_rn(A, B, C);
    float f0 = __fmaf_rn(a[i], b[i], c[i]), f1 = __fmaf_rn(a[i + 1], b[i + 1], c[i + 1]);
    float2 m2 = __fmul2_rn(A, B);
    float2 s2 = __fadd2_rn(A, C);
    if (__float_as_uint(f2.x) != __float_as_uint(f0) || __float_as_uint(f2.y) != __float_as_uint(f1)) atomicAdd(&bad[0], 1u);
    if (__float_as_uint(m2.x) != __float_as_uint(__fmul_rn(a[i], b[i])) || __float_as_uint(m2.y) != __float_as_uint(__fmul_rn(a[i + 1], b[i + 1]))) atomicAdd(&bad[1], 1u);
    if (__float_as_uint(s2.x) != __float_as_uint(__fadd_rn(a[i], c[i])) || __float_as_uint(s2.y) != __float_as_uint(__fadd_rn(a[i + 1], c[i + 1]))) atomicAdd(&bad[2], 1u);
}
int main()
{
    const int n = 1 << 24;
    float *h = new float[3 * (size_t)n];
    uint64_t s = 88172645463325252ull;
    for (size_t i = 0; i < 3 * (size_t)n; ++i) {
        s ^= s << 13; s ^= s >> 7; s ^= s << 17;
        float u = (float)((s >> 11) * (1.0 / 9007199254740992.0));
        h[i] = (i % 3 == 1) ? (float)((int)(u * 16) - 8) / 8.0f : (i % 7 == 0 ? -u * 3.f : u * 5.f);
    }
    float *d; unsigned *bad;
    cudaMalloc(&d, 3 * (size_t)n * 4); cudaMalloc(&bad, 12); cudaMemset(bad, 0, 12);
    cudaMemcpy(d, h, 3 * (size_t)n * 4, cudaMemcpyHostToDevice);
    k<<<n / 2 / 256, 256>>>(d, d + n, d + 2 * (size_t)n, n, bad);
    unsigned hb[3];
    cudaMemcpy(hb, bad, 12, cudaMemcpyDeviceToHost);
    printf("pairs=%d ffma2_mismatch=%u fmul2_mismatch=%u fadd2_mismatch=%u (%s)\n", n / 2, hb[0], hb[1], hb[2],
           cudaGetErrorString(cudaGetLastError()));
    return 0;
}

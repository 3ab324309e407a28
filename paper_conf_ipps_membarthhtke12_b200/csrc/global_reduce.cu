// global_reduce.cu -- global operators ("global operators
// (e.g., reduction operators) produce one output for the operator applied to
// all pixels of the image (e.g., compute the sum of all pixels)"; SURVEY §8(f)
// N3 "global reductions (sum/min/max)"): SUM, MIN or MAX over the pixels of a
// region of interest (all frames of a batch).
//
// Deterministic: a fixed number of CTAs (kGlobalParts, independent of the GPU)
// each reduce a fixed contiguous block of rows -- every thread a fixed set of
// columns, in a fixed order, accumulating in double (f32) or int64 (u8 SUM) --
// then a fixed tree in shared memory; the last CTA to finish combines the
// parts in a fixed tree.  The same input always gives the same bits.
// Bound: HBM (the image is read once).
#include <cuda_runtime.h>
#include <stdint.h>

#include "kernels.h"
#include "lop_params.h"

namespace lop {

namespace glob {
constexpr int NT = 256;
}

template <int OP> __device__ __forceinline__ double comb(double a, double b)
{
    return OP == RED_MIN ? fmin(a, b) : (OP == RED_MAX ? fmax(a, b) : a + b);
}

// CTA c reduces rows [c * R / P, (c + 1) * R / P) of the R = batch * roi_h
// region rows; thread t the 16-byte column groups t, t + NT, ... of each row.
template <typename T, int OP>
__global__ void __launch_bounds__(glob::NT) global_partial_kernel(const __grid_constant__ GlobalReduce p)
{
    const Common &c = p.c;
    const int64_t rows = (int64_t)c.batch * c.roi_h;
    const int64_t r0 = rows * blockIdx.x / kGlobalParts, r1 = rows * (blockIdx.x + 1) / kGlobalParts;
    constexpr bool F = sizeof(T) == 4;
    // per-thread accumulators in the cheapest exact form: f32 SUM in double;
    // f32 MIN / MAX in float (exact); u8 SUM in int32 by byte dot products
    // (IDP4A); u8 MIN / MAX on packed bytes (__vminu4 / __vmaxu4)
    double dacc = 0.0;
    float facc = OP == RED_MIN ? __int_as_float(0x7f800000) : -__int_as_float(0x7f800000);
    unsigned int iacc = 0;
    uint32_t bacc = OP == RED_MIN ? 0xFFFFFFFFu : 0u;
    auto add_word = [&](uint32_t w, int nbytes) {                // u8: 4 packed pixels
        if (nbytes < 4) {                                         // pad with the identity
            const uint32_t keep = nbytes == 0 ? 0u : (0xFFFFFFFFu >> (8 * (4 - nbytes)));
            w = OP == RED_MIN ? (w | ~keep) : (w & keep);
        }
        if (OP == RED_SUM) iacc = __dp4a(w, 0x01010101u, iacc);   // unsigned bytes, exact
        else bacc = OP == RED_MIN ? __vminu4(bacc, w) : __vmaxu4(bacc, w);
    };
    auto add_f = [&](float v) {
        if (OP == RED_SUM) dacc += (double)v;
        else facc = OP == RED_MIN ? fminf(facc, v) : fmaxf(facc, v);
    };
    constexpr int V = 16 / (int)sizeof(T);                       // elements per 16-B load
#pragma unroll 2
    for (int64_t r = r0; r < r1; ++r) {
        const int b = (int)(r / c.roi_h), y = c.roi_y0 + (int)(r - (int64_t)b * c.roi_h);
        const T *row = reinterpret_cast<const T *>(c.in.data + (int64_t)b * c.in.bstride +
                                                   (int64_t)y * c.in.stride) + c.roi_x0;
        const bool vec = (reinterpret_cast<uintptr_t>(row) % 16) == 0;               // row-uniform
#pragma unroll 4
        for (int x = V * threadIdx.x; x < c.roi_w; x += V * glob::NT) {
            const int n = min(V, c.roi_w - x);
            if (vec && n == V) {                                 // one 16-B load, in column order
                const uint4 q = __ldg(reinterpret_cast<const uint4 *>(row + x));
                if constexpr (F) {
                    add_f(__uint_as_float(q.x)); add_f(__uint_as_float(q.y));
                    add_f(__uint_as_float(q.z)); add_f(__uint_as_float(q.w));
                } else {
                    add_word(q.x, 4); add_word(q.y, 4); add_word(q.z, 4); add_word(q.w, 4);
                }
            } else {
                for (int j = 0; j < n; ++j) {
                    if constexpr (F) add_f(__ldg(row + x + j));
                    else add_word((uint32_t)__ldg(row + x + j), 1);
                }
            }
        }
    }
    double acc;
    if constexpr (F) acc = OP == RED_SUM ? dacc : (double)facc;
    else if (OP == RED_SUM) acc = (double)iacc;                   // exact (partials < 2^31)
    else {
        uint32_t m = bacc & 0xFF;
#pragma unroll
        for (int j = 1; j < 4; ++j) {
            const uint32_t v = (bacc >> (8 * j)) & 0xFF;
            m = OP == RED_MIN ? min(m, v) : max(m, v);
        }
        acc = (double)m;
    }
    __shared__ double sh[glob::NT];
    sh[threadIdx.x] = acc;
    __syncthreads();
#pragma unroll
    for (int s = glob::NT / 2; s > 0; s >>= 1) {                 // fixed tree
        if ((int)threadIdx.x < s) sh[threadIdx.x] = comb<OP>(sh[threadIdx.x], sh[threadIdx.x + s]);
        __syncthreads();
    }
    // The last CTA to finish combines the parts (fixed tree over the part index,
    // so the result does not depend on which CTA is last); the arrival counter
    // lives in work[kGlobalParts] and is reset for the next call.
    __shared__ bool last;
    if (threadIdx.x == 0) {
        p.work[blockIdx.x] = sh[0];
        __threadfence();
        unsigned int *count = reinterpret_cast<unsigned int *>(p.work + kGlobalParts);
        last = atomicAdd(count, 1u) == kGlobalParts - 1;
    }
    __syncthreads();
    if (!last) return;
    __threadfence();
    constexpr int PER = kGlobalParts / glob::NT;                 // parts per thread
    double a = __ldcg(p.work + threadIdx.x * PER);
#pragma unroll
    for (int i = 1; i < PER; ++i) a = comb<OP>(a, __ldcg(p.work + threadIdx.x * PER + i));
    sh[threadIdx.x] = a;
    __syncthreads();
#pragma unroll
    for (int s = glob::NT / 2; s > 0; s >>= 1) {
        if ((int)threadIdx.x < s) sh[threadIdx.x] = comb<OP>(sh[threadIdx.x], sh[threadIdx.x + s]);
        __syncthreads();
    }
    if (threadIdx.x == 0) {
        *p.result = sh[0];
        *reinterpret_cast<unsigned int *>(p.work + kGlobalParts) = 0u;
    }
}

namespace {
template <typename T, int OP>
cudaError_t launch_global_t(const GlobalReduce &p, cudaStream_t stream)
{
    global_partial_kernel<T, OP><<<kGlobalParts, glob::NT, 0, stream>>>(p);
    return cudaGetLastError();
}

template <typename T>
cudaError_t launch_global_op(const GlobalReduce &p, cudaStream_t stream)
{
    switch (p.op) {
    case RED_SUM: return launch_global_t<T, RED_SUM>(p, stream);
    case RED_MIN: return launch_global_t<T, RED_MIN>(p, stream);
    case RED_MAX: return launch_global_t<T, RED_MAX>(p, stream);
    default: return cudaErrorNotSupported;
    }
}
}  // namespace

cudaError_t launch_global_reduce(const GlobalReduce &p, cudaStream_t stream)
{
    return p.u8 ? launch_global_op<uint8_t>(p, stream) : launch_global_op<float>(p, stream);
}

}  // namespace lop

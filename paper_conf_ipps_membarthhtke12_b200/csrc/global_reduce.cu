// global_reduce.cu -- global operators ("global operators
// (e.g., reduction operators) produce one output for the operator applied to
// all pixels of the image (e.g., compute the sum of all pixels)"; SURVEY §8(f)
// N3 "global reductions (sum/min/max)"): SUM, MIN, MAX or SUMSQ over the pixels
// of a region of interest (all frames of a batch).  SUMSQ is the merge
// a, b -> a^2 + b^2 of PAPER.md L956-L959 ("operations that merge/reduce two
// pixels"; reading c26): f32 squares are exact in double, u8 squares are
// byte dot products of a word with itself (IDP4A), exact.
//
// Deterministic: a fixed number of CTAs (kGlobalParts, independent of the GPU)
// each reduce a fixed contiguous block of rows -- every thread a fixed set of
// columns, in a fixed order, accumulating in double (f32) or int64 (u8 SUM) --
// then a fixed tree (warp butterflies, then the warp sums); the last CTA to finish combines the
// parts in a fixed tree.  The same input always gives the same bits.
// Bound: HBM (the image is read once).
#include <cuda_runtime.h>
#include <stdint.h>

#include "kernels.h"
#include "lop_params.h"

namespace lop {

#ifndef LOP_GLOBAL_U
#define LOP_GLOBAL_U 8
#endif

namespace glob {
constexpr int NT = 256;
}

template <int OP> __device__ __forceinline__ double comb(double a, double b)
{
    return OP == RED_MIN ? fmin(a, b) : (OP == RED_MAX ? fmax(a, b) : a + b);
}

// A ragged or unaligned column group: its n < V (or misaligned) elements
// loaded one by one into the identity-padded group `q` (kept out of line).
template <typename T>
__device__ __noinline__ uint4 glob_partial_group(const T *src, int n, uint4 q)
{
    uint32_t w[4] = {q.x, q.y, q.z, q.w};
    for (int j = 0; j < n; ++j) {
        if constexpr (sizeof(T) == 4) {
            w[j] = __float_as_uint(__ldg(src + j));
        } else {
            const int k = j >> 2, s = 8 * (j & 3);
            w[k] = (w[k] & ~(0xFFu << s)) | ((uint32_t)__ldg(src + j) << s);
        }
    }
    return make_uint4(w[0], w[1], w[2], w[3]);
}

// CTA c reduces rows [c * R / P, (c + 1) * R / P) of the R = batch * roi_h
// region rows; thread t the items t, t + NT, ... of its (row, 16-byte column group) list.
template <typename T, int OP>
__global__ void __launch_bounds__(glob::NT) global_partial_kernel(const __grid_constant__ GlobalReduce p)
{
    const Common &c = p.c;
    const int64_t rows = (int64_t)c.batch * c.roi_h;
    const int64_t r0 = rows * blockIdx.x / kGlobalParts, r1 = rows * (blockIdx.x + 1) / kGlobalParts;
    constexpr bool F = sizeof(T) == 4;
    // per-thread accumulators in the cheapest exact form: f32 SUM / SUMSQ in
    // double; f32 MIN / MAX in float (exact); u8 SUM in int32 by byte dot
    // products (IDP4A); u8 SUMSQ by dot products of a word with itself, per
    // batch of loads in 32 bits (<= 128 x 255^2) then in 64; u8 MIN / MAX on
    // bytes in 16-bit lanes
    constexpr bool SQ = OP == RED_SUMSQ;
    double dacc = 0.0;
    float facc = OP == RED_MIN ? __int_as_float(0x7f800000) : -__int_as_float(0x7f800000);
    unsigned int iacc = 0;
    unsigned long long lacc = 0;
    // u8 MIN / MAX: even and odd bytes in the 16-bit lanes of two accumulators
    // (native VIMNMX.U16x2; __vminu4 / __vmaxu4 are emulated on sm_100)
    uint32_t eacc = OP == RED_MIN ? 0x00FF00FFu : 0u, oacc = eacc;
    auto add_word = [&](uint32_t w, int nbytes) {                // u8: 4 packed pixels
        if (nbytes < 4) {                                         // pad with the identity
            const uint32_t keep = nbytes == 0 ? 0u : (0xFFFFFFFFu >> (8 * (4 - nbytes)));
            w = OP == RED_MIN ? (w | ~keep) : (w & keep);
        }
        if (OP == RED_SUM) iacc = __dp4a(w, 0x01010101u, iacc);   // unsigned bytes, exact
        else if (SQ) iacc = __dp4a(w, w, iacc);                    // sum of the 4 squares
        else {
            const uint32_t e = w & 0x00FF00FFu, o = (w >> 8) & 0x00FF00FFu;
            eacc = OP == RED_MIN ? __vminu2(eacc, e) : __vmaxu2(eacc, e);
            oacc = OP == RED_MIN ? __vminu2(oacc, o) : __vmaxu2(oacc, o);
        }
    };
    auto add_f = [&](float v) {
        if (OP == RED_SUM) dacc += (double)v;
        else if (SQ) dacc = fma((double)v, (double)v, dacc);      // exact square, one rounding
        else facc = OP == RED_MIN ? fminf(facc, v) : fmaxf(facc, v);
    };
    constexpr int V = 16 / (int)sizeof(T);                       // elements per 16-B load
    // The CTA's rows form (row, column group) items in row-major order; thread t
    // takes items t, t + NT, ... in that order.  U items are fetched before any
    // is accumulated (U independent 16-B loads in flight per thread: the first
    // version read one row at a time and stalled on memory latency).  The item
    // -> (frame, row, group) walk is incremental: one division per thread.
    const int G = max((c.roi_w + V - 1) / V, 1);                 // column groups per row
    const int dr = glob::NT / G, dg = glob::NT % G;
    int64_t r = c.roi_w > 0 ? r0 + threadIdx.x / G : r1;         // empty region: no items
    int g = (int)(threadIdx.x % G);
    const int64_t rr = r < r1 ? r : 0;
    int b = c.roi_h > 0 ? (int)(rr / c.roi_h) : 0, y = (int)(rr - (int64_t)b * c.roi_h);
    auto row_at = [&](int bb, int yy) {
        return c.in.data + (int64_t)bb * c.in.bstride + (int64_t)(c.roi_y0 + yy) * c.in.stride +
               (int64_t)c.roi_x0 * (int64_t)sizeof(T);
    };
    const char *rowp = row_at(b, y);
    // Identity element of the operator (partial groups are padded with it).
    const float fid = OP == RED_SUM || SQ ? 0.0f : (OP == RED_MIN ? __int_as_float(0x7f800000)
                                                           : -__int_as_float(0x7f800000));
    const uint32_t bid = OP == RED_MIN ? 0xFFFFFFFFu : 0u;
    const uint32_t idw = F ? __float_as_uint(fid) : bid;
    constexpr int U = LOP_GLOBAL_U;                              // 16-B groups in flight per thread
    while (r < r1) {
        uint4 q[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            q[u] = make_uint4(idw, idw, idw, idw);
            if (r < r1) {
                const int x = g * V;
                const char *src = rowp + (int64_t)x * (int64_t)sizeof(T);
                if (x + V <= c.roi_w && (reinterpret_cast<uintptr_t>(src) % 16) == 0)
                    q[u] = __ldg(reinterpret_cast<const uint4 *>(src));
                else                                              // ragged / unaligned
                    q[u] = glob_partial_group<T>(reinterpret_cast<const T *>(src),
                                                 min(V, c.roi_w - x), q[u]);
                g += dg;
                int adv = dr;
                if (g >= G) { g -= G; ++adv; }
                r += adv; y += adv;
                if (y < c.roi_h) {
                    rowp += (int64_t)adv * c.in.stride;
                } else {
                    while (y >= c.roi_h) { y -= c.roi_h; ++b; }
                    rowp = row_at(b, y);
                }
            }
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {                             // in item and column order
            if constexpr (F) {
                add_f(__uint_as_float(q[u].x)); add_f(__uint_as_float(q[u].y));
                add_f(__uint_as_float(q[u].z)); add_f(__uint_as_float(q[u].w));
            } else {
                add_word(q[u].x, 4); add_word(q[u].y, 4); add_word(q[u].z, 4); add_word(q[u].w, 4);
            }
        }
        if constexpr (!F && SQ) { lacc += iacc; iacc = 0; }
    }
    double acc;
    if constexpr (F) acc = OP == RED_SUM || SQ ? dacc : (double)facc;
    else if (OP == RED_SUM) acc = (double)iacc;                   // exact (partials < 2^31)
    else if (SQ) acc = (double)lacc;                              // exact (partials < 2^53)
    else {
        const uint32_t l = OP == RED_MIN ? __vminu2(eacc, oacc) : __vmaxu2(eacc, oacc);
        const uint32_t m = OP == RED_MIN ? min(l & 0xFFFFu, l >> 16) : max(l & 0xFFFFu, l >> 16);
        acc = (double)m;
    }
    // Fixed trees: a shuffle butterfly within each warp, then warp 0 over the
    // NT / 32 warp sums (fewer barriers than a shared-memory tree).
    __shared__ double sh[glob::NT / 32];
    auto cta_reduce = [&](double v) {
#pragma unroll
        for (int s = 16; s > 0; s >>= 1) v = comb<OP>(v, __shfl_xor_sync(0xFFFFFFFFu, v, s));
        if ((threadIdx.x & 31) == 0) sh[threadIdx.x >> 5] = v;
        __syncthreads();
        double t = sh[0];
#pragma unroll
        for (int w = 1; w < glob::NT / 32; ++w) t = comb<OP>(t, sh[w]);
        return t;                                                 // same bits in every thread
    };
    const double part = cta_reduce(acc);
    if constexpr (OP == RED_MIN || OP == RED_MAX) {
        // MIN / MAX are order-independent: each CTA folds its part into one word
        // with an integer atomic (an order-preserving encoding, identity 0, in the
        // high half of work[kGlobalCounter]); the last CTA decodes it -- no
        // 512-part read and tree at the end.  Same value as the tree, any order.
        __shared__ bool lastm;
        unsigned int *count = reinterpret_cast<unsigned int *>(p.work + kGlobalCounter);
        if (threadIdx.x == 0) {
            uint32_t enc;
            if constexpr (F) {
                const uint32_t bits = __float_as_uint((float)part);
                const uint32_t ord = (bits >> 31) ? ~bits : (bits | 0x80000000u);   // monotone in the value
                enc = OP == RED_MAX ? ord : ~ord;
            } else {
                enc = OP == RED_MAX ? (uint32_t)part : 255u - (uint32_t)part;
            }
            atomicMax(count + 1, enc);
            __threadfence();
            lastm = atomicAdd(count, 1u) == kGlobalParts - 1;
        }
        __syncthreads();
        if (!lastm || threadIdx.x != 0) return;
        __threadfence();
        const uint32_t enc = atomicExch(count + 1, 0u);                // read and reset
        double total;
        if constexpr (F) {
            const uint32_t ord = OP == RED_MAX ? enc : ~enc;
            total = (double)__uint_as_float((ord & 0x80000000u) ? (ord ^ 0x80000000u) : ~ord);
        } else {
            total = (double)(OP == RED_MAX ? enc : 255u - enc);
        }
        *p.result = total;
        *count = 0u;
        return;
    }
    // The last CTA to finish combines the parts (fixed tree over the part index,
    // so the result does not depend on which CTA is last); the arrival counter
    // lives in work[kGlobalCounter] and is reset for the next call.
    __shared__ bool last;
    if (threadIdx.x == 0) {
        p.work[blockIdx.x] = part;
        __threadfence();
        unsigned int *count = reinterpret_cast<unsigned int *>(p.work + kGlobalCounter);
        last = atomicAdd(count, 1u) == kGlobalParts - 1;
    }
    __syncthreads();
    if (!last) return;
    __threadfence();
    constexpr int PER = kGlobalParts / glob::NT;                 // parts per thread
    double a = __ldcg(p.work + threadIdx.x * PER);
#pragma unroll
    for (int i = 1; i < PER; ++i) a = comb<OP>(a, __ldcg(p.work + threadIdx.x * PER + i));
    __syncthreads();                                              // sh reused
    const double total = cta_reduce(a);
    if (threadIdx.x == 0) {
        *p.result = total;
        *reinterpret_cast<unsigned int *>(p.work + kGlobalCounter) = 0u;
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
    case RED_SUMSQ: return launch_global_t<T, RED_SUMSQ>(p, stream);
    default: return cudaErrorNotSupported;
    }
}
}  // namespace

cudaError_t launch_global_reduce(const GlobalReduce &p, cudaStream_t stream)
{
    return p.u8 ? launch_global_op<uint8_t>(p, stream) : launch_global_op<float>(p, stream);
}

}  // namespace lop

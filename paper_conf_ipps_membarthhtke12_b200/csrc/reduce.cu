// reduce.cu -- local MIN / MAX reductions over a mask domain: the
// convolve(mask, <reduction>, f) form of Listing 9 (the
// paper writes it with the SUM reduction, which is lop_convolve_execute) with
// the reductions MIN and MAX -- grey-value erosion / dilation with a
// structuring element, a local operator in the paper's sense (every output a
// reduction over a (2m+1)x(2n+1) window, L274-L282) with the same boundary
// handling (Table I).  Exact for f32 and u8: the result is one of
// the input values (or the constant), whatever the evaluation order.
//
//  * reduce_tiled_kernel<T, OP, R>: full square windows up to 9x9 -- the
//    domain is a rectangle, so min/max is separable (row reduction, then
//    column reduction).  Tile staging as the convolution kernels (stage.cuh:
//    one cp.async.bulk per row, boundary resolved at staging time).  u8: two
//    pixels per instruction in 16-bit lanes with the native 3-input
//    VIMNMX3.U16x2 (pixels q, q+2 per register, as the SWAR convolution);
//    f32: FMNMX per pixel.  HBM-bound (2 or 8 bytes per pixel).
//  * reduce_generic_kernel: any domain up to 63x63 (one bit per tap), one
//    thread per output pixel, per-tap boundary resolution.
#include <cuda_runtime.h>
#include <stdint.h>

#include <cstdlib>

#include "boundary.cuh"
#include "kernels.h"
#include "launch_cache.h"
#include "lop_params.h"
#include "stage.cuh"

namespace lop {

namespace red {
constexpr int NT = 128;
template <typename T, int TS_ = (sizeof(T) == 4 ? 8 : 16)> struct Shape {
    static constexpr int PX = sizeof(T) == 4 ? 4 : 8;        // columns per thread
    static constexpr int TWE = NT * PX;                      // tile width (elements)
    static constexpr int PADE = 16 / (int)sizeof(T);         // 16-B pad each side (>= R)
    static constexpr int SWE = TWE + 2 * PADE;               // smem row pitch
    static constexpr int TS = TS_;                           // output rows per tile
};
}  // namespace red

template <int OP> __device__ __forceinline__ float red_f(float a, float b)
{
    return OP == RED_MIN ? fminf(a, b) : fmaxf(a, b);
}
// u8 pixels in 16-bit lanes: native VIMNMX.U16x2 / VIMNMX3.U16x2 (3-input)
// on sm_100 (the byte-SIMD __vminu4 is emulated with ~7 instructions).
template <int OP> __device__ __forceinline__ uint32_t red2(uint32_t a, uint32_t b)
{
    return OP == RED_MIN ? __vminu2(a, b) : __vmaxu2(a, b);
}
template <int OP> __device__ __forceinline__ uint32_t red3(uint32_t a, uint32_t b, uint32_t c)
{
    return OP == RED_MIN ? __vimin3_u16x2(a, b, c) : __vimax3_u16x2(a, b, c);
}
// reduction of x[0..N-1] with 3-input instructions
template <int OP, int N> __device__ __forceinline__ uint32_t red_n(const uint32_t *x)
{
    uint32_t m = N >= 3 ? red3<OP>(x[0], x[1], x[2]) : (N == 2 ? red2<OP>(x[0], x[1]) : x[0]);
#pragma unroll
    for (int i = 3; i < N; i += 2) m = i + 1 < N ? red3<OP>(m, x[i], x[i + 1]) : red2<OP>(m, x[i]);
    return m;
}

// Filter one staged tile (thread: PX columns streamed down the tile).  FULL:
// all TS + 2R staged rows present (no per-row bound check); VEC: the CTA's
// whole tile row is inside the iteration space and aligned (every thread
// stores whole vectors, no per-row divergent store branch).  Output rows are
// addressed by a running pointer.
template <typename T, int OP, int R, int TS_, bool FULL, bool VEC>
__device__ __forceinline__ void reduce_compute(const Common &c, const T *tile, int srows, char *obase,
                                               int ox0, int roi_x1, bool ovec)
{
    using S = red::Shape<T, TS_>;
    constexpr int PX = S::PX, SWE = S::SWE, PADE = S::PADE, TS = S::TS, P = 2 * R + 1;
    const T *tcol = tile + PADE + threadIdx.x * PX;
    if constexpr (sizeof(T) == 1) {
        // staged words W0..W3 = bytes -4..11 of this thread's 8 columns; sources
        // S[q + R] = bytes (q, q+2) in the two 16-bit lanes (as conv_u8_swar)
        uint32_t h[P][4];                                        // lanes (0,2) (1,3) (4,6) (5,7)
#pragma unroll
        for (int k = 0; k < TS + 2 * R; ++k) {
            if (!FULL && k >= srows) break;
            const uint8_t *rp = reinterpret_cast<const uint8_t *>(tcol) + k * SWE;
            const uint2 cv = *reinterpret_cast<const uint2 *>(rp);
            const uint32_t W[4] = {*reinterpret_cast<const uint32_t *>(rp - 4), cv.x, cv.y,
                                   *reinterpret_cast<const uint32_t *>(rp + 8)};
            uint32_t E[4], O[4];
#pragma unroll
            for (int i = 0; i < 4; ++i) {
                E[i] = __byte_perm(W[i], 0u, 0x4240);
                O[i] = __byte_perm(W[i], 0u, 0x4341);
            }
            uint32_t Sx[6 + 2 * R];
#pragma unroll
            for (int q = -R; q <= 5 + R; ++q) {
                const int wi = (q + 4) >> 2, sh = (q + 4) & 3;
                if (sh == 0) Sx[q + R] = E[wi];
                else if (sh == 1) Sx[q + R] = O[wi];
                else if (sh == 2) Sx[q + R] = __byte_perm(E[wi], E[wi + 1], 0x5412);
                else Sx[q + R] = __byte_perm(O[wi], O[wi + 1], 0x5412);
            }
            constexpr int J[4] = {0, 1, 4, 5};
#pragma unroll
            for (int jj = 0; jj < 4; ++jj) h[k % P][jj] = red_n<OP, P>(Sx + J[jj]);
            const int o = k - 2 * R;
            if (o < 0) continue;
            uint32_t q4[4];
#pragma unroll
            for (int jj = 0; jj < 4; ++jj) {
                uint32_t col[P];
#pragma unroll
                for (int t = 0; t < P; ++t) col[t] = h[(o + t) % P][jj];
                q4[jj] = red_n<OP, P>(col);
            }
            const uint32_t lo = __byte_perm(q4[0], q4[1], 0x6240), hi = __byte_perm(q4[2], q4[3], 0x6240);
            uint8_t *op = reinterpret_cast<uint8_t *>(obase) + ox0;
            obase += c.out.stride;
            if (VEC || ovec) {
                *reinterpret_cast<uint2 *>(op) = make_uint2(lo, hi);
            } else {
#pragma unroll
                for (int j = 0; j < 8; ++j)
                    if (ox0 + j < roi_x1) op[j] = (uint8_t)((j < 4 ? lo : hi) >> (8 * (j & 3)));
            }
        }
    } else {
        float h[P][PX];
#pragma unroll
        for (int k = 0; k < TS + 2 * R; ++k) {
            if (!FULL && k >= srows) break;
            const float *rp = reinterpret_cast<const float *>(tcol) + k * SWE;
            const float4 cv = *reinterpret_cast<const float4 *>(rp);
            const float4 l = *reinterpret_cast<const float4 *>(rp - 4);
            const float4 r = *reinterpret_cast<const float4 *>(rp + 4);
            const float v[12] = {l.x, l.y, l.z, l.w, cv.x, cv.y, cv.z, cv.w, r.x, r.y, r.z, r.w};
#pragma unroll
            for (int j = 0; j < PX; ++j) {
                float m = v[4 + j];
#pragma unroll
                for (int s = 1; s <= R; ++s) m = red_f<OP>(red_f<OP>(m, v[4 + j - s]), v[4 + j + s]);
                h[k % P][j] = m;
            }
            const int o = k - 2 * R;
            if (o < 0) continue;
            float q[PX];
#pragma unroll
            for (int j = 0; j < PX; ++j) {
                float m = h[o % P][j];
#pragma unroll
                for (int t = 1; t < P; ++t) m = red_f<OP>(m, h[(o + t) % P][j]);
                q[j] = m;
            }
            float *op = reinterpret_cast<float *>(obase) + ox0;
            obase += c.out.stride;
            if (VEC || ovec) {
                *reinterpret_cast<float4 *>(op) = make_float4(q[0], q[1], q[2], q[3]);
            } else {
#pragma unroll
                for (int j = 0; j < PX; ++j)
                    if (ox0 + j < roi_x1) op[j] = q[j];
            }
        }
    }
}

template <typename T, int OP, int R, int TS_>
__global__ void __launch_bounds__(red::NT) reduce_tiled_kernel(const __grid_constant__ ReduceParams p)
{
    using S = red::Shape<T, TS_>;
    constexpr int PX = S::PX, SWE = S::SWE, PADE = S::PADE, TS = S::TS;
    static_assert(R >= 1 && R <= 4, "halo must fit the 16-B pad");
    extern __shared__ __align__(16) unsigned char smem_raw[];
    __shared__ __align__(8) uint64_t bar;
    T *tile = reinterpret_cast<T *>(smem_raw);
    const Common &c = p.c;
    const int b = blockIdx.z;
    const int tx0 = c.roi_x0 + blockIdx.x * S::TWE, ty0 = c.roi_y0 + blockIdx.y * TS;
    const int roi_x1 = c.roi_x0 + c.roi_w;
    const int nrows = min(TS, c.roi_y0 + c.roi_h - ty0), srows = nrows + 2 * R;
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared.b64 [%0], 1;" ::"r"(smem_addr(&bar)));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    stage_rows<T, SWE, red::NT>(c, b, tx0 + c.off_x - PADE, ty0 + c.off_y - R, srows, tile, &bar);
    __syncthreads();
    mbar_wait(&bar, 0);

    const int ox0 = tx0 + threadIdx.x * PX;
    if (ox0 >= roi_x1) return;
    char *obase = c.out.data + (int64_t)b * c.out.bstride + (int64_t)ty0 * c.out.stride;
    const bool ovec = (ox0 + PX <= roi_x1) && (ox0 % PX == 0) &&
                      (((reinterpret_cast<uintptr_t>(obase) | (uintptr_t)c.out.stride) %
                        (sizeof(T) * PX)) == 0);
    const bool full = srows == TS + 2 * R;
    const bool cta_vec = tx0 + S::TWE <= roi_x1 &&
                         ((reinterpret_cast<uintptr_t>(obase) | (uintptr_t)c.out.stride) % 16) == 0;
    if (full && cta_vec) reduce_compute<T, OP, R, TS_, true, true>(c, tile, srows, obase, ox0, roi_x1, ovec);
    else if (full) reduce_compute<T, OP, R, TS_, true, false>(c, tile, srows, obase, ox0, roi_x1, ovec);
    else reduce_compute<T, OP, R, TS_, false, false>(c, tile, srows, obase, ox0, roi_x1, ovec);
}

template <int OP>
__global__ void __launch_bounds__(256) reduce_generic_kernel(const __grid_constant__ ReduceParams p)
{
    const Common &c = p.c;
    const int ox = c.roi_x0 + blockIdx.x * blockDim.x + threadIdx.x;
    const int oy = c.roi_y0 + blockIdx.y * blockDim.y + threadIdx.y;
    const int b = blockIdx.z;
    if (ox >= c.roi_x0 + c.roi_w || oy >= c.roi_y0 + c.roi_h) return;
    const int ix = ox + c.off_x, iy = oy + c.off_y;
    char *orow = c.out.data + (int64_t)b * c.out.bstride + (int64_t)oy * c.out.stride;
    float mf = 0.f;
    uint32_t mi = 0;
    bool first = true;
    for (int yf = -c.ry; yf <= c.ry; ++yf) {
        uint64_t bits = p.dom[yf + c.ry];
        if (!bits) continue;
        int row;
        const bool row_ok = resolve_row(iy + yf, c.in, c.mode, row);
        while (bits) {
            const int xf = __ffsll((long long)bits) - 1 - c.rx;
            bits &= bits - 1;
            int col;
            const bool ok = row_ok && resolve_col(ix + xf, c.in, c.mode, col);
            if (p.u8) {
                const uint32_t v = ok ? (uint32_t)__ldg(row_ptr<uint8_t>(c.in, b, row) + col)
                                      : (uint32_t)c.cval_i;
                mi = first ? v : (OP == RED_MIN ? min(mi, v) : max(mi, v));
            } else {
                const float v = ok ? __ldg(row_ptr<float>(c.in, b, row) + col) : c.cval_f;
                mf = first ? v : red_f<OP>(mf, v);
            }
            first = false;
        }
    }
    if (p.u8) reinterpret_cast<uint8_t *>(orow)[ox] = (uint8_t)mi;
    else reinterpret_cast<float *>(orow)[ox] = mf;
}

namespace {

template <typename T, int OP, int R, int TS>
cudaError_t launch_tiled_ts(const ReduceParams &p, cudaStream_t stream)
{
    using S = red::Shape<T, TS>;
    const size_t smem = (size_t)(S::TS + 2 * R) * S::SWE * sizeof(T);
    static PerDevice configured;
    const cudaError_t e = ensure_smem(reduce_tiled_kernel<T, OP, R, TS>, smem, configured);
    if (e != cudaSuccess) return e;
    dim3 grid((p.c.roi_w + S::TWE - 1) / S::TWE, (p.c.roi_h + S::TS - 1) / S::TS, p.c.batch);
    reduce_tiled_kernel<T, OP, R, TS><<<grid, red::NT, smem, stream>>>(p);
    return cudaGetLastError();
}

// output rows per tile: default f32 8, u8 16; LOP_REDUCE_TS (4 / 8 / 16) overrides
template <typename T, int OP, int R>
cudaError_t launch_tiled_r(const ReduceParams &p, cudaStream_t stream)
{
    int ts = sizeof(T) == 4 ? 8 : 16;
    if (const char *env = std::getenv("LOP_REDUCE_TS")) ts = std::atoi(env);
    if (ts == 4) return launch_tiled_ts<T, OP, R, 4>(p, stream);
    if (ts == 16) return launch_tiled_ts<T, OP, R, 16>(p, stream);
    return launch_tiled_ts<T, OP, R, 8>(p, stream);
}

template <typename T, int OP>
cudaError_t launch_tiled_op(const ReduceParams &p, cudaStream_t stream)
{
    switch (p.c.rx) {
    case 1: return launch_tiled_r<T, OP, 1>(p, stream);
    case 2: return launch_tiled_r<T, OP, 2>(p, stream);
    case 3: return launch_tiled_r<T, OP, 3>(p, stream);
    case 4: return launch_tiled_r<T, OP, 4>(p, stream);
    default: return cudaErrorNotSupported;
    }
}

}  // namespace

cudaError_t launch_reduce(const ReduceParams &p, bool allow_tiled, cudaStream_t stream)
{
    const bool tiled = allow_tiled && p.full && p.c.rx == p.c.ry && p.c.rx >= 1 && p.c.rx <= 4;
    if (tiled) {
        if (p.u8) return p.op == RED_MIN ? launch_tiled_op<uint8_t, RED_MIN>(p, stream)
                                         : launch_tiled_op<uint8_t, RED_MAX>(p, stream);
        return p.op == RED_MIN ? launch_tiled_op<float, RED_MIN>(p, stream)
                               : launch_tiled_op<float, RED_MAX>(p, stream);
    }
    dim3 block(32, 8);
    dim3 grid((p.c.roi_w + 31) / 32, (p.c.roi_h + 7) / 8, p.c.batch);
    if (p.op == RED_MIN) reduce_generic_kernel<RED_MIN><<<grid, block, 0, stream>>>(p);
    else reduce_generic_kernel<RED_MAX><<<grid, block, 0, stream>>>(p);
    return cudaGetLastError();
}

}  // namespace lop

// conv_pair.cu -- two local operators on one input with a point-operator
// epilogue combining them, in one pass ("point operators in
// the prologue or epilogue"; PAPER.md L107-L122 on point / local operators):
//   out(x,y) = combine(A(x,y), B(x,y)),  A = Ma (*) I,  B = Mb (*) I
// e.g. the Sobel gradient magnitude sqrt(gx^2 + gy^2) (Sobel: Table IX,
// L847-L849).  A and B are computed exactly like lop_convolve_execute (same
// separable factorisation, same operations in the same order), so the result
// equals combine() applied to two separate convolution passes bit for bit;
// the input is read once and A, B never reach HBM.
//
//  * conv_pair_kernel<T, TO, R, CMB>: both masks exactly separable with the
//    same radius R <= 2; tile staging as the convolution kernels (stage.cuh);
//    per staged row the horizontal sums of both masks go to two register
//    rings, the vertical sums give A and B, the epilogue combines them.
//  * conv_pair_generic_kernel: any two masks (2D sums in conv_generic order).
#include <cuda_runtime.h>
#include <stdint.h>

#include <type_traits>

#include "boundary.cuh"
#include "kernels.h"
#include "lop_params.h"
#include "stage.cuh"

namespace lop {

namespace cpair {
constexpr int NT = 128;
template <typename T> struct Shape {
    static constexpr int PX = sizeof(T) == 4 ? 4 : 8;        // columns per thread
    static constexpr int TWE = NT * PX;                      // tile width (elements)
    static constexpr int PADE = 16 / (int)sizeof(T);         // 16-B pad each side
    static constexpr int SWE = TWE + 2 * PADE;               // smem row pitch
    static constexpr int TS = 8;                             // output rows per tile
};
}  // namespace cpair

// The point-operator epilogue (exact IEEE f32 operations in a fixed order /
// exact integers).
template <int CMB> __device__ __forceinline__ float combine_f(float a, float b)
{
    if (CMB == PAIR_L1) return __fadd_rn(fabsf(a), fabsf(b));
    const float s = __fadd_rn(__fmul_rn(a, a), __fmul_rn(b, b));
    return CMB == PAIR_L2 ? __fsqrt_rn(s) : s;
}
template <int CMB> __device__ __forceinline__ int combine_i(int a, int b)
{
    return CMB == PAIR_L1 ? abs(a) + abs(b) : a * a + b * b;
}

// One staged tile (see conv_tiled.cu conv_compute): FULL = all TS + 2R staged
// rows present (no per-row bound check), VEC = the CTA's tile row lies in the
// iteration space and is 16-B aligned (whole-vector stores, no per-row
// divergent store branch); output rows by a running pointer.
template <typename T, typename TO, int R, int CMB, bool FULL, bool VEC>
__device__ __forceinline__ void conv_pair_compute(const ConvPair &p, const T *tile, int srows, char *obase,
                                                  int ox0, int roi_x1, bool ovec)
{
    using S = cpair::Shape<T>;
    constexpr int PX = S::PX, SWE = S::SWE, PADE = S::PADE, TS = S::TS, P = 2 * R + 1;
    constexpr bool F = sizeof(T) == 4;
    using A = typename std::conditional<F, float, int>::type;
    const Common &c = p.a.c;
    const T *tcol = tile + PADE + threadIdx.x * PX;
    A ha[P][PX], hb[P][PX];                                      // horizontal sums, rings
#pragma unroll
    for (int k = 0; k < TS + 2 * R; ++k) {
        if (!FULL && k >= srows) break;
        A v[PX + 2 * R];
        if constexpr (F) {
            const float *rp = reinterpret_cast<const float *>(tcol) + k * SWE;
            const float4 cv = *reinterpret_cast<const float4 *>(rp);
            const float4 l = *reinterpret_cast<const float4 *>(rp - 4);
            const float4 r = *reinterpret_cast<const float4 *>(rp + 4);
            const float lv[4] = {l.x, l.y, l.z, l.w}, rv[4] = {r.x, r.y, r.z, r.w};
            v[R + 0] = cv.x; v[R + 1] = cv.y; v[R + 2] = cv.z; v[R + 3] = cv.w;
#pragma unroll
            for (int j = 0; j < R; ++j) { v[j] = lv[4 - R + j]; v[R + PX + j] = rv[j]; }
        } else {
            const uint8_t *rp = reinterpret_cast<const uint8_t *>(tcol) + k * SWE;
            const uint2 cv = *reinterpret_cast<const uint2 *>(rp);
            const uint32_t w[2] = {cv.x, cv.y};
            const uint32_t l = *reinterpret_cast<const uint32_t *>(rp - 4);
            const uint32_t r = *reinterpret_cast<const uint32_t *>(rp + 8);
#pragma unroll
            for (int j = 0; j < 8; ++j) v[R + j] = (int)((w[j >> 2] >> (8 * (j & 3))) & 0xFF);
#pragma unroll
            for (int j = 0; j < R; ++j) {
                v[j] = (int)((l >> (8 * (4 - R + j))) & 0xFF);
                v[R + PX + j] = (int)((r >> (8 * j)) & 0xFF);
            }
        }
        // horizontal sums of both masks (the operations of conv_sep_kernel)
#pragma unroll
        for (int j = 0; j < PX; ++j) {
            A sa, sb;
            if constexpr (F) {
                sa = __fmul_rn(p.a.rf[0], v[j]);
                sb = __fmul_rn(p.b.rf[0], v[j]);
#pragma unroll
                for (int t = 1; t <= 2 * R; ++t) {
                    sa = __fmaf_rn(p.a.rf[t], v[j + t], sa);
                    sb = __fmaf_rn(p.b.rf[t], v[j + t], sb);
                }
            } else {
                sa = p.a.ri[0] * v[j];
                sb = p.b.ri[0] * v[j];
#pragma unroll
                for (int t = 1; t <= 2 * R; ++t) {
                    sa += p.a.ri[t] * v[j + t];
                    sb += p.b.ri[t] * v[j + t];
                }
            }
            ha[k % P][j] = sa;
            hb[k % P][j] = sb;
        }
        const int o = k - 2 * R;
        if (o < 0) continue;
        TO out[PX];
#pragma unroll
        for (int j = 0; j < PX; ++j) {
            A sa, sb;
            if constexpr (F) {
                sa = __fmul_rn(p.a.cf[0], ha[o % P][j]);
                sb = __fmul_rn(p.b.cf[0], hb[o % P][j]);
#pragma unroll
                for (int t = 1; t <= 2 * R; ++t) {
                    sa = __fmaf_rn(p.a.cf[t], ha[(o + t) % P][j], sa);
                    sb = __fmaf_rn(p.b.cf[t], hb[(o + t) % P][j], sb);
                }
                out[j] = combine_f<CMB>(sa, sb);
            } else {
                sa = p.a.ci[0] * ha[o % P][j];
                sb = p.b.ci[0] * hb[o % P][j];
#pragma unroll
                for (int t = 1; t <= 2 * R; ++t) {
                    sa += p.a.ci[t] * ha[(o + t) % P][j];
                    sb += p.b.ci[t] * hb[(o + t) % P][j];
                }
                out[j] = combine_i<CMB>(sa, sb);
            }
        }
        TO *op = reinterpret_cast<TO *>(obase) + ox0;                // output row o (running pointer)
        obase += c.out.stride;
        if (VEC || ovec) {
#pragma unroll
            for (int q = 0; q < PX / 4; ++q)
                *reinterpret_cast<typename std::conditional<F, float4, int4>::type *>(op + 4 * q) =
                    {out[4 * q], out[4 * q + 1], out[4 * q + 2], out[4 * q + 3]};
        } else {
#pragma unroll
            for (int j = 0; j < PX; ++j)
                if (ox0 + j < roi_x1) op[j] = out[j];
        }
    }
}

template <typename T, typename TO, int R, int CMB>
__global__ void __launch_bounds__(cpair::NT) conv_pair_kernel(const __grid_constant__ ConvPair p)
{
    using S = cpair::Shape<T>;
    constexpr int PX = S::PX, SWE = S::SWE, PADE = S::PADE, TS = S::TS;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    __shared__ __align__(8) uint64_t bar;
    T *tile = reinterpret_cast<T *>(smem_raw);
    const Common &c = p.a.c;
    const int b = blockIdx.z;
    const int tx0 = c.roi_x0 + blockIdx.x * S::TWE, ty0 = c.roi_y0 + blockIdx.y * TS;
    const int roi_x1 = c.roi_x0 + c.roi_w;
    const int nrows = min(TS, c.roi_y0 + c.roi_h - ty0), srows = nrows + 2 * R;
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared.b64 [%0], 1;" ::"r"(smem_addr(&bar)));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    stage_rows<T, SWE, cpair::NT>(c, b, tx0 + c.off_x - PADE, ty0 + c.off_y - R, srows, tile, &bar);
    __syncthreads();
    mbar_wait(&bar, 0);

    const int ox0 = tx0 + threadIdx.x * PX;
    if (ox0 >= roi_x1) return;
    char *obase = c.out.data + (int64_t)b * c.out.bstride + (int64_t)ty0 * c.out.stride;
    const bool ovec = (ox0 + PX <= roi_x1) && (ox0 % PX == 0) &&
                      (((reinterpret_cast<uintptr_t>(obase) | (uintptr_t)c.out.stride) % 16) == 0);
    const bool full = srows == TS + 2 * R;
    const bool cta_vec = tx0 + S::TWE <= roi_x1 &&
                         ((reinterpret_cast<uintptr_t>(obase) | (uintptr_t)c.out.stride) % 16) == 0;
    // f32: full-tile / whole-vector instances (Sobel magnitude 29.0 -> 27.6 us at 4096^2);
    // u8 -> i32 keeps the checked form, which measured faster for it (19.5 vs 22.7 us)
    if (sizeof(T) == 4 && full && cta_vec)
        conv_pair_compute<T, TO, R, CMB, true, true>(p, tile, srows, obase, ox0, roi_x1, ovec);
    else if (sizeof(T) == 4 && full)
        conv_pair_compute<T, TO, R, CMB, true, false>(p, tile, srows, obase, ox0, roi_x1, ovec);
    else
        conv_pair_compute<T, TO, R, CMB, false, false>(p, tile, srows, obase, ox0, roi_x1, ovec);
}

// Any two masks: one thread per output, both 2D sums in conv_generic_kernel's
// order (yf outer, xf inner, per-tap boundary resolution), then the epilogue.
template <int CMB>
__global__ void __launch_bounds__(256) conv_pair_generic_kernel(const __grid_constant__ ConvPairGeneric p)
{
    const Common &c = p.c;
    const int ox = c.roi_x0 + blockIdx.x * blockDim.x + threadIdx.x;
    const int oy = c.roi_y0 + blockIdx.y * blockDim.y + threadIdx.y;
    const int b = blockIdx.z;
    if (ox >= c.roi_x0 + c.roi_w || oy >= c.roi_y0 + c.roi_h) return;
    const int ix = ox + c.off_x, iy = oy + c.off_y;
    const int sx = 2 * c.rx + 1;
    char *orow = c.out.data + (int64_t)b * c.out.bstride + (int64_t)oy * c.out.stride;
    if (!p.u8) {
        float sa = 0.0f, sb = 0.0f;
        for (int yf = -c.ry; yf <= c.ry; ++yf) {
            int row;
            const bool row_ok = resolve_row(iy + yf, c.in, c.mode, row);
            for (int xf = -c.rx; xf <= c.rx; ++xf) {
                int col;
                float v = c.cval_f;
                if (row_ok && resolve_col(ix + xf, c.in, c.mode, col)) v = __ldg(row_ptr<float>(c.in, b, row) + col);
                const int m = (yf + c.ry) * sx + xf + c.rx;
                sa = __fmaf_rn(p.ma[m], v, sa);
                sb = __fmaf_rn(p.mb[m], v, sb);
            }
        }
        reinterpret_cast<float *>(orow)[ox] = combine_f<CMB>(sa, sb);
    } else {
        int sa = 0, sb = 0;
        for (int yf = -c.ry; yf <= c.ry; ++yf) {
            int row;
            const bool row_ok = resolve_row(iy + yf, c.in, c.mode, row);
            for (int xf = -c.rx; xf <= c.rx; ++xf) {
                int col;
                int v = c.cval_i;
                if (row_ok && resolve_col(ix + xf, c.in, c.mode, col)) v = __ldg(row_ptr<uint8_t>(c.in, b, row) + col);
                const int m = (yf + c.ry) * sx + xf + c.rx;
                sa += p.ia[m] * v;
                sb += p.ib[m] * v;
            }
        }
        reinterpret_cast<int32_t *>(orow)[ox] = combine_i<CMB>(sa, sb);
    }
}

namespace {

template <typename T, typename TO, int R, int CMB>
cudaError_t launch_pair_cfg(const ConvPair &p, cudaStream_t stream)
{
    using S = cpair::Shape<T>;
    const size_t smem = (size_t)(S::TS + 2 * R) * S::SWE * sizeof(T);
    const Common &c = p.a.c;
    dim3 grid((c.roi_w + S::TWE - 1) / S::TWE, (c.roi_h + S::TS - 1) / S::TS, c.batch);
    conv_pair_kernel<T, TO, R, CMB><<<grid, cpair::NT, smem, stream>>>(p);
    return cudaGetLastError();
}

template <typename T, typename TO, int CMB>
cudaError_t launch_pair_r(const ConvPair &p, cudaStream_t stream)
{
    switch (p.a.c.rx) {
    case 1: return launch_pair_cfg<T, TO, 1, CMB>(p, stream);
    case 2: return launch_pair_cfg<T, TO, 2, CMB>(p, stream);
    default: return cudaErrorNotSupported;
    }
}

template <typename T, typename TO>
cudaError_t launch_pair_t(const ConvPair &p, cudaStream_t stream)
{
    switch (p.combine) {
    case PAIR_L2: return launch_pair_r<T, TO, PAIR_L2>(p, stream);
    case PAIR_L1: return launch_pair_r<T, TO, PAIR_L1>(p, stream);
    case PAIR_SUMSQ: return launch_pair_r<T, TO, PAIR_SUMSQ>(p, stream);
    default: return cudaErrorNotSupported;
    }
}

}  // namespace

cudaError_t launch_conv_pair(const ConvPair &p, cudaStream_t stream)
{
    if (p.a.c.rx != p.a.c.ry || p.a.c.rx < 1 || p.a.c.rx > 2) return cudaErrorNotSupported;
    if (p.u8) {
        if (p.combine == PAIR_L2) return cudaErrorNotSupported;
        return launch_pair_t<uint8_t, int32_t>(p, stream);
    }
    return launch_pair_t<float, float>(p, stream);
}

cudaError_t launch_conv_pair_generic(const ConvPairGeneric &p, cudaStream_t stream)
{
    dim3 block(32, 8);
    dim3 grid((p.c.roi_w + 31) / 32, (p.c.roi_h + 7) / 8, p.c.batch);
    switch (p.combine) {
    case PAIR_L2: conv_pair_generic_kernel<PAIR_L2><<<grid, block, 0, stream>>>(p); break;
    case PAIR_L1: conv_pair_generic_kernel<PAIR_L1><<<grid, block, 0, stream>>>(p); break;
    case PAIR_SUMSQ: conv_pair_generic_kernel<PAIR_SUMSQ><<<grid, block, 0, stream>>>(p); break;
    default: return cudaErrorNotSupported;
    }
    return cudaGetLastError();
}

}  // namespace lop

// conv_chain.cu -- fused two-stage local operator ("chaining
// Gaussian -> Sobel in one pass with halo recompute"): out = M2 (*) (M1 (*) I),
// both stages with the same BoundaryCondition, exactly the result of two
// lop_convolve_execute passes (bit for bit), without the intermediate image
// making a round trip through HBM.
//
// Per CTA (128 threads):
//   1. stage the input footprint (output tile + R1 + R2 halo) into smem with the
//      bulk-copy staging of the convolution kernels (stage.cuh);
//   2. compute the intermediate G over the output tile + R2 halo into smem with
//      the same separable arithmetic as conv_sep_kernel (pass 1); G positions
//      outside the image follow pass 2's boundary condition on G (constant, or
//      G at the per-axis mapped position, recomputed from global memory);
//   3. stream the output rows from the G tile (pass 2) and store them.
// Tile: f32 4 columns/thread (G 512 wide, output 504), u8 8 columns/thread
// (G 1024 wide, output 992: 16-B aligned input origin); TS = 8 output rows.
#include <cuda_runtime.h>
#include <stdint.h>

#include <cstdlib>
#include <type_traits>

#include "boundary.cuh"
#include "kernels.h"
#include "lop_params.h"
#include "stage.cuh"

namespace lop {

namespace chain {
constexpr int NT = 128;
constexpr int kDefTS_f32 = 8, kDefTS_u8 = 8;   // output rows per tile (tools/tune_chain)

template <typename T> struct Shape {
    static constexpr int PX = sizeof(T) == 4 ? 4 : 8;      // columns per thread
    static constexpr int GW = NT * PX;                     // intermediate tile width
    static constexpr int HALO = 16 / sizeof(T);            // G halo per side (>= R2): keeps the
                                                           // input origin 16-B aligned
    static constexpr int OW = GW - 2 * HALO;               // output tile width
    static constexpr int IPAD = 16 / sizeof(T);            // input pad beyond G (>= R1), 16 B
    static constexpr int ISW = GW + 2 * IPAD;              // input smem pitch (elements)
};
}  // namespace chain

// PX + 2R values starting R before column `col` of a smem row (pitch-aligned
// vector loads, as in conv_sep_kernel).
template <typename T, int R, typename A>
__device__ __forceinline__ void chain_gather(const T *rp, A *v)
{
    constexpr int PX = chain::Shape<T>::PX;
    if constexpr (sizeof(T) == 4) {
        const float4 cv = *reinterpret_cast<const float4 *>(rp);
        v[R + 0] = cv.x; v[R + 1] = cv.y; v[R + 2] = cv.z; v[R + 3] = cv.w;
        if constexpr (R > 0) {
            const float4 l = *reinterpret_cast<const float4 *>(rp - 4);
            const float4 r = *reinterpret_cast<const float4 *>(rp + 4);
            const float lv[4] = {l.x, l.y, l.z, l.w}, rv[4] = {r.x, r.y, r.z, r.w};
#pragma unroll
            for (int j = 0; j < R; ++j) {
                v[j] = lv[4 - R + j];
                v[R + PX + j] = rv[j];
            }
        }
    } else {
        const uint2 cv = *reinterpret_cast<const uint2 *>(rp);
        const uint32_t w[2] = {cv.x, cv.y};
#pragma unroll
        for (int j = 0; j < 8; ++j) v[R + j] = (int)((w[j >> 2] >> (8 * (j & 3))) & 0xFF);
        if constexpr (R > 0) {
            const uint32_t l = *reinterpret_cast<const uint32_t *>(rp - 4);
            const uint32_t r = *reinterpret_cast<const uint32_t *>(rp + 8);
#pragma unroll
            for (int j = 0; j < R; ++j) {
                v[j] = (int)((l >> (8 * (4 - R + j))) & 0xFF);
                v[R + PX + j] = (int)((r >> (8 * j)) & 0xFF);
            }
        }
    }
}

// Separable arithmetic of conv_sep_kernel: horizontal then vertical pass.
template <typename A, int R>
__device__ __forceinline__ A sep_h(const ConvSep &s, const A *v)
{
    A acc;
    if constexpr (std::is_same<A, float>::value) {
        acc = __fmul_rn(s.rf[0], v[0]);
#pragma unroll
        for (int t = 1; t <= 2 * R; ++t) acc = __fmaf_rn(s.rf[t], v[t], acc);
    } else {
        acc = s.ri[0] * v[0];
#pragma unroll
        for (int t = 1; t <= 2 * R; ++t) acc += s.ri[t] * v[t];
    }
    return acc;
}

template <typename A, int R>
__device__ __forceinline__ A sep_v(const ConvSep &s, const A *h)
{
    A acc;
    if constexpr (std::is_same<A, float>::value) {
        acc = __fmul_rn(s.cf[0], h[0]);
#pragma unroll
        for (int t = 1; t <= 2 * R; ++t) acc = __fmaf_rn(s.cf[t], h[t], acc);
    } else {
        acc = s.ci[0] * h[0];
#pragma unroll
        for (int t = 1; t <= 2 * R; ++t) acc += s.ci[t] * h[t];
    }
    return acc;
}

// Pass-1 value (before quantisation) at in-image (x, y), reading the input with
// its boundary condition from global memory -- for G positions outside the
// image, which take G at their mapped position (pass 2's boundary on G).
// Rarely executed (border tiles only): kept out of line and rolled so that the
// hot path's instruction footprint stays small.
template <typename T, typename A, int R1>
__device__ __noinline__ A sep_point(const ConvSep &s, const Common &c, int b, int x, int y)
{
    A h[2 * R1 + 1];
#pragma unroll
    for (int t = 0; t <= 2 * R1; ++t) {
        A v[2 * R1 + 1];
#pragma unroll
        for (int k = 0; k <= 2 * R1; ++k) {
            if constexpr (sizeof(T) == 4)
                v[k] = read_f32(c.in, b, x + k - R1, y + t - R1, c.mode, c.cval_f);
            else
                v[k] = read_u8(c.in, b, x + k - R1, y + t - R1, c.mode, c.cval_i);
        }
        h[t] = sep_h<A, R1>(s, v);
    }
    return sep_v<A, R1>(s, h);
}

template <typename A, typename TG>
__device__ __forceinline__ TG to_g(A v, int shift)
{
    if constexpr (std::is_same<TG, float>::value) return v;
    else return (TG)min(max(quantize_shift(v, shift), 0), 255);
}

// One output row of PX values (vector store when aligned, else per element).
template <typename TO, int PX, typename A>
__device__ __forceinline__ void store_row(char *orow, int ox0, int roi_x1, bool ovec,
                                          const A *out, int shift)
{
    if constexpr (std::is_same<TO, float>::value) {
        float *op = reinterpret_cast<float *>(orow) + ox0;
        if (ovec) {
            *reinterpret_cast<float4 *>(op) = make_float4(out[0], out[1], out[2], out[3]);
        } else {
            for (int j = 0; j < PX; ++j)
                if (ox0 + j < roi_x1) op[j] = out[j];
        }
    } else if constexpr (sizeof(TO) == 1) {
        uint32_t w[2] = {0u, 0u};
#pragma unroll
        for (int j = 0; j < PX; ++j) {
            const int q = min(max(quantize_shift(out[j], shift), 0), 255);
            w[j >> 2] |= (uint32_t)q << (8 * (j & 3));
        }
        uint8_t *op = reinterpret_cast<uint8_t *>(orow) + ox0;
        if (ovec) {
            *reinterpret_cast<uint2 *>(op) = make_uint2(w[0], w[1]);
        } else {
            for (int j = 0; j < PX; ++j)
                if (ox0 + j < roi_x1) op[j] = (uint8_t)(w[j >> 2] >> (8 * (j & 3)));
        }
    } else {
        int32_t *op = reinterpret_cast<int32_t *>(orow) + ox0;
        int q[PX];
#pragma unroll
        for (int j = 0; j < PX; ++j) q[j] = quantize_shift(out[j], shift);
        if (ovec) {
            *reinterpret_cast<int4 *>(op) = make_int4(q[0], q[1], q[2], q[3]);
            *reinterpret_cast<int4 *>(op + 4) = make_int4(q[4], q[5], q[6], q[7]);
        } else {
            for (int j = 0; j < PX; ++j)
                if (ox0 + j < roi_x1) op[j] = q[j];
        }
    }
}

template <typename T, typename TO, int R1, int R2, int TS>
__global__ void __launch_bounds__(chain::NT) conv_chain_kernel(const __grid_constant__ ConvChain p)
{
    using S = chain::Shape<T>;
    constexpr int PX = S::PX, GW = S::GW, HALO = S::HALO, OW = S::OW, IPAD = S::IPAD,
                  ISW = S::ISW;
    constexpr bool F = sizeof(T) == 4;
    using A = typename std::conditional<F, float, int>::type;
    using TG = T;                                                   // intermediate type
    static_assert(R1 <= IPAD && R2 <= 4 && R2 <= HALO, "halo");
    const Common &c = p.s1.c;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    __shared__ __align__(8) uint64_t bar;
    T *itile = reinterpret_cast<T *>(smem_raw);                     // ni x ISW
    const int b = blockIdx.z;
    const int tx0 = c.roi_x0 + blockIdx.x * OW;
    const int ty0 = c.roi_y0 + blockIdx.y * TS;
    const int roi_x1 = c.roi_x0 + c.roi_w, roi_y1 = c.roi_y0 + c.roi_h;
    const int nrows = min(TS, roi_y1 - ty0);
    const int ng = nrows + 2 * R2, ni = ng + 2 * R1;
    TG *gtile = reinterpret_cast<TG *>(smem_raw + (size_t)(TS + 2 * R1 + 2 * R2) * ISW * sizeof(T));
    const int gx0 = tx0 + c.off_x - HALO;                           // input col of G col 0
    const int gy0 = ty0 + c.off_y - R2;                             // input row of G row 0

    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared.b64 [%0], 1;" ::"r"(smem_addr(&bar)));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    // columns the outputs of this tile need: G [x_lo, x_hi), input up to x_hi + R1
    const int x_lo = HALO - R2;
    const int x_hi = min(GW, HALO + (min(roi_x1, tx0 + OW) - tx0) + R2);
    constexpr int V16 = 16 / sizeof(T);
    const int icols = min(ISW, (IPAD + x_hi + R1 + V16 - 1) / V16 * V16);
    stage_rows<T, ISW, chain::NT>(c, b, gx0 - IPAD, gy0 - R1, ni, itile, &bar, icols);
    __syncthreads();
    mbar_wait(&bar, 0);

    // ---- pass 1: G over the tile + R2 halo (thread: PX columns, all G rows).
    // The row loop is rolled in groups of one ring period (2R1+1 rows) so the
    // ring slots stay compile-time register indices while the code stays small.
    if (threadIdx.x * PX < x_hi) {
        constexpr int P = 2 * R1 + 1;
        const T *tcol = itile + IPAD + threadIdx.x * PX;
        A h[P][PX];
#pragma unroll 1
        for (int k0 = 0; k0 < ni; k0 += P) {
#pragma unroll
            for (int i = 0; i < P; ++i) {
                const int k = k0 + i;
                if (k >= ni) break;
                A v[PX + 2 * R1];
                chain_gather<T, R1, A>(tcol + k * ISW, v);
#pragma unroll
                for (int j = 0; j < PX; ++j) h[i][j] = sep_h<A, R1>(p.s1, v + j);
                const int g = k - 2 * R1;
                if (g < 0) continue;
                TG out[PX];
#pragma unroll
                for (int j = 0; j < PX; ++j) {
                    A col[P];
#pragma unroll
                    for (int t = 0; t < P; ++t) col[t] = h[(i + 1 + t) % P][j];   // rows g..k
                    out[j] = to_g<A, TG>(sep_v<A, R1>(p.s1, col), p.s1.shift);
                }
                TG *gp = gtile + g * GW + threadIdx.x * PX;
                if constexpr (F) {
                    *reinterpret_cast<float4 *>(gp) = make_float4(out[0], out[1], out[2], out[3]);
                } else {
                    uint32_t w[2] = {0u, 0u};
#pragma unroll
                    for (int j = 0; j < 8; ++j) w[j >> 2] |= (uint32_t)out[j] << (8 * (j & 3));
                    *reinterpret_cast<uint2 *>(gp) = make_uint2(w[0], w[1]);
                }
            }
        }
    }
    // ---- G positions outside the image: pass 2's boundary condition on G.
    // Only the G positions the tile's outputs read are fixed up (columns
    // [x_lo, x_hi), all G rows).  A mapped position that lies inside this tile
    // (clamp, mirror, and repeat for narrow images) is copied from the tile;
    // otherwise (repeat across the image) it is recomputed from global memory.
    const int GH = c.in.GH, IW = c.in.W;
    const bool border = gx0 + x_lo < 0 || gx0 + x_hi > IW || gy0 < 0 || gy0 + ng > GH;
    if (border) {
        __syncthreads();                      // all in-tile G values written
        const int span = x_hi - x_lo;
        for (int i = threadIdx.x; i < ng * span; i += chain::NT) {
            const int r = i / span, x = x_lo + (i - r * span);
            const int gx = gx0 + x, gy = gy0 + r;
            if ((unsigned)gx < (unsigned)IW && (unsigned)gy < (unsigned)GH) continue;
            TG val;
            if (c.mode == M_CONSTANT) {
                val = F ? (TG)c.cval_f : (TG)c.cval_i;
            } else {
                const int mx = map_axis(gx, IW, c.mode), my = map_axis(gy, GH, c.mode);
                const int tx = mx - gx0, ty = my - gy0;
                if (tx >= 0 && tx < GW && ty >= 0 && ty < ng)
                    val = gtile[ty * GW + tx];                         // computed in pass 1
                else
                    val = to_g<A, TG>(sep_point<T, A, R1>(p.s1, c, b, mx, my), p.s1.shift);
            }
            gtile[r * GW + x] = val;
        }
    }
    __syncthreads();

    // ---- pass 2: output rows from the G tile
    const int ox0 = tx0 + threadIdx.x * PX;
    if (threadIdx.x * PX >= OW || ox0 >= roi_x1) return;
    char *obase = c.out.data + (int64_t)b * c.out.bstride;
    const bool ovec = (ox0 + PX <= roi_x1) && (ox0 % PX == 0) &&
                      (((reinterpret_cast<uintptr_t>(obase) | (uintptr_t)c.out.stride) %
                        (sizeof(TO) * PX > 16 ? 16 : sizeof(TO) * PX)) == 0);
    const TG *gcol = gtile + HALO + threadIdx.x * PX;
    constexpr int P2 = 2 * R2 + 1;
    A h[P2][PX];
#pragma unroll 1
    for (int k0 = 0; k0 < ng; k0 += P2) {
#pragma unroll
        for (int i = 0; i < P2; ++i) {
            const int k = k0 + i;
            if (k >= ng) break;
            A v[PX + 2 * R2];
            chain_gather<TG, R2, A>(gcol + k * GW, v);
#pragma unroll
            for (int j = 0; j < PX; ++j) h[i][j] = sep_h<A, R2>(p.s2, v + j);
            const int o = k - 2 * R2;
            if (o < 0) continue;
            A out[PX];
#pragma unroll
            for (int j = 0; j < PX; ++j) {
                A col[P2];
#pragma unroll
                for (int t = 0; t < P2; ++t) col[t] = h[(i + 1 + t) % P2][j];   // rows o..k
                out[j] = sep_v<A, R2>(p.s2, col);
            }
            store_row<TO, PX>(obase + (int64_t)(ty0 + o) * c.out.stride, ox0, roi_x1, ovec, out,
                              p.s2.shift);
        }
    }
}

namespace {

template <typename T, typename TO, int R1, int R2, int TS>
cudaError_t launch_chain_cfg(const ConvChain &p, cudaStream_t stream)
{
    using S = chain::Shape<T>;
    const size_t smem = (size_t)(TS + 2 * R1 + 2 * R2) * S::ISW * sizeof(T) +
                        (size_t)(TS + 2 * R2) * S::GW * sizeof(T);
    static bool configured = false;
    if (!configured) {
        cudaError_t e = cudaFuncSetAttribute(conv_chain_kernel<T, TO, R1, R2, TS>,
                                             cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
        configured = true;
    }
    const Common &c = p.s1.c;
    dim3 grid((c.roi_w + S::OW - 1) / S::OW, (c.roi_h + TS - 1) / TS, c.batch);
    conv_chain_kernel<T, TO, R1, R2, TS><<<grid, chain::NT, smem, stream>>>(p);
    return cudaGetLastError();
}

// output rows per tile: LOP_CHAIN_TS overrides (tuning); default per type
template <typename T, typename TO, int R1, int R2>
cudaError_t launch_chain_rr(const ConvChain &p, cudaStream_t stream)
{
    int ts = sizeof(T) == 4 ? chain::kDefTS_f32 : chain::kDefTS_u8;
    if (const char *env = std::getenv("LOP_CHAIN_TS")) ts = std::atoi(env);
    switch (ts) {
    case 4: return launch_chain_cfg<T, TO, R1, R2, 4>(p, stream);
    case 16: return launch_chain_cfg<T, TO, R1, R2, 16>(p, stream);
    default: return launch_chain_cfg<T, TO, R1, R2, 8>(p, stream);
    }
}

template <typename T, typename TO>
cudaError_t launch_chain_t(const ConvChain &p, cudaStream_t stream)
{
    const int r1 = p.s1.c.rx, r2 = p.s2.c.rx;
    if (r1 == 1 && r2 == 1) return launch_chain_rr<T, TO, 1, 1>(p, stream);
    if (r1 == 1 && r2 == 2) return launch_chain_rr<T, TO, 1, 2>(p, stream);
    if (r1 == 2 && r2 == 1) return launch_chain_rr<T, TO, 2, 1>(p, stream);
    if (r1 == 2 && r2 == 2) return launch_chain_rr<T, TO, 2, 2>(p, stream);
    return cudaErrorNotSupported;
}

}  // namespace

cudaError_t launch_conv_chain(const ConvChain &p, cudaStream_t stream)
{
    switch (p.kind) {
    case 0: return launch_chain_t<float, float>(p, stream);
    case 1: return launch_chain_t<uint8_t, uint8_t>(p, stream);
    case 2: return launch_chain_t<uint8_t, int32_t>(p, stream);
    default: return cudaErrorNotSupported;
    }
}

}  // namespace lop

// bilateral.cu -- bilateral filter kernels for sm_100a.
//
// Method: Algorithm 1 with the precomputed closeness
// Mask of Listing 5 (L379-L416): one exp per tap, p/d normalisation.
// B200 design:
//  * bilateral_generic: one thread per output pixel, per-tap boundary
//    resolution, mask in the (large) kernel parameter block.  Any window up
//    to 63x63.  Fallback and cross-check: it uses the same per-tap helpers as
//    the tiled kernels, so the outputs are bit-identical.
//  * bilateral_sep_kernel<RX> (hot kernel, closeness from sigma_d): Eq. (1) is
//    separable, c(xf,yf) = cy[yf] * 2^lx[xf] (Listing 1 l.21 computes it as a
//    product of two 1D exps).  lx is folded into the exponent of each tap as a
//    compile-time-indexed constant-bank operand; cy multiplies the per-row
//    partial sums once per window row.  No mask traffic through shared memory.
//  * bilateral_tiled_kernel<RX> (user closeness Mask, Listing 4/5): the log2
//    mask row is read from shared memory (broadcast LDS) each window row.
//  Both tiled kernels: a CTA owns a 128 x 32 output tile; tile + halo are
//  staged once into shared memory with boundary handling resolved at staging
//  time (interior CTAs take an unchecked 128-bit path -- the paper's
//  nine-region idea, Fig. 3 / Listing 8, reduced to interior vs border CTAs);
//  each thread owns 4 horizontally adjacent outputs (and, in the sep kernel,
//  2 output rows that share every staged row they read); one MUFU.EX2 per tap.
//  The kernels are SFU-bound by construction (DESIGN.md §6 roofline).
#include <cuda_runtime.h>
#include <stdint.h>

#include "boundary.cuh"
#include "lop_params.h"

namespace lop {

// ------------------------------------------------------------------ generic
__global__ void __launch_bounds__(256) bilateral_generic_kernel(const __grid_constant__ BilateralGeneric p)
{
    const Common &c = p.c;
    const int ox = c.roi_x0 + blockIdx.x * blockDim.x + threadIdx.x;
    const int oy = c.roi_y0 + blockIdx.y * blockDim.y + threadIdx.y;
    const int b = blockIdx.z;
    if (ox >= c.roi_x0 + c.roi_w || oy >= c.roi_y0 + c.roi_h) return;
    const int ix = ox + c.off_x, iy = oy + c.off_y;
    // centre Input(): the pixel itself (for offset accessors it is read
    // through the boundary condition like every other tap)
    const bool sc = p.scaled != 0;
    float centre = read_f32(c.in, b, ix, iy, c.mode, c.cval_f);
    if (sc) centre = __fmul_rn(centre, p.alpha);
    const int sx = 2 * c.rx + 1;
    float d = 0.0f, pacc = 0.0f;
    for (int yf = -c.ry; yf <= c.ry; ++yf) {
        int row;
        const bool row_ok = resolve_row(iy + yf, c.in, c.mode, row);
        const float *rp = row_ok ? row_ptr<float>(c.in, b, row) : nullptr;
        if (p.sep) {
            float rd = 0.f, rpp = 0.f;
            for (int xf = -c.rx; xf <= c.rx; ++xf) {
                int col;
                float v = c.cval_f;
                if (row_ok && resolve_col(ix + xf, c.in, c.mode, col)) v = __ldg(rp + col);
                const float lx = p.lx[xf + c.rx];
                const bool poly = xf + c.rx < p.npoly;
                if (sc) {
                    v = __fmul_rn(v, p.alpha);
                    if (xf == -c.rx) bilateral_row_first<false, true>(v, centre, lx, p.nk, rd, rpp);
                    else bilateral_row_tap<false, true>(v, centre, lx, p.nk, rd, rpp);
                } else if (xf == -c.rx) {
                    if (poly) bilateral_row_first<true>(v, centre, lx, p.nk, rd, rpp);
                    else bilateral_row_first<false>(v, centre, lx, p.nk, rd, rpp);
                } else {
                    if (poly) bilateral_row_tap<true>(v, centre, lx, p.nk, rd, rpp);
                    else bilateral_row_tap<false>(v, centre, lx, p.nk, rd, rpp);
                }
            }
            bilateral_row_fold(p.cy[yf + c.ry], rd, rpp, d, pacc);
        } else {
            const float *lc = p.lc + (yf + c.ry) * sx + c.rx;
            for (int xf = -c.rx; xf <= c.rx; ++xf) {
                int col;
                float v = c.cval_f;
                if (row_ok && resolve_col(ix + xf, c.in, c.mode, col)) v = __ldg(rp + col);
                if (sc) bilateral_tap<true>(__fmul_rn(v, p.alpha), centre, lc[xf], p.nk, d, pacc);
                else bilateral_tap<false>(v, centre, lc[xf], p.nk, d, pacc);
            }
        }
    }
    float *orow = reinterpret_cast<float *>(c.out.data + (int64_t)b * c.out.bstride +
                                            (int64_t)oy * c.out.stride);
    orow[ox] = sc ? bilateral_finish_scaled(d, pacc, p.inv_alpha) : bilateral_finish(d, pacc);
}

cudaError_t launch_bilateral_generic(const BilateralGeneric &p, cudaStream_t stream)
{
    dim3 block(32, 8, 1);
    dim3 grid((p.c.roi_w + 31) / 32, (p.c.roi_h + 7) / 8, p.c.batch);
    bilateral_generic_kernel<<<grid, block, 0, stream>>>(p);
    return cudaGetLastError();
}

// -------------------------------------------------------------------- tiled
namespace tiled {
constexpr int TW = 128;       // outputs per tile row (32 lanes x 4)
constexpr int TH = 32;        // output rows per tile
constexpr int NT = 256;       // threads per CTA (8 warps)

template <int RX> struct Shape {
    static constexpr int PAD = (RX + 3) & ~3;                 // left halo, 16-B aligned
    static constexpr int SW = TW + 2 * PAD;                   // smem row pitch (floats)
    static constexpr int NV = (PAD + 3 + RX) / 4 + 1;         // float4 per thread per row
    static constexpr int MV = (2 * RX + 1 + 3) / 4;           // float4 per mask row
    static constexpr int VOFF = PAD - RX;                     // first used value
};
}  // namespace tiled

// Stage the input footprint of one output tile into shared memory:
// (nrows + 2ry) rows x SW columns starting at input (ix0, iy0).  Boundary
// handling is resolved here, once per staged pixel (§8(a) a2/a3).  Only the
// rows the tile's outputs need are staged (a partial last tile must not touch
// rows beyond the validated band + halo).
// SCALE: store alpha * I (the range-scaled values of the scaled-difference
// form, boundary.cuh bilateral_weight_scaled) instead of I.
template <int SW, bool SCALE = false>
__device__ __forceinline__ void stage_tile(const Common &c, int b, int ix0, int iy0, int srows,
                                           float *tile, float alpha = 1.0f)
{
    constexpr int NT = tiled::NT;
    const Geom &g = c.in;
    const int gy_lo = iy0 + g.gy0;
    const bool interior = ix0 >= 0 && ix0 + SW <= g.W && gy_lo >= 0 && gy_lo + srows <= g.GH;
    const char *fbase = g.data + (int64_t)b * g.bstride;
    if (interior && ((ix0 & 3) == 0) && ((g.stride & 15) == 0) &&
        ((reinterpret_cast<uintptr_t>(fbase) & 15) == 0)) {
        constexpr int V = SW / 4;                               // float4 per smem row
        float4 *t4 = reinterpret_cast<float4 *>(tile);
        for (int i = threadIdx.x; i < srows * V; i += NT) {
            const int r = i / V, v = i - r * V;
            const float4 *src = reinterpret_cast<const float4 *>(
                fbase + (int64_t)(iy0 + r) * g.stride) + (ix0 >> 2) + v;
            float4 q = __ldg(src);
            if (SCALE) {
                q.x = __fmul_rn(q.x, alpha); q.y = __fmul_rn(q.y, alpha);
                q.z = __fmul_rn(q.z, alpha); q.w = __fmul_rn(q.w, alpha);
            }
            t4[r * V + v] = q;
        }
    } else if (interior) {
        for (int i = threadIdx.x; i < srows * SW; i += NT) {
            const int r = i / SW, x = i - r * SW;
            const float q = __ldg(reinterpret_cast<const float *>(fbase + (int64_t)(iy0 + r) * g.stride) +
                                  ix0 + x);
            tile[i] = SCALE ? __fmul_rn(q, alpha) : q;
        }
    } else {
        for (int i = threadIdx.x; i < srows * SW; i += NT) {
            const int r = i / SW, x = i - r * SW;
            const float q = read_f32(g, b, ix0 + x, iy0 + r, c.mode, c.cval_f);
            tile[i] = SCALE ? __fmul_rn(q, alpha) : q;
        }
    }
}

__device__ __forceinline__ void store4(const Common &c, int b, int oy, int x_out, const float res[4])
{
    const int roi_x1 = c.roi_x0 + c.roi_w;
    char *fb = c.out.data + (int64_t)b * c.out.bstride;
    float *orow = reinterpret_cast<float *>(fb + (int64_t)oy * c.out.stride);
    if (x_out + 3 < roi_x1 && ((x_out & 3) == 0) && ((c.out.stride & 15) == 0) &&
        ((reinterpret_cast<uintptr_t>(fb) & 15) == 0)) {
        *reinterpret_cast<float4 *>(orow + x_out) = make_float4(res[0], res[1], res[2], res[3]);
    } else {
#pragma unroll
        for (int j = 0; j < 4; ++j)
            if (x_out + j < roi_x1) orow[x_out + j] = res[j];
    }
}

template <int NV>
__device__ __forceinline__ void load_row(const float4 *rowv, float *v)
{
#pragma unroll
    for (int k = 0; k < NV; ++k) {
        const float4 q = rowv[k];
        v[4 * k + 0] = q.x; v[4 * k + 1] = q.y; v[4 * k + 2] = q.z; v[4 * k + 3] = q.w;
    }
}

// ------------------------------------------------- user-mask tiled kernel
// One window row of taps for the 4 outputs of a thread with the mask row m
// (log2 coefficients) from shared memory.
template <int RX, int VOFF, bool SC>
__device__ __forceinline__ void mask_row(const float *v, const float cen[4], const float *m,
                                         float nk, float d[4], float pp[4])
{
#pragma unroll
    for (int xf = 0; xf <= 2 * RX; ++xf)
#pragma unroll
        for (int j = 0; j < 4; ++j) bilateral_tap<SC>(v[VOFF + xf + j], cen[j], m[xf], nk, d[j], pp[j]);
}

template <int RX, bool SC>
__global__ void __launch_bounds__(tiled::NT, 3) bilateral_tiled_kernel(const __grid_constant__ BilateralTiled p)
{
    using S = tiled::Shape<RX>;
    constexpr int TW = tiled::TW, TH = tiled::TH, NT = tiled::NT;
    constexpr int SW = S::SW, PAD = S::PAD, NV = S::NV, MV = S::MV;
    const Common &c = p.c;
    const int ry = c.ry;
    const int SH = TH + 2 * ry;

    extern __shared__ float4 smem4[];
    float *tile = reinterpret_cast<float *>(smem4);          // SH x SW
    float *msk = tile + SH * SW;                               // (2ry+1) x (4*MV)

    const int b = blockIdx.z;
    const int tx0 = c.roi_x0 + blockIdx.x * TW;                // output tile origin
    const int ty0 = c.roi_y0 + blockIdx.y * TH;
    const int roi_y1 = c.roi_y0 + c.roi_h;

    for (int i = threadIdx.x; i < (2 * ry + 1) * 4 * MV; i += NT) {
        const int r = i / (4 * MV), k = i - r * (4 * MV);
        msk[i] = k < 2 * RX + 1 ? p.lc[r * kTiledMaskPitch + k] : 0.0f;
    }
    stage_tile<SW, SC>(c, b, tx0 + c.off_x - PAD, ty0 + c.off_y - ry,
                       min(TH, roi_y1 - ty0) + 2 * ry, tile, p.alpha);
    __syncthreads();

    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int x_out = tx0 + 4 * lane;
    const float nk = p.nk;
    const float4 *mrow = reinterpret_cast<const float4 *>(msk);
    // pairs of output rows (r0, r0+1) share every staged row they read
    for (int r0 = 2 * warp; r0 < TH; r0 += 2 * (NT / 32)) {
        const int oy = ty0 + r0;
        if (oy >= roi_y1) break;
        const float4 c0 = smem4[((r0 + ry) * SW + PAD) / 4 + lane];
        const float4 c1 = smem4[((r0 + 1 + ry) * SW + PAD) / 4 + lane];
        const float cen0[4] = {c0.x, c0.y, c0.z, c0.w}, cen1[4] = {c1.x, c1.y, c1.z, c1.w};
        float d0[4] = {0.f, 0.f, 0.f, 0.f}, p0[4] = {0.f, 0.f, 0.f, 0.f};
        float d1[4] = {0.f, 0.f, 0.f, 0.f}, p1[4] = {0.f, 0.f, 0.f, 0.f};
        const float4 *rowv = smem4 + (r0 * SW) / 4 + lane;
        float v[4 * NV], m[4 * MV];
        load_row<NV>(rowv, v);
        load_row<MV>(mrow, m);
        mask_row<RX, S::VOFF, SC>(v, cen0, m, nk, d0, p0);                  // yf = 0 of r0
#pragma unroll 1
        for (int r = 1; r <= 2 * ry; ++r) {
            load_row<NV>(rowv + r * (SW / 4), v);
            float m1[4 * MV];
            load_row<MV>(mrow + (r - 1) * MV, m1);
            load_row<MV>(mrow + r * MV, m);
            mask_row<RX, S::VOFF, SC>(v, cen0, m, nk, d0, p0);              // r0, yf = r
            mask_row<RX, S::VOFF, SC>(v, cen1, m1, nk, d1, p1);             // r0+1, yf = r-1
        }
        load_row<NV>(rowv + (2 * ry + 1) * (SW / 4), v);
        load_row<MV>(mrow + 2 * ry * MV, m);
        mask_row<RX, S::VOFF, SC>(v, cen1, m, nk, d1, p1);                  // yf = 2ry of r0+1
        float res[4];
#pragma unroll
        for (int j = 0; j < 4; ++j)
            res[j] = SC ? bilateral_finish_scaled(d0[j], p0[j], p.inv_alpha) : bilateral_finish(d0[j], p0[j]);
        store4(c, b, oy, x_out, res);
        if (oy + 1 < roi_y1) {
#pragma unroll
            for (int j = 0; j < 4; ++j)
                res[j] = SC ? bilateral_finish_scaled(d1[j], p1[j], p.inv_alpha) : bilateral_finish(d1[j], p1[j]);
            store4(c, b, oy + 1, x_out, res);
        }
    }
}

// -------------------------------------- separable-closeness tiled kernel
// One window row of taps for the 4 outputs of a thread (lx from the
// constant bank, compile-time indexed), folded with cy.
template <int RX, int VOFF, int NP, bool SC>
__device__ __forceinline__ void sep_row(const float *v, const float cen[4], const float *lx,
                                        float nk, float cy, float d[4], float pp[4])
{
    float rd[4], rp[4];
#pragma unroll
    for (int j = 0; j < 4; ++j)
        bilateral_row_first<(NP > 0), SC>(v[VOFF + j], cen[j], lx[0], nk, rd[j], rp[j]);
#pragma unroll
    for (int xf = 1; xf <= 2 * RX; ++xf)
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            if (xf < NP)   // resolved at compile time after unrolling
                bilateral_row_tap<true, SC>(v[VOFF + xf + j], cen[j], lx[xf], nk, rd[j], rp[j]);
            else
                bilateral_row_tap<false, SC>(v[VOFF + xf + j], cen[j], lx[xf], nk, rd[j], rp[j]);
        }
#pragma unroll
    for (int j = 0; j < 4; ++j) bilateral_row_fold(cy, rd[j], rp[j], d[j], pp[j]);
}

template <int RX, int NP, bool SC>
__global__ void __launch_bounds__(tiled::NT, 3) bilateral_sep_kernel(const __grid_constant__ BilateralSep p)
{
    using S = tiled::Shape<RX>;
    constexpr int TW = tiled::TW, TH = tiled::TH, NT = tiled::NT;
    constexpr int SW = S::SW, PAD = S::PAD, NV = S::NV;
    const Common &c = p.c;
    const int ry = c.ry;
    const int SH = TH + 2 * ry;

    extern __shared__ float4 smem4[];
    float *tile = reinterpret_cast<float *>(smem4);          // SH x SW
    float *scy = tile + SH * SW;                               // 2ry+1 floats

    const int b = blockIdx.z;
    const int tx0 = c.roi_x0 + blockIdx.x * TW;
    const int ty0 = c.roi_y0 + blockIdx.y * TH;
    const int roi_y1 = c.roi_y0 + c.roi_h;

    for (int i = threadIdx.x; i <= 2 * ry; i += NT) scy[i] = p.cy[i];
    stage_tile<SW, SC>(c, b, tx0 + c.off_x - PAD, ty0 + c.off_y - ry,
                       min(TH, roi_y1 - ty0) + 2 * ry, tile, p.alpha);
    __syncthreads();

    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int x_out = tx0 + 4 * lane;
    const float nk = p.nk;
    // each warp: pairs of output rows (r0, r0+1); every staged row read once
    // serves both outputs (window rows yf and yf-1)
    for (int r0 = 2 * warp; r0 < TH; r0 += 2 * (NT / 32)) {
        const int oy = ty0 + r0;
        if (oy >= roi_y1) break;
        const float4 c0 = smem4[((r0 + ry) * SW + PAD) / 4 + lane];
        const float4 c1 = smem4[((r0 + 1 + ry) * SW + PAD) / 4 + lane];
        const float cen0[4] = {c0.x, c0.y, c0.z, c0.w}, cen1[4] = {c1.x, c1.y, c1.z, c1.w};
        float d0[4] = {0.f, 0.f, 0.f, 0.f}, p0[4] = {0.f, 0.f, 0.f, 0.f};
        float d1[4] = {0.f, 0.f, 0.f, 0.f}, p1[4] = {0.f, 0.f, 0.f, 0.f};
        const float4 *rowv = smem4 + (r0 * SW) / 4 + lane;
        float v[4 * NV];
        // staged row 0: window row 0 of output r0 only
        load_row<NV>(rowv, v);
        sep_row<RX, S::VOFF, NP, SC>(v, cen0, p.lx, nk, scy[0], d0, p0);
#pragma unroll 1
        for (int r = 1; r <= 2 * ry; ++r) {
            load_row<NV>(rowv + r * (SW / 4), v);
            sep_row<RX, S::VOFF, NP, SC>(v, cen0, p.lx, nk, scy[r], d0, p0);       // output r0, yf = r
            sep_row<RX, S::VOFF, NP, SC>(v, cen1, p.lx, nk, scy[r - 1], d1, p1);   // output r0+1, yf = r-1
        }
        // staged row 2ry+1: last window row of output r0+1
        load_row<NV>(rowv + (2 * ry + 1) * (SW / 4), v);
        sep_row<RX, S::VOFF, NP, SC>(v, cen1, p.lx, nk, scy[2 * ry], d1, p1);
        float res[4];
#pragma unroll
        for (int j = 0; j < 4; ++j)
            res[j] = SC ? bilateral_finish_scaled(d0[j], p0[j], p.inv_alpha) : bilateral_finish(d0[j], p0[j]);
        store4(c, b, oy, x_out, res);
        if (oy + 1 < roi_y1) {
#pragma unroll
            for (int j = 0; j < 4; ++j)
                res[j] = SC ? bilateral_finish_scaled(d1[j], p1[j], p.inv_alpha) : bilateral_finish(d1[j], p1[j]);
            store4(c, b, oy + 1, x_out, res);
        }
    }
}

// ------------------------------------------------------------- launchers
template <typename P, typename K>
static cudaError_t launch_tiled(K kernel, const P &p, size_t smem, cudaStream_t stream,
                                size_t &configured)
{
    if (smem > 48 * 1024 && smem > configured) {
        cudaError_t e = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                             (int)smem);
        if (e != cudaSuccess) return e;
        configured = smem;
    }
    dim3 grid((p.c.roi_w + tiled::TW - 1) / tiled::TW, (p.c.roi_h + tiled::TH - 1) / tiled::TH,
              p.c.batch);
    kernel<<<grid, tiled::NT, smem, stream>>>(p);
    return cudaGetLastError();
}

template <int RX, bool SC>
static cudaError_t launch_tiled_rx_sc(const BilateralTiled &p, cudaStream_t stream)
{
    using S = tiled::Shape<RX>;
    static size_t configured = 0;
    const size_t smem = (size_t)((tiled::TH + 2 * p.c.ry) * S::SW + (2 * p.c.ry + 1) * 4 * S::MV) *
                        sizeof(float);
    return launch_tiled(bilateral_tiled_kernel<RX, SC>, p, smem, stream, configured);
}

template <int RX>
static cudaError_t launch_tiled_rx(const BilateralTiled &p, cudaStream_t stream)
{
    return p.scaled ? launch_tiled_rx_sc<RX, true>(p, stream) : launch_tiled_rx_sc<RX, false>(p, stream);
}

template <int RX, int NP, bool SC>
static cudaError_t launch_sep_rx_np(const BilateralSep &p, cudaStream_t stream)
{
    using S = tiled::Shape<RX>;
    static size_t configured = 0;
    const size_t smem = (size_t)((tiled::TH + 2 * p.c.ry) * S::SW + ((2 * p.c.ry + 1 + 3) & ~3)) *
                        sizeof(float);
    return launch_tiled(bilateral_sep_kernel<RX, NP, SC>, p, smem, stream, configured);
}

// instances: npoly 0 (scaled or not) for every width; npoly 1 (unscaled) for
// windows >= 9 wide (kept for the tuning sweep).
template <int RX>
static cudaError_t launch_sep_rx(const BilateralSep &p, cudaStream_t stream)
{
    if (p.npoly == 0)
        return p.scaled ? launch_sep_rx_np<RX, 0, true>(p, stream)
                        : launch_sep_rx_np<RX, 0, false>(p, stream);
    if constexpr (RX >= 4) {
        if (p.npoly == 1 && !p.scaled) return launch_sep_rx_np<RX, 1, false>(p, stream);
    }
    return cudaErrorInvalidValue;
}

int bilateral_sep_max_npoly(int rx) { return rx >= 4 ? 1 : 0; }

cudaError_t launch_bilateral_tiled(const BilateralTiled &p, cudaStream_t stream)
{
    switch (p.c.rx) {
    case 0: return launch_tiled_rx<0>(p, stream);
    case 1: return launch_tiled_rx<1>(p, stream);
    case 2: return launch_tiled_rx<2>(p, stream);
    case 3: return launch_tiled_rx<3>(p, stream);
    case 4: return launch_tiled_rx<4>(p, stream);
    case 5: return launch_tiled_rx<5>(p, stream);
    case 6: return launch_tiled_rx<6>(p, stream);
    case 7: return launch_tiled_rx<7>(p, stream);
    default: return cudaErrorInvalidValue;
    }
}

cudaError_t launch_bilateral_sep(const BilateralSep &p, cudaStream_t stream)
{
    switch (p.c.rx) {
    case 0: return launch_sep_rx<0>(p, stream);
    case 1: return launch_sep_rx<1>(p, stream);
    case 2: return launch_sep_rx<2>(p, stream);
    case 3: return launch_sep_rx<3>(p, stream);
    case 4: return launch_sep_rx<4>(p, stream);
    case 5: return launch_sep_rx<5>(p, stream);
    case 6: return launch_sep_rx<6>(p, stream);
    case 7: return launch_sep_rx<7>(p, stream);
    default: return cudaErrorInvalidValue;
    }
}

}  // namespace lop

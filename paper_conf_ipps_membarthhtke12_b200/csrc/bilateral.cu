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

#include <algorithm>
#include <cstdlib>

#include "boundary.cuh"
#include "launch_cache.h"
#include "lop_params.h"

namespace lop {

// ------------------------------------------------------------------ generic
// pair kernel lane groups (see bilateral_pair_kernel): floor(t / 4), and
// the dx of the first partner value of receiving column jr (owner push)
__host__ __device__ constexpr int pair_floor4(int t) { return t >= 0 ? t / 4 : -((-t + 3) / 4); }
__host__ __device__ constexpr int pair_first_dx(int jr, int dx0, int R)
{
    return pair_floor4(jr - dx0) == 0 ? dx0
                                      : (jr - 4 * pair_floor4(jr - dx0) < R ? jr - 4 * pair_floor4(jr - dx0) : R);
}

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
    if (p.pair) {
        // Pair-sharing order of bilateral_pair_kernel (below): the same 169
        // weights, each computed by the pair's owner p with q = p + (dx, dy),
        // dy > 0 or (dy = 0, dx > 0), as ex2(lx[dx] - (J(q) - J(p))^2), and the
        // same per-row partial sums folded in the same order:
        //   rows above (partner side, dy = R..1), own row (own, then partner),
        //   rows below (own side, dy = 1..R).
        const int R = c.rx;
        auto J = [&](int x, int y) { return __fmul_rn(read_f32(c.in, b, x, y, c.mode, c.cval_f), p.alpha); };
        // partner terms of a row in dx order; a run of dx whose owners sit in
        // another lane of the pair kernel (column group floor(x / 4)) is
        // pre-summed by that lane and added as one value (owner push)
        const int jr = ox & 3;
        auto partner_row = [&](int dy, int dx0) {
            float qd = 0.f, qp = 0.f;
            for (int dx = dx0; dx <= R;) {
                const int o = pair_floor4(jr - dx);
                const int dx_end = o == 0 ? dx : min(jr - 4 * o, R);
                float sd = 0.f, sp = 0.f;
                for (int k = dx; k <= dx_end; ++k) {
                    const float jp = J(ix - k, iy - dy);
                    const float w = bilateral_weight<false, true>(centre, jp, p.lx[k + R], p.nk);
                    if (k == dx) { sd = w; sp = __fmul_rn(w, jp); }
                    else { sd = __fadd_rn(sd, w); sp = __fmaf_rn(w, jp, sp); }
                }
                if (dx == dx0) { qd = sd; qp = sp; }
                else if (o == 0) {
                    // in-lane term: accumulated like an own term
                    const float jp = J(ix - dx, iy - dy);
                    const float w = bilateral_weight<false, true>(centre, jp, p.lx[dx + R], p.nk);
                    qd = __fadd_rn(qd, w); qp = __fmaf_rn(w, jp, qp);
                } else { qd = __fadd_rn(qd, sd); qp = __fadd_rn(qp, sp); }
                dx = dx_end + 1;
            }
            bilateral_row_fold(p.cy[dy + R], qd, qp, d, pacc);
        };
        auto own_row = [&](int dy, int dx0) {
            float rd = 0.f, rp = 0.f;
            for (int dx = dx0; dx <= R; ++dx) {
                const float jq = J(ix + dx, iy + dy);
                const float w = bilateral_weight<false, true>(jq, centre, p.lx[dx + R], p.nk);
                if (dx == dx0) { rd = w; rp = __fmul_rn(w, jq); }
                else { rd = __fadd_rn(rd, w); rp = __fmaf_rn(w, jq, rp); }
            }
            bilateral_row_fold(p.cy[dy + R], rd, rp, d, pacc);
        };
        for (int dy = R; dy >= 1; --dy) partner_row(dy, -R);
        own_row(0, 0);
        partner_row(0, 1);
        for (int dy = 1; dy <= R; ++dy) own_row(dy, -R);
        float *orow = reinterpret_cast<float *>(c.out.data + (int64_t)b * c.out.bstride +
                                                (int64_t)oy * c.out.stride);
        orow[ox] = bilateral_finish_scaled(d, pacc, p.inv_alpha);
        return;
    }
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

// Store the outputs of lane columns x_out .. x_out + 3 that lie in [xs0, xs1).
__device__ __forceinline__ void pair_store_span(const Common &c, int b, int s, int x_out, int xs0, int xs1,
                                                const float res[4])
{
    if (xs0 == x_out && xs1 == x_out + 4) {
        store4(c, b, s, x_out, res);
        return;
    }
    float *orow = reinterpret_cast<float *>(c.out.data + (int64_t)b * c.out.bstride + (int64_t)s * c.out.stride);
#pragma unroll
    for (int j = 0; j < 4; ++j)
        if (x_out + j >= xs0 && x_out + j < xs1) orow[x_out + j] = res[j];
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
        if (x_out >= c.roi_x0 + c.roi_w) continue;   // no division for columns past the ROI
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
        if (x_out >= c.roi_x0 + c.roi_w) continue;   // no division for columns past the ROI
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

// --------------------------------------- pair-sharing separable kernel
// The range weight is symmetric: w(p, q) = c(q - p) s(J(q) - J(p)) = w(q, p)
// (c is even in both axes, (J(q) - J(p))^2 = (J(p) - J(q))^2 exactly), so the
// 168 exps of a 13x13 window are 84 distinct ones per pixel (SURVEY.md §8(d)
// "symmetric pair-sharing").  Each pair {p, q} is evaluated once by its owner
// p, with q = p + (dx, dy) in the half window dy > 0 or (dy = 0, dx > 0), and
// contributes (w, w J(q)) to p and (w, w J(p)) to q.
//  * A warp owns a 128-column frame (lane L: columns 4L..4L+3) and streams
//    down T output rows.  Partner contributions to columns of other lanes
//    travel by SHFL; the frame's HLN outer lanes each side are halo (they own
//    pairs, but their own outputs would miss partners outside the frame), so
//    a warp writes OW = 128 - 8 HLN columns.
//  * Partner contributions to rows below (dy > 0) go to a register ring of
//    per-row accumulators D/P[0..R]; row s is complete after step s.  The
//    warp starts R rows early (warm-up steps evaluate only the pairs that
//    reach row >= y0).
//  * Input rows stream through a per-warp ring of R+2 rows in shared memory
//    (alpha * I, boundary resolved at staging); no block-level barriers.
// Summation order per output (mirrored by bilateral_generic_kernel, p.pair):
// partner rows dy = R..1, own row (own, partner), own rows dy = 1..R, each a
// left-to-right partial sum folded with cy[dy].
#ifndef LOP_PAIR_NW
#define LOP_PAIR_NW 2
#endif
#ifndef LOP_PAIR_MAXREG
#define LOP_PAIR_MAXREG 160   // 160 / 164 / 168: same 12 warps/SM; 160 schedules best (profiles/r02)
#endif
#ifndef LOP_PAIR_DY_UNROLL
#define LOP_PAIR_DY_UNROLL 1
#endif
namespace pair {
constexpr int NW = LOP_PAIR_NW;                        // warps per CTA
constexpr int kDyUnroll = LOP_PAIR_DY_UNROLL;          // packed row-pair loop unroll (1: rolled)
template <int R> struct Shape {
    static constexpr int HLN = (R + 3) / 4;            // halo lanes each side
    static constexpr int HL = 4 * HLN;                 // halo columns each side
    static constexpr int OW = 128 - 2 * HL;            // output columns per warp
    // the TMEM kernel's TIGHT geometry: frame columns [R, R + OWT) are complete
    // (every partner of them is owned inside the frame); OWT a multiple of 4 so
    // frame starts stay at x = 0 mod 4; lanes straddling the output edge store
    // their inner columns (13x13: 116 of 128 columns instead of 112)
    static constexpr int OWT = (128 - 2 * R) & ~3;
    static constexpr int PAD = HL;                     // smem columns left of frame column 0
    static constexpr int SW = 128 + 2 * PAD;           // smem row (floats)
    static constexpr int NV = PAD / 2 + 1;             // float4 per lane per row: 4L-PAD .. 4L+3+PAD
    static constexpr int NR = R + 2;                   // ring slots
    // per-warp shared memory (floats): interleaved row-pair ring (slot k holds
    // rows (r, r+1) as (J(r,x), J(r+1,x)) pairs), plain row ring, staging row,
    // column map (ints)
    static constexpr int RING2 = NR * SW * 2, RING1 = NR * SW;
    static constexpr int WARP_FLOATS = RING2 + RING1 + SW + SW;   // + staging row, column map
};
}  // namespace pair

// Value x of lane (this lane + o); o is a compile-time constant after unrolling.
__device__ __forceinline__ float lane_shift(float x, int o)
{
    if (o == 0) return x;
    if (o > 0) return __shfl_down_sync(0xffffffffu, x, o);
    return __shfl_up_sync(0xffffffffu, x, -o);
}

// Partner-side exchange (owner push).  Owner column j of this lane pairs with
// q at column c = j + dx (relative to the lane's first column).  A partner in
// this lane (0 <= c <= 3) takes (w, w J(p)) directly; one in another lane is
// served by an outgoing sum per destination column, accumulated by the owner
// over the dx that reach c (owners j = c - dx, dx ascending) and sent with one
// SHFL per value when complete (at dx = min(c, R)) -- 2 SHFL per destination
// column and row instead of one per pair.  The receiver (column jr = c - 4o of
// lane L + o, o = floor(c / 4)) adds the sums in dx order of its partner terms,
// each off-lane run of dx as one pre-summed value.
// pair_first_dx: dx at which receiver column jr gets its first partner value,
// for partner dx running dx0 .. R.
// One window row dy of the half window for this lane's 4 owners (scalar; DY0:
// dy = 0, own side dx = 0..R with the centre, partner side dx = 1..R): own
// sums (rd, rp) and partner sums (qd, qp) of the receiving columns.
// wc: the centre tap's weight ex2(lx[R]) (difference exactly 0), computed once
// per thread instead of per pixel -- the same bits as evaluating it here.
template <int R, int PAD, bool DY0>
__device__ __forceinline__ void pair_row1(const float *v, const float cen[4], const float *lx, float nk,
                                          float wc, float rd[4], float rp[4], float qd[4], float qp[4])
{
    constexpr int dx0 = DY0 ? 0 : -R;             // own side: first dx of this row
    constexpr int px0 = DY0 ? 1 : -R;             // partner side: first dx of this row
    float od[2 * R + 4], op[2 * R + 4];           // outgoing sums, index c + R
#pragma unroll
    for (int dx = dx0; dx <= R; ++dx) {
        float w[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            const float jq = v[PAD + j + dx];
            w[j] = DY0 && dx == 0 ? wc : bilateral_weight<false, true>(jq, cen[j], lx[dx + R], nk);
            if (dx == dx0) { rd[j] = w[j]; rp[j] = __fmul_rn(w[j], jq); }
            else { rd[j] = __fadd_rn(rd[j], w[j]); rp[j] = __fmaf_rn(w[j], jq, rp[j]); }
        }
        if (DY0 && dx == 0) continue;             // centre tap: no partner
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            const int c = j + dx;
            if (c >= 0 && c <= 3) {
                if (dx == pair_first_dx(c, px0, R)) { qd[c] = w[j]; qp[c] = __fmul_rn(w[j], cen[j]); }
                else { qd[c] = __fadd_rn(qd[c], w[j]); qp[c] = __fmaf_rn(w[j], cen[j], qp[c]); }
            } else {
                const int first = c - 3 > px0 ? c - 3 : px0;
                if (dx == first) { od[c + R] = w[j]; op[c + R] = __fmul_rn(w[j], cen[j]); }
                else { od[c + R] = __fadd_rn(od[c + R], w[j]); op[c + R] = __fmaf_rn(w[j], cen[j], op[c + R]); }
            }
        }
        // destinations complete at this dx: c = dx (c < 0), or c >= 4 with min(c, R) == dx
#pragma unroll
        for (int c = -R; c <= R + 3; ++c) {
            if (c >= 0 && c <= 3) continue;
            if ((c < R ? c : R) != dx) continue;
            const int o = pair_floor4(c), jr = c - 4 * o;
            const float a = lane_shift(od[c + R], -o), bq = lane_shift(op[c + R], -o);
            if (dx == pair_first_dx(jr, px0, R)) { qd[jr] = a; qp[jr] = bq; }
            else { qd[jr] = __fadd_rn(qd[jr], a); qp[jr] = __fadd_rn(qp[jr], bq); }
        }
    }
}

__device__ __forceinline__ void fold4(float cy, const float rd[4], const float rp[4], float d[4], float pp[4])
{
#pragma unroll
    for (int j = 0; j < 4; ++j) {
        d[j] = __fmaf_rn(cy, rd[j], d[j]);
        pp[j] = __fmaf_rn(cy, rp[j], pp[j]);
    }
}

// Packed form of pair_row1 for two window rows (a, b) = (s+dy, s+dy+1) at
// once: v[i] = (J(a, col i), J(b, col i)) from the interleaved ring; each
// FADD2 / FFMA2 lane does exactly the scalar arithmetic of its row (same
// rounding), so packing changes no result bit.  cen / J(p) enter as scalar
// broadcast operands, (lx, lx) as a broadcast pair.
template <int R, int PAD>
__device__ __forceinline__ void pair_row2(const float2 *v, const float cen[4], const float *lx,
                                          float2 rd[4], float2 rp[4], float2 qd[4], float2 qp[4])
{
    float2 od[2 * R + 4], op[2 * R + 4];
#pragma unroll
    for (int dx = -R; dx <= R; ++dx) {
        float2 w[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            const float2 jq = v[PAD + j + dx];
            const float2 diff = __fadd2_rn(jq, make_float2(-cen[j], -cen[j]));
            const float2 e = __ffma2_rn(make_float2(-diff.x, -diff.y), diff, make_float2(lx[dx + R], lx[dx + R]));
            w[j] = make_float2(ex2_approx(e.x), ex2_approx(e.y));
            if (dx == -R) { rd[j] = w[j]; rp[j] = __fmul2_rn(w[j], jq); }
            else { rd[j] = __fadd2_rn(rd[j], w[j]); rp[j] = __ffma2_rn(w[j], jq, rp[j]); }
        }
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            const int c = j + dx;
            const float2 cj = make_float2(cen[j], cen[j]);
            if (c >= 0 && c <= 3) {
                if (dx == pair_first_dx(c, -R, R)) { qd[c] = w[j]; qp[c] = __fmul2_rn(w[j], cj); }
                else { qd[c] = __fadd2_rn(qd[c], w[j]); qp[c] = __ffma2_rn(w[j], cj, qp[c]); }
            } else {
                const int first = c - 3 > -R ? c - 3 : -R;
                if (dx == first) { od[c + R] = w[j]; op[c + R] = __fmul2_rn(w[j], cj); }
                else { od[c + R] = __fadd2_rn(od[c + R], w[j]); op[c + R] = __ffma2_rn(w[j], cj, op[c + R]); }
            }
        }
#pragma unroll
        for (int c = -R; c <= R + 3; ++c) {
            if (c >= 0 && c <= 3) continue;
            if ((c < R ? c : R) != dx) continue;
            const int o = pair_floor4(c), jr = c - 4 * o;
            const float2 a = make_float2(lane_shift(od[c + R].x, -o), lane_shift(od[c + R].y, -o));
            const float2 bq = make_float2(lane_shift(op[c + R].x, -o), lane_shift(op[c + R].y, -o));
            if (dx == pair_first_dx(jr, -R, R)) { qd[jr] = a; qp[jr] = bq; }
            else { qd[jr] = __fadd2_rn(qd[jr], a); qp[jr] = __fadd2_rn(qp[jr], bq); }
        }
    }
}

__device__ __forceinline__ void cp_async16(void *smem_dst, const void *gsrc)
{
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_addr(smem_dst)), "l"(gsrc)
                 : "memory");
}

__device__ __forceinline__ void cp_async4(void *smem_dst, const void *gsrc)
{
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(smem_addr(smem_dst)), "l"(gsrc)
                 : "memory");
}

// Column map of a warp's frame, resolved once per kernel (columns do not
// change from row to row): cm[i] = input column read for smem column i, or -1
// where CONSTANT substitutes the constant (Table I).  Columns no
// stored output reads (beyond the iteration space's footprint, e.g. the part
// of the last strip past the image edge) are -1 too: they are not fetched
// (their value only reaches outputs that are not stored).
template <int SW>
__device__ __forceinline__ void pair_colmap(const Common &c, int ix0, int *cm, int lane)
{
    const int lo = c.roi_x0 + c.off_x - c.rx, hi = c.roi_x0 + c.roi_w - 1 + c.off_x + c.rx;
#pragma unroll
    for (int i = lane; i < SW; i += 32) {
        int col;
        const int ix = ix0 + i;
        cm[i] = ix >= lo && ix <= hi && resolve_col(ix, c.in, c.mode, col) ? col : -1;
    }
}

// Row fetch, part 1: raw I of input row iy (smem columns 0 .. SW-1) goes
// global -> dst asynchronously: 16-B chunks wholly inside the image as one
// LDGSTS.128, border chunks element-wise through the column map (LDGSTS.32).
// Nothing is fetched for a CONSTANT row.  Border warps thus never wait on a
// synchronous load, and the per-element boundary arithmetic (the modulo of
// REPEAT / MIRROR) is paid once per kernel, not per row (mode invariance, E5).
template <int SW>
__device__ __forceinline__ void pair_issue_row(const Common &c, int b, int iy, int ix0, float4 *dst,
                                               const int *cm, int lane, bool vec_ok)
{
    const Geom &g = c.in;
    int row;
    if (resolve_row(iy, g, c.mode, row)) {
        const float *rp = row_ptr<float>(g, b, row);
#pragma unroll
        for (int k = lane; k < SW / 4; k += 32) {
            const int ix = ix0 + 4 * k;
            if (vec_ok && ix >= 0 && ix + 3 < g.W) {
                cp_async16(dst + k, rp + ix);
            } else {
                float *d = reinterpret_cast<float *>(dst + k);
#pragma unroll
                for (int jj = 0; jj < 4; ++jj)
                    if (cm[4 * k + jj] >= 0) cp_async4(d + jj, rp + cm[4 * k + jj]);
            }
        }
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
}

// Part 2 (after cp.async.wait_all): chunk values alpha * I (fetched chunks
// from src, CONSTANT elements substituted) written to the plain ring slot of
// the row (may alias src: each lane reads its chunk before writing it), the
// first half of its interleaved slot and the second half of the previous
// row's interleaved slot.
template <int SW, bool PLAIN = true>
__device__ __forceinline__ void pair_put_row(const Common &c, int iy, int ix0, float alpha,
                                             const float4 *src, float4 *plain, float2 *first,
                                             float2 *second, const int *cm, int lane, bool vec_ok)
{
    const Geom &g = c.in;
    int row;
    const bool row_ok = resolve_row(iy, g, c.mode, row);
#pragma unroll
    for (int k = lane; k < SW / 4; k += 32) {
        const int ix = ix0 + 4 * k;
        float4 q;
        if (row_ok && vec_ok && ix >= 0 && ix + 3 < g.W) {
            q = src[k];
        } else {
            const float4 r = src[k];
            q.x = (row_ok && cm[4 * k + 0] >= 0) ? r.x : c.cval_f;
            q.y = (row_ok && cm[4 * k + 1] >= 0) ? r.y : c.cval_f;
            q.z = (row_ok && cm[4 * k + 2] >= 0) ? r.z : c.cval_f;
            q.w = (row_ok && cm[4 * k + 3] >= 0) ? r.w : c.cval_f;
        }
        q.x = __fmul_rn(q.x, alpha); q.y = __fmul_rn(q.y, alpha);
        q.z = __fmul_rn(q.z, alpha); q.w = __fmul_rn(q.w, alpha);
        if (PLAIN) plain[k] = q;
        // interleaved slot, swizzled: float4 i of a slot lives at i ^ ((i >> 3) & 1),
        // so the LDS.128 of 8 lanes reading float4 2L + k (2 x 16 B apart) hit 8
        // distinct 16-B bank groups (no 2-way conflict); columns 4k..4k+3 are
        // float4 2k, 2k+1, swapped when bit 3 of 2k (= bit 2 of k) is set
        const int a = ((k >> 2) & 1) ? 4 : 0, a2 = 4 - a;
        float *f = reinterpret_cast<float *>(first + 4 * k);
        f[a + 0] = q.x; f[a + 2] = q.y; f[a2 + 0] = q.z; f[a2 + 2] = q.w;
        if (second) {
            float *sc = reinterpret_cast<float *>(second + 4 * k) + 1;
            sc[a + 0] = q.x; sc[a + 2] = q.y; sc[a2 + 0] = q.z; sc[a2 + 2] = q.w;
        }
    }
}

template <int R>
__global__ void __maxnreg__(LOP_PAIR_MAXREG) bilateral_pair_kernel(const __grid_constant__ BilateralSep p)
{
    using S = pair::Shape<R>;
    constexpr int SW = S::SW, SW4 = S::SW / 4, NV = S::NV, NR = S::NR, PAD = S::PAD, HLN = S::HLN;
    const Common &c = p.c;
    const Geom &g = c.in;
    extern __shared__ float4 smem4[];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    float *wbase = reinterpret_cast<float *>(smem4) + warp * S::WARP_FLOATS;
    float2 *ring2 = reinterpret_cast<float2 *>(wbase);                    // NR x SW pairs
    float4 *ring1 = reinterpret_cast<float4 *>(wbase + S::RING2);          // NR x SW
    float4 *stg = reinterpret_cast<float4 *>(wbase + S::RING2 + S::RING1); // SW
    int *cm = reinterpret_cast<int *>(wbase + S::RING2 + S::RING1 + SW);   // SW
    const int b = blockIdx.z;
    // lane column groups are anchored to x = 0 mod 4 of the output (not to
    // the ROI), so that every pixel's summation order -- and result -- is
    // independent of the iteration space (owner push groups by lane)
    const int ox0 = (c.roi_x0 & ~3) + blockIdx.x * S::OW;        // first output column of the warp
    const int T = p.pair_rows;
    const float wc = ex2_approx(p.lx[R]);                        // centre weight (see pair_row1)
    const int y0 = c.roi_y0 + (blockIdx.y * pair::NW + warp) * T;
    const int roi_y1 = c.roi_y0 + c.roi_h;
    if (y0 >= roi_y1) return;                                    // warp-uniform; warps are independent
    const int yend = min(y0 + T, roi_y1);
    const int ix0 = ox0 - S::HL + c.off_x - PAD;                 // input column of smem column 0
    const bool vec_ok = ((ix0 & 3) == 0) && ((g.stride & 15) == 0) &&
                        ((reinterpret_cast<uintptr_t>(g.data + (int64_t)b * g.bstride) & 15) == 0);
    pair_colmap<SW>(c, ix0, cm, lane);
    __syncwarp();
    for (int r = 0; r <= R; ++r)                                 // rows y0-R .. y0 -> slots 0..R
        pair_issue_row<SW>(c, b, y0 - R + r + c.off_y, ix0, ring1 + r * SW4, cm, lane, vec_ok);
    asm volatile("cp.async.wait_all;" ::: "memory");
    for (int r = 0; r <= R; ++r)
        pair_put_row<SW>(c, y0 - R + r + c.off_y, ix0, p.alpha, ring1 + r * SW4, ring1 + r * SW4,
                         ring2 + r * SW, r > 0 ? ring2 + (r - 1) * SW : nullptr, cm, lane, vec_ok);
    __syncwarp();

    float D[R + 1][4], P[R + 1][4];                              // D/P[k]: row s + k
#pragma unroll
    for (int k = 0; k <= R; ++k)
#pragma unroll
        for (int j = 0; j < 4; ++j) D[k][j] = P[k][j] = 0.0f;
    const int x_out = ox0 + 4 * (lane - HLN);
    const bool store_lane = lane >= HLN && lane < 32 - HLN && x_out < c.roi_x0 + c.roi_w &&
                            x_out + 3 >= c.roi_x0;
    int slot0 = 0;                                               // ring slot of row s
#pragma unroll 1
    for (int s = y0 - R; s < yend; ++s) {
        // prefetch row s + R + 1 (its slot = that of row s - 1, not read by step s)
        const bool pre = s + 1 < yend;
        if (pre) pair_issue_row<SW>(c, b, s + R + 1 + c.off_y, ix0, stg, cm, lane, vec_ok);

        const int kmin = y0 - s;                                 // warm-up: rows < y0 are not outputs
        float u[4 * NV];
        load_row<NV>(ring1 + slot0 * SW4 + lane, u);
        const float cen[4] = {u[PAD], u[PAD + 1], u[PAD + 2], u[PAD + 3]};
        if (kmin <= 0) {                                         // dy = 0: own row (scalar)
            float rd[4], rp[4], qd[4], qp[4];
            pair_row1<R, PAD, true>(u, cen, p.lx, p.nk, wc, rd, rp, qd, qp);
            const float cy = p.cy[R];
            fold4(cy, rd, rp, D[0], P[0]);
            fold4(cy, qd, qp, D[0], P[0]);
        }
#pragma unroll pair::kDyUnroll
        for (int dy = 1; dy + 1 <= R; dy += 2) {                 // row pairs (dy, dy+1): packed
            if (dy + 1 < kmin) continue;
            const int sl = slot0 + dy >= NR ? slot0 + dy - NR : slot0 + dy;
            float2 v[4 * NV];
            {
                const float4 *src = reinterpret_cast<const float4 *>(ring2 + sl * SW);
#pragma unroll
                for (int k = 0; k < 2 * NV; ++k) {
                    const int i = 2 * lane + k;                          // swizzled (pair_put_row)
                    const float4 q = src[i ^ ((i >> 3) & 1)];
                    v[2 * k] = make_float2(q.x, q.y);
                    v[2 * k + 1] = make_float2(q.z, q.w);
                }
            }
            float2 rd[4], rp[4], qd[4], qp[4];
            pair_row2<R, PAD>(v, cen, p.lx, rd, rp, qd, qp);
            const float cya = p.cy[dy + R], cyb = p.cy[dy + 1 + R];
            float ta[4], tb[4], sa[4], sb[4];
#pragma unroll
            for (int j = 0; j < 4; ++j) { ta[j] = rd[j].x; sa[j] = rp[j].x; tb[j] = rd[j].y; sb[j] = rp[j].y; }
            fold4(cya, ta, sa, D[0], P[0]);
            fold4(cyb, tb, sb, D[0], P[0]);
#pragma unroll
            for (int j = 0; j < 4; ++j) { ta[j] = qd[j].x; sa[j] = qp[j].x; tb[j] = qd[j].y; sb[j] = qp[j].y; }
            switch (dy) {                                        // partner rows: register ring
#define LOP_PAIR_FOLD(K) case K: if constexpr (K + 1 <= R) { fold4(cya, ta, sa, D[K], P[K]); fold4(cyb, tb, sb, D[K + 1], P[K + 1]); } break;
            LOP_PAIR_FOLD(1) LOP_PAIR_FOLD(3) LOP_PAIR_FOLD(5)
#undef LOP_PAIR_FOLD
            default: break;
            }
        }
        if constexpr (R % 2 == 1) {                              // odd R: last row dy = R (scalar)
            const int sl = slot0 + R >= NR ? slot0 + R - NR : slot0 + R;
            float v[4 * NV];
            load_row<NV>(ring1 + sl * SW4 + lane, v);
            float rd[4], rp[4], qd[4], qp[4];
            pair_row1<R, PAD, false>(v, cen, p.lx, p.nk, wc, rd, rp, qd, qp);
            const float cy = p.cy[2 * R];
            fold4(cy, rd, rp, D[0], P[0]);
            fold4(cy, qd, qp, D[R], P[R]);
        }
        // lanes of the frame outside the iteration space skip the division as well:
        // an out-of-image pixel under CONSTANT 0 has P = 0 there, which sends
        // __fdiv_rn to its slow path (the right edge strip then set the kernel's
        // tail: CONSTANT 0 was 4.4 % slower than the other modes)
        if (s >= y0 && store_lane) {
            float res[4];
#pragma unroll
            for (int j = 0; j < 4; ++j) res[j] = bilateral_finish_scaled(D[0][j], P[0][j], p.inv_alpha);
            {
                if (x_out >= c.roi_x0) {
                    store4(c, b, s, x_out, res);
                } else {                                         // group straddling the ROI start
                    float *orow = reinterpret_cast<float *>(c.out.data + (int64_t)b * c.out.bstride +
                                                            (int64_t)s * c.out.stride);
#pragma unroll
                    for (int j = 0; j < 4; ++j)
                        if (x_out + j >= c.roi_x0 && x_out + j < c.roi_x0 + c.roi_w) orow[x_out + j] = res[j];
                }
            }
        }
#pragma unroll
        for (int k = 0; k < R; ++k)
#pragma unroll
            for (int j = 0; j < 4; ++j) { D[k][j] = D[k + 1][j]; P[k][j] = P[k + 1][j]; }
#pragma unroll
        for (int j = 0; j < 4; ++j) D[R][j] = P[R][j] = 0.0f;
        if (pre) {
            const int sn = slot0 + R + 1 >= NR ? slot0 + R + 1 - NR : slot0 + R + 1;
            const int sp = slot0 + R >= NR ? slot0 + R - NR : slot0 + R;
            asm volatile("cp.async.wait_all;" ::: "memory");
            pair_put_row<SW>(c, s + R + 1 + c.off_y, ix0, p.alpha, stg, ring1 + sn * SW4,
                             ring2 + sn * SW, ring2 + sp * SW, cm, lane, vec_ok);
        }
        __syncwarp();
        slot0 = slot0 + 1 == NR ? 0 : slot0 + 1;
    }
}

// ------------------------- pair-sharing kernel, partner ring in TMEM
// Same arithmetic, order and results as bilateral_pair_kernel (bit-identical,
// tested), with two storage changes that free registers and shared memory so
// that 16 warps fit on an SM instead of 12 (the kernel is latency-bound:
// ncu "wait" / MIO stalls with 3 warps per scheduler):
//  * the per-row partner accumulators D/P[1..R] (8(R+1) floats per thread,
//    the largest live register set) live in tensor memory: TMEM lane
//    32 (warp % 4) + lane, 8 columns per ring slot (D[0..3], P[0..3]), the
//    slot of row s is s mod (R+1), so the per-step ring shift of the
//    register version becomes an index rotation.  Each row pair loads its two
//    partner slots (tcgen05.ld 32x32b.x8), folds, and stores them back
//    (tcgen05.st); the own row's slot is loaded once per step.  One warp of
//    the CTA allocates 64 columns (<= 8 CTAs per SM: 512 columns).
//  * no plain (non-interleaved) row ring: the own row dy = 0 and the odd last
//    row are read as the .x halves of the interleaved row-pair slots.
#ifndef LOP_PAIR_TM_MAXREG
#define LOP_PAIR_TM_MAXREG 128
#endif
#ifndef LOP_PAIR_TM_DY_UNROLL
#define LOP_PAIR_TM_DY_UNROLL 1   // packed row-pair loop of the TMEM kernel (1: rolled)
#endif
namespace pair {
constexpr int kTmemCols = 64;                          // per CTA; >= 8 (R + 1) for R <= 7
constexpr int kTmDyUnroll = LOP_PAIR_TM_DY_UNROLL;
constexpr int kTmemMinSmem = 25600;                    // dynamic smem floor: <= 8 CTAs / SM
template <int R> struct ShapeTM {
    static constexpr int WARP_FLOATS = Shape<R>::RING2 + 2 * Shape<R>::SW;   // ring2, staging, column map
};
}  // namespace pair

__device__ __forceinline__ void tm_ld8(uint32_t ta, float v[8])
{
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8];"
                 : "=f"(v[0]), "=f"(v[1]), "=f"(v[2]), "=f"(v[3]), "=f"(v[4]), "=f"(v[5]), "=f"(v[6]),
                   "=f"(v[7])
                 : "r"(ta));
}
// wait for the outstanding tcgen05.ld; the values become valid here (the
// registers are in/out operands so no use is scheduled above the wait)
__device__ __forceinline__ void tm_wait_ld8(float v[8])
{
    asm volatile("tcgen05.wait::ld.sync.aligned;"
                 : "+f"(v[0]), "+f"(v[1]), "+f"(v[2]), "+f"(v[3]), "+f"(v[4]), "+f"(v[5]), "+f"(v[6]),
                   "+f"(v[7]));
}
__device__ __forceinline__ void tm_wait_ld16(float a[8], float b[8])
{
    asm volatile("tcgen05.wait::ld.sync.aligned;"
                 : "+f"(a[0]), "+f"(a[1]), "+f"(a[2]), "+f"(a[3]), "+f"(a[4]), "+f"(a[5]), "+f"(a[6]),
                   "+f"(a[7]), "+f"(b[0]), "+f"(b[1]), "+f"(b[2]), "+f"(b[3]), "+f"(b[4]), "+f"(b[5]),
                   "+f"(b[6]), "+f"(b[7]));
}
__device__ __forceinline__ void tm_st8(uint32_t ta, const float v[8])
{
    asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8};"
                 ::"r"(ta), "f"(v[0]), "f"(v[1]), "f"(v[2]), "f"(v[3]), "f"(v[4]), "f"(v[5]), "f"(v[6]),
                   "f"(v[7]));
}
__device__ __forceinline__ void tm_wait_st() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }

// The .x halves (row r) of this lane's 4 NV columns of an interleaved slot.
template <int NV>
__device__ __forceinline__ void load_row_x(const float2 *slot, int lane, float *u)
{
    const float4 *src = reinterpret_cast<const float4 *>(slot);
#pragma unroll
    for (int k = 0; k < 2 * NV; ++k) {
        const int i = 2 * lane + k;                          // swizzled (pair_put_row)
        const float4 q = src[i ^ ((i >> 3) & 1)];
        u[2 * k] = q.x;
        u[2 * k + 1] = q.z;
    }
}

// TIGHT: frames of OWT output columns (launches that span several waves, where
// fewer frames mean fewer waves); otherwise the lane-aligned OW of the register
// kernel (its simpler store path measured faster within one wave).  The frame
// geometry never changes a result: every pixel's order depends on x mod 4 only.
template <int R, bool TIGHT>
__global__ void __maxnreg__(LOP_PAIR_TM_MAXREG) bilateral_pair_tm_kernel(const __grid_constant__ BilateralSep p)
{
    using S = pair::Shape<R>;
    constexpr int SW = S::SW, NV = S::NV, NR = S::NR, PAD = S::PAD;
    constexpr int NT = R + 1;                                    // TMEM ring slots
    const Common &c = p.c;
    const Geom &g = c.in;
    extern __shared__ float4 smem4[];
    __shared__ uint32_t tm_base_sh;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    float *wbase = reinterpret_cast<float *>(smem4) + warp * pair::ShapeTM<R>::WARP_FLOATS;
    float2 *ring2 = reinterpret_cast<float2 *>(wbase);                    // NR x SW pairs
    float4 *stg = reinterpret_cast<float4 *>(wbase + S::RING2);           // SW
    int *cm = reinterpret_cast<int *>(wbase + S::RING2 + SW);             // SW
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;"
                     ::"r"(smem_addr(&tm_base_sh)), "n"(pair::kTmemCols) : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t tbase = tm_base_sh + ((uint32_t)(32 * (warp & 3)) << 16);
    const int b = blockIdx.z;
    const int ox0 = TIGHT ? ((c.roi_x0 - R) & ~3) + blockIdx.x * S::OWT + R   // frame start + R
                          : (c.roi_x0 & ~3) + blockIdx.x * S::OW;             // frame start + HL
    const int T = p.pair_rows;
    const float wc = ex2_approx(p.lx[R]);                        // centre weight (see pair_row1)
    const int y0 = c.roi_y0 + (blockIdx.y * pair::NW + warp) * T;
    const int roi_y1 = c.roi_y0 + c.roi_h;
    if (y0 < roi_y1) {                                           // warp-uniform
        const int yend = min(y0 + T, roi_y1);
        const int ix0 = ox0 - (TIGHT ? R : S::HL) + c.off_x - PAD;
        const bool vec_ok = ((ix0 & 3) == 0) && ((g.stride & 15) == 0) &&
                            ((reinterpret_cast<uintptr_t>(g.data + (int64_t)b * g.bstride) & 15) == 0);
        pair_colmap<SW>(c, ix0, cm, lane);
        __syncwarp();
        // rows y0-R .. y0 -> interleaved slots 0..R; raw row r is fetched into
        // the storage of slot r + 1 (not written until row r + 1 is put)
        for (int r = 0; r <= R; ++r)
            pair_issue_row<SW>(c, b, y0 - R + r + c.off_y, ix0, reinterpret_cast<float4 *>(ring2 + (r + 1) * SW),
                               cm, lane, vec_ok);
        asm volatile("cp.async.wait_all;" ::: "memory");
        for (int r = 0; r <= R; ++r) {
            pair_put_row<SW, false>(c, y0 - R + r + c.off_y, ix0, p.alpha,
                                    reinterpret_cast<const float4 *>(ring2 + (r + 1) * SW), nullptr,
                                    ring2 + r * SW, r > 0 ? ring2 + (r - 1) * SW : nullptr, cm, lane, vec_ok);
            __syncwarp();
        }
        const float zero8[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
#pragma unroll
        for (int k = 0; k < NT; ++k) tm_st8(tbase + 8 * k, zero8);
        // this lane's stored columns [xs0, xs1): TIGHT frames store the frame columns
        // [R, R + OWT) (straddling lanes partly); aligned frames whole lanes
        // [HLN, 32 - HLN) (the register kernel's store path)
        const int x_out = TIGHT ? ox0 - R + 4 * lane : ox0 + 4 * (lane - S::HLN);
        int xs0 = 0, xs1 = 0;
        bool store_lane;
        if constexpr (TIGHT) {
            xs0 = max(x_out, max(ox0, c.roi_x0));
            xs1 = min(x_out + 4, min(ox0 + S::OWT, c.roi_x0 + c.roi_w));
            store_lane = xs1 > xs0;
        } else {
            store_lane = lane >= S::HLN && lane < 32 - S::HLN && x_out < c.roi_x0 + c.roi_w && x_out + 3 >= c.roi_x0;
        }
        int slot0 = 0, ts0 = 0;                                  // ring slot / TMEM slot of row s
#pragma unroll 1
        for (int s = y0 - R; s < yend; ++s) {
            const bool pre = s + 1 < yend;
            if (pre) pair_issue_row<SW>(c, b, s + R + 1 + c.off_y, ix0, stg, cm, lane, vec_ok);
            const int kmin = y0 - s;
            float u[4 * NV];
            load_row_x<NV>(ring2 + slot0 * SW, lane, u);
            const float cen[4] = {u[PAD], u[PAD + 1], u[PAD + 2], u[PAD + 3]};
            tm_wait_st();                                        // last step's stores have landed
            float DP[8];                                         // row s: D[0..3], P[0..3]
            tm_ld8(tbase + 8 * ts0, DP);
            tm_wait_ld8(DP);
            float *D0 = DP, *P0 = DP + 4;
            if (kmin <= 0) {                                     // dy = 0: own row (scalar)
                float rd[4], rp[4], qd[4], qp[4];
                pair_row1<R, PAD, true>(u, cen, p.lx, p.nk, wc, rd, rp, qd, qp);
                const float cy = p.cy[R];
                fold4(cy, rd, rp, D0, P0);
                fold4(cy, qd, qp, D0, P0);
            }
#pragma unroll pair::kTmDyUnroll
            for (int dy = 1; dy + 1 <= R; dy += 2) {             // row pairs (dy, dy+1): packed
                if (dy + 1 < kmin) continue;
                const int sl = slot0 + dy >= NR ? slot0 + dy - NR : slot0 + dy;
                float2 v[4 * NV];
                {
                    const float4 *src = reinterpret_cast<const float4 *>(ring2 + sl * SW);
#pragma unroll
                    for (int k = 0; k < 2 * NV; ++k) {
                        const int i = 2 * lane + k;
                        const float4 q = src[i ^ ((i >> 3) & 1)];
                        v[2 * k] = make_float2(q.x, q.y);
                        v[2 * k + 1] = make_float2(q.z, q.w);
                    }
                }
                float2 rd[4], rp[4], qd[4], qp[4];
                pair_row2<R, PAD>(v, cen, p.lx, rd, rp, qd, qp);
                const float cya = p.cy[dy + R], cyb = p.cy[dy + 1 + R];
                float ta[4], tb[4], sa[4], sb[4];
#pragma unroll
                for (int j = 0; j < 4; ++j) { ta[j] = rd[j].x; sa[j] = rp[j].x; tb[j] = rd[j].y; sb[j] = rp[j].y; }
                fold4(cya, ta, sa, D0, P0);
                fold4(cyb, tb, sb, D0, P0);
#pragma unroll
                for (int j = 0; j < 4; ++j) { ta[j] = qd[j].x; sa[j] = qp[j].x; tb[j] = qd[j].y; sb[j] = qp[j].y; }
                const int ka = ts0 + dy >= NT ? ts0 + dy - NT : ts0 + dy;
                const int kb = ka + 1 >= NT ? ka + 1 - NT : ka + 1;
                float A[8], B[8];                                // partner rows s+dy, s+dy+1
                tm_ld8(tbase + 8 * ka, A);
                tm_ld8(tbase + 8 * kb, B);
                tm_wait_ld16(A, B);
                fold4(cya, ta, sa, A, A + 4);
                fold4(cyb, tb, sb, B, B + 4);
                tm_st8(tbase + 8 * ka, A);
                tm_st8(tbase + 8 * kb, B);
            }
            if constexpr (R % 2 == 1) {                          // odd R: last row dy = R (scalar)
                const int sl = slot0 + R >= NR ? slot0 + R - NR : slot0 + R;
                float v[4 * NV];
                load_row_x<NV>(ring2 + sl * SW, lane, v);
                float rd[4], rp[4], qd[4], qp[4];
                pair_row1<R, PAD, false>(v, cen, p.lx, p.nk, wc, rd, rp, qd, qp);
                const float cy = p.cy[2 * R];
                fold4(cy, rd, rp, D0, P0);
                const int kr = ts0 + R >= NT ? ts0 + R - NT : ts0 + R;
                float A[8];
                tm_ld8(tbase + 8 * kr, A);
                tm_wait_ld8(A);
                fold4(cy, qd, qp, A, A + 4);
                tm_st8(tbase + 8 * kr, A);
            }
            if (s >= y0 && store_lane) {
                float res[4];
#pragma unroll
                for (int j = 0; j < 4; ++j) res[j] = bilateral_finish_scaled(D0[j], P0[j], p.inv_alpha);
                if (TIGHT) {
                    pair_store_span(c, b, s, x_out, xs0, xs1, res);
                } else if (x_out >= c.roi_x0) {
                    store4(c, b, s, x_out, res);
                } else {
                    float *orow = reinterpret_cast<float *>(c.out.data + (int64_t)b * c.out.bstride +
                                                            (int64_t)s * c.out.stride);
#pragma unroll
                    for (int j = 0; j < 4; ++j)
                        if (x_out + j >= c.roi_x0 && x_out + j < c.roi_x0 + c.roi_w) orow[x_out + j] = res[j];
                }
            }
            tm_st8(tbase + 8 * ts0, zero8);                      // the slot now serves row s + R + 1
            if (pre) {
                const int sn = slot0 + R + 1 >= NR ? slot0 + R + 1 - NR : slot0 + R + 1;
                const int sp = slot0 + R >= NR ? slot0 + R - NR : slot0 + R;
                asm volatile("cp.async.wait_all;" ::: "memory");
                pair_put_row<SW, false>(c, s + R + 1 + c.off_y, ix0, p.alpha, stg, nullptr, ring2 + sn * SW,
                                        ring2 + sp * SW, cm, lane, vec_ok);
            }
            __syncwarp();
            slot0 = slot0 + 1 == NR ? 0 : slot0 + 1;
            ts0 = ts0 + 1 == NT ? 0 : ts0 + 1;
        }
        tm_wait_st();
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (warp == 0) {
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tm_base_sh),
                     "n"(pair::kTmemCols) : "memory");
    }
}

// ------------------------------------------------------------- launchers
template <typename P, typename K>
static cudaError_t launch_tiled(K kernel, const P &p, size_t smem, cudaStream_t stream,
                                PerDevice &configured)
{
    cudaError_t e = ensure_smem(kernel, smem, configured);
    if (e != cudaSuccess) return e;
    dim3 grid((p.c.roi_w + tiled::TW - 1) / tiled::TW, (p.c.roi_h + tiled::TH - 1) / tiled::TH,
              p.c.batch);
    kernel<<<grid, tiled::NT, smem, stream>>>(p);
    return cudaGetLastError();
}

template <int RX, bool SC>
static cudaError_t launch_tiled_rx_sc(const BilateralTiled &p, cudaStream_t stream)
{
    using S = tiled::Shape<RX>;
    static PerDevice configured;
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
    static PerDevice configured;
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

// Pair kernel: rows per warp T from a wave-quantisation model (the paper's
// Alg. 2 idea -- pick the configuration from occupancy -- on B200 terms):
// cost(T) = waves(T) * (T + warm-up), waves = ceil(CTAs / resident CTAs);
// LOP_PAIR_ROWS overrides.
#ifndef LOP_PAIR_TMEM
#define LOP_PAIR_TMEM 1       // default kernel: 1 = partner ring in TMEM (bilateral_pair_tm_kernel)
#endif
static bool pair_tmem_enabled()
{
    static const int v = [] {
        const char *env = std::getenv("LOP_PAIR_TMEM");
        return env ? std::atoi(env) : LOP_PAIR_TMEM;
    }();
    return v != 0;
}

template <int R>
static cudaError_t launch_pair_r(const BilateralSep &p0, cudaStream_t stream)
{
    using S = pair::Shape<R>;
    // TMEM kernel for launches of at least 1024^2 pixels: below that the launch is
    // latency-bound and the TMEM allocation / barriers / ring clearing cost more
    // than the occupancy buys (config 1, 256^2 3x3: 4.5 -> 6.1 us per launch).
    // Both kernels give the same bits, so the choice is free to depend on size.
    // and windows of 9 x 9 and up: for 3 x 3 the register kernel is faster (4096^2: 82 vs
    // 98 us), 5 x 5 / 7 x 7 tie (profiles/r02/sweep_bilateral_pair_vs_sep_tm.jsonl)
    const bool tm = pair_tmem_enabled() && R >= 4 &&
                    (double)p0.c.in.W * (double)p0.c.in.GH * (double)p0.c.batch >= 1024.0 * 1024.0;
    static PerDevice smem_set, resident_cache, smem_set_tm, resident_cache_tm;
    const size_t smem = tm ? std::max((size_t)pair::NW * pair::ShapeTM<R>::WARP_FLOATS * sizeof(float),
                                      (size_t)pair::kTmemMinSmem)
                           : (size_t)pair::NW * S::WARP_FLOATS * sizeof(float);
    auto kern = tm ? bilateral_pair_tm_kernel<R, false> : bilateral_pair_kernel<R>;
    cudaError_t e;
    const int64_t resident =
        tm ? resident_ctas_tmem(kern, pair::NW * 32, smem, pair::kTmemCols, smem_set_tm, resident_cache_tm, e)
           : resident_ctas(kern, pair::NW * 32, smem, smem_set, resident_cache, e);
    if (e != cudaSuccess) return e;
    e = ensure_smem(kern, smem, tm ? smem_set_tm : smem_set);
    if (e != cudaSuccess) return e;
    BilateralSep p = p0;
    // rows per warp T from the wave model, for a frame geometry of `strips` frames
    auto plan = [&](int64_t strips, double &best) {
        int T = 0;
        best = 0;
        const int tmax = std::max(1, p.c.roi_h);
        for (int t = 1; t <= tmax; ++t) {
            const int64_t segs = (p.c.roi_h + t - 1) / t;
            const int64_t ctas = strips * ((segs + pair::NW - 1) / pair::NW) * p.c.batch;
            const double cost = (double)((ctas + resident - 1) / resident) * (t + 0.55 * R);
            if (T == 0 || cost < best) { best = cost; T = t; }
            if (segs == 1) break;
        }
        return T;
    };
    // lane-aligned frames of OW output columns, or (TMEM kernel) TIGHT frames of OWT
    const int64_t strips_a = ((p.c.roi_x0 & 3) + p.c.roi_w + S::OW - 1) / S::OW;
    const int64_t first_t = ((p.c.roi_x0 - R) & ~3) + R;
    const int64_t strips_t = (p.c.roi_x0 + p.c.roi_w - first_t + S::OWT - 1) / S::OWT;
    int T = 0;
    if (const char *env = std::getenv("LOP_PAIR_ROWS")) T = std::atoi(env);
    static thread_local int64_t memo_key[4] = {-1, -1, -1, -1};
    static thread_local int memo_T = 0, memo_tight = 0;
    int tight = 0;
    if (T <= 0 && memo_key[0] == p.c.roi_h && memo_key[1] == strips_a * 4096 + p.c.roi_w % 4096 &&
        memo_key[2] == p.c.batch && memo_key[3] == resident * 2 + tm) {
        T = memo_T;
        tight = memo_tight;
    } else if (T <= 0) {
        // every T from 1 to the ROI height: waves of resident CTAs x rows per warp
        // (+ warm-up); a partial wave costs a full one (few warps per SM
        // cannot saturate the SFU).  Small images take small T: the row steps of
        // a warp are serial (one global row fetch each), so a launch that fits
        // in one wave is latency-bound by T + R steps (config 1: T = 1).
        // TIGHT frames when they cut the modelled time by more than the ~2 % their
        // store path costs (launches spanning several waves: config 4's 1024-column
        // frames, config 5's 32768-column bands); same results either way.
        double cost_a = 0, cost_t = 0;
        T = plan(strips_a, cost_a);
        if (tm) {
            const int Tt = plan(strips_t, cost_t);
            if (cost_t < 0.97 * cost_a) { T = Tt; tight = 1; }
        }
        memo_key[0] = p.c.roi_h; memo_key[1] = strips_a * 4096 + p.c.roi_w % 4096;
        memo_key[2] = p.c.batch; memo_key[3] = resident * 2 + tm;
        memo_T = T;
        memo_tight = tight;
    }
    if (const char *env = std::getenv("LOP_PAIR_TIGHT")) tight = tm && std::atoi(env) != 0;   // A/B
    p.pair_rows = T;
    const int64_t strips = tight ? strips_t : strips_a;
    const int64_t segs = (p.c.roi_h + T - 1) / T;
    dim3 grid((unsigned)strips, (unsigned)((segs + pair::NW - 1) / pair::NW), p.c.batch);
    if (tight) kern = bilateral_pair_tm_kernel<R, true>;
    kern<<<grid, pair::NW * 32, smem, stream>>>(p);
    return cudaGetLastError();
}

cudaError_t launch_bilateral_pair(const BilateralSep &p, cudaStream_t stream)
{
    switch (p.c.rx) {
    case 1: return launch_pair_r<1>(p, stream);
    case 2: return launch_pair_r<2>(p, stream);
    case 3: return launch_pair_r<3>(p, stream);
    case 4: return launch_pair_r<4>(p, stream);
    case 5: return launch_pair_r<5>(p, stream);
    case 6: return launch_pair_r<6>(p, stream);
    case 7: return launch_pair_r<7>(p, stream);
    default: return cudaErrorInvalidValue;
    }
}

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

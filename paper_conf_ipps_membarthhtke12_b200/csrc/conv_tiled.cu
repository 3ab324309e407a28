// conv_tiled.cu -- HBM-bound tiled convolution kernels (Gaussian / Sobel and
// any separable mask up to 9x9): Tables VIII-IX, Sobel
// "same implementation" (L847-L849).
//
// Design:
//  * the mask is separable (factorised exactly on the host): M = c r^T, so
//    each output is sum_t c[t] * (sum_xf r[xf] * I(x+xf, y+t-RY)).  The u8
//    path is exact integer arithmetic, hence bit-identical to the 2D
//    definition (reading c13); the f32 path is within rounding of it.
//  * a CTA (128 threads) owns an output tile of 128*PX columns x TS rows
//    (f32: 512 x 16, u8: 1024 x 16).  Its input footprint, TS + 2RY rows of
//    128*PX + 2*PAD bytes-aligned columns, is staged into shared memory with
//    one cp.async.bulk (TMA bulk copy, SASS UBLKCP) per row completing on an
//    mbarrier -- every row of the tile in flight at once, each input byte read
//    from DRAM once.  Border tiles (image edge, band edge without halo,
//    unaligned views) stage element by element with the boundary resolved at
//    staging time instead (the paper's nine-region idea, Fig. 3 / Listing 8,
//    reduced to interior vs border CTAs).
//  * each thread then streams its PX columns down the tile from shared
//    memory, keeps the horizontal sums of the last 2RY+1 rows in registers and
//    writes every output row with one 16-B (f32, i32) / 8-B (u8) store.
//  * coefficients are kernel parameters (constant-bank operands of FFMA/IMAD),
//    the dynamic constant-memory variant of §IV-C (L563-L605).
#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <type_traits>

#include "boundary.cuh"
#include "stage.cuh"
#include "kernels.h"
#include "launch_cache.h"
#include "lop_params.h"

namespace lop {

namespace convt {
constexpr int NT = 128;      // threads per CTA
}  // namespace convt

template <typename T> struct Px;
template <> struct Px<float> { static constexpr int N = 4; };
template <> struct Px<uint8_t> { static constexpr int N = 8; };

template <typename T> struct TileShape {
    static constexpr int PX = Px<T>::N;
    static constexpr int TWE = convt::NT * PX;                 // output columns per tile
    static constexpr int PADE = 16 / sizeof(T);                // left/right pad (elements), 16 B
    static constexpr int SWE = TWE + 2 * PADE;                 // smem row pitch (elements)
    static constexpr int ROW_BYTES = SWE * sizeof(T);          // multiple of 16
};


// u8 -> u8 with non-negative coefficients whose sums fit 16 bits: SWAR on two
// 16-bit lanes per 32-bit register (pixels q and q+2), so every IMAD does two
// exact integer MACs.  Exactness conditions are checked on the host
// (launch_conv_tiled).  MODE bits: SW_SYM -- both factors are palindromes
// (every Gaussian): taps t and 2R-t are added first (IADD, ALU pipe) and
// multiplied once (IMAD, FMA pipe), R+1 instead of 2R+1 IMADs per sum;
// SW_SH8 -- shift 8 (5x5 binomial): the rounded result of each lane is its
// byte 1, so two PRMTs pack 8 outputs with no shift or mask.
// Sources: each staged word W splits into E(W) = lanes (b0, b2) and O(W) =
// lanes (b1, b3) (PRMT with a zero source); the lanes (q, q+2) that straddle
// two words are one PRMT of two E (or O) words.  All integer arithmetic is
// exact, so every MODE gives the same bits.
// SW_I32 -- u8 -> i32 with signed coefficients (Sobel): every lane starts from
// a bias (sw_bias_h per row sum, sw_bias_v per column sum) chosen on the host
// so that the final value of each 16-bit lane lies in [0, 65535] -- the 32-bit
// arithmetic is modular, so borrows between lanes in intermediate steps cancel
// once the final low lane is in range -- and S = lane - sw_off exactly.
// SW_BIN5 -- both factors are the binomial [1 4 6 4 1] (the 5x5 Gaussian):
// the coefficients are compile-time constants (the paper's outlook, L946-L950:
// "propagate the constants of the filter masks"), so a sum is
// (a + e) + 4 (b + d) + 6 c -- two adds, a shift-add and one IMAD.
enum { SW_ON = 1, SW_SYM = 2, SW_SH8 = 4, SW_I32 = 8, SW_BIN5 = 16 };

// FULL: the tile has all TS + 2R staged rows (every tile but a partial last
// one), so the unrolled row loop carries no per-row bound check (the check made
// the compiler wrap every row in a divergence region).
template <int R, int TS, int MODE, bool FULL, bool VEC>
__device__ __forceinline__ void conv_u8_swar(const ConvSep &p, const uint8_t *tcol, int srows,
                                             char *orow0, int64_t ostride, int ox0, int roi_x1,
                                             bool ovec)
{
    constexpr int SWE = TileShape<uint8_t>::SWE;
    constexpr uint32_t M = 0x00FF00FFu;
    constexpr bool SYM = (MODE & SW_SYM) != 0, SH8 = (MODE & SW_SH8) != 0, I32 = (MODE & SW_I32) != 0;
    constexpr bool BIN5 = (MODE & SW_BIN5) != 0;
    static_assert(!BIN5 || (R == 2 && SYM && SH8), "binomial 5x5 constants");
    static_assert(R <= 3, "SWAR sources cover bytes -4..11");
    const uint32_t rnd = I32 ? (uint32_t)p.sw_bias_v * 0x00010001u
                             : (p.shift > 0 ? (1u << (p.shift - 1)) * 0x00010001u : 0u);
    const uint32_t hb = I32 ? (uint32_t)p.sw_bias_h * 0x00010001u : 0u;
    uint32_t h[2 * R + 1][4];                     // pairs (0,2) (1,3) (4,6) (5,7)
#pragma unroll
    for (int k = 0; k < TS + 2 * R; ++k) {
        if (!FULL && k >= srows) break;
        const uint8_t *rp = tcol + k * SWE;
        const uint2 cv = *reinterpret_cast<const uint2 *>(rp);
        const uint32_t W[4] = {*reinterpret_cast<const uint32_t *>(rp - 4), cv.x, cv.y,
                               *reinterpret_cast<const uint32_t *>(rp + 8)};
        uint32_t E[4], O[4];
#pragma unroll
        for (int i = 0; i < 4; ++i) {
            E[i] = __byte_perm(W[i], 0u, 0x4240);            // bytes 0, 2 -> lanes
            O[i] = __byte_perm(W[i], 0u, 0x4341);            // bytes 1, 3 -> lanes
        }
        uint32_t S[6 + 2 * R];                    // S[q + R] = lanes (q, q+2), q in [-R, 5+R]
#pragma unroll
        for (int q = -R; q <= 5 + R; ++q) {
            const int wi = (q + 4) >> 2, sh = (q + 4) & 3;
            if (sh == 0) S[q + R] = E[wi];
            else if (sh == 1) S[q + R] = O[wi];
            else if (sh == 2) S[q + R] = __byte_perm(E[wi], E[wi + 1], 0x5412);   // (b2, b4')
            else S[q + R] = __byte_perm(O[wi], O[wi + 1], 0x5412);                // (b3, b5')
        }
        uint32_t *hk = h[k % (2 * R + 1)];
        constexpr int J[4] = {0, 1, 4, 5};
#pragma unroll
        for (int jj = 0; jj < 4; ++jj) {
            uint32_t s;
            if constexpr (BIN5) {
                const uint32_t *x = S + J[jj];
                s = (x[0] + x[4]) + ((x[1] + x[3]) << 2) + 6u * x[2];
            } else if constexpr (SYM) {
                s = (uint32_t)p.ri[R] * S[J[jj] + R];
#pragma unroll
                for (int t = 0; t < R; ++t) s += (uint32_t)p.ri[t] * (S[J[jj] + t] + S[J[jj] + 2 * R - t]);
            } else {
                s = (uint32_t)p.ri[0] * S[J[jj]] + hb;
#pragma unroll
                for (int t = 1; t <= 2 * R; ++t) s += (uint32_t)p.ri[t] * S[J[jj] + t];
            }
            hk[jj] = s;
        }
        const int o = k - 2 * R;
        if (o < 0) continue;
        uint32_t q4[4];
#pragma unroll
        for (int jj = 0; jj < 4; ++jj) {
            uint32_t s;
            if constexpr (BIN5) {
                const uint32_t h0 = h[o % 5][jj], h1 = h[(o + 1) % 5][jj], h2 = h[(o + 2) % 5][jj],
                               h3 = h[(o + 3) % 5][jj], h4 = h[(o + 4) % 5][jj];
                s = (h0 + h4 + rnd) + ((h1 + h3) << 2) + 6u * h2;
            } else if constexpr (SYM) {
                s = (uint32_t)p.ci[R] * h[(o + R) % (2 * R + 1)][jj] + rnd;    // rounding folded in
#pragma unroll
                for (int t = 0; t < R; ++t)
                    s += (uint32_t)p.ci[t] * (h[(o + t) % (2 * R + 1)][jj] + h[(o + 2 * R - t) % (2 * R + 1)][jj]);
            } else {
                s = (uint32_t)p.ci[0] * h[o % (2 * R + 1)][jj] + rnd;
#pragma unroll
                for (int t = 1; t <= 2 * R; ++t) s += (uint32_t)p.ci[t] * h[(o + t) % (2 * R + 1)][jj];
            }
            q4[jj] = (SH8 || I32) ? s : (s >> p.shift) & M;
        }
        if constexpr (I32) {
            // lanes -> S = lane - sw_off, then (S + 2^(k-1)) >> k (quantize_shift)
            int v[8];
#pragma unroll
            for (int jj = 0; jj < 4; ++jj) {
                const int px = J[jj];                                // lanes: pixels px, px + 2
                v[px] = quantize_shift((int)(q4[jj] & 0xFFFFu) - p.sw_off, p.shift);
                v[px + 2] = quantize_shift((int)(q4[jj] >> 16) - p.sw_off, p.shift);
            }
            int32_t *op = reinterpret_cast<int32_t *>(orow0) + ox0;   // output row o (running pointer)
            orow0 += ostride;
            if (VEC || ovec) {
                *reinterpret_cast<int4 *>(op) = make_int4(v[0], v[1], v[2], v[3]);
                *reinterpret_cast<int4 *>(op + 4) = make_int4(v[4], v[5], v[6], v[7]);
            } else {
#pragma unroll
                for (int j = 0; j < 8; ++j)
                    if (ox0 + j < roi_x1) op[j] = v[j];
            }
            continue;
        }
        // lo = pixels 0..3 = lanes of q4[0] (0, 2) and q4[1] (1, 3); hi likewise
        const uint32_t lo = SH8 ? __byte_perm(q4[0], q4[1], 0x7351) : __byte_perm(q4[0], q4[1], 0x6240);
        const uint32_t hi = SH8 ? __byte_perm(q4[2], q4[3], 0x7351) : __byte_perm(q4[2], q4[3], 0x6240);
        uint8_t *op = reinterpret_cast<uint8_t *>(orow0) + ox0;    // output row o (running pointer)
        orow0 += ostride;
        if (VEC || ovec) {
            *reinterpret_cast<uint2 *>(op) = make_uint2(lo, hi);
        } else {
#pragma unroll
            for (int j = 0; j < 8; ++j)
                if (ox0 + j < roi_x1) op[j] = (uint8_t)((j < 4 ? lo : hi) >> (8 * (j & 3)));
        }
    }
}

// f32 separable pass with sm_100 packed FP32 for the vertical half: the ring
// holds the horizontal sums of two adjacent columns as a register pair, so
// (o[j], o[j+1]) = c0 (h[o][j], h[o][j+1]) + sum_t c[t] (...) is one FMUL2 /
// FFMA2 per tap with the coefficient as a broadcast pair.  Each lane performs
// exactly the scalar operation of its column (same operands, same order,
// round-to-nearest), so the result is the scalar kernel's bit for bit.
template <int R, int TS, bool FULL, bool VEC>
__device__ __forceinline__ void conv_f32_packed(const ConvSep &p, const float *tcol, int srows,
                                                char *orow0, int64_t ostride, int ox0, int roi_x1,
                                                bool ovec)
{
    constexpr int SWE = TileShape<float>::SWE;
    constexpr int P = 2 * R + 1;
    float2 h[P][2];                                                 // (h0,h1), (h2,h3) ring
#pragma unroll
    for (int k = 0; k < TS + 2 * R; ++k) {
        if (!FULL && k >= srows) break;
        const float *rp = tcol + k * SWE;
        float v[4 + 2 * R];
        const float4 cv = *reinterpret_cast<const float4 *>(rp);
        v[R + 0] = cv.x; v[R + 1] = cv.y; v[R + 2] = cv.z; v[R + 3] = cv.w;
        if constexpr (R > 0) {
            const float4 l = *reinterpret_cast<const float4 *>(rp - 4);
            const float4 r = *reinterpret_cast<const float4 *>(rp + 4);
            const float lv[4] = {l.x, l.y, l.z, l.w}, rv[4] = {r.x, r.y, r.z, r.w};
#pragma unroll
            for (int j = 0; j < R; ++j) {
                v[j] = lv[4 - R + j];
                v[R + 4 + j] = rv[j];
            }
        }
        // horizontal: scalar (packing it would need a register pair per odd shift),
        // results written straight into the pair registers of the ring
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            float a = __fmul_rn(p.rf[0], v[j]);
#pragma unroll
            for (int t = 1; t <= 2 * R; ++t) a = __fmaf_rn(p.rf[t], v[j + t], a);
            if (j & 1) h[k % P][j >> 1].y = a;
            else h[k % P][j >> 1].x = a;
        }
        const int o = k - 2 * R;
        if (o < 0) continue;
        float2 out[2];
#pragma unroll
        for (int q = 0; q < 2; ++q) {
            float2 a = __fmul2_rn(h[o % P][q], make_float2(p.cf[0], p.cf[0]));
#pragma unroll
            for (int t = 1; t <= 2 * R; ++t)
                a = __ffma2_rn(h[(o + t) % P][q], make_float2(p.cf[t], p.cf[t]), a);
            out[q] = a;
        }
        float *op = reinterpret_cast<float *>(orow0) + ox0;        // output row o (running pointer)
        orow0 += ostride;
        if (VEC || ovec) {
            *reinterpret_cast<float4 *>(op) = make_float4(out[0].x, out[0].y, out[1].x, out[1].y);
        } else {
            const float w[4] = {out[0].x, out[0].y, out[1].x, out[1].y};
#pragma unroll
            for (int j = 0; j < 4; ++j)
                if (ox0 + j < roi_x1) op[j] = w[j];
        }
    }
}

// Tile geometry of tile index `t` (row-major over column tiles, row tiles, frames).
struct ConvTile {
    int b, tx0, ty0, nrows;
};

// Tile (blockIdx.x, blockIdx.y) of frame blockIdx.z (one tile per CTA): no
// integer division (the linear form below costs two division sequences per warp).
template <typename T, int TS>
__device__ __forceinline__ ConvTile conv_tile_grid(const Common &c)
{
    using S = TileShape<T>;
    ConvTile ct;
    ct.b = blockIdx.z;
    ct.tx0 = c.roi_x0 + (int)blockIdx.x * S::TWE;
    ct.ty0 = c.roi_y0 + (int)blockIdx.y * TS;
    ct.nrows = min(TS, c.roi_y0 + c.roi_h - ct.ty0);
    return ct;
}

template <typename T, int TS>
__device__ __forceinline__ ConvTile conv_tile_at(const Common &c, int t)
{
    using S = TileShape<T>;
    const int ntx = (c.roi_w + S::TWE - 1) / S::TWE, nty = (c.roi_h + TS - 1) / TS;
    ConvTile ct;
    ct.b = t / (ntx * nty);
    const int r = t - ct.b * ntx * nty;
    const int ty = r / ntx, tx = r - ty * ntx;
    ct.tx0 = c.roi_x0 + tx * S::TWE;
    ct.ty0 = c.roi_y0 + ty * TS;
    ct.nrows = min(TS, c.roi_y0 + c.roi_h - ct.ty0);
    return ct;
}

// Stage the input footprint of tile `ct` into `tile`: every staged row whose
// source row exists (in-image, halo, or mapped by the boundary mode) is copied
// by one cp.async.bulk of its 16-B aligned in-image column span completing on
// `bar` (thread 0 arms it with the byte count; 0 bytes completes at once); the
// out-of-image columns and CONSTANT rows are filled element by element with
// the boundary resolved per column (visible after the caller's __syncthreads).
template <typename T, int R>
__device__ __forceinline__ void conv_stage(const Common &c, const ConvTile &ct, T *tile,
                                           uint64_t *bar)
{
    using S = TileShape<T>;
    stage_rows<T, S::SWE, convt::NT>(c, ct.b, ct.tx0 + c.off_x - S::PADE, ct.ty0 + c.off_y - R,
                                     ct.nrows + 2 * R, tile, bar);
}


// Filter one staged tile: each thread streams its PX columns down the tile.
template <typename T, typename TO, int R, int TS, bool FULL, bool VEC>
__device__ __forceinline__ void conv_scalar(const ConvSep &p, const T *tcol, int srows, char *obase, int ty0,
                                            int ox0, int roi_x1, bool ovec);

// FULL: all TS + 2R staged rows present; VEC: the CTA's whole tile row lies in
// the iteration space and the output is 16-B aligned (whole-vector stores by
// every thread, no per-row divergent store branch).
template <typename T, typename TO, int R, int SWAR, int TS, bool FULL, bool VEC>
__device__ __forceinline__ void conv_compute(const ConvSep &p, const ConvTile &ct, const T *tile)
{
    constexpr int RY = R;
    using S = TileShape<T>;
    constexpr int PX = S::PX, PADE = S::PADE;
    constexpr bool F = sizeof(T) == 4;
    const Common &c = p.c;
    const int b = ct.b, ty0 = ct.ty0;
    const int srows = ct.nrows + 2 * RY;
    const int roi_x1 = c.roi_x0 + c.roi_w;
    const int ox0 = ct.tx0 + threadIdx.x * PX;
    if (ox0 >= roi_x1) return;
    char *obase = c.out.data + (int64_t)b * c.out.bstride;
    const bool ovec = (ox0 + PX <= roi_x1) && (ox0 % PX == 0) &&
                      (((reinterpret_cast<uintptr_t>(obase) | (uintptr_t)c.out.stride) %
                        (sizeof(TO) * PX > 16 ? 16 : sizeof(TO) * PX)) == 0);
    const T *tcol = tile + PADE + threadIdx.x * PX;              // this thread's centre column
    if constexpr (SWAR != 0) {
        static_assert(SWAR == 0 || sizeof(T) == 1, "SWAR is for u8 inputs");
        char *orow0 = obase + (int64_t)ty0 * c.out.stride;
        conv_u8_swar<R, TS, SWAR, FULL, VEC>(p, reinterpret_cast<const uint8_t *>(tcol), srows, orow0,
                                             c.out.stride, ox0, roi_x1, ovec);
        return;
    }
    if constexpr (F) {
        conv_f32_packed<R, TS, FULL, VEC>(p, reinterpret_cast<const float *>(tcol), srows,
                               obase + (int64_t)ty0 * c.out.stride, c.out.stride, ox0, roi_x1, ovec);
        return;
    }
    if constexpr (SWAR == 0 && !F) conv_scalar<T, TO, R, TS, FULL, VEC>(p, tcol, srows, obase, ty0, ox0, roi_x1, ovec);
}

// Scalar (unpacked integer) path: u8 -> u8 without SWAR, u8 -> i32.
template <typename T, typename TO, int R, int TS, bool FULL, bool VEC>
__device__ __forceinline__ void conv_scalar(const ConvSep &p, const T *tcol, int srows, char *obase, int ty0,
                                            int ox0, int roi_x1, bool ovec)
{
    constexpr int RX = R, RY = R;
    using S = TileShape<T>;
    constexpr int PX = S::PX, SWE = S::SWE;
    constexpr bool F = sizeof(T) == 4;
    using A = typename std::conditional<F, float, int>::type;   // accumulator type
    const Common &c = p.c;
    A h[2 * RY + 1][PX];                                          // horizontal sums, ring
#pragma unroll
    for (int k = 0; k < TS + 2 * RY; ++k) {
        if (!FULL && k >= srows) break;
        // ---- gather PX + 2RX values of staged row k
        A v[PX + 2 * RX];
        const T *rp = tcol + k * SWE;
        if constexpr (F) {
            const float4 cv = *reinterpret_cast<const float4 *>(rp);
            v[RX + 0] = cv.x; v[RX + 1] = cv.y; v[RX + 2] = cv.z; v[RX + 3] = cv.w;
            if constexpr (RX > 0) {
                const float4 l = *reinterpret_cast<const float4 *>(rp - 4);
                const float4 r = *reinterpret_cast<const float4 *>(rp + 4);
                const float lv[4] = {l.x, l.y, l.z, l.w}, rv[4] = {r.x, r.y, r.z, r.w};
#pragma unroll
                for (int j = 0; j < RX; ++j) {
                    v[j] = lv[4 - RX + j];
                    v[RX + PX + j] = rv[j];
                }
            }
        } else {
            const uint2 cv = *reinterpret_cast<const uint2 *>(rp);
            const uint32_t w[2] = {cv.x, cv.y};
#pragma unroll
            for (int j = 0; j < 8; ++j) v[RX + j] = (int)((w[j >> 2] >> (8 * (j & 3))) & 0xFF);
            if constexpr (RX > 0) {
                const uint32_t l = *reinterpret_cast<const uint32_t *>(rp - 4);
                const uint32_t r = *reinterpret_cast<const uint32_t *>(rp + 8);
#pragma unroll
                for (int j = 0; j < RX; ++j) {
                    v[j] = (int)((l >> (8 * (4 - RX + j))) & 0xFF);
                    v[RX + PX + j] = (int)((r >> (8 * j)) & 0xFF);
                }
            }
        }
        // ---- horizontal pass
        A *hk = h[k % (2 * RY + 1)];
#pragma unroll
        for (int j = 0; j < PX; ++j) {
            A s;
            if constexpr (F) {
                s = __fmul_rn(p.rf[0], v[j]);
#pragma unroll
                for (int t = 1; t <= 2 * RX; ++t) s = __fmaf_rn(p.rf[t], v[j + t], s);
            } else {
                s = p.ri[0] * v[j];
#pragma unroll
                for (int t = 1; t <= 2 * RX; ++t) s += p.ri[t] * v[j + t];
            }
            hk[j] = s;
        }
        // ---- vertical pass: output row o = k - 2RY is complete
        const int o = k - 2 * RY;
        if (o < 0) continue;
        A out[PX];
#pragma unroll
        for (int j = 0; j < PX; ++j) {
            A s;
            if constexpr (F) {
                s = __fmul_rn(p.cf[0], h[o % (2 * RY + 1)][j]);
#pragma unroll
                for (int t = 1; t <= 2 * RY; ++t)
                    s = __fmaf_rn(p.cf[t], h[(o + t) % (2 * RY + 1)][j], s);
            } else {
                s = p.ci[0] * h[o % (2 * RY + 1)][j];
#pragma unroll
                for (int t = 1; t <= 2 * RY; ++t) s += p.ci[t] * h[(o + t) % (2 * RY + 1)][j];
            }
            out[j] = s;
        }
        char *orow = obase + (int64_t)(ty0 + o) * c.out.stride;
        if constexpr (F) {
            float *op = reinterpret_cast<float *>(orow) + ox0;
            if (VEC || ovec) {
                *reinterpret_cast<float4 *>(op) = make_float4(out[0], out[1], out[2], out[3]);
            } else {
#pragma unroll
                for (int j = 0; j < PX; ++j)
                    if (ox0 + j < roi_x1) op[j] = out[j];
            }
        } else if constexpr (sizeof(TO) == 1) {
            uint32_t w[2] = {0u, 0u};
#pragma unroll
            for (int j = 0; j < PX; ++j) {
                const int q = min(max(quantize_shift(out[j], p.shift), 0), 255);
                w[j >> 2] |= (uint32_t)q << (8 * (j & 3));
            }
            uint8_t *op = reinterpret_cast<uint8_t *>(orow) + ox0;
            if (VEC || ovec) {
                *reinterpret_cast<uint2 *>(op) = make_uint2(w[0], w[1]);
            } else {
#pragma unroll
                for (int j = 0; j < PX; ++j)
                    if (ox0 + j < roi_x1) op[j] = (uint8_t)(w[j >> 2] >> (8 * (j & 3)));
            }
        } else {
            int32_t *op = reinterpret_cast<int32_t *>(orow) + ox0;
            int q[PX];
#pragma unroll
            for (int j = 0; j < PX; ++j) q[j] = quantize_shift(out[j], p.shift);
            if (VEC || ovec) {
                *reinterpret_cast<int4 *>(op) = make_int4(q[0], q[1], q[2], q[3]);
                *reinterpret_cast<int4 *>(op + 4) = make_int4(q[4], q[5], q[6], q[7]);
            } else {
#pragma unroll
                for (int j = 0; j < PX; ++j)
                    if (ox0 + j < roi_x1) op[j] = q[j];
            }
        }
    }
}

// NBUF = 2: persistent kernel -- each CTA walks tiles blockIdx.x,
// blockIdx.x + gridDim.x, ...; the next tile's rows are in flight
// (cp.async.bulk into the other smem buffer) while the current tile is
// filtered.  NBUF = 1: one tile per CTA (grid = #tiles), latency hidden by
// co-resident CTAs.  TS = output rows per tile.  (Configuration space of the
// paper's §V-D exploration, re-done for sm_100a: tools/tune_conv.py.)
template <typename T, typename TO, int R, int SWAR, int TS, int NBUF>
__global__ void __launch_bounds__(convt::NT) conv_sep_kernel(const __grid_constant__ ConvSep p)
{
    using S = TileShape<T>;
    static_assert(R <= 4, "halo must fit the 16-B pad");
    constexpr int BUF_ELEMS = (TS + 2 * R) * S::SWE;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    __shared__ __align__(8) uint64_t bar[2];
    T *buf0 = reinterpret_cast<T *>(smem_raw);
    T *buf1 = NBUF == 2 ? buf0 + BUF_ELEMS : buf0;
    const Common &c = p.c;
    const int ntiles = ((c.roi_w + S::TWE - 1) / S::TWE) * ((c.roi_h + TS - 1) / TS) * c.batch;
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared.b64 [%0], 1;" ::"r"(smem_addr(&bar[0])));
        asm volatile("mbarrier.init.shared.b64 [%0], 1;" ::"r"(smem_addr(&bar[1])));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if constexpr (NBUF == 1) {                      // 3D grid: one tile per CTA
        const ConvTile ct = conv_tile_grid<T, TS>(c);
        conv_stage<T, R>(c, ct, buf0, &bar[0]);
        __syncthreads();
        mbar_wait(&bar[0], 0);
        // full tiles (all but a partial last row of tiles) without per-row bound checks;
        // whole-vector stores when the tile row lies in the iteration space, aligned
        using S = TileShape<T>;
        const char *ob = c.out.data + (int64_t)ct.b * c.out.bstride;
        const bool cta_vec = ct.tx0 + S::TWE <= c.roi_x0 + c.roi_w && (ct.tx0 % S::PX) == 0 &&
                             ((reinterpret_cast<uintptr_t>(ob) | (uintptr_t)c.out.stride) % 16) == 0;
        if (ct.nrows == TS && cta_vec) conv_compute<T, TO, R, SWAR, TS, true, true>(p, ct, buf0);
        else if (ct.nrows == TS) conv_compute<T, TO, R, SWAR, TS, true, false>(p, ct, buf0);
        else conv_compute<T, TO, R, SWAR, TS, false, false>(p, ct, buf0);
        return;
    }
    int t = blockIdx.x;
    if (t < ntiles) conv_stage<T, R>(c, conv_tile_at<T, TS>(c, t), buf0, &bar[0]);
    for (int it = 0; t < ntiles; t += gridDim.x, ++it) {
        const int cur = it & 1;
        __syncthreads();        // tile it-1 fully consumed; element fills of tile it visible
        const int tn = t + gridDim.x;
        if (tn < ntiles)
            conv_stage<T, R>(c, conv_tile_at<T, TS>(c, tn), cur ? buf0 : buf1, &bar[cur ^ 1]);
        mbar_wait(&bar[cur], (it >> 1) & 1);
        conv_compute<T, TO, R, SWAR, TS, false, false>(p, conv_tile_at<T, TS>(c, t), cur ? buf1 : buf0);
    }
}

// -------------------------------------------------------------- host side
namespace {

int64_t gcd64(int64_t a, int64_t b)
{
    a = a < 0 ? -a : a;
    b = b < 0 ? -b : b;
    while (b) { int64_t t = a % b; a = b; b = t; }
    return a;
}

bool verify_f32(const float *M, int sx, int sy, const float *cf, const float *rf)
{
    for (int i = 0; i < sy; ++i)
        for (int j = 0; j < sx; ++j)
            if ((double)cf[i] * (double)rf[j] != (double)M[i * sx + j]) return false;
    return true;
}

// Exact rank-1 factorisation M = c r^T (integer or float); false if none.
bool factor(const ConvGeneric &p, ConvSep &s)
{
    const int sx = 2 * p.c.rx + 1, sy = 2 * p.c.ry + 1;
    if (sx > 9 || sy > 9) return false;
    for (int t = 0; t < 9; ++t) { s.rf[t] = s.cf[t] = 0.f; s.ri[t] = s.ci[t] = 0; }
    int i0 = -1, j0 = -1;
    for (int i = 0; i < sy && i0 < 0; ++i)
        for (int j = 0; j < sx; ++j) {
            const bool nz = p.kind == CONV_F32 ? p.m.f[i * sx + j] != 0.0f : p.m.i[i * sx + j] != 0;
            if (nz) { i0 = i; j0 = j; break; }
        }
    if (i0 < 0) return true;             // all-zero mask
    if (p.kind == CONV_F32) {
        const float *M = p.m.f;
        // (a) r = row i0, c = column j0 / M[i0][j0];  (b) r = row i0 / M[i0][j0], c = column j0
        for (int j = 0; j < sx; ++j) s.rf[j] = M[i0 * sx + j];
        for (int i = 0; i < sy; ++i) s.cf[i] = M[i * sx + j0] / M[i0 * sx + j0];
        if (verify_f32(M, sx, sy, s.cf, s.rf)) return true;
        for (int j = 0; j < sx; ++j) s.rf[j] = M[i0 * sx + j] / M[i0 * sx + j0];
        for (int i = 0; i < sy; ++i) s.cf[i] = M[i * sx + j0];
        return verify_f32(M, sx, sy, s.cf, s.rf);
    }
    const int32_t *M = p.m.i;
    int64_t g = 0;
    for (int j = 0; j < sx; ++j) g = gcd64(g, M[i0 * sx + j]);
    for (int j = 0; j < sx; ++j) s.ri[j] = (int32_t)(M[i0 * sx + j] / g);
    const int64_t rj0 = s.ri[j0];
    for (int i = 0; i < sy; ++i) {
        if (M[i * sx + j0] % rj0) return false;
        s.ci[i] = (int32_t)(M[i * sx + j0] / rj0);
    }
    for (int i = 0; i < sy; ++i)
        for (int j = 0; j < sx; ++j)
            if ((int64_t)s.ci[i] * s.ri[j] != (int64_t)M[i * sx + j]) return false;
    // partial sums must stay exact in int32 (255 * sum|r| * sum|c|)
    int64_t lr = 0, lc = 0;
    for (int j = 0; j < sx; ++j) lr += s.ri[j] < 0 ? -(int64_t)s.ri[j] : s.ri[j];
    for (int i = 0; i < sy; ++i) lc += s.ci[i] < 0 ? -(int64_t)s.ci[i] : s.ci[i];
    return 255 * lr * lc + (1ll << 30) < (1ll << 31);
}

template <typename T, typename TO, int R, int SWAR, int TS, int NBUF>
cudaError_t launch_cfg(const ConvSep &s, cudaStream_t stream)
{
    using S = TileShape<T>;
    size_t smem = (size_t)NBUF * (TS + 2 * R) * S::ROW_BYTES;
    // LOP_CONV_SMEM_PAD (exploration): extra dynamic shared memory per CTA, which caps
    // the co-resident CTAs (more, staggered waves instead of one lock-step wave)
    if (const char *env = std::getenv("LOP_CONV_SMEM_PAD")) smem += (size_t)std::max(0, std::atoi(env));
    static PerDevice smem_set, resident;
    cudaError_t e;
    int64_t grid_max = resident_ctas(conv_sep_kernel<T, TO, R, SWAR, TS, NBUF>, convt::NT, smem,
                                     smem_set, resident, e);
    if (e != cudaSuccess) return e;
    e = ensure_smem(conv_sep_kernel<T, TO, R, SWAR, TS, NBUF>, smem, smem_set);
    if (e != cudaSuccess) return e;
    // persistent (NBUF = 2) grid: LOP_CONV_CTAS_PER_SM caps the resident CTAs so
    // that each walks several tiles (otherwise a 4096^2 u8 image -- 1024 tiles --
    // fits in one wave and the double buffer never pipelines)
    if (const char *env = std::getenv("LOP_CONV_CTAS_PER_SM")) {
        int sms = 0;
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, current_device());
        const int cap = std::atoi(env);
        if (cap > 0 && (int64_t)sms * cap < grid_max) grid_max = (int64_t)sms * cap;
    }
    const long ntiles = (long)((s.c.roi_w + S::TWE - 1) / S::TWE) * ((s.c.roi_h + TS - 1) / TS) *
                        s.c.batch;
    dim3 grid;
    if (NBUF == 1)
        grid = dim3((s.c.roi_w + S::TWE - 1) / S::TWE, (s.c.roi_h + TS - 1) / TS, s.c.batch);
    else
        grid = dim3((unsigned)(ntiles < grid_max ? ntiles : grid_max));
    conv_sep_kernel<T, TO, R, SWAR, TS, NBUF><<<grid, convt::NT, smem, stream>>>(s);
    return cudaGetLastError();
}

// Tile configuration: (TS, NBUF) from LOP_CONV_CFG="TS:NBUF" (tuning sweep),
// else the default measured best on B200.  The sweep space is
// instantiated for radii 1 and 2 (Sobel 3x3, Gaussian 5x5); other radii use
// the default.
// f32 / other: 8 rows per tile (round 1); 4 rows for radii <= 2 (f32 Gaussian 5x5 23.8 -> 22.4 us
// at 4096^2 once the full-tile instances dropped the per-row checks, tools/time_conv_all.py)
constexpr int kDefTS = 8, kDefTSSmallR = 4, kDefTSSwar = 16, kDefNBUF = 1;
// u8 -> i32 (Sobel): 4 rows per tile -- a 4096^2 image is then 4096 tiles (~2 waves), so
// CTAs in their store phase overlap CTAs in their load phase (0.0180 vs 0.0192 ms at 8
// rows; profiles/r01_tune_conv.jsonl)
constexpr int kDefTSI32 = 4;

template <typename T, typename TO, int R, int SWAR = 0>
cudaError_t launch_sep(const ConvSep &s, cudaStream_t stream)
{
    int ts = SWAR ? kDefTSSwar : (sizeof(T) == 1 && sizeof(TO) == 4 ? kDefTSI32 : (R <= 2 ? kDefTSSmallR : kDefTS));
    int nbuf = kDefNBUF;
    if (const char *env = std::getenv("LOP_CONV_CFG")) std::sscanf(env, "%d:%d", &ts, &nbuf);
    if constexpr (R == 1 || R == 2) {
        if (ts == 4 && nbuf == 1) return launch_cfg<T, TO, R, SWAR, 4, 1>(s, stream);
        if (ts == 16 && nbuf == 1) return launch_cfg<T, TO, R, SWAR, 16, 1>(s, stream);
        if (ts == 8 && nbuf == 2) return launch_cfg<T, TO, R, SWAR, 8, 2>(s, stream);
        if (ts == 16 && nbuf == 2) return launch_cfg<T, TO, R, SWAR, 16, 2>(s, stream);
        if (ts == 32 && nbuf == 1) return launch_cfg<T, TO, R, SWAR, 32, 1>(s, stream);
        if (ts == 32 && nbuf == 2) return launch_cfg<T, TO, R, SWAR, 32, 2>(s, stream);
    }
    return launch_cfg<T, TO, R, SWAR, kDefTS, kDefNBUF>(s, stream);
}

template <typename T, typename TO>
cudaError_t dispatch_r(const ConvSep &s, cudaStream_t stream)
{
    switch (s.c.rx) {
    case 0: return launch_sep<T, TO, 0>(s, stream);
    case 1: return launch_sep<T, TO, 1>(s, stream);
    case 2: return launch_sep<T, TO, 2>(s, stream);
    case 3: return launch_sep<T, TO, 3>(s, stream);
    case 4: return launch_sep<T, TO, 4>(s, stream);
    default: return cudaErrorNotSupported;
    }
}

// SWAR eligibility (u8 -> u8): non-negative factors, sum fits a 16-bit lane,
// no saturation (sum r * sum c <= 2^shift) and the lane shift stays in-lane.
// Signed SWAR eligibility (u8 -> i32) and its lane biases: row sums biased by
// 255 * sum of the negative row factors, column sums by max_h * sum of the
// negative column factors; both lanes' final values must stay below 2^16.
bool swar_i32_prepare(ConvSep &s)
{
    // opt-in (LOP_CONV_SWAR_I32=1): measured slower than the unpacked kernel for the
    // Sobel u8 -> i32 on B200 (22.5 vs 19.3 us at 4096^2) -- the i32
    // stores and the lane extraction dominate, not the multiply-adds
    const char *on = std::getenv("LOP_CONV_SWAR_I32");
    if (!on || std::atoi(on) != 1) return false;
    if (s.kind != CONV_U8_I32 || s.c.rx < 1 || s.c.rx > 3) return false;
    int64_t rneg = 0, rpos = 0, cneg = 0, cpos = 0, csum = 0;
    for (int t = 0; t <= 2 * s.c.rx; ++t) {
        (s.ri[t] < 0 ? rneg : rpos) += s.ri[t] < 0 ? -(int64_t)s.ri[t] : s.ri[t];
        (s.ci[t] < 0 ? cneg : cpos) += s.ci[t] < 0 ? -(int64_t)s.ci[t] : s.ci[t];
        csum += s.ci[t];
    }
    const int64_t bias_h = 255 * rneg, max_h = bias_h + 255 * rpos;
    const int64_t bias_v = max_h * cneg, max_v = bias_v + max_h * cpos;
    if (max_h > 65535 || max_v > 65535) return false;
    s.sw_bias_h = (int32_t)bias_h;
    s.sw_bias_v = (int32_t)bias_v;
    s.sw_off = (int32_t)(bias_v + bias_h * csum);
    return true;
}

bool swar_ok(const ConvSep &s)
{
    if (s.kind != CONV_U8_U8 || s.c.rx < 1 || s.c.rx > 3 || s.shift > 8) return false;
    int64_t lr = 0, lc = 0;
    for (int t = 0; t <= 2 * s.c.rx; ++t) {
        if (s.ri[t] < 0 || s.ci[t] < 0) return false;
        lr += s.ri[t];
        lc += s.ci[t];
    }
    const int64_t rnd = s.shift > 0 ? (1ll << (s.shift - 1)) : 0;
    return lr * lc <= (1ll << s.shift) && 255 * lr * lc + rnd < 65536;
}

// SWAR variant (conv_u8_swar): palindromic factors with shift 8 (the 5x5
// binomial) take SW_SYM | SW_SH8; everything else the plain variant.  Measured
// on B200 (profiles/r01_session4/u8_swar_ab.txt): SYM|SH8 is 3.6 % faster than
// plain for the 5x5 Gaussian, while SYM alone is 14 % slower than plain for the
// 3x3 one (the compiler moves the pre-adds onto the FMA pipe as IMAD.IADD).
// LOP_CONV_SWAR=1 forces the plain variant (A/B, parity).
int swar_mode(const ConvSep &s)
{
    if (const char *env = std::getenv("LOP_CONV_SWAR"))
        if (std::atoi(env) == 1) return SW_ON;
    const int n = 2 * s.c.rx;
    bool sym = true;
    for (int t = 0; t <= n; ++t) sym = sym && s.ri[t] == s.ri[n - t] && s.ci[t] == s.ci[n - t];
    if (!(sym && s.shift == 8)) return SW_ON;
    bool bin5 = s.c.rx == 2;
    const int b5[5] = {1, 4, 6, 4, 1};
    for (int t = 0; t < 5 && bin5; ++t) bin5 = s.ri[t] == b5[t] && s.ci[t] == b5[t];
    if (const char *env = std::getenv("LOP_CONV_SWAR"))
        if (std::atoi(env) == 7) bin5 = false;                      // runtime-coefficient variant
    return bin5 ? (SW_ON | SW_SYM | SW_SH8 | SW_BIN5) : (SW_ON | SW_SYM | SW_SH8);
}

// u8 Gaussian 5x5 (SW_BIN5), 16 pixels per thread: the SWAR arithmetic of
// conv_u8_swar<2, ., BIN5> (same integer operations per pixel, so the same
// bytes) on four staged words per thread and row instead of two, which halves
// the per-pixel share of the halo words, their unpacking and the per-warp
// set-up.  A CTA (128 threads) owns 2048 columns x TS16 rows.
namespace conv16 {
constexpr int NT = 128, PX = 16, TWE = NT * PX, PADE = 16, SWE = TWE + 2 * PADE;
}

template <int TS, bool FULL, bool VEC>
__device__ __forceinline__ void conv_u8_bin5_x16_rows(const uint8_t *tcol, int srows, char *orow, int64_t ostride,
                                                      int ox0, int roi_x1, bool ovec)
{
    constexpr int SWE = conv16::SWE, R = 2;
    constexpr uint32_t rnd = 0x00800080u;                       // 2^7 per lane (shift 8)
    uint32_t h[2 * R + 1][8];                                   // lanes (q, q+2), q in J
    constexpr int J[8] = {0, 1, 4, 5, 8, 9, 12, 13};
#pragma unroll
    for (int k = 0; k < TS + 2 * R; ++k) {
        if (!FULL && k >= srows) break;
        const uint8_t *rp = tcol + k * SWE;
        const uint4 cv = *reinterpret_cast<const uint4 *>(rp);
        const uint32_t W[6] = {*reinterpret_cast<const uint32_t *>(rp - 4), cv.x, cv.y, cv.z, cv.w,
                               *reinterpret_cast<const uint32_t *>(rp + 16)};
        uint32_t E[6], O[6];
#pragma unroll
        for (int i = 0; i < 6; ++i) {
            E[i] = __byte_perm(W[i], 0u, 0x4240);                // bytes 0, 2 -> lanes
            O[i] = __byte_perm(W[i], 0u, 0x4341);                // bytes 1, 3 -> lanes
        }
        uint32_t S[14 + 2 * R];                                 // S[q + R] = lanes (q, q+2), q in [-R, 13+R]
#pragma unroll
        for (int q = -R; q <= 13 + R; ++q) {
            const int wi = (q + 4) >> 2, sh = (q + 4) & 3;
            if (sh == 0) S[q + R] = E[wi];
            else if (sh == 1) S[q + R] = O[wi];
            else if (sh == 2) S[q + R] = __byte_perm(E[wi], E[wi + 1], 0x5412);
            else S[q + R] = __byte_perm(O[wi], O[wi + 1], 0x5412);
        }
        uint32_t *hk = h[k % (2 * R + 1)];
#pragma unroll
        for (int jj = 0; jj < 8; ++jj) {
            const uint32_t *x = S + J[jj];
            hk[jj] = (x[0] + x[4]) + ((x[1] + x[3]) << 2) + 6u * x[2];
        }
        const int o = k - 2 * R;
        if (o < 0) continue;
        uint32_t q8[8];
#pragma unroll
        for (int jj = 0; jj < 8; ++jj) {
            const uint32_t h0 = h[o % 5][jj], h1 = h[(o + 1) % 5][jj], h2 = h[(o + 2) % 5][jj],
                           h3 = h[(o + 3) % 5][jj], h4 = h[(o + 4) % 5][jj];
            q8[jj] = (h0 + h4 + rnd) + ((h1 + h3) << 2) + 6u * h2;
        }
        const uint4 outw = make_uint4(__byte_perm(q8[0], q8[1], 0x7351), __byte_perm(q8[2], q8[3], 0x7351),
                                      __byte_perm(q8[4], q8[5], 0x7351), __byte_perm(q8[6], q8[7], 0x7351));
        uint8_t *op = reinterpret_cast<uint8_t *>(orow) + ox0;      // output row o (running pointer)
        orow += ostride;
        if (VEC || ovec) {
            *reinterpret_cast<uint4 *>(op) = outw;
        } else {
            const uint32_t w4[4] = {outw.x, outw.y, outw.z, outw.w};
#pragma unroll
            for (int j = 0; j < 16; ++j)
                if (ox0 + j < roi_x1) op[j] = (uint8_t)(w4[j >> 2] >> (8 * (j & 3)));
        }
    }
}

template <int TS>
__global__ void __launch_bounds__(conv16::NT) conv_u8_bin5_x16_kernel(const __grid_constant__ ConvSep p)
{
    constexpr int R = 2, SWE = conv16::SWE;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    __shared__ __align__(8) uint64_t bar;
    uint8_t *tile = smem_raw;
    const Common &c = p.c;
    const int b = blockIdx.z;
    const int tx0 = c.roi_x0 + (int)blockIdx.x * conv16::TWE, ty0 = c.roi_y0 + (int)blockIdx.y * TS;
    const int nrows = min(TS, c.roi_y0 + c.roi_h - ty0), srows = nrows + 2 * R;
    const int roi_x1 = c.roi_x0 + c.roi_w;
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared.b64 [%0], 1;" ::"r"(smem_addr(&bar)));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    stage_rows<uint8_t, SWE, conv16::NT>(c, b, tx0 + c.off_x - conv16::PADE, ty0 + c.off_y - R, srows, tile, &bar);
    __syncthreads();
    mbar_wait(&bar, 0);
    const int ox0 = tx0 + threadIdx.x * conv16::PX;
    if (ox0 >= roi_x1) return;
    char *obase = c.out.data + (int64_t)b * c.out.bstride;
    const bool ovec = ox0 + conv16::PX <= roi_x1 && (ox0 % 16) == 0 &&
                      ((reinterpret_cast<uintptr_t>(obase) | (uintptr_t)c.out.stride) % 16) == 0;
    const bool cta_vec = tx0 + conv16::TWE <= roi_x1 && (tx0 % 16) == 0 &&
                         ((reinterpret_cast<uintptr_t>(obase) | (uintptr_t)c.out.stride) % 16) == 0;
    const uint8_t *tcol = tile + conv16::PADE + threadIdx.x * conv16::PX;
    char *orow = obase + (int64_t)ty0 * c.out.stride;
    if (nrows == TS && cta_vec)
        conv_u8_bin5_x16_rows<TS, true, true>(tcol, srows, orow, c.out.stride, ox0, roi_x1, ovec);
    else if (nrows == TS)
        conv_u8_bin5_x16_rows<TS, true, false>(tcol, srows, orow, c.out.stride, ox0, roi_x1, ovec);
    else
        conv_u8_bin5_x16_rows<TS, false, false>(tcol, srows, orow, c.out.stride, ox0, roi_x1, ovec);
}

template <int TS>
cudaError_t launch_bin5_x16(const ConvSep &s, cudaStream_t stream)
{
    const size_t smem = (size_t)(TS + 4) * conv16::SWE;
    static PerDevice smem_set;
    cudaError_t e = ensure_smem(conv_u8_bin5_x16_kernel<TS>, smem, smem_set);
    if (e != cudaSuccess) return e;
    dim3 grid((s.c.roi_w + conv16::TWE - 1) / conv16::TWE, (s.c.roi_h + TS - 1) / TS, s.c.batch);
    conv_u8_bin5_x16_kernel<TS><<<grid, conv16::NT, smem, stream>>>(s);
    return cudaGetLastError();
}

// LOP_CONV_X16: 0 = the 8-pixel kernel; 4 / 8 / 16 = the 16-pixel kernel with that many rows
// per tile.  4096^2 (tools/time_conv_all.py): 8-pixel kernel 11.15 us; 16 pixels x 4 / 8 / 16
// rows 11.6 / 10.8 / 11.6 us -- 8 rows (1024 CTAs) is the default.
static int bin5_x16_rows()
{
    static const int v = [] {
        const char *env = std::getenv("LOP_CONV_X16");
        return env ? std::atoi(env) : 8;
    }();
    return v;
}

template <int R>
cudaError_t dispatch_swar_r(const ConvSep &s, cudaStream_t stream)
{
    const int mode = swar_mode(s);
    if constexpr (R == 2) {
        if (mode == (SW_ON | SW_SYM | SW_SH8 | SW_BIN5)) {
            if (!std::getenv("LOP_CONV_CFG")) {                 // (a tile-config sweep keeps the 8-px kernel)
                if (bin5_x16_rows() == 16) return launch_bin5_x16<16>(s, stream);
                if (bin5_x16_rows() == 8) return launch_bin5_x16<8>(s, stream);
                if (bin5_x16_rows() == 4) return launch_bin5_x16<4>(s, stream);
            }
            return launch_sep<uint8_t, uint8_t, R, SW_ON | SW_SYM | SW_SH8 | SW_BIN5>(s, stream);
        }
    }
    if (mode & SW_SH8)
        return launch_sep<uint8_t, uint8_t, R, SW_ON | SW_SYM | SW_SH8>(s, stream);
    return launch_sep<uint8_t, uint8_t, R, SW_ON>(s, stream);
}

cudaError_t dispatch_swar_i32(const ConvSep &s, cudaStream_t stream)
{
    switch (s.c.rx) {
    case 1: return launch_sep<uint8_t, int32_t, 1, SW_ON | SW_I32>(s, stream);
    case 2: return launch_sep<uint8_t, int32_t, 2, SW_ON | SW_I32>(s, stream);
    case 3: return launch_sep<uint8_t, int32_t, 3, SW_ON | SW_I32>(s, stream);
    default: return cudaErrorNotSupported;
    }
}

cudaError_t dispatch_swar(const ConvSep &s, cudaStream_t stream)
{
    switch (s.c.rx) {
    case 1: return dispatch_swar_r<1>(s, stream);
    case 2: return dispatch_swar_r<2>(s, stream);
    case 3: return dispatch_swar_r<3>(s, stream);
    default: return cudaErrorNotSupported;
    }
}

}  // namespace

bool conv_factor(const ConvGeneric &p, ConvSep &s) { return factor(p, s); }

bool conv_tiled_supported(const ConvGeneric &p)
{
    if (p.c.rx != p.c.ry || p.c.rx > 4) return false;
    static thread_local ConvSep s;
    return factor(p, s);
}

cudaError_t launch_conv_tiled(const ConvGeneric &p, cudaStream_t stream)
{
    static thread_local ConvSep s;
    if (p.c.rx != p.c.ry || p.c.rx > 4 || !factor(p, s)) return cudaErrorNotSupported;
    s.c = p.c;
    s.kind = p.kind;
    s.shift = p.shift;
    switch (p.kind) {
    case CONV_F32: return dispatch_r<float, float>(s, stream);
    case CONV_U8_U8:
        return swar_ok(s) ? dispatch_swar(s, stream) : dispatch_r<uint8_t, uint8_t>(s, stream);
    case CONV_U8_I32:
        return swar_i32_prepare(s) ? dispatch_swar_i32(s, stream) : dispatch_r<uint8_t, int32_t>(s, stream);
    default: return cudaErrorNotSupported;
    }
}

}  // namespace lop

// boundary.cuh -- boundary handling by index adjustment (PAPER.md L340-L357,
// Table I, Fig. 2) and the per-tap arithmetic shared by
// every kernel variant, so that the generic and tiled kernels produce
// bit-identical outputs (the same instruction sequence per tap, in the same
// yf-major / xf-minor order as Algorithm 1).
#pragma once
#include <stdint.h>

#include "lop_params.h"

namespace lop {

enum { M_UNDEFINED = 0, M_CLAMP = 1, M_REPEAT = 2, M_MIRROR = 3, M_CONSTANT = 4 };

// Per-axis index adjustment of i into [0, n).  UNDEFINED is served as CLAMP
// so that the kernels never read outside the image (reading c9).
__device__ __forceinline__ int map_axis(int i, int n, int mode)
{
    if ((unsigned)i < (unsigned)n) return i;
    if (mode == M_REPEAT) {
        int q = i % n;
        return q < 0 ? q + n : q;
    }
    if (mode == M_MIRROR) {
        int period = 2 * n;
        int q = i % period;
        if (q < 0) q += period;
        return q < n ? q : period - 1 - q;
    }
    return i < 0 ? 0 : n - 1;
}

// Resolve a band-local input row iy (global row iy + gy0) to the band-local
// row that is physically read; returns false for a CONSTANT read.
//  * rows inside the global image are read where they are stored (own rows
//    or halo rows, which the host validated to be present);
//  * out-of-image rows under REPEAT that are physically present are a ring
//    halo supplied by the neighbour band: read as stored;
//  * otherwise the global row is adjusted per mode (Table I).
__device__ __forceinline__ bool resolve_row(int iy, const Geom &g, int mode, int &row)
{
    const int gy = iy + g.gy0;
    if ((unsigned)gy < (unsigned)g.GH) { row = iy; return true; }
    if (mode == M_CONSTANT) return false;
    if (mode == M_REPEAT && iy >= -g.halo_top && iy < g.H + g.halo_bottom) { row = iy; return true; }
    row = map_axis(gy, g.GH, mode) - g.gy0;
    return true;
}

__device__ __forceinline__ bool resolve_col(int ix, const Geom &g, int mode, int &col)
{
    if ((unsigned)ix < (unsigned)g.W) { col = ix; return true; }
    if (mode == M_CONSTANT) return false;
    col = map_axis(ix, g.W, mode);
    return true;
}

template <typename T>
__device__ __forceinline__ const T *row_ptr(const Geom &g, int b, int row)
{
    return reinterpret_cast<const T *>(g.data + (int64_t)b * g.bstride + (int64_t)row * g.stride);
}

// Read(ix, iy) of frame b with boundary handling (generic, per tap).
__device__ __forceinline__ float read_f32(const Geom &g, int b, int ix, int iy, int mode, float cval)
{
    int row, col;
    if (!resolve_row(iy, g, mode, row) || !resolve_col(ix, g, mode, col)) return cval;
    return __ldg(row_ptr<float>(g, b, row) + col);
}

__device__ __forceinline__ int read_u8(const Geom &g, int b, int ix, int iy, int mode, int cval)
{
    int row, col;
    if (!resolve_row(iy, g, mode, row) || !resolve_col(ix, g, mode, col)) return cval;
    return (int)__ldg(row_ptr<uint8_t>(g, b, row) + col);
}

__device__ __forceinline__ uint32_t smem_addr(const void *p)
{
    return (uint32_t)__cvta_generic_to_shared(p);
}

// Wait for phase `parity` of an mbarrier (try_wait loop; hardware sleep).
// LOP_MBAR_SUSPEND_NS: a suspend-time hint for try_wait (the thread sleeps up
// to that long unless the phase completes first), so waiting warps do not
// spin on the issue slots of the warps that are computing; 0 = no hint.
#ifndef LOP_MBAR_SUSPEND_NS
#define LOP_MBAR_SUSPEND_NS 0
#endif
__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity)
{
#if LOP_MBAR_SUSPEND_NS > 0
    asm volatile(
        "{\n\t.reg .pred P;\n"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared.b64 P, [%0], %1, %2;\n\t"
        "@!P bra WAIT_%=;\n}" ::"r"(smem_addr(bar)), "r"(parity), "n"(LOP_MBAR_SUSPEND_NS) : "memory");
#else
    asm volatile(
        "{\n\t.reg .pred P;\n"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared.b64 P, [%0], %1;\n\t"
        "@!P bra WAIT_%=;\n}" ::"r"(smem_addr(bar)), "r"(parity) : "memory");
#endif
}

__device__ __forceinline__ float ex2_approx(float x)
{
    float y;
    asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}

// One bilateral tap (Alg. 1 lines 8-11 / Listing 5 l.7-12) in the log2 domain:
//   w = c(xf,yf) * exp(-(v - centre)^2 / (2 sigma_r^2))
//     = ex2(lc + nk * (v - centre)^2),  lc = log2 c,  nk = -log2(e)/(2 sigma_r^2)
//   d += w;  p += w * v
// Explicit _rn intrinsics: never contracted or reassociated by the compiler.
// SCALED: v, centre are alpha * I (see bilateral_weight below): exponent
// lc - (v - centre)^2 without the FMUL by nk.
template <bool SCALED = false>
__device__ __forceinline__ void bilateral_tap(float v, float centre, float lc, float nk,
                                              float &d, float &p)
{
    const float diff = __fsub_rn(v, centre);
    float e;
    if (SCALED) {
        e = __fmaf_rn(-diff, diff, lc);
    } else {
        const float t = __fmul_rn(diff, diff);
        e = __fmaf_rn(t, nk, lc);
    }
    const float w = ex2_approx(e);
    d = __fadd_rn(d, w);
    p = __fmaf_rn(w, v, p);
}

// 2^x on the FMA pipe (Cody-Waite split + degree-5 polynomial), used for a
// fixed subset of taps to offload the MUFU (SFU) pipe, which bounds the
// bilateral kernel.  x <= 0 here (log2 of a product of weights <= 1); values
// below -126 return 2^-126 (weights that small are below f32 resolution of the
// sums).  Relative error <= 2.1e-7 in f32 (ex2.approx: <= 2^-22 ~ 2.4e-7).
__device__ __forceinline__ float ex2_poly(float x)
{
    x = fmaxf(x, -126.0f);
    const float t = __fadd_rn(x, 12582912.0f);          // 1.5 * 2^23: j = round(x) in the low bits
    const float j = __fsub_rn(t, 12582912.0f);
    const float f = __fsub_rn(x, j);                    // f in [-0.5, 0.5]
    float p = __fmaf_rn(1.3277444522827864e-3f, f, 9.675883688032627e-3f);
    p = __fmaf_rn(p, f, 5.550713092088699e-2f);
    p = __fmaf_rn(p, f, 2.4022112786769867e-1f);
    p = __fmaf_rn(p, f, 6.931469440460205e-1f);
    p = __fmaf_rn(p, f, 1.0000001192092896f);
    return __int_as_float(__float_as_int(p) + (__float_as_int(t) << 23));   // p * 2^j
}

// Separable-closeness form (Eq. 1 is a product of two 1D Gaussians, Listing 1
// l.21): c(xf,yf) = cy[yf] * 2^lx[xf].  Per window row the taps accumulate
//   rd = sum_xf w',  rp = sum_xf w' v,   w' = ex2(lx[xf] + nk * (v - centre)^2)
// (first tap initialises), then the row is folded in with one FFMA each:
//   d += cy[yf] * rd,  p += cy[yf] * rp.
// Same operation count per tap as bilateral_tap, no per-tap mask operand from
// shared memory, and per-row partial sums (better accuracy).
// SCALED = scaled-difference form: v and centre are alpha * I with
// alpha^2 = log2(e) / (2 sigma_r^2), so the exponent is lx - (v - centre)^2
// (one FFMA with a negated operand, no FMUL); p then accumulates alpha * I and
// the result is divided by alpha at the end (bilateral_finish_scaled).
template <bool POLY = false, bool SCALED = false>
__device__ __forceinline__ float bilateral_weight(float v, float centre, float lx, float nk)
{
    const float diff = __fsub_rn(v, centre);
    float e;
    if (SCALED) {
        e = __fmaf_rn(-diff, diff, lx);
    } else {
        const float t = __fmul_rn(diff, diff);
        e = __fmaf_rn(t, nk, lx);
    }
    return POLY ? ex2_poly(e) : ex2_approx(e);
}

template <bool POLY = false, bool SCALED = false>
__device__ __forceinline__ void bilateral_row_first(float v, float centre, float lx, float nk,
                                                    float &rd, float &rp)
{
    const float w = bilateral_weight<POLY, SCALED>(v, centre, lx, nk);
    rd = w;
    rp = __fmul_rn(w, v);
}

template <bool POLY = false, bool SCALED = false>
__device__ __forceinline__ void bilateral_row_tap(float v, float centre, float lx, float nk,
                                                  float &rd, float &rp)
{
    const float w = bilateral_weight<POLY, SCALED>(v, centre, lx, nk);
    rd = __fadd_rn(rd, w);
    rp = __fmaf_rn(w, v, rp);
}

__device__ __forceinline__ float bilateral_finish_scaled(float d, float p, float inv_alpha)
{
    return __fmul_rn(__fdiv_rn(p, d), inv_alpha);
}

__device__ __forceinline__ void bilateral_row_fold(float cy, float rd, float rp, float &d, float &p)
{
    d = __fmaf_rn(cy, rd, d);
    p = __fmaf_rn(cy, rp, p);
}

__device__ __forceinline__ float bilateral_finish(float d, float p)
{
    return __fdiv_rn(p, d);   // Alg. 1 line 14: output = p / k
}

// Integer output quantisation (reading c12): (S + 2^(k-1)) >> k, arithmetic.
__device__ __forceinline__ int quantize_shift(int s, int shift)
{
    return shift > 0 ? (s + (1 << (shift - 1))) >> shift : s;
}

}  // namespace lop

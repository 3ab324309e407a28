// conv_stream.cu -- register-streaming separable convolution (no shared memory).
//
// Each warp owns a column strip of 32 lanes x PX columns (f32: PX = 4, one
// 16-B load per lane and row; u8: PX = 16, one 16-B load per lane and row) and
// streams S output rows down the image:
//   * input rows are loaded straight from global memory with LDG.128 and kept
//     in a register queue P = 2R+1 rows deep (the next P rows are in flight
//     while the current ones are filtered);
//   * the horizontal halo comes from the neighbouring lanes by warp shuffle
//     (lanes 0 and 31 load the 16 B beyond the strip themselves);
//   * horizontal pass -> register ring of 2R+1 row sums -> vertical pass ->
//     one vector store per lane and output row (the arithmetic of
//     conv_sep_kernel, so the result is bit-identical to the tiled kernel);
//   * u8 -> u8 with non-negative factors uses SWAR (two exact 16-bit lanes per
//     register) like the tiled kernel.
// Warps whose strip touches the image border in x, or whose rows are not
// 16-B aligned, take a per-element path with the boundary resolved per pixel.
// Rows are resolved per row (uniform across the warp).  Compared with the
// tiled kernel: every input row is read once per strip (S + 2R rows for S
// outputs instead of TS + 2R per TS), no staging barrier, no smem traffic.
#include <cuda_runtime.h>
#include <stdint.h>

#include <cstdlib>
#include <type_traits>

#include "boundary.cuh"
#include "kernels.h"
#include "lop_params.h"

namespace lop {

namespace cstream {
constexpr int NW = 4;                 // warps per CTA (side by side)
constexpr int NT = 32 * NW;
}  // namespace cstream

template <typename T> struct SPx;
template <> struct SPx<float> { static constexpr int N = 4; };
template <> struct SPx<uint8_t> { static constexpr int N = 16; };

// One lane's raw row: the 16-B centre vector + (lanes 0 / 31) the 16 B to the
// left / right of the strip.
struct RawRow {
    uint4 cen;
    uint4 ext;
};

// Full row window of one lane: f32 -> 4 left, PX centre, 4 right floats;
// u8 -> 1 left word, 4 centre words, 1 right word.
template <typename T> struct RowWin;
template <> struct RowWin<float> { float v[12]; };
template <> struct RowWin<uint8_t> { uint32_t w[6]; };

__device__ __forceinline__ uint4 ldg16(const void *p)
{
    return __ldg(reinterpret_cast<const uint4 *>(p));
}

// Assemble the window from raw rows: shuffles give the neighbours' edges.
template <typename T>
__device__ __forceinline__ void assemble(const RawRow &r, int lane, RowWin<T> &win)
{
    if constexpr (sizeof(T) == 4) {
        const float c[4] = {__uint_as_float(r.cen.x), __uint_as_float(r.cen.y),
                            __uint_as_float(r.cen.z), __uint_as_float(r.cen.w)};
        const float e[4] = {__uint_as_float(r.ext.x), __uint_as_float(r.ext.y),
                            __uint_as_float(r.ext.z), __uint_as_float(r.ext.w)};
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            const float l = __shfl_up_sync(0xffffffffu, c[k], 1);
            const float rr = __shfl_down_sync(0xffffffffu, c[k], 1);
            win.v[k] = lane == 0 ? e[k] : l;
            win.v[4 + k] = c[k];
            win.v[8 + k] = lane == 31 ? e[k] : rr;
        }
    } else {
        const uint32_t l = __shfl_up_sync(0xffffffffu, r.cen.w, 1);
        const uint32_t rr = __shfl_down_sync(0xffffffffu, r.cen.x, 1);
        win.w[0] = lane == 0 ? r.ext.w : l;
        win.w[1] = r.cen.x;
        win.w[2] = r.cen.y;
        win.w[3] = r.cen.z;
        win.w[4] = r.cen.w;
        win.w[5] = lane == 31 ? r.ext.x : rr;
    }
}

// Per-element window for edge strips: every value through the boundary condition.
template <typename T>
__device__ __forceinline__ void load_slow(const Common &c, int b, int ix0, int iy, RowWin<T> &win)
{
    const Geom &g = c.in;
    int row;
    const bool row_ok = resolve_row(iy, g, c.mode, row);
    if constexpr (sizeof(T) == 4) {
        const float *rp = row_ok ? row_ptr<float>(g, b, row) : nullptr;
#pragma unroll
        for (int k = 0; k < 12; ++k) {
            int col;
            win.v[k] = (row_ok && resolve_col(ix0 - 4 + k, g, c.mode, col)) ? __ldg(rp + col)
                                                                           : c.cval_f;
        }
    } else {
        const uint8_t *rp = row_ok ? row_ptr<uint8_t>(g, b, row) : nullptr;
#pragma unroll
        for (int w = 0; w < 6; ++w) {
            uint32_t word = 0;
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                int col;
                const uint32_t byte = (row_ok && resolve_col(ix0 - 4 + 4 * w + k, g, c.mode, col))
                                          ? (uint32_t)__ldg(rp + col)
                                          : (uint32_t)c.cval_i;
                word |= byte << (8 * k);
            }
            win.w[w] = word;
        }
    }
}

// Fast-path raw load of input row iy (lane's centre + strip-edge extras).
template <typename T>
__device__ __forceinline__ void load_fast(const Common &c, int b, int ix0, int iy, int lane,
                                          RawRow &r)
{
    const Geom &g = c.in;
    int row;
    if (!resolve_row(iy, g, c.mode, row)) {           // CONSTANT row
        uint32_t cv;
        if constexpr (sizeof(T) == 4) cv = __float_as_uint(c.cval_f);
        else cv = (uint32_t)c.cval_i * 0x01010101u;
        r.cen = make_uint4(cv, cv, cv, cv);
        r.ext = r.cen;
        return;
    }
    const char *rp = reinterpret_cast<const char *>(row_ptr<T>(g, b, row)) + (int64_t)ix0 * sizeof(T);
    r.cen = ldg16(rp);
    if (lane == 0) r.ext = ldg16(rp - 16);
    else if (lane == 31) r.ext = ldg16(rp + 16);
}

// Horizontal pass of one row window into PX (f32) / PX/2 SWAR words or PX ints.
template <typename T, int R, bool SWAR>
struct HRow;
template <int R> struct HRow<float, R, false> { float h[4]; };
template <int R> struct HRow<uint8_t, R, true> { uint32_t h[8]; };
template <int R> struct HRow<uint8_t, R, false> { int h[16]; };

template <typename T, int R, bool SWAR>
__device__ __forceinline__ void hpass(const ConvSep &p, const RowWin<T> &win, HRow<T, R, SWAR> &o)
{
    if constexpr (sizeof(T) == 4) {
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            float s = __fmul_rn(p.rf[0], win.v[4 - R + j]);
#pragma unroll
            for (int t = 1; t <= 2 * R; ++t) s = __fmaf_rn(p.rf[t], win.v[4 - R + j + t], s);
            o.h[j] = s;
        }
    } else if constexpr (SWAR) {
        constexpr uint32_t M = 0x00FF00FFu;
        uint32_t S[14 + 2 * R];                   // S[q + R] = lanes (q, q+2), q in [-R, 13+R]
#pragma unroll
        for (int q = -R; q <= 13 + R; ++q) {
            const int wi = (q + 4) >> 2, sh = (q + 4) & 3;
            if (sh == 0) S[q + R] = __byte_perm(win.w[wi], 0u, 0x4240);
            else if (sh == 1) S[q + R] = __byte_perm(win.w[wi], 0u, 0x4341);
            else S[q + R] = __funnelshift_r(win.w[wi], win.w[wi + 1], 8 * sh) & M;
        }
        constexpr int J[8] = {0, 1, 4, 5, 8, 9, 12, 13};
#pragma unroll
        for (int jj = 0; jj < 8; ++jj) {
            uint32_t s = (uint32_t)p.ri[0] * S[J[jj]];
#pragma unroll
            for (int t = 1; t <= 2 * R; ++t) s += (uint32_t)p.ri[t] * S[J[jj] + t];
            o.h[jj] = s;
        }
    } else {
        int v[16 + 2 * R];
#pragma unroll
        for (int k = 0; k < 16 + 2 * R; ++k) {
            const int byte = 4 - R + k;                    // position in the 24-byte window
            v[k] = (int)((win.w[byte >> 2] >> (8 * (byte & 3))) & 0xFF);
        }
#pragma unroll
        for (int j = 0; j < 16; ++j) {
            int s = p.ri[0] * v[j];
#pragma unroll
            for (int t = 1; t <= 2 * R; ++t) s += p.ri[t] * v[j + t];
            o.h[j] = s;
        }
    }
}

// Vertical pass + store of output row `oy` from ring rows (oldest first).
template <typename T, typename TO, int R, bool SWAR>
__device__ __forceinline__ void vpass_store(const ConvSep &p, const HRow<T, R, SWAR> *ring[],
                                            char *orow, int ox0, int roi_x1, bool ovec)
{
    constexpr int PX = SPx<T>::N;
    if constexpr (sizeof(T) == 4) {
        float out[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            float s = __fmul_rn(p.cf[0], ring[0]->h[j]);
#pragma unroll
            for (int t = 1; t <= 2 * R; ++t) s = __fmaf_rn(p.cf[t], ring[t]->h[j], s);
            out[j] = s;
        }
        float *op = reinterpret_cast<float *>(orow) + ox0;
        if (ovec) {
            *reinterpret_cast<float4 *>(op) = make_float4(out[0], out[1], out[2], out[3]);
        } else {
            for (int j = 0; j < 4; ++j)
                if (ox0 + j < roi_x1) op[j] = out[j];
        }
    } else if constexpr (SWAR) {
        constexpr uint32_t M = 0x00FF00FFu;
        const uint32_t rnd = p.shift > 0 ? (1u << (p.shift - 1)) * 0x00010001u : 0u;
        uint32_t q[8];
#pragma unroll
        for (int jj = 0; jj < 8; ++jj) {
            uint32_t s = (uint32_t)p.ci[0] * ring[0]->h[jj] + rnd;
#pragma unroll
            for (int t = 1; t <= 2 * R; ++t) s += (uint32_t)p.ci[t] * ring[t]->h[jj];
            q[jj] = (s >> p.shift) & M;
        }
        const uint4 w = make_uint4(__byte_perm(q[0], q[1], 0x6240), __byte_perm(q[2], q[3], 0x6240),
                                   __byte_perm(q[4], q[5], 0x6240), __byte_perm(q[6], q[7], 0x6240));
        uint8_t *op = reinterpret_cast<uint8_t *>(orow) + ox0;
        if (ovec) {
            *reinterpret_cast<uint4 *>(op) = w;
        } else {
            const uint32_t ws[4] = {w.x, w.y, w.z, w.w};
            for (int j = 0; j < 16; ++j)
                if (ox0 + j < roi_x1) op[j] = (uint8_t)(ws[j >> 2] >> (8 * (j & 3)));
        }
    } else {
        int qv[PX];
#pragma unroll
        for (int j = 0; j < PX; ++j) {
            int s = p.ci[0] * ring[0]->h[j];
#pragma unroll
            for (int t = 1; t <= 2 * R; ++t) s += p.ci[t] * ring[t]->h[j];
            qv[j] = quantize_shift(s, p.shift);
        }
        if constexpr (sizeof(TO) == 1) {
            uint32_t ws[4] = {0u, 0u, 0u, 0u};
#pragma unroll
            for (int j = 0; j < 16; ++j)
                ws[j >> 2] |= (uint32_t)min(max(qv[j], 0), 255) << (8 * (j & 3));
            uint8_t *op = reinterpret_cast<uint8_t *>(orow) + ox0;
            if (ovec) {
                *reinterpret_cast<uint4 *>(op) = make_uint4(ws[0], ws[1], ws[2], ws[3]);
            } else {
                for (int j = 0; j < 16; ++j)
                    if (ox0 + j < roi_x1) op[j] = (uint8_t)(ws[j >> 2] >> (8 * (j & 3)));
            }
        } else {
            int32_t *op = reinterpret_cast<int32_t *>(orow) + ox0;
            if (ovec) {
#pragma unroll
                for (int k = 0; k < 4; ++k)
                    reinterpret_cast<int4 *>(op)[k] =
                        make_int4(qv[4 * k], qv[4 * k + 1], qv[4 * k + 2], qv[4 * k + 3]);
            } else {
                for (int j = 0; j < 16; ++j)
                    if (ox0 + j < roi_x1) op[j] = qv[j];
            }
        }
    }
}

template <typename T, typename TO, int R, bool SWAR, int S>
__global__ void __launch_bounds__(cstream::NT) conv_stream_kernel(const __grid_constant__ ConvSep p)
{
    constexpr int PX = SPx<T>::N, P = 2 * R + 1;
    static_assert(R <= 4, "halo must fit the 16-B edge vectors");
    const Common &c = p.c;
    const Geom &g = c.in;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int b = blockIdx.z;
    const int sx0 = c.roi_x0 + (blockIdx.x * cstream::NW + warp) * 32 * PX;   // strip origin
    const int roi_x1 = c.roi_x0 + c.roi_w, roi_y1 = c.roi_y0 + c.roi_h;
    if (sx0 >= roi_x1) return;
    const int oy0 = c.roi_y0 + blockIdx.y * S;
    const int nout = min(S, roi_y1 - oy0);
    const int nin = nout + 2 * R;                         // input rows streamed
    const int ox0 = sx0 + lane * PX;                      // this lane's first output column
    const int ix0 = ox0 + c.off_x;                        // ... and input column
    const int iy0 = oy0 + c.off_y - R;                    // first input row
    const int sxi = sx0 + c.off_x;                        // strip input origin
    const char *fbase = g.data + (int64_t)b * g.bstride;
    // fast path: the strip +- 16 B lies inside the image rows and is 16-B aligned
    const bool fast = sxi * (int)sizeof(T) >= 16 &&
                      (sxi + 32 * PX) * (int)sizeof(T) + 16 <= g.W * (int)sizeof(T) &&
                      ((reinterpret_cast<uintptr_t>(fbase) | (uintptr_t)g.stride |
                        (uintptr_t)(sxi * (int)sizeof(T))) % 16 == 0);
    char *obase = c.out.data + (int64_t)b * c.out.bstride;
    const bool ovec = (ox0 + PX <= roi_x1) &&
                      (((reinterpret_cast<uintptr_t>(obase) | (uintptr_t)c.out.stride |
                         (uintptr_t)(ox0 * (int)sizeof(TO))) % 16) == 0);

    HRow<T, R, SWAR> ring[P];
    RawRow q[P];                                          // in-flight input rows
    if (fast) {
#pragma unroll
        for (int i = 0; i < P; ++i)
            if (i < nin) load_fast<T>(c, b, ix0, iy0 + i, lane, q[i]);
    }
#pragma unroll 1
    for (int k0 = 0; k0 < nin; k0 += P) {
#pragma unroll
        for (int i = 0; i < P; ++i) {
            const int k = k0 + i;
            if (k >= nin) break;
            RowWin<T> win;
            if (fast) {
                assemble<T>(q[i], lane, win);
                if (k + P < nin) load_fast<T>(c, b, ix0, iy0 + k + P, lane, q[i]);
            } else {
                load_slow<T>(c, b, ix0, iy0 + k, win);
            }
            hpass<T, R, SWAR>(p, win, ring[i]);
            const int o = k - 2 * R;
            if (o < 0) continue;
            const HRow<T, R, SWAR> *rows[P];
#pragma unroll
            for (int t = 0; t < P; ++t) rows[t] = &ring[(i + 1 + t) % P];   // rows o .. k
            if (ox0 < roi_x1)
                vpass_store<T, TO, R, SWAR>(p, rows, obase + (int64_t)(oy0 + o) * c.out.stride,
                                            ox0, roi_x1, ovec);
        }
    }
}

namespace {

constexpr int kStreamRows = 32;   // output rows per strip (tools/tune_conv.py)

template <typename T, typename TO, int R, bool SWAR, int S>
cudaError_t launch_stream_s(const ConvSep &s, cudaStream_t stream)
{
    constexpr int PX = SPx<T>::N;
    const int strips = (s.c.roi_w + 32 * PX - 1) / (32 * PX);
    dim3 grid((strips + cstream::NW - 1) / cstream::NW, (s.c.roi_h + S - 1) / S, s.c.batch);
    conv_stream_kernel<T, TO, R, SWAR, S><<<grid, cstream::NT, 0, stream>>>(s);
    return cudaGetLastError();
}

template <typename T, typename TO, int R, bool SWAR>
cudaError_t launch_stream_r(const ConvSep &s, cudaStream_t stream)
{
    int rows = kStreamRows;
    if (const char *env = std::getenv("LOP_CONV_STREAM_ROWS")) rows = std::atoi(env);
    switch (rows) {
    case 16: return launch_stream_s<T, TO, R, SWAR, 16>(s, stream);
    case 64: return launch_stream_s<T, TO, R, SWAR, 64>(s, stream);
    default: return launch_stream_s<T, TO, R, SWAR, 32>(s, stream);
    }
}

template <typename T, typename TO, bool SWAR>
cudaError_t dispatch_stream(const ConvSep &s, cudaStream_t stream)
{
    switch (s.c.rx) {
    case 0: if constexpr (!SWAR) return launch_stream_r<T, TO, 0, false>(s, stream); break;
    case 1: return launch_stream_r<T, TO, 1, SWAR>(s, stream);
    case 2: return launch_stream_r<T, TO, 2, SWAR>(s, stream);
    case 3: return launch_stream_r<T, TO, 3, SWAR>(s, stream);
    case 4: if constexpr (!SWAR) return launch_stream_r<T, TO, 4, false>(s, stream); break;
    default: break;
    }
    return cudaErrorNotSupported;
}

}  // namespace

cudaError_t launch_conv_stream(const ConvSep &s, bool swar, cudaStream_t stream)
{
    switch (s.kind) {
    case CONV_F32: return dispatch_stream<float, float, false>(s, stream);
    case CONV_U8_U8:
        return swar ? dispatch_stream<uint8_t, uint8_t, true>(s, stream)
                    : dispatch_stream<uint8_t, uint8_t, false>(s, stream);
    case CONV_U8_I32: return dispatch_stream<uint8_t, int32_t, false>(s, stream);
    default: return cudaErrorNotSupported;
    }
}

}  // namespace lop

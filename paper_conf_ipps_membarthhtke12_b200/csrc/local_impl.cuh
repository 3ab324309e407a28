// local_impl.cuh -- local operator over several Accessors with a per-tap function
// (include/lop.h lop_local_execute):
//   PAPER.md L556-L558  "In case multiple Accessors are used within one
//                        kernel, the largest window size specified is taken"
//   Listing 9 L961-L964 convolve(cMask, SUM, [&] () { return cMask() *
//                        Input(cMask); }) -- a reduction over the mask's taps
//                        of a per-tap function (reading c22: a fixed set).
//   out(x, y) = op_{k, yf, xf} f(M_k(xf, yf), Read_k(x + ox_k + xf,
//                                 y + oy_k + yf), Read_k(x + ox_k, y + oy_k))
// with an optional point-operator prologue per accessor (
// reading c27): Read'_k = a_k Read_k + b_k, applied once per staged element
// (tiled kernels: in shared memory after staging, so the boundary constant is
// mapped too) or per read (generic kernel) -- the same value either way.
//
// Two kernels with the same per-output arithmetic in the same order (so the
// outputs are bit-identical, tested):
//  * local_tiled_kernel: every accessor's footprint (tile + its own window +
//    offset) is staged once into shared memory with the boundary resolved at
//    staging time (interior CTAs: unchecked loads; border CTAs: per element,
//    Table I) -- the B200 form of the paper's nine-region kernels (Fig. 3);
//    a thread computes one column x 4 rows, so consecutive lanes read
//    consecutive shared-memory words (no bank conflicts) and every staged row
//    a thread loads serves up to 4 outputs.
//  * local_generic_kernel: one thread per output, per-tap boundary resolution
//    (interior CTAs skip it).
// The CTA shape of both comes from Algorithm 2 (select.cpp): occupancy from
// cudaOccupancyMaxActiveBlocksPerMultiprocessor, then the fewest threads in
// border CTAs with y-preferred tilings.
// Summation order (SUM, f32): per accessor one FMA chain from +0 over its
// taps, window rows top to bottom and taps left to right; the accessors'
// sums added in order (FADD).  MIN / MAX: exact, taps with M != 0.
// Instantiated by local_f32.cu and local_u8.cu (two translation units, so the
// ~70 kernel instances each compile in parallel).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <climits>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <type_traits>

#include "boundary.cuh"
#include "kernels.h"
#include "launch_cache.h"
#include "lop_params.h"
#include "select.h"

namespace lop {

namespace local {
constexpr int OUT_Y = 4;                     // output rows per thread (tiled kernel)
enum { FN_PRODUCT = 0, FN_ABSDIFF = 1, FN_SQDIFF = 2, FN_SQUARE = 3 };
}  // namespace local

// g(v, c) of the per-tap function f = M * g
template <int FN>
__device__ __forceinline__ float tap_g(float v, float c)
{
    if (FN == local::FN_ABSDIFF) return fabsf(__fsub_rn(v, c));
    if (FN == local::FN_SQDIFF) { const float d = __fsub_rn(v, c); return __fmul_rn(d, d); }
    if (FN == local::FN_SQUARE) return __fmul_rn(v, v);
    return v;
}
template <int FN>
__device__ __forceinline__ int tap_g(int v, int c)
{
    if (FN == local::FN_ABSDIFF) return abs(v - c);
    if (FN == local::FN_SQDIFF) return (v - c) * (v - c);
    if (FN == local::FN_SQUARE) return v * v;
    return v;
}

// Per-output accumulator: SUM keeps (total, running accessor sum);
// MIN / MAX a running extreme initialised to the identity.
template <typename V, int OP>
struct LocalAccum {
    V total, acck, rs;
    __device__ __forceinline__ void init()
    {
        if constexpr (std::is_same<V, float>::value)
            total = OP == RED_MIN ? INFINITY : (OP == RED_MAX ? -INFINITY : 0.0f);
        else
            total = OP == RED_MIN ? INT_MAX : (OP == RED_MAX ? INT_MIN : 0);
        acck = rs = (V)0;
    }
    // tap xf of a window row (first: the row's first tap)
    template <int FN>
    __device__ __forceinline__ void tap(V M, V v, V c, bool first)
    {
        const V g = tap_g<FN>(v, c);
        if (OP == RED_SUM) {
            // every tap an FMA into the row partial sum, which starts at +0 (so the
            // first tap is M*g exactly, up to the sign of a zero product)
            if (std::is_same<V, float>::value) rs = __fmaf_rn(M, g, rs);
            else rs = rs + M * g;
        } else if (M != (V)0) {
            const V f = std::is_same<V, float>::value ? (V)__fmul_rn(M, g) : M * g;
            total = OP == RED_MIN ? min(total, f) : max(total, f);
        }
    }
    // one FMA chain per accessor over its taps (yf outer, xf inner); the
    // accessors' sums are added in order
    __device__ __forceinline__ void end_row(bool) {}
    __device__ __forceinline__ void end_accessor(bool first_acc)
    {
        if (OP == RED_SUM) {
            total = first_acc ? rs : (std::is_same<V, float>::value ? (V)__fadd_rn(total, rs) : total + rs);
            rs = (V)0;
        }
    }
};

template <bool U8>
__device__ __forceinline__ void local_store(const Common &c, int b, int x, int y, float vf, int vi)
{
    char *orow = c.out.data + (int64_t)b * c.out.bstride + (int64_t)y * c.out.stride;
    if (U8) reinterpret_cast<int32_t *>(orow)[x] = vi;
    else reinterpret_cast<float *>(orow)[x] = vf;
}

template <bool U8>
__device__ __forceinline__ auto local_read(const LocalAcc &a, int b, int ix, int iy)
{
    if constexpr (U8) return read_u8(a.in, b, ix, iy, a.mode, a.cval_i);
    else return read_f32(a.in, b, ix, iy, a.mode, a.cval_f);
}

// Point-operator prologue (reading c27): f32 one FMA (a, b rounded to f32),
// u8 exact int32 (|a|, |b| <= 2^16 checked by the API).
__device__ __forceinline__ float local_point(const LocalAcc &a, float v) { return __fmaf_rn(a.pa_f, v, a.pb_f); }
__device__ __forceinline__ int local_point(const LocalAcc &a, int v) { return a.pa_i * v + a.pb_i; }

// Map the n staged elements t[0..n) of accessor a in place (all threads of
// the CTA; the caller synchronises before and after).
template <typename V>
__device__ __forceinline__ void local_point_stage(const LocalAcc &a, V *t, int n)
{
    const int tid = threadIdx.y * blockDim.x + threadIdx.x, nthr = blockDim.x * blockDim.y;
    for (int i = tid; i < n; i += nthr) t[i] = local_point(a, t[i]);
}

// Is accessor a's footprint of output rectangle [x0, x0+w) x [y0, y0+h)
// inside the image (global rows, columns)?  Then no boundary handling.
__device__ __forceinline__ bool local_interior(const LocalAcc &a, int x0, int y0, int w, int h)
{
    const int ix0 = x0 + a.off_x - a.rx, iy0 = y0 + a.off_y - a.ry;
    const int gy = iy0 + a.in.gy0;
    return ix0 >= 0 && ix0 + w + 2 * a.rx <= a.in.W && gy >= 0 && gy + h + 2 * a.ry <= a.in.GH;
}

// Stage rows [r_lo, r_hi) x pitch columns of accessor a's footprint (input
// origin (ix0, iy0)) into t (row pitch `pitch`, in elements).  Warps take
// rows, lanes columns (no per-element division); interior tiles load without
// boundary handling, 16 bytes at a time when aligned.
template <bool U8>
__device__ __forceinline__ void local_stage(const LocalAcc &a, int b, int ix0, int iy0, int r_lo,
                                            int r_hi, int pitch, bool interior,
                                            typename std::conditional<U8, int, float>::type *t)
{
    using V = typename std::conditional<U8, int, float>::type;
    const int lane = (threadIdx.y * blockDim.x + threadIdx.x) & 31;
    const int warp = (threadIdx.y * blockDim.x + threadIdx.x) >> 5;
    const int nwarps = (blockDim.x * blockDim.y + 31) >> 5;
    const char *fb = a.in.data + (int64_t)b * a.in.bstride;
    const bool vec = interior && (pitch & 3) == 0 && (ix0 & 3) == 0 && (a.in.stride & (U8 ? 3 : 15)) == 0 &&
                     ((reinterpret_cast<uintptr_t>(fb) & (U8 ? 3 : 15)) == 0);
    if constexpr (!U8) {
        if (vec) {
            // f32 interior: 16-byte asynchronous copies (LDGSTS), all in flight at
            // once, waited for here (the caller's __syncthreads follows)
            const int nv = pitch >> 2, tid = threadIdx.y * blockDim.x + threadIdx.x;
            const int nthr = blockDim.x * blockDim.y, total = (r_hi - r_lo) * nv;
            int r = r_lo + tid / nv, x4 = tid % nv;               // one division per thread
            const int dr = nthr / nv, dx = nthr % nv;
            for (int i = tid; i < total; i += nthr) {
                const char *src = fb + (int64_t)(iy0 + r) * a.in.stride + (int64_t)(ix0 + 4 * x4) * 4;
                const uint32_t dst = (uint32_t)__cvta_generic_to_shared(t + r * pitch + 4 * x4);
                asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst), "l"(src) : "memory");
                r += dr;
                x4 += dx;
                if (x4 >= nv) { x4 -= nv; ++r; }
            }
            asm volatile("cp.async.commit_group;\n\tcp.async.wait_all;" ::: "memory");
            return;
        }
    }
    if (U8 && interior && vec && pitch <= 256) {
        // u8 interior, rows up to 256 bytes: each lane fetches its words of 4 rows
        // before storing any (8 independent loads in flight per lane; one row per
        // iteration made every row a dependent DRAM round trip of the warp)
        for (int r0 = r_lo + warp; r0 < r_hi; r0 += 4 * nwarps) {
            uint32_t w[4][2];
#pragma unroll
            for (int u = 0; u < 4; ++u) {
                const int r = r0 + u * nwarps;
                const char *rp = fb + (int64_t)(iy0 + r) * a.in.stride + ix0;
#pragma unroll
                for (int h = 0; h < 2; ++h) {
                    const int x = 4 * lane + 128 * h;
                    w[u][h] = r < r_hi && x < pitch ? __ldg(reinterpret_cast<const uint32_t *>(rp + x)) : 0u;
                }
            }
#pragma unroll
            for (int u = 0; u < 4; ++u) {
                const int r = r0 + u * nwarps;
#pragma unroll
                for (int h = 0; h < 2; ++h) {
                    const int x = 4 * lane + 128 * h;
                    if (r < r_hi && x < pitch)
                        *reinterpret_cast<int4 *>(t + r * pitch + x) =
                            make_int4(w[u][h] & 0xFF, (w[u][h] >> 8) & 0xFF, (w[u][h] >> 16) & 0xFF, w[u][h] >> 24);
                }
            }
        }
        return;
    }
    for (int r = r_lo + warp; r < r_hi; r += nwarps) {
        V *trow = t + r * pitch;
        if (interior) {
            const char *rp = fb + (int64_t)(iy0 + r) * a.in.stride;
            if (vec) {                                   // u8: 4-byte words, 4 in flight per lane
                for (int x = 4 * lane; x < pitch; x += 512) {
                    uint32_t w[4];
#pragma unroll
                    for (int u = 0; u < 4; ++u)
                        w[u] = x + 128 * u < pitch
                                   ? __ldg(reinterpret_cast<const uint32_t *>(rp + ix0 + x + 128 * u)) : 0u;
#pragma unroll
                    for (int u = 0; u < 4; ++u)
                        if (x + 128 * u < pitch)
                            *reinterpret_cast<int4 *>(trow + x + 128 * u) =
                                make_int4(w[u] & 0xFF, (w[u] >> 8) & 0xFF, (w[u] >> 16) & 0xFF, w[u] >> 24);
                }
            } else {
                for (int x = lane; x < pitch; x += 32) {
                    if constexpr (U8) trow[x] = (int)__ldg(reinterpret_cast<const uint8_t *>(rp) + ix0 + x);
                    else trow[x] = __ldg(reinterpret_cast<const float *>(rp) + ix0 + x);
                }
            }
        } else {
            for (int x = lane; x < pitch; x += 32) trow[x] = local_read<U8>(a, b, ix0 + x, iy0 + r);
        }
    }
}

// ------------------------------------------------------------------ tiled
template <bool U8, int OP, int FN>
__global__ void __launch_bounds__(1024) local_tiled_kernel(const __grid_constant__ LocalParams p)
{
    using V = typename std::conditional<U8, int, float>::type;
    constexpr int OY = local::OUT_Y;
    extern __shared__ float4 smem4[];
    V *sm = reinterpret_cast<V *>(smem4);
    const Common &c = p.c;
    const int tw = blockDim.x, th = OY * blockDim.y;
    const int b = blockIdx.z;
    const int tx0 = c.roi_x0 + blockIdx.x * tw, ty0 = c.roi_y0 + blockIdx.y * th;
    const int roi_x1 = c.roi_x0 + c.roi_w, roi_y1 = c.roi_y0 + c.roi_h;
    const int rows = min(th, roi_y1 - ty0);               // output rows of this tile
    // stage every accessor's footprint (only the rows the tile's outputs need)
    int base = 0;
    for (int k = 0; k < p.n; ++k) {
        const LocalAcc &a = p.acc[k];
        const int sw = tw + 2 * a.rx, sh = rows + 2 * a.ry;
        const int ix0 = tx0 + a.off_x - a.rx, iy0 = ty0 + a.off_y - a.ry;
        local_stage<U8>(a, b, ix0, iy0, 0, sh, sw, local_interior(a, tx0, ty0, tw, rows), sm + base);
        base += sw * sh;
    }
    __syncthreads();
    if (p.any_point) {                                     // point-operator prologue
        base = 0;
        for (int k = 0; k < p.n; ++k) {
            const LocalAcc &a = p.acc[k];
            const int n = (tw + 2 * a.rx) * (rows + 2 * a.ry);
            if (a.point) local_point_stage(a, sm + base, n);
            base += n;
        }
        __syncthreads();
    }

    const int x = tx0 + threadIdx.x;
    const int y0 = OY * threadIdx.y;                       // first output row (tile-relative)
    const int nj = min(OY, rows - y0);
    if (x >= roi_x1 || nj <= 0) return;
    LocalAccum<V, OP> acc[OY];
#pragma unroll
    for (int j = 0; j < OY; ++j) acc[j].init();
    base = 0;
    for (int k = 0; k < p.n; ++k) {
        const LocalAcc &a = p.acc[k];
        const int sw = tw + 2 * a.rx, sh = rows + 2 * a.ry;
        const int sx = 2 * a.rx + 1;
        const V *t = sm + base + threadIdx.x + a.rx;      // column of this thread's outputs
        V cen[OY];
#pragma unroll
        for (int j = 0; j < OY; ++j) cen[j] = j < nj ? t[(y0 + j + a.ry) * sw] : (V)0;
        const V *mk = (const V *)(U8 ? (const void *)(p.m.i + a.moff) : (const void *)(p.m.f + a.moff));
        // staged row r feeds output j with window row yf = r - j - ry
        for (int r = 0; r < nj + 2 * a.ry; ++r) {
            const V *row = t + (y0 + r) * sw;
            for (int xf = -a.rx; xf <= a.rx; ++xf) {
                const V v = row[xf];
#pragma unroll
                for (int j = 0; j < OY; ++j) {
                    const int yf = r - j - a.ry;
                    if (j < nj && yf >= -a.ry && yf <= a.ry)
                        acc[j].template tap<FN>(mk[(yf + a.ry) * sx + xf + a.rx], v, cen[j], xf == -a.rx);
                }
            }
#pragma unroll
            for (int j = 0; j < OY; ++j) {
                const int yf = r - j - a.ry;
                if (j < nj && yf >= -a.ry && yf <= a.ry) acc[j].end_row(yf == -a.ry);
            }
        }
#pragma unroll
        for (int j = 0; j < OY; ++j) acc[j].end_accessor(k == 0);
        base += sw * sh;
    }
#pragma unroll
    for (int j = 0; j < OY; ++j)
        if (j < nj) local_store<U8>(c, b, x, ty0 + y0 + j, (float)acc[j].total, (int)acc[j].total);
}

// ----------------------------------------------------- small-window tiled
// Every accessor's window <= 7 x 7 (the common case: 3x3, 5x5 stencils).
// Register blocking: a thread computes 4 columns x 4 rows.  Per accessor k and
// window row yf (runtime, warp-uniform loop) the 7 coefficients of the row are
// read once (uniform, from the kernel parameter block: the mask embedded in a
// 7 x 7 slot), then for each of the 4 output rows the staged row segment of
// 12 values (columns c0 .. c0 + 11 = c0 - 4 .. c0 + 7 of the input) comes in
// as 3 LDS.128 and feeds 7 x 4 taps, the tap loop unrolled over the slot with
// warp-uniform predicates for the accessor's own window.  Each output sees
// exactly the generic kernel's sequence of operations (accessor, window row,
// left-to-right taps).  Staging: per accessor the tile's rows +- ry_k and
// columns +- 4; rows past the iteration space are zero-filled, not fetched.
namespace local {
constexpr int SR = kLocalSmallR, SW = kLocalSmallW;
constexpr int SX = 4;                        // output columns per thread
// staged columns left / right for a launch whose largest x radius is <= RXM
// (>= RXM, a multiple of 4 so that rows stay 16-byte aligned)
template <int RXM> struct Halo { static constexpr int HX = (RXM + 3) & ~3; };
inline int rxm_bucket(int rx) { return rx <= 1 ? 1 : rx <= 2 ? 2 : rx <= 3 ? 3 : 7; }
}  // namespace local

template <bool U8, int OP, int FN, int RXM>
__global__ void __launch_bounds__(256) local_small_kernel(const __grid_constant__ LocalParams p)
{
    using V = typename std::conditional<U8, int, float>::type;
    using V4 = typename std::conditional<U8, int4, float4>::type;
    constexpr int OY = local::OUT_Y, SR = local::SR, SW = local::SW, SX = local::SX;
    constexpr int HX = local::Halo<RXM>::HX, NV = (SX + 2 * HX) / 4;    // float4 per row segment
    extern __shared__ float4 smem4[];
    V *sm = reinterpret_cast<V *>(smem4);
    const Common &c = p.c;
    const int tw = SX * blockDim.x, th = OY * blockDim.y;
    const int pitch = tw + 2 * HX;
    const int b = blockIdx.z;
    const int tx0 = c.roi_x0 + blockIdx.x * tw, ty0 = c.roi_y0 + blockIdx.y * th;
    const int roi_x1 = c.roi_x0 + c.roi_w, roi_y1 = c.roi_y0 + c.roi_h;
    const int rows = min(th, roi_y1 - ty0);
    const int tid = threadIdx.y * blockDim.x + threadIdx.x;
    // f32 interior footprints: one cp.async.bulk per staged row (TMA bulk
    // engine, rows spread over the threads), completing on the accessor's own
    // mbarrier, so accessor k's taps start as soon as its rows have landed while
    // the later accessors' rows are still in flight; the rest element-wise
    __shared__ __align__(8) uint64_t sbar[kLocalMaxAcc];
    if (tid == 0) {
        for (int k = 0; k < p.n; ++k) asm volatile("mbarrier.init.shared.b64 [%0], 1;" ::"r"(smem_addr(&sbar[k])));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    auto bulk_ok = [&](const LocalAcc &a, int ix0, int iy0, int sh) {
        if constexpr (U8) return false;
        const char *fb = a.in.data + (int64_t)b * a.in.bstride;
        const int gy = iy0 + a.in.gy0;
        return ix0 >= 0 && ix0 + pitch <= a.in.W && gy >= 0 && gy + sh <= a.in.GH && (ix0 & 3) == 0 &&
               (a.in.stride & 15) == 0 && (reinterpret_cast<uintptr_t>(fb) & 15) == 0;
    };
    if (tid == 0) {
        for (int k = 0; k < p.n; ++k) {
            const LocalAcc &a = p.acc[k];
            const int ix0 = tx0 + a.off_x - HX, iy0 = ty0 + a.off_y - a.ry, sh = rows + 2 * a.ry;
            const uint32_t nbytes = bulk_ok(a, ix0, iy0, sh) ? (uint32_t)(sh * pitch * 4) : 0u;
            asm volatile("mbarrier.arrive.expect_tx.shared.b64 _, [%0], %1;" ::"r"(smem_addr(&sbar[k])),
                         "r"(nbytes) : "memory");
        }
    }
    int base = 0;
#pragma unroll 1
    for (int k = 0; k < p.n; ++k) {
        const LocalAcc &a = p.acc[k];
        const int ix0 = tx0 + a.off_x - HX, iy0 = ty0 + a.off_y - a.ry;
        const int sh = rows + 2 * a.ry;                                 // fetched rows
        if (bulk_ok(a, ix0, iy0, sh)) {
            {                                                        // rows spread over the threads
                const char *src = a.in.data + (int64_t)b * a.in.bstride + (int64_t)iy0 * a.in.stride +
                                  (int64_t)ix0 * 4;
                for (int r = tid; r < sh; r += blockDim.x * blockDim.y)
                    asm volatile(
                        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                        ::"r"(smem_addr(sm + base + r * pitch)), "l"(src + (int64_t)r * a.in.stride),
                          "r"(pitch * 4), "r"(smem_addr(&sbar[k]))
                        : "memory");
            }
        } else {
            const int gy = iy0 + a.in.gy0;
            const bool interior = ix0 >= 0 && ix0 + pitch <= a.in.W && gy >= 0 && gy + sh <= a.in.GH;
            local_stage<U8>(a, b, ix0, iy0, 0, sh, pitch, interior, sm + base);
        }
        // rows of a partial last tile row: zero (computed, never stored)
        for (int i = tid + sh * pitch; i < (th + 2 * a.ry) * pitch; i += blockDim.x * blockDim.y)
            sm[base + i] = (V)0;
        base += (th + 2 * a.ry) * pitch;
    }
    __syncthreads();                                       // element-wise staging visible
    if (p.any_point) {                                     // point-operator prologue
        for (int k = 0; k < p.n; ++k) mbar_wait(&sbar[k], 0);
        base = 0;
        for (int k = 0; k < p.n; ++k) {
            const LocalAcc &a = p.acc[k];
            const int n = (th + 2 * a.ry) * pitch;
            if (a.point) local_point_stage(a, sm + base, n);
            base += n;
        }
        __syncthreads();
    }

    const int c0 = SX * threadIdx.x;                       // tile-relative first column
    const int r0 = OY * threadIdx.y;                       // tile-relative first row
    const int x0 = tx0 + c0;
    LocalAccum<V, OP> acc[OY][SX];
#pragma unroll
    for (int j = 0; j < OY; ++j)
#pragma unroll
        for (int q = 0; q < SX; ++q) acc[j][q].init();
    base = 0;
#pragma unroll 1
    for (int k = 0; k < p.n; ++k) {
        const LocalAcc &a = p.acc[k];
        const int rx = a.rx, ry = a.ry;
        mbar_wait(&sbar[k], 0);                             // accessor k's bulk rows have landed
        const V *t = sm + base + c0;                        // column c0 - HX of the input
        const V *mk = (const V *)(U8 ? (const void *)p.ms.i[k] : (const void *)p.ms.f[k]);
        V cen[OY][SX];
        if (FN == local::FN_ABSDIFF || FN == local::FN_SQDIFF) {
#pragma unroll
            for (int j = 0; j < OY; ++j) {
                const V4 w = *reinterpret_cast<const V4 *>(t + (r0 + j + ry) * pitch + HX);
                cen[j][0] = w.x; cen[j][1] = w.y; cen[j][2] = w.z; cen[j][3] = w.w;
            }
        }
#pragma unroll 1
        for (int yf = -ry; yf <= ry; ++yf) {
            V M[2 * RXM + 1];
#pragma unroll
            for (int xf = -RXM; xf <= RXM; ++xf) M[xf + RXM] = mk[(yf + SR) * SW + xf + SR];
#pragma unroll
            for (int j = 0; j < OY; ++j) {
                const V4 *rp = reinterpret_cast<const V4 *>(t + (r0 + j + yf + ry) * pitch);
                V v[4 * NV];
#pragma unroll
                for (int i = 0; i < NV; ++i) {
                    const V4 w = rp[i];
                    v[4 * i] = w.x; v[4 * i + 1] = w.y; v[4 * i + 2] = w.z; v[4 * i + 3] = w.w;
                }
#pragma unroll
                for (int xf = -RXM; xf <= RXM; ++xf) {
                    if (xf < -rx || xf > rx) continue;               // warp-uniform
#pragma unroll
                    for (int q = 0; q < SX; ++q)
                        acc[j][q].template tap<FN>(M[xf + RXM], v[HX + q + xf], cen[j][q], xf == -rx);
                }
#pragma unroll
                for (int q = 0; q < SX; ++q) acc[j][q].end_row(yf == -ry);
            }
        }
#pragma unroll
        for (int j = 0; j < OY; ++j)
#pragma unroll
            for (int q = 0; q < SX; ++q) acc[j][q].end_accessor(k == 0);
        base += (th + 2 * ry) * pitch;
    }
    if (x0 >= roi_x1) return;
    const bool vec = x0 + SX <= roi_x1 && ((x0 & 3) == 0) && ((c.out.stride & 15) == 0) &&
                     ((reinterpret_cast<uintptr_t>(c.out.data + (int64_t)b * c.out.bstride) & 15) == 0);
#pragma unroll
    for (int j = 0; j < OY; ++j) {
        if (r0 + j >= rows) break;
        const int y = ty0 + r0 + j;
        char *orow = c.out.data + (int64_t)b * c.out.bstride + (int64_t)y * c.out.stride;
        if (vec) {
            if constexpr (U8) *reinterpret_cast<int4 *>(reinterpret_cast<int32_t *>(orow) + x0) =
                make_int4(acc[j][0].total, acc[j][1].total, acc[j][2].total, acc[j][3].total);
            else *reinterpret_cast<float4 *>(reinterpret_cast<float *>(orow) + x0) =
                make_float4(acc[j][0].total, acc[j][1].total, acc[j][2].total, acc[j][3].total);
        } else {
#pragma unroll
            for (int q = 0; q < SX; ++q)
                if (x0 + q < roi_x1) local_store<U8>(c, b, x0 + q, y, (float)acc[j][q].total, (int)acc[j][q].total);
        }
    }
}

// ---------------------------------------------------------------- generic
template <bool U8, int OP, int FN>
__global__ void __launch_bounds__(1024) local_generic_kernel(const __grid_constant__ LocalParams p)
{
    using V = typename std::conditional<U8, int, float>::type;
    const Common &c = p.c;
    const int bx0 = c.roi_x0 + blockIdx.x * blockDim.x, by0 = c.roi_y0 + blockIdx.y * blockDim.y;
    const int x = bx0 + threadIdx.x, y = by0 + threadIdx.y;
    const int b = blockIdx.z;
    if (x >= c.roi_x0 + c.roi_w || y >= c.roi_y0 + c.roi_h) return;
    LocalAccum<V, OP> acc;
    acc.init();
    for (int k = 0; k < p.n; ++k) {
        const LocalAcc &a = p.acc[k];
        const int sx = 2 * a.rx + 1;
        const int ix = x + a.off_x, iy = y + a.off_y;
        // CTAs whose footprint stays inside the image skip the per-tap
        // boundary resolution (Algorithm 2 counts the others' threads)
        const bool interior = local_interior(a, bx0, by0, blockDim.x, blockDim.y);
        const char *fb = a.in.data + (int64_t)b * a.in.bstride;
        auto rd0 = [&](int xx, int yy) -> V {
            if (interior) {
                const char *rp = fb + (int64_t)yy * a.in.stride;
                if constexpr (U8) return (int)__ldg(reinterpret_cast<const uint8_t *>(rp) + xx);
                else return __ldg(reinterpret_cast<const float *>(rp) + xx);
            }
            return local_read<U8>(a, b, xx, yy);
        };
        auto rd = [&](int xx, int yy) -> V {
            const V v = rd0(xx, yy);
            return a.point ? local_point(a, v) : v;
        };
        const V cen = rd(ix, iy);
        const V *mk = (const V *)(U8 ? (const void *)(p.m.i + a.moff) : (const void *)(p.m.f + a.moff));
        for (int yf = -a.ry; yf <= a.ry; ++yf) {
            for (int xf = -a.rx; xf <= a.rx; ++xf)
                acc.template tap<FN>(mk[(yf + a.ry) * sx + xf + a.rx], rd(ix + xf, iy + yf), cen, xf == -a.rx);
            acc.end_row(yf == -a.ry);
        }
        acc.end_accessor(k == 0);
    }
    local_store<U8>(c, b, x, y, (float)acc.total, (int)acc.total);
}

// --------------------------------------------------------------- launcher
namespace {

size_t small_smem(const LocalParams &p, int bx, int by)
{
    const int rxm = local::rxm_bucket(p.c.rx), hx = (rxm + 3) & ~3;
    size_t n = 0;
    for (int k = 0; k < p.n; ++k)
        n += (size_t)(local::SX * bx + 2 * hx) * (local::OUT_Y * by + 2 * p.acc[k].ry);
    return n * 4;
}

size_t tiled_smem(const LocalParams &p, int bx, int by)
{
    size_t n = 0;
    for (int k = 0; k < p.n; ++k)
        n += (size_t)(bx + 2 * p.acc[k].rx) * (local::OUT_Y * by + 2 * p.acc[k].ry);
    return n * 4;
}

// Algorithm 2 over the thread counts 32, 64, ..., 1024 (multiples of the
// SIMD width): tiling y-preferred (32 x T/32) with border handling, x-preferred
// (T x 1) without; resource limits from the kernel's attributes and the
// device's opt-in shared memory; occupancy from the CUDA occupancy API.
// tiled: 0 generic (1 x 1 outputs per thread), 1 tiled (1 x 4), 2 small (2 x 4)
template <typename K>
cudaError_t choose_config(K kernel, const LocalParams &p, int tiled, int &bx, int &by)
{
    const int dev = current_device();
    cudaFuncAttributes fa;
    cudaError_t e = cudaFuncGetAttributes(&fa, kernel);
    int smem_max = 0, max_thr_sm = 0;
    if (e == cudaSuccess) e = cudaDeviceGetAttribute(&smem_max, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
    if (e == cudaSuccess) e = cudaDeviceGetAttribute(&max_thr_sm, cudaDevAttrMaxThreadsPerMultiProcessor, dev);
    if (e != cudaSuccess) return e;
    int fx = 0, fy = 0;                                   // footprint radii (window + offset)
    for (int k = 0; k < p.n; ++k) {
        fx = max(fx, p.acc[k].rx + abs(p.acc[k].off_x));
        fy = max(fy, p.acc[k].ry + abs(p.acc[k].off_y));
    }
    const bool border = fx > 0 || fy > 0;
    lop_config_candidate cand[32];
    int n = 0;
    for (int t = 32; t <= 1024; t += 32) {
        lop_config_candidate &cd = cand[n++];
        cd.block_x = border ? 32 : t;
        cd.block_y = border ? t / 32 : 1;
        cd.out_x = tiled == 2 ? local::SX : 1;
        cd.out_y = tiled ? local::OUT_Y : 1;
        const size_t smem = tiled == 2 ? small_smem(p, cd.block_x, cd.block_y)
                                       : (tiled ? tiled_smem(p, cd.block_x, cd.block_y) : 0);
        cd.valid = t <= fa.maxThreadsPerBlock && smem <= (size_t)smem_max;
        cd.occupancy = 0.0;
        if (cd.valid) {
            if (smem > 48 * 1024) {
                e = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
                if (e != cudaSuccess) return e;
            }
            int blocks = 0;
            e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&blocks, kernel, t, smem);
            if (e != cudaSuccess) return e;
            cd.occupancy = (double)blocks * t / max_thr_sm;
            cd.valid = blocks > 0;
        }
    }
    const int i = alg2_select(cand, n, 32, p.c.roi_w, p.c.roi_h, fx, fy, nullptr);
    if (i < 0) return cudaErrorInvalidConfiguration;
    bx = cand[i].block_x;
    by = cand[i].block_y;
    return cudaSuccess;
}

// the small-window instance for the launch's largest x radius
template <bool U8, int OP, int FN>
auto small_kernel_ptr(const LocalParams &p) -> decltype(&local_small_kernel<U8, OP, FN, 1>)
{
    switch (local::rxm_bucket(p.c.rx)) {
    case 1: return local_small_kernel<U8, OP, FN, 1>;
    case 2: return local_small_kernel<U8, OP, FN, 2>;
    case 3: return local_small_kernel<U8, OP, FN, 3>;
    default: return local_small_kernel<U8, OP, FN, 7>;
    }
}

template <bool U8, int OP, int FN>
cudaError_t launch_local_t(const LocalParams &p, bool tiled_ok, cudaStream_t stream)
{
    const int kind = !tiled_ok ? 0 : (p.small ? 2 : 1);
    // configuration cache: the last geometry per (thread, instance)
    struct Key { int dev, w, h, batch, n, kind; int r[4 * kLocalMaxAcc]; };
    static thread_local Key last{};
    static thread_local int last_bx = 0, last_by = 0;
    Key key{};
    key.dev = current_device(); key.w = p.c.roi_w; key.h = p.c.roi_h; key.batch = p.c.batch;
    key.n = p.n; key.kind = kind;
    for (int k = 0; k < p.n; ++k) {
        key.r[4 * k] = p.acc[k].rx; key.r[4 * k + 1] = p.acc[k].ry;
        key.r[4 * k + 2] = p.acc[k].off_x; key.r[4 * k + 3] = p.acc[k].off_y;
    }
    int bx = 0, by = 0;
    if (const char *env = std::getenv("LOP_LOCAL_CFG")) {          // exploration (Fig. 4 sweep)
        if (std::sscanf(env, "%d:%d", &bx, &by) != 2 || bx < 1 || by < 1 || bx * by > 1024) bx = by = 0;
    }
    if (bx) {
    } else if (last_bx && !memcmp(&key, &last, sizeof key)) {
        bx = last_bx; by = last_by;
    } else {
        cudaError_t e = kind == 2 ? choose_config(small_kernel_ptr<U8, OP, FN>(p), p, 2, bx, by)
                      : kind == 1 ? choose_config(local_tiled_kernel<U8, OP, FN>, p, 1, bx, by)
                                  : choose_config(local_generic_kernel<U8, OP, FN>, p, 0, bx, by);
        if (e != cudaSuccess) return e;
        last = key; last_bx = bx; last_by = by;
        if (std::getenv("LOP_DEBUG_SELECT"))
            fprintf(stderr, "[lop] local kernel %d: Algorithm 2 chose %d x %d threads for %d x %d\n",
                    kind, bx, by, p.c.roi_w, p.c.roi_h);
    }
    if (kind == 2) {
        const size_t smem = small_smem(p, bx, by);
        auto kern = small_kernel_ptr<U8, OP, FN>(p);
        static PerDevice configured_b[8];                       // one cache per instance (bucket)
        cudaError_t e = ensure_smem(kern, smem, configured_b[local::rxm_bucket(p.c.rx)]);
        if (e != cudaSuccess) return e;
        const int tw = local::SX * bx, th = local::OUT_Y * by;
        dim3 grid((p.c.roi_w + tw - 1) / tw, (p.c.roi_h + th - 1) / th, p.c.batch);
        kern<<<grid, dim3(bx, by), smem, stream>>>(p);
    } else if (kind == 1) {
        const size_t smem = tiled_smem(p, bx, by);
        static PerDevice configured;
        cudaError_t e = ensure_smem(local_tiled_kernel<U8, OP, FN>, smem, configured);
        if (e != cudaSuccess) return e;
        dim3 grid((p.c.roi_w + bx - 1) / bx, (p.c.roi_h + local::OUT_Y * by - 1) / (local::OUT_Y * by),
                  p.c.batch);
        local_tiled_kernel<U8, OP, FN><<<grid, dim3(bx, by), smem, stream>>>(p);
    } else {
        dim3 grid((p.c.roi_w + bx - 1) / bx, (p.c.roi_h + by - 1) / by, p.c.batch);
        local_generic_kernel<U8, OP, FN><<<grid, dim3(bx, by), 0, stream>>>(p);
    }
    return cudaGetLastError();
}

template <bool U8, int OP>
cudaError_t launch_local_op(const LocalParams &p, bool tiled, cudaStream_t s)
{
    switch (p.fn) {
    case local::FN_PRODUCT: return launch_local_t<U8, OP, local::FN_PRODUCT>(p, tiled, s);
    case local::FN_ABSDIFF: return launch_local_t<U8, OP, local::FN_ABSDIFF>(p, tiled, s);
    case local::FN_SQDIFF: return launch_local_t<U8, OP, local::FN_SQDIFF>(p, tiled, s);
    case local::FN_SQUARE: return launch_local_t<U8, OP, local::FN_SQUARE>(p, tiled, s);
    default: return cudaErrorInvalidValue;
    }
}

template <bool U8>
cudaError_t launch_local_u8(const LocalParams &p, bool tiled, cudaStream_t s)
{
    switch (p.op) {
    case RED_SUM: return launch_local_op<U8, RED_SUM>(p, tiled, s);
    case RED_MIN: return launch_local_op<U8, RED_MIN>(p, tiled, s);
    case RED_MAX: return launch_local_op<U8, RED_MAX>(p, tiled, s);
    default: return cudaErrorInvalidValue;
    }
}

}  // namespace

}  // namespace lop

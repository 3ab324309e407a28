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

#include <algorithm>
#include <cstdlib>
#include <type_traits>

#include "boundary.cuh"
#include "kernels.h"
#include "launch_cache.h"
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

// One output tile (tx0, ty0) of at most TS rows, ending before row ry1 (the
// iteration space's end, or a band's); every thread of the CTA takes part
// (block barriers inside).
// One output row of PX values at ox, per element, only columns in [x0, x1).
template <typename TO, int PX, typename A>
__device__ __forceinline__ void store_row_masked(char *orow, int ox, int x0, int x1, const A *out,
                                                 int shift)
{
    TO *op = reinterpret_cast<TO *>(orow);
#pragma unroll
    for (int j = 0; j < PX; ++j) {
        if (ox + j < x0 || ox + j >= x1) continue;
        if constexpr (std::is_same<TO, float>::value) op[ox + j] = out[j];
        else if constexpr (sizeof(TO) == 1) op[ox + j] = (TO)min(max(quantize_shift(out[j], shift), 0), 255);
        else op[ox + j] = quantize_shift(out[j], shift);
    }
}

template <typename T, typename TO, int R1, int R2, int TS>
__device__ __forceinline__ void chain_tile(const ConvChain &p, int b, int tx0, int ty0, int ry1,
                                           unsigned char *smem_raw, uint64_t &bar)
{
    using S = chain::Shape<T>;
    constexpr int PX = S::PX, GW = S::GW, HALO = S::HALO, OW = S::OW, IPAD = S::IPAD,
                  ISW = S::ISW;
    constexpr bool F = sizeof(T) == 4;
    using A = typename std::conditional<F, float, int>::type;
    using TG = T;                                                   // intermediate type
    static_assert(R1 <= IPAD && R2 <= 4 && R2 <= HALO, "halo");
    const Common &c = p.s1.c;
    T *itile = reinterpret_cast<T *>(smem_raw);                     // ni x ISW
    const int roi_x1 = c.roi_x0 + c.roi_w;
    const int nrows = min(TS, ry1 - ty0);
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

template <typename T, typename TO, int R1, int R2, int TS>
__global__ void __launch_bounds__(chain::NT) conv_chain_kernel(const __grid_constant__ ConvChain p)
{
    extern __shared__ __align__(16) unsigned char smem_raw[];
    __shared__ __align__(8) uint64_t bar;
    const Common &c = p.s1.c;
    chain_tile<T, TO, R1, R2, TS>(p, blockIdx.z, c.roi_x0 + blockIdx.x * chain::Shape<T>::OW,
                                  c.roi_y0 + blockIdx.y * TS, c.roi_y0 + c.roi_h, smem_raw, bar);
}

// ------------------------------------------------ row-streaming fused chain
// Each warp owns a frame of 32 lanes x PX G columns (lane L: G columns
// gxb + PX L .. + PX-1) and streams down T output rows; the outer lane on each
// side is halo (its G values feed its neighbour's pass 2; its own outputs are
// not stored), so a warp writes OWS = 30 PX columns.  Per input row:
//   cp.async of the row PD rows ahead into a per-warp smem ring (16-B chunks;
//   chunks outside the image: REPEAT fetches the wrapped chunk, the other
//   modes fill from the row itself / the constant once the row has landed),
//   pass-1 horizontal sums into a register ring, pass-1 vertical -> one G row
//   (kept in registers, quantised like a u8 pass), G columns outside the image
//   per pass 2's boundary condition (edge frames: constant, or the G value at
//   the mapped column fetched by shuffle; REPEAT: the naive G there already
//   equals G at the wrapped column), the G neighbours of the pass-2 window by
//   shuffles, pass-2 horizontal sums into a second register ring, pass-2
//   vertical -> one output row.  No block barrier, no G tile, no HBM round
//   trip of G.  The arithmetic (sep_h / sep_v, the same operations in the same
//   order) is that of two conv_sep_kernel passes, so the result is bit-identical
//   to two lop_convolve_execute calls.  The output rows whose pass 2 reads G
//   rows outside the image (the top and bottom R2 rows) are tiles of chain_tile
//   in the same launch.
namespace chain {
template <typename T> struct SShape {
    static constexpr int PX = sizeof(T) == 4 ? 4 : 8;          // G columns per lane
    static constexpr int FW = 32 * PX;                         // frame width (G columns)
    static constexpr int OWS = FW - 2 * PX;                    // output columns per warp
    static constexpr int PAD = PX;                             // input columns beyond the frame
    static constexpr int SW = FW + 2 * PAD;                    // smem ring row (elements)
    static constexpr int V16 = 16 / (int)sizeof(T);            // elements per 16-B chunk
    static constexpr int NCH = SW / V16;                       // chunks per row
    static constexpr int PD = 6;                               // prefetch distance (rows)
    static constexpr int NS = PD + 1;                          // ring slots
    static constexpr int RING_BYTES = NS * SW * (int)sizeof(T);
    static constexpr int WARP_BYTES = RING_BYTES + SW * 4;     // + column map
};
constexpr int NW = NT / 32;          // warps per CTA
constexpr int TSB = 2;               // rows per band tile
}  // namespace chain

__device__ __forceinline__ void chain_cp_async16(void *smem_dst, const void *gsrc)
{
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_addr(smem_dst)), "l"(gsrc)
                 : "memory");
}

// G[e] of lane m / PX for a warp-uniform frame column m (clamped into the frame).
template <typename A, int PX>
__device__ __forceinline__ A chain_frame_value(const A (&G)[PX], int m)
{
    m = min(max(m, 0), 32 * PX - 1);
    const int e = m % PX;
    A x = G[0];
#pragma unroll
    for (int j = 1; j < PX; ++j) x = e == j ? G[j] : x;
    return __shfl_sync(0xffffffffu, x, m / PX);
}

// Rare paths of the streaming loop, out of line so that the unrolled loop body
// stays small (I-cache): the row index of an input row outside the image, and
// the fill of a landed ring row (CONSTANT rows; out-of-image columns of edge
// frames from the row itself or the constant).
__device__ __noinline__ bool chain_row_outside(int iy, const Geom &g, int mode, int &row)
{
    return resolve_row(iy, g, mode, row);
}

template <typename T>
__device__ __noinline__ void chain_fill_row(T *row, int lane, int ix0, int IW, const int *cm,
                                            bool row_ok, T cval)
{
    constexpr int SW = chain::SShape<T>::SW;
    for (int e = lane; e < SW; e += 32) {
        if (!row_ok) { row[e] = cval; continue; }
        if ((unsigned)(ix0 + e) < (unsigned)IW) continue;
        row[e] = cm[e] >= 0 ? row[cm[e] - ix0] : cval;
    }
}

// Per-warp geometry of the streaming path.
struct ChainWarp {
    int y0, nsteps;          // first output row, input rows streamed (T + 2 (R1 + R2))
    int ix0, gxb, iy0;       // input column of smem column 0 / of lane 0's G column 0; input row of step 0
    int ox;                  // this lane's first output column
    bool col_edge, rows_inside;
};

// The streaming loop.  SIMPLE: every input row inside the image and no frame
// column outside it (all but the edge warps) -- no row resolution, no fills,
// no G boundary, one running source pointer.
template <typename T, typename TO, int R1, int R2, bool SIMPLE>
__device__ __forceinline__ void chain_stream_run(const ConvChain &p, int b, const ChainWarp &cw,
                                                 unsigned char *wsmem)
{
    using S = chain::SShape<T>;
    constexpr int PX = S::PX, PAD = S::PAD, SW = S::SW, V16 = S::V16, NCH = S::NCH,
                  PD = S::PD, NS = S::NS;
    constexpr bool F = sizeof(T) == 4;
    using A = typename std::conditional<F, float, int>::type;
    constexpr int P1 = 2 * R1 + 1, P2 = 2 * R2 + 1;
    const Common &c = p.s1.c;
    const Geom &g = c.in;
    const int lane = threadIdx.x & 31;
    const int IW = g.W, mode = c.mode, nsteps = cw.nsteps, ix0 = cw.ix0, iy0 = cw.iy0;
    T *ring = reinterpret_cast<T *>(wsmem);
    const int *cm = reinterpret_cast<const int *>(wsmem + S::RING_BYTES);
    const T cval = F ? (T)c.cval_f : (T)c.cval_i;
    const bool fill_cols = !SIMPLE && cw.col_edge && mode != M_REPEAT;
    // this lane's chunks (q = lane, lane + 32): source column, or -1 (filled after landing)
    int src0 = -1, src1 = -1;
    {
        const int ixa = ix0 + lane * V16, ixb = ixa + 32 * V16;
        if (lane >= NCH) {                                        // u8: 17 chunks per row
        } else if ((unsigned)ixa < (unsigned)IW) src0 = ixa;
        else if (!SIMPLE && mode == M_REPEAT) src0 = cm[lane * V16];
        if (NCH > 32 && lane + 32 < NCH) {
            if ((unsigned)ixb < (unsigned)IW) src1 = ixb;
            else if (!SIMPLE && mode == M_REPEAT) src1 = cm[(lane + 32) * V16];
        }
    }
    const char *fbase = g.data + (int64_t)b * g.bstride;
    const T *srow = reinterpret_cast<const T *>(fbase + (int64_t)iy0 * g.stride);   // SIMPLE: row of step k
    const uint32_t sdst = smem_addr(ring + lane * V16);
    // input row iy0 + k into ring slot sl (one commit group per call)
    auto issue = [&](int k, int sl, const T *rp) {
        if (k < nsteps) {
            bool ok = true;
            if (!SIMPLE) {
                int row = iy0 + k;
                if ((unsigned)row >= (unsigned)g.H) ok = chain_row_outside(row, g, mode, row);
                rp = reinterpret_cast<const T *>(fbase + (int64_t)row * g.stride);
            }
            if (ok) {
                const uint32_t d = sdst + sl * (SW * (int)sizeof(T));
                if (src0 >= 0)
                    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(d), "l"(rp + src0) : "memory");
                if (NCH > 32 && src1 >= 0)
                    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(d + 32 * 16), "l"(rp + src1)
                                 : "memory");
            }
        }
        asm volatile("cp.async.commit_group;" ::: "memory");
    };
    const int64_t sstride = g.stride / (int64_t)sizeof(T);
#pragma unroll
    for (int k = 0; k < PD; ++k) issue(k, k, srow + k * sstride);
    const T *pre = srow + PD * sstride;                           // SIMPLE: row of step k + PD

    // frame columns of G at the mapped positions of G columns -1-t and IW+t
    int gml[R2], gmr[R2];
#pragma unroll
    for (int t = 0; t < R2; ++t) {
        gml[t] = fill_cols ? map_axis(-1 - t, IW, mode) - cw.gxb : 0;
        gmr[t] = fill_cols ? map_axis(IW + t, IW, mode) - cw.gxb : 0;
    }
    char *obase = c.out.data + (int64_t)b * c.out.bstride;
    const int roi_x0 = c.roi_x0, roi_x1 = c.roi_x0 + c.roi_w;
    const int ox = cw.ox;
    const bool out_lane = lane >= 1 && lane <= 30 && ox + PX > roi_x0 && ox < roi_x1;
    const bool ovec = out_lane && ox >= roi_x0 && ox + PX <= roi_x1 &&
                      (((reinterpret_cast<uintptr_t>(obase) | (uintptr_t)c.out.stride) %
                        (sizeof(TO) * PX > 16 ? 16 : sizeof(TO) * PX)) == 0);
    const T *lrow = ring + PAD + lane * PX;                      // gather base in slot 0
    char *orow = obase + (int64_t)cw.y0 * c.out.stride;          // output row of the next output
    A h1[P1][PX], h2[P2][PX];
    int slot = 0, islot = PD;                                    // slot of row k, of row k + PD
    // Register rings of P1 (pass 1) and P2 (pass 2) rows with compile-time slot
    // indices: the SIMPLE loop is unrolled by the common period of both; the
    // general loop (edge warps, larger code) by P1 only, with pass 2 as a
    // shift register (h2[P2-1] newest) so that its body stays short (I-cache).
    constexpr int UNR = SIMPLE ? (P1 == P2 ? P1 : P1 * P2) : P1;
    constexpr bool H2RING = UNR % P2 == 0;
#pragma unroll 1
    for (int k0 = 0; k0 < nsteps; k0 += UNR) {
#pragma unroll
        for (int i = 0; i < UNR; ++i) {
            const int k = k0 + i;
            if (k >= nsteps) break;
            // row k has landed once at most PD - 1 younger groups are pending;
            // after the barrier every lane is also done with slot k - 1,
            // which takes row k + PD
            asm volatile("cp.async.wait_group %0;" ::"n"(PD - 1) : "memory");
            __syncwarp();
            issue(k + PD, islot, pre);
            pre += sstride;
            islot = islot + 1 == NS ? 0 : islot + 1;
            if (!SIMPLE) {
                int r;
                const int iy = iy0 + k;
                const bool rok = (unsigned)iy < (unsigned)g.H || chain_row_outside(iy, g, mode, r);
                if (fill_cols || !rok) {
                    chain_fill_row<T>(ring + slot * SW, lane, ix0, IW, cm, rok, cval);
                    __syncwarp();
                }
            }
            // ---- pass 1, horizontal
            {
                A v[PX + 2 * R1];
                chain_gather<T, R1, A>(lrow + slot * SW, v);
#pragma unroll
                for (int j = 0; j < PX; ++j) h1[i % P1][j] = sep_h<A, R1>(p.s1, v + j);
            }
            slot = slot + 1 == NS ? 0 : slot + 1;
            if (k < 2 * R1) continue;
            // ---- pass 1, vertical: G row k - 2 R1 (quantised like a u8 pass)
            A G[PX];
#pragma unroll
            for (int j = 0; j < PX; ++j) {
                A col[P1];
#pragma unroll
                for (int t = 0; t < P1; ++t) col[t] = h1[(i + 1 + t) % P1][j];
                G[j] = (A)to_g<A, T>(sep_v<A, R1>(p.s1, col), p.s1.shift);
            }
            if (fill_cols) {                                         // pass 2's boundary on G
                const int gx = cw.gxb + PX * lane;
                if (mode == M_CONSTANT) {
#pragma unroll
                    for (int j = 0; j < PX; ++j)
                        if ((unsigned)(gx + j) >= (unsigned)IW) G[j] = (A)cval;
                } else {
                    A lv[R2], rv[R2];
#pragma unroll
                    for (int t = 0; t < R2; ++t) {
                        lv[t] = chain_frame_value<A, PX>(G, gml[t]);
                        rv[t] = chain_frame_value<A, PX>(G, gmr[t]);
                    }
#pragma unroll
                    for (int j = 0; j < PX; ++j)
#pragma unroll
                        for (int t = 0; t < R2; ++t) {
                            if (gx + j == -1 - t) G[j] = lv[t];
                            if (gx + j == IW + t) G[j] = rv[t];
                        }
                }
            }
            // ---- pass 2, horizontal: the R2 G columns of each neighbour lane by shuffles
            const int i2 = H2RING ? (((i - 2 * R1) % P2) + P2) % P2 : P2 - 1;   // slot of this G row
            if (!H2RING) {
#pragma unroll
                for (int t = 0; t + 1 < P2; ++t)
#pragma unroll
                    for (int j = 0; j < PX; ++j) h2[t][j] = h2[t + 1][j];
            }
            {
                A v2[PX + 2 * R2];
#pragma unroll
                for (int j = 0; j < PX; ++j) v2[R2 + j] = G[j];
#pragma unroll
                for (int t = 0; t < R2; ++t) {
                    v2[t] = __shfl_up_sync(0xffffffffu, G[PX - R2 + t], 1);
                    v2[R2 + PX + t] = __shfl_down_sync(0xffffffffu, G[t], 1);
                }
#pragma unroll
                for (int j = 0; j < PX; ++j) h2[i2][j] = sep_h<A, R2>(p.s2, v2 + j);
            }
            if (k < 2 * (R1 + R2)) continue;
            // ---- pass 2, vertical: output row
            A out[PX];
#pragma unroll
            for (int j = 0; j < PX; ++j) {
                A col[P2];
#pragma unroll
                for (int t = 0; t < P2; ++t) col[t] = h2[H2RING ? (i2 + 1 + t) % P2 : t][j];   // rows o .. o + 2 R2
                out[j] = sep_v<A, R2>(p.s2, col);
            }
            if (ovec) store_row<TO, PX>(orow, ox, roi_x1, true, out, p.s2.shift);
            else if (!SIMPLE && out_lane) store_row_masked<TO, PX>(orow, ox, roi_x0, roi_x1, out, p.s2.shift);
            orow += c.out.stride;
        }
    }
    asm volatile("cp.async.wait_all;" ::: "memory");
}

template <typename T, typename TO, int R1, int R2>
__device__ __forceinline__ void chain_stream_warp(const ConvChain &p, int b, int w,
                                                  unsigned char *wsmem)
{
    using S = chain::SShape<T>;
    const Common &c = p.s1.c;
    const ChainPlan &pl = p.plan;
    const Geom &g = c.in;
    const int lane = threadIdx.x & 31;
    const int f = w % pl.nframes, seg = w / pl.nframes;
    ChainWarp cw;
    cw.y0 = pl.sy0 + seg * pl.T;
    if (seg >= pl.nseg || cw.y0 >= pl.sy1) return;               // warp-uniform
    const int y1 = min(cw.y0 + pl.T, pl.sy1);
    const int ox0 = pl.ox_base + f * S::OWS;       // output column of lane 1, element 0
    cw.gxb = ox0 + c.off_x - S::PX;                // input column of lane 0's first G column
    cw.ix0 = cw.gxb - S::PAD;                      // input column of smem column 0
    cw.ox = ox0 + S::PX * (lane - 1);
    cw.iy0 = cw.y0 + c.off_y - R2 - R1;
    cw.nsteps = (y1 - cw.y0) + 2 * (R1 + R2);
    cw.col_edge = cw.ix0 < 0 || cw.ix0 + S::SW > g.W;
    cw.rows_inside = cw.iy0 >= 0 && cw.iy0 + cw.nsteps <= g.H;
    // output columns partly outside the iteration space also take the general path
    const bool roi_inner = ox0 >= c.roi_x0 && ox0 + S::OWS <= c.roi_x0 + c.roi_w;
    if (cw.col_edge) {
        int *cm = reinterpret_cast<int *>(wsmem + S::RING_BYTES);
        for (int i = lane; i < S::SW; i += 32) {
            int col;
            cm[i] = resolve_col(cw.ix0 + i, g, c.mode, col) ? col : -1;
        }
        __syncwarp();
    }
    if (!cw.col_edge && cw.rows_inside && roi_inner)
        chain_stream_run<T, TO, R1, R2, true>(p, b, cw, wsmem);
    else
        chain_stream_run<T, TO, R1, R2, false>(p, b, cw, wsmem);
}

template <typename T, typename TO, int R1, int R2>
__global__ void __launch_bounds__(chain::NT) conv_chain_stream_kernel(const __grid_constant__ ConvChain p)
{
    extern __shared__ __align__(16) unsigned char smem_raw[];
    __shared__ __align__(8) uint64_t bar;
    const ChainPlan &pl = p.plan;
    const int b = blockIdx.z;
    if ((int)blockIdx.x < pl.stream_ctas) {                      // block-uniform
        const int warp = threadIdx.x >> 5;
        chain_stream_warp<T, TO, R1, R2>(p, b, blockIdx.x * chain::NW + warp,
                                         smem_raw + warp * chain::SShape<T>::WARP_BYTES);
        return;
    }
    const Common &c = p.s1.c;
    const int t = blockIdx.x - pl.stream_ctas;
    const int ty = t / pl.ntx, tx = t - ty * pl.ntx;
    const int tx0 = c.roi_x0 + tx * chain::Shape<T>::OW;
    int ty0, ry1;
    if (ty < pl.top_rows) { ty0 = c.roi_y0 + ty * chain::TSB; ry1 = pl.sy0; }
    else { ty0 = pl.sy1 + (ty - pl.top_rows) * chain::TSB; ry1 = c.roi_y0 + c.roi_h; }
    chain_tile<T, TO, R1, R2, chain::TSB>(p, b, tx0, ty0, ry1, smem_raw, bar);
}

namespace {

template <typename T, typename TO, int R1, int R2, int TS>
cudaError_t launch_chain_cfg(const ConvChain &p, cudaStream_t stream)
{
    using S = chain::Shape<T>;
    const size_t smem = (size_t)(TS + 2 * R1 + 2 * R2) * S::ISW * sizeof(T) +
                        (size_t)(TS + 2 * R2) * S::GW * sizeof(T);
    static PerDevice configured;
    const cudaError_t e = ensure_smem(conv_chain_kernel<T, TO, R1, R2, TS>, smem, configured);
    if (e != cudaSuccess) return e;
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

// Row-streaming launch (conv_chain_stream_kernel) when the geometry allows it:
// 16-B aligned input rows, chunk-aligned frames (W and off_x multiples of 16 B),
// outputs that read the image through their own column (roi + off_x inside the
// image, so every G column outside it is within R2 of an edge), images at least
// two frames wide and enough streamed rows.  Rows per warp T from the wave
// model of the pair kernel: cost(T) = waves(T) x (T + warm-up rows).
// T >= 16 (measured best).  Returns false when not selected or not eligible.
template <typename T, typename TO, int R1, int R2>
bool launch_chain_stream(const ConvChain &p0, cudaStream_t stream, cudaError_t &err)
{
    using S = chain::SShape<T>;
    // opt-in (LOP_CHAIN_STREAM=1): measured slower than the tile kernel on B200
    // (DESIGN.md §6 conv_chain, profiles/r01_session4/chain_stream.txt)
    const char *env = std::getenv("LOP_CHAIN_STREAM");
    if (!env || std::atoi(env) == 0) return false;
    const Common &c = p0.s1.c;
    const Geom &g = c.in;
    constexpr int V16 = S::V16;
    if (((reinterpret_cast<uintptr_t>(g.data) | (uintptr_t)g.stride | (uintptr_t)g.bstride) & 15) ||
        g.W % V16 || ((c.off_x % V16) + V16) % V16 || g.W < 2 * S::FW)
        return false;
    if (c.roi_x0 + c.off_x < 0 || c.roi_x0 + c.roi_w - 1 + c.off_x > g.W - 1) return false;
    const int sy0 = std::max(c.roi_y0, R2 - c.off_y);
    const int sy1 = std::min(c.roi_y0 + c.roi_h, g.GH - R2 - c.off_y);
    if (sy1 - sy0 < 16) return false;
    static PerDevice smem_set, resident_cache;
    constexpr size_t smem_stream = (size_t)chain::NW * S::WARP_BYTES;
    using TS = chain::Shape<T>;
    constexpr size_t smem_tile = (size_t)(chain::TSB + 2 * R1 + 2 * R2) * TS::ISW * sizeof(T) +
                                 (size_t)(chain::TSB + 2 * R2) * TS::GW * sizeof(T);
    constexpr size_t smem = smem_stream > smem_tile ? smem_stream : smem_tile;
    auto kern = conv_chain_stream_kernel<T, TO, R1, R2>;
    cudaError_t e;
    const int64_t resident = resident_ctas(kern, chain::NT, smem, smem_set, resident_cache, e);
    if (e == cudaSuccess) e = ensure_smem(kern, smem, smem_set);
    if (e != cudaSuccess) { err = e; return true; }
    ConvChain p = p0;
    ChainPlan &pl = p.plan;
    pl.sy0 = sy0;
    pl.sy1 = sy1;
    pl.ox_base = c.roi_x0 & ~(V16 - 1);
    pl.nframes = (c.roi_x0 + c.roi_w - pl.ox_base + S::OWS - 1) / S::OWS;
    const int rows = sy1 - sy0, warm = 2 * (R1 + R2);
    int tr = 0;
    if (const char *env = std::getenv("LOP_CHAIN_ROWS")) tr = std::atoi(env);
    if (tr <= 0) {
        double best = 0;
        for (int t = 16; t <= rows; ++t) {
            const int64_t segs = (rows + t - 1) / t;
            const int64_t ctas = (segs * pl.nframes + chain::NW - 1) / chain::NW * c.batch;
            const double cost = (double)((ctas + resident - 1) / resident) * (t + warm);
            if (tr == 0 || cost < best) { best = cost; tr = t; }
            if (segs == 1) break;
        }
        if (tr == 0) tr = rows;
    }
    pl.T = tr;
    pl.nseg = (rows + tr - 1) / tr;
    pl.stream_ctas = (pl.nseg * pl.nframes + chain::NW - 1) / chain::NW;
    pl.ntx = (c.roi_w + TS::OW - 1) / TS::OW;
    pl.top_rows = (sy0 - c.roi_y0 + chain::TSB - 1) / chain::TSB;
    pl.bot_rows = (c.roi_y0 + c.roi_h - sy1 + chain::TSB - 1) / chain::TSB;
    dim3 grid((unsigned)(pl.stream_ctas + pl.ntx * (pl.top_rows + pl.bot_rows)), 1, c.batch);
    kern<<<grid, chain::NT, smem, stream>>>(p);
    err = cudaGetLastError();
    return true;
}

template <typename T, typename TO, int R1, int R2>
cudaError_t launch_chain_any(const ConvChain &p, cudaStream_t stream)
{
    cudaError_t e = cudaSuccess;
    if (launch_chain_stream<T, TO, R1, R2>(p, stream, e)) return e;
    return launch_chain_rr<T, TO, R1, R2>(p, stream);
}

template <typename T, typename TO>
cudaError_t launch_chain_t(const ConvChain &p, cudaStream_t stream)
{
    const int r1 = p.s1.c.rx, r2 = p.s2.c.rx;
    if (r1 == 1 && r2 == 1) return launch_chain_any<T, TO, 1, 1>(p, stream);
    if (r1 == 1 && r2 == 2) return launch_chain_any<T, TO, 1, 2>(p, stream);
    if (r1 == 2 && r2 == 1) return launch_chain_any<T, TO, 2, 1>(p, stream);
    if (r1 == 2 && r2 == 2) return launch_chain_any<T, TO, 2, 2>(p, stream);
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

// pyramid.cu -- Laplacian-pyramid REDUCE / EXPAND kernels of the
// multiresolution filter ("a
// multiresolution filter (see [7]) is applied to an image: the image gets
// upsampled multiple times", with Mirror borders; reading c28 in DESIGN.md).
//   w = [1 4 6 4 1] / 16
//   REDUCE  G'(x, y) = sum_{i,j} w(i) w(j) Read_G(2x + i, 2y + j)
//   EXPAND  E(x, y)  = sum 4 w(i) w(j) Read_G'((x - i) / 2, (y - j) / 2)
//                      over even x - i, y - j; per axis the even phase is
//                      (g[u-1] + 6 g[u] + g[u+1]) / 8, the odd phase
//                      (g[u] + g[u+1]) / 2
//   out = addend + sign * E   (band-pass: sign -1; reconstruction: +1)
// Both are HBM-bound: a thread computes a 4 x 2 output block from its input
// footprint, loaded directly with vector loads (the footprints of
// neighbouring threads overlap by a few columns / rows; those re-reads hit L1),
// border threads per element with the boundary resolved (Table I); 16-byte
// stores.  Algorithmic bytes: REDUCE
// 4 B read per fine pixel + 4 B written per coarse pixel (5 B per fine
// pixel); EXPAND with an addend 4 B read + 4 B written per fine pixel + 4 B
// read per coarse pixel (9 B per fine pixel).
#include <cuda_runtime.h>
#include <stdint.h>

#include "boundary.cuh"
#include "kernels.h"
#include "lop_params.h"

namespace lop {

namespace pyr {
constexpr int BX = 32, BY = 8;                  // threads per CTA (x, y)
// EXPAND: a thread computes 4 fine columns x 2 fine rows (tile 128 x 16)
}  // namespace pyr

__device__ __forceinline__ float pyr_b5(float a, float b, float c, float d, float e)
{
    return __fmaf_rn(6.0f, c, __fmaf_rn(4.0f, b + d, a + e));     // binomial taps x 16
}

__device__ __forceinline__ bool pyr_vec_ok(const Geom &g, int b)
{
    return (g.stride & 15) == 0 && (reinterpret_cast<uintptr_t>(g.data + (int64_t)b * g.bstride) & 15) == 0;
}

// REDUCE.  Lane t of a warp owns coarse columns 2t, 2t + 1 of the warp's 64
// (fine columns 4t .. 4t + 3: one 16-byte load per fine row, a warp reads 512
// contiguous bytes) and streams 7 fine rows for 2 coarse rows; the two fine
// columns left and the one right of its quad are loaded by the lane too (L1
// hits), every load issued before the first use.  Per fine row the horizontal sums
// at the two even columns enter a 5-row register window; a coarse row is
// complete every second fine row.  CTAs whose footprint leaves the image (or
// an unaligned view) read every element through the boundary mode (Table I).
namespace pyr {
constexpr int RW = 32, RWARPS = 8, RROWS = 2;   // REDUCE: lanes, warps, coarse rows per warp
}

__global__ void __launch_bounds__(pyr::RW * pyr::RWARPS) pyr_reduce_kernel(const __grid_constant__ PyrParams p)
{
    const Geom &g = p.in;
    const int b = blockIdx.z;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int bx0 = blockIdx.x * 128;                                  // block's first fine column
    const int cy0 = (blockIdx.y * pyr::RWARPS + warp) * pyr::RROWS;    // warp's first coarse row
    const int by0 = 2 * blockIdx.y * pyr::RWARPS * pyr::RROWS - 2;     // block's first fine row
    const int fx = bx0 + 4 * lane, fy0 = 2 * cy0 - 2;
    const bool inside = bx0 - 2 >= 0 && bx0 + 130 <= g.W && by0 >= 0 &&
                        by0 + 2 * pyr::RWARPS * pyr::RROWS + 3 <= g.H && pyr_vec_ok(g, b);
    const int cx = fx / 2;                                             // first coarse column
    char *ob = p.out.data + (int64_t)b * p.out.bstride;
    const bool ovec = cx + 1 < p.out.W && (p.out.stride & 7) == 0 && (reinterpret_cast<uintptr_t>(ob) & 7) == 0;
    constexpr int NF = 2 * pyr::RROWS + 3;                            // fine rows per warp
    // all of the warp's row loads are issued before any is used (7 x 512 B in
    // flight per warp; a load-use chain per row left the kernel latency-bound)
    // the two columns left and the one right of the quad are loaded by every lane
    // as well (L1 hits: the neighbouring lanes' quads), all before the first use --
    // the edge lanes' loads are no longer a dependent round trip per row
    float4 qs[NF];
    float2 ls[NF];
    float rs[NF];
    if (inside) {
#pragma unroll
        for (int i = 0; i < NF; ++i) {
            const float *rp = row_ptr<float>(g, b, fy0 + i) + fx;
            qs[i] = __ldg(reinterpret_cast<const float4 *>(rp));
            ls[i] = __ldg(reinterpret_cast<const float2 *>(rp - 2));
            rs[i] = __ldg(rp + 4);
        }
    }
    // border CTAs: the 7 columns of the lane resolved once (Table I; -1 = the
    // CONSTANT value), each row resolved once per row
    int cols[7];
    if (!inside) {
#pragma unroll
        for (int k = 0; k < 7; ++k) cols[k] = resolve_col(fx - 2 + k, g, p.mode, cols[k]) ? cols[k] : -1;
    }
    float w0[5], w1[5];                                                // last 5 rows' sums (even cols)
#pragma unroll
    for (int i = 0; i < NF; ++i) {
        const int fy = fy0 + i;
        float f[7];                                                    // fine columns fx - 2 .. fx + 4
        if (inside) {
            const float4 q = qs[i];
            f[0] = ls[i].x; f[1] = ls[i].y; f[2] = q.x; f[3] = q.y; f[4] = q.z; f[5] = q.w; f[6] = rs[i];
        } else {
            int row;
            const bool row_ok = resolve_row(fy, g, p.mode, row);
            const float *rp = row_ok ? row_ptr<float>(g, b, row) : nullptr;
#pragma unroll
            for (int k = 0; k < 7; ++k) f[k] = row_ok && cols[k] >= 0 ? __ldg(rp + cols[k]) : p.cval;
        }
#pragma unroll
        for (int k = 0; k < 4; ++k) { w0[k] = w0[k + 1]; w1[k] = w1[k + 1]; }
        w0[4] = pyr_b5(f[0], f[1], f[2], f[3], f[4]);
        w1[4] = pyr_b5(f[2], f[3], f[4], f[5], f[6]);
        if (i >= 4 && (i & 1) == 0) {                                  // coarse row cy0 + (i - 4) / 2
            const int oy = cy0 + (i - 4) / 2;
            if (oy < p.out.H && cx < p.out.W) {
                const float v0 = pyr_b5(w0[0], w0[1], w0[2], w0[3], w0[4]) * (1.0f / 256.0f);
                const float v1 = pyr_b5(w1[0], w1[1], w1[2], w1[3], w1[4]) * (1.0f / 256.0f);
                float *orow = reinterpret_cast<float *>(ob + (int64_t)oy * p.out.stride);
                if (ovec) {
                    *reinterpret_cast<float2 *>(orow + cx) = make_float2(v0, v1);
                } else {
                    orow[cx] = v0;
                    if (cx + 1 < p.out.W) orow[cx + 1] = v1;
                }
            }
        }
    }
}

// EXPAND (+ addend).  Coarse footprint of the thread: rows gy - 1 .. gy + 1,
// columns 2 gx - 1 .. 2 gx + 2 (direct loads, L1 absorbs the overlap; border
// threads per element with the mode resolved).  Per coarse row the 4 fine
// columns' phases, then the 2 fine rows' phases; the addend rows are loaded
// before the arithmetic (they do not depend on it).
__global__ void __launch_bounds__(pyr::BX * pyr::BY) pyr_expand_kernel(const __grid_constant__ PyrParams p)
{
    const Geom &g = p.in;
    const int b = blockIdx.z;
    const int gx = blockIdx.x * pyr::BX + threadIdx.x, gy = blockIdx.y * pyr::BY + threadIdx.y;
    const int x0 = 4 * gx, y0 = 2 * gy;                           // first fine output
    if (x0 >= p.out.W || y0 >= p.out.H) return;
    char *ob = p.out.data + (int64_t)b * p.out.bstride;
    const bool ovec = x0 + 3 < p.out.W && (p.out.stride & 15) == 0 && (reinterpret_cast<uintptr_t>(ob) & 15) == 0 &&
                      (!p.add || ((p.add_stride & 15) == 0 &&
                                  (reinterpret_cast<uintptr_t>(p.add + (int64_t)b * p.add_bstride) & 15) == 0));
    const int ny = min(2, p.out.H - y0);
    float add[2][4] = {{0.f, 0.f, 0.f, 0.f}, {0.f, 0.f, 0.f, 0.f}};
    if (p.add) {
#pragma unroll
        for (int j = 0; j < 2; ++j) {
            if (j >= ny) break;
            const float *arow = reinterpret_cast<const float *>(p.add + (int64_t)b * p.add_bstride +
                                                                (int64_t)(y0 + j) * p.add_stride);
            if (ovec) {
                const float4 a = *reinterpret_cast<const float4 *>(arow + x0);   // may alias the output
                add[j][0] = a.x; add[j][1] = a.y; add[j][2] = a.z; add[j][3] = a.w;
            } else {
#pragma unroll
                for (int k = 0; k < 4; ++k)
                    if (x0 + k < p.out.W) add[j][k] = arow[x0 + k];
            }
        }
    }
    const int u0 = 2 * gx - 1, v0 = gy - 1;                       // coarse footprint origin
    const bool inside = u0 >= 0 && u0 + 3 < g.W && v0 >= 0 && v0 + 2 < g.H && (g.stride & 7) == 0 &&
                        (reinterpret_cast<uintptr_t>(g.data + (int64_t)b * g.bstride) & 7) == 0;
    int cols[4];                                                  // border threads: resolved columns
    if (!inside) {
#pragma unroll
        for (int k = 0; k < 4; ++k) cols[k] = resolve_col(u0 + k, g, p.mode, cols[k]) ? cols[k] : -1;
    }
    float h[3][4];
#pragma unroll
    for (int r = 0; r < 3; ++r) {
        float c[4];                                               // coarse u0 .. u0 + 3
        if (inside) {
            const float *rp = row_ptr<float>(g, b, v0 + r) + u0 - 1;   // 8-byte aligned (u0 - 1 even)
            const float2 a = __ldg(reinterpret_cast<const float2 *>(rp));
            const float2 m = __ldg(reinterpret_cast<const float2 *>(rp + 2));
            c[0] = a.y; c[1] = m.x; c[2] = m.y; c[3] = __ldg(rp + 4);
        } else {
            int row;
            const bool row_ok = resolve_row(v0 + r, g, p.mode, row);
            const float *rp = row_ok ? row_ptr<float>(g, b, row) : nullptr;
#pragma unroll
            for (int k = 0; k < 4; ++k) c[k] = row_ok && cols[k] >= 0 ? __ldg(rp + cols[k]) : p.cval;
        }
        h[r][0] = 0.125f * __fmaf_rn(6.0f, c[1], c[0] + c[2]);   // x = 4 gx     (even)
        h[r][1] = 0.5f * (c[1] + c[2]);                            // x = 4 gx + 1 (odd)
        h[r][2] = 0.125f * __fmaf_rn(6.0f, c[2], c[1] + c[3]);   // x = 4 gx + 2 (even)
        h[r][3] = 0.5f * (c[2] + c[3]);                            // x = 4 gx + 3 (odd)
    }
#pragma unroll
    for (int j = 0; j < 2; ++j) {
        if (j >= ny) break;
        float v[4];
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            const float e = j == 0 ? 0.125f * __fmaf_rn(6.0f, h[1][k], h[0][k] + h[2][k])   // even row
                                   : 0.5f * (h[1][k] + h[2][k]);                            // odd row
            v[k] = p.add ? add[j][k] + p.sign * e : p.sign * e;
        }
        float *orow = reinterpret_cast<float *>(ob + (int64_t)(y0 + j) * p.out.stride);
        if (ovec) {
            *reinterpret_cast<float4 *>(orow + x0) = make_float4(v[0], v[1], v[2], v[3]);
        } else {
#pragma unroll
            for (int k = 0; k < 4; ++k)
                if (x0 + k < p.out.W) orow[x0 + k] = v[k];
        }
    }
}

cudaError_t launch_pyr_reduce(const PyrParams &p, cudaStream_t stream)
{
    dim3 grid((p.out.W + 63) / 64, (p.out.H + pyr::RWARPS * pyr::RROWS - 1) / (pyr::RWARPS * pyr::RROWS), p.batch);
    pyr_reduce_kernel<<<grid, pyr::RW * pyr::RWARPS, 0, stream>>>(p);
    return cudaGetLastError();
}

cudaError_t launch_pyr_expand(const PyrParams &p, cudaStream_t stream)
{
    dim3 grid((p.out.W + 4 * pyr::BX - 1) / (4 * pyr::BX), (p.out.H + 2 * pyr::BY - 1) / (2 * pyr::BY), p.batch);
    pyr_expand_kernel<<<grid, dim3(pyr::BX, pyr::BY), 0, stream>>>(p);
    return cudaGetLastError();
}

}  // namespace lop

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
// Both are HBM-bound: a CTA stages its input footprint once into shared
// memory (interior tiles by 16-byte cp.async, border tiles per element with
// the boundary resolved at staging time, Table I), runs the separable passes
// from shared memory and writes coalesced rows.  Algorithmic bytes: REDUCE
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
constexpr int NT = 256;
constexpr int TX = 64, TY = 16;                 // output tile (both kernels)
// REDUCE: fine footprint columns 2 tx0 - 4 .. 2 tx0 + 2 TX + 3 (aligned to 4),
// rows 2 ty0 - 2 .. 2 ty0 + 2 TY + 2
constexpr int RSW = 2 * TX + 8, RSH = 2 * TY + 3;
// EXPAND: coarse footprint columns tx0/2 - 4 .. tx0/2 + TX/2 + 3, rows
// ty0/2 - 1 .. ty0/2 + TY/2
constexpr int ESW = TX / 2 + 8, ESH = TY / 2 + 2;
}  // namespace pyr

__device__ __forceinline__ void pyr_cp16(float *dst, const float *src)
{
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_addr(dst)), "l"(src) : "memory");
}

// Stage rows iy0 .. iy0 + nh - 1, columns ix0 .. ix0 + nw - 1 (nw a multiple
// of 4, ix0 a multiple of 4) of frame b into t (pitch nw): whole interior
// 16-byte chunks asynchronously, everything else per element (Table I).
__device__ __forceinline__ void pyr_stage(const PyrParams &p, int b, int ix0, int iy0, int nw, int nh,
                                          float *t)
{
    const Geom &g = p.in;
    const bool vec = (g.stride & 15) == 0 && (reinterpret_cast<uintptr_t>(g.data + (int64_t)b * g.bstride) & 15) == 0;
    const int nv = nw / 4;
    for (int i = threadIdx.x; i < nh * nv; i += pyr::NT) {
        const int r = i / nv, q = i - r * nv;
        const int iy = iy0 + r, ix = ix0 + 4 * q;
        float *d = t + r * nw + 4 * q;
        if (vec && iy >= 0 && iy < g.H && ix >= 0 && ix + 3 < g.W) {
            pyr_cp16(d, row_ptr<float>(g, b, iy) + ix);
        } else {
#pragma unroll
            for (int k = 0; k < 4; ++k) d[k] = read_f32(g, b, ix + k, iy, p.mode, p.cval);
        }
    }
    asm volatile("cp.async.commit_group;\n\tcp.async.wait_all;" ::: "memory");
}

__global__ void __launch_bounds__(pyr::NT) pyr_reduce_kernel(const __grid_constant__ PyrParams p)
{
    __shared__ __align__(16) float s[pyr::RSH * pyr::RSW];
    __shared__ float h[pyr::RSH * pyr::TX];
    const int b = blockIdx.z;
    const int tx0 = blockIdx.x * pyr::TX, ty0 = blockIdx.y * pyr::TY;
    pyr_stage(p, b, 2 * tx0 - 4, 2 * ty0 - 2, pyr::RSW, pyr::RSH, s);
    __syncthreads();
    // horizontal: h[r][x] = sum_i w(i) s[r][2x + i] around fine column 2 (tx0 + x)
    for (int i = threadIdx.x; i < pyr::RSH * pyr::TX; i += pyr::NT) {
        const int r = i / pyr::TX, x = i - r * pyr::TX;
        const float *q = s + r * pyr::RSW + 2 * x + 2;          // fine column 2 (tx0 + x) - 2
        h[i] = __fmaf_rn(6.0f, q[2], __fmaf_rn(4.0f, q[1] + q[3], q[0] + q[4]));
    }
    __syncthreads();
    const int x = threadIdx.x & (pyr::TX - 1);
    const int ox = tx0 + x;
    if (ox >= p.out.W) return;
#pragma unroll
    for (int k = 0; k < pyr::TY / (pyr::NT / pyr::TX); ++k) {
        const int y = (threadIdx.x / pyr::TX) + k * (pyr::NT / pyr::TX);
        const int oy = ty0 + y;
        if (oy >= p.out.H) break;
        const float *q = h + 2 * y * pyr::TX + x;                // staged row 2y = fine row 2 oy - 2
        const float v = __fmaf_rn(6.0f, q[2 * pyr::TX],
                                  __fmaf_rn(4.0f, q[pyr::TX] + q[3 * pyr::TX], q[0] + q[4 * pyr::TX]));
        float *orow = reinterpret_cast<float *>(p.out.data + (int64_t)b * p.out.bstride + (int64_t)oy * p.out.stride);
        orow[ox] = v * (1.0f / 256.0f);
    }
}

__global__ void __launch_bounds__(pyr::NT) pyr_expand_kernel(const __grid_constant__ PyrParams p)
{
    __shared__ __align__(16) float s[pyr::ESH * pyr::ESW];
    __shared__ float h[pyr::ESH * pyr::TX];
    const int b = blockIdx.z;
    const int tx0 = blockIdx.x * pyr::TX, ty0 = blockIdx.y * pyr::TY;
    const int cx0 = tx0 / 2 - 4, cy0 = ty0 / 2 - 1;             // coarse origin of the footprint
    pyr_stage(p, b, cx0, cy0, pyr::ESW, pyr::ESH, s);
    __syncthreads();
    // horizontal: fine column x = tx0 + xl, u = x / 2 (coarse, smem column u - cx0)
    for (int i = threadIdx.x; i < pyr::ESH * pyr::TX; i += pyr::NT) {
        const int r = i / pyr::TX, xl = i - r * pyr::TX;
        const float *q = s + r * pyr::ESW + (xl >> 1) + 4;       // coarse u = tx0/2 + xl/2
        h[i] = (xl & 1) ? 0.5f * (q[0] + q[1]) : 0.125f * __fmaf_rn(6.0f, q[0], q[-1] + q[1]);
    }
    __syncthreads();
    const int xl = threadIdx.x & (pyr::TX - 1);
    const int ox = tx0 + xl;
    if (ox >= p.out.W) return;
#pragma unroll
    for (int k = 0; k < pyr::TY / (pyr::NT / pyr::TX); ++k) {
        const int yl = (threadIdx.x / pyr::TX) + k * (pyr::NT / pyr::TX);
        const int oy = ty0 + yl;
        if (oy >= p.out.H) break;
        const float *q = h + ((yl >> 1) + 1) * pyr::TX + xl;    // coarse row ty0/2 + yl/2
        const float e = (yl & 1) ? 0.5f * (q[0] + q[pyr::TX])
                                 : 0.125f * __fmaf_rn(6.0f, q[0], q[-pyr::TX] + q[pyr::TX]);
        float *orow = reinterpret_cast<float *>(p.out.data + (int64_t)b * p.out.bstride + (int64_t)oy * p.out.stride);
        float v = p.sign * e;
        if (p.add) {
            const float *arow = reinterpret_cast<const float *>(p.add + (int64_t)b * p.add_bstride +
                                                                (int64_t)oy * p.add_stride);
            v = arow[ox] + v;                                     // may alias orow (in place)
        }
        orow[ox] = v;
    }
}

cudaError_t launch_pyr_reduce(const PyrParams &p, cudaStream_t stream)
{
    dim3 grid((p.out.W + pyr::TX - 1) / pyr::TX, (p.out.H + pyr::TY - 1) / pyr::TY, p.batch);
    pyr_reduce_kernel<<<grid, pyr::NT, 0, stream>>>(p);
    return cudaGetLastError();
}

cudaError_t launch_pyr_expand(const PyrParams &p, cudaStream_t stream)
{
    dim3 grid((p.out.W + pyr::TX - 1) / pyr::TX, (p.out.H + pyr::TY - 1) / pyr::TY, p.batch);
    pyr_expand_kernel<<<grid, pyr::NT, 0, stream>>>(p);
    return cudaGetLastError();
}

}  // namespace lop

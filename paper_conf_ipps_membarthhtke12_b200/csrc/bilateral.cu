// bilateral.cu -- bilateral filter kernels for sm_100a.
//
// Method: Algorithm 1 with the precomputed closeness
// Mask of Listing 5 (L379-L416): one exp per tap, p/d normalisation.
// B200 design:
//  * bilateral_generic: one thread per output pixel, per-tap boundary
//    resolution, mask in the (large) kernel parameter block.  Any window up
//    to 63x63.  Reference-quality fallback and the cross-check for the tiled
//    kernel (bit-identical arithmetic via lop::bilateral_tap).
//  * bilateral_tiled<RX>: the hot kernel.  A CTA owns a 128 x 32 output tile;
//    the tile plus its (2RX+1)x(2RY+1) halo is staged once into shared memory
//    with boundary handling resolved at staging time (interior tiles take an
//    unchecked 128-bit path -- the paper's nine-region idea, Fig. 3 /
//    Listing 8, reduced to interior vs border CTAs).  Each thread owns 4
//    horizontally adjacent outputs, reads its window rows with 128-bit LDS
//    and the log2 mask row with broadcast LDS, and issues one MUFU.EX2 per
//    tap (ex2.approx.ftz) with the closeness folded into the exponent.
//    The kernel is SFU-bound by construction.
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
    // centre Input(): the pixel itself (always inside the image for offset 0;
    // for offset accessors it is read through the boundary condition too)
    const float centre = read_f32(c.in, b, ix, iy, c.mode, c.cval_f);
    const int sx = 2 * c.rx + 1;
    float d = 0.0f, pacc = 0.0f;
    for (int yf = -c.ry; yf <= c.ry; ++yf) {
        int row;
        const bool row_ok = resolve_row(iy + yf, c.in, c.mode, row);
        const float *rp = row_ok ? row_ptr<float>(c.in, b, row) : nullptr;
        const float *lc = p.lc + (yf + c.ry) * sx + c.rx;
        for (int xf = -c.rx; xf <= c.rx; ++xf) {
            int col;
            float v = c.cval_f;
            if (row_ok && resolve_col(ix + xf, c.in, c.mode, col)) v = __ldg(rp + col);
            bilateral_tap(v, centre, lc[xf], p.nk, d, pacc);
        }
    }
    float *orow = reinterpret_cast<float *>(c.out.data + (int64_t)b * c.out.bstride +
                                            (int64_t)oy * c.out.stride);
    orow[ox] = bilateral_finish(d, pacc);
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

__host__ __device__ inline int smem_rows(int ry) { return TH + 2 * ry; }
}  // namespace tiled

template <int RX>
__global__ void __launch_bounds__(tiled::NT, 4) bilateral_tiled_kernel(const __grid_constant__ BilateralTiled p)
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
    const int ix0 = tx0 + c.off_x - PAD;                       // input coords of smem (0,0)
    const int iy0 = ty0 + c.off_y - ry;
    const Geom &g = c.in;

    // ---- stage the mask (log2 closeness), rows padded to 4*MV floats
    for (int i = threadIdx.x; i < (2 * ry + 1) * 4 * MV; i += NT) {
        const int r = i / (4 * MV), k = i - r * (4 * MV);
        msk[i] = k < 2 * RX + 1 ? p.lc[r * kTiledMaskPitch + k] : 0.0f;
    }

    // ---- stage tile + halo; boundary handling resolved here (§8(a) a2/a3).
    // Only the rows this tile's outputs need are staged (a partial last tile
    // must not touch rows beyond the validated band + halo).
    const int roi_y1 = c.roi_y0 + c.roi_h;
    const int SHn = min(TH, roi_y1 - ty0) + 2 * ry;
    const int gy_lo = iy0 + g.gy0;
    const bool interior = ix0 >= 0 && ix0 + SW <= g.W && gy_lo >= 0 && gy_lo + SHn <= g.GH;
    const char *fbase = g.data + (int64_t)b * g.bstride;
    if (interior && ((ix0 & 3) == 0) && ((g.stride & 15) == 0) &&
        ((reinterpret_cast<uintptr_t>(fbase) & 15) == 0)) {
        constexpr int V = SW / 4;                               // float4 per smem row
        for (int i = threadIdx.x; i < SHn * V; i += NT) {
            const int r = i / V, v = i - r * V;
            const float4 *src = reinterpret_cast<const float4 *>(
                fbase + (int64_t)(iy0 + r) * g.stride) + (ix0 >> 2) + v;
            smem4[r * V + v] = __ldg(src);
        }
    } else if (interior) {
        for (int i = threadIdx.x; i < SHn * SW; i += NT) {
            const int r = i / SW, x = i - r * SW;
            tile[i] = __ldg(reinterpret_cast<const float *>(fbase + (int64_t)(iy0 + r) * g.stride) +
                            ix0 + x);
        }
    } else {
        for (int i = threadIdx.x; i < SHn * SW; i += NT) {
            const int r = i / SW, x = i - r * SW;
            tile[i] = read_f32(g, b, ix0 + x, iy0 + r, c.mode, c.cval_f);
        }
    }
    __syncthreads();

    // ---- window reduction: 4 outputs per thread, yf rolled, xf unrolled
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int x_out = tx0 + 4 * lane;
    const int roi_x1 = c.roi_x0 + c.roi_w;
    const float nk = p.nk;
    for (int r = warp; r < TH; r += NT / 32) {
        const int oy = ty0 + r;
        if (oy >= roi_y1) break;
        const float4 cen4 = smem4[((r + ry) * SW + PAD) / 4 + lane];
        const float cen[4] = {cen4.x, cen4.y, cen4.z, cen4.w};
        float d[4] = {0.f, 0.f, 0.f, 0.f}, pp[4] = {0.f, 0.f, 0.f, 0.f};
        const float4 *rowv = smem4 + (r * SW) / 4 + lane;
        const float4 *mrow = reinterpret_cast<const float4 *>(msk);
#pragma unroll 1
        for (int yf = 0; yf <= 2 * ry; ++yf) {
            float v[4 * NV];
#pragma unroll
            for (int k = 0; k < NV; ++k) {
                const float4 q = rowv[yf * (SW / 4) + k];
                v[4 * k + 0] = q.x; v[4 * k + 1] = q.y; v[4 * k + 2] = q.z; v[4 * k + 3] = q.w;
            }
            float m[4 * MV];
#pragma unroll
            for (int k = 0; k < MV; ++k) {
                const float4 q = mrow[yf * MV + k];
                m[4 * k + 0] = q.x; m[4 * k + 1] = q.y; m[4 * k + 2] = q.z; m[4 * k + 3] = q.w;
            }
#pragma unroll
            for (int xf = 0; xf <= 2 * RX; ++xf)
#pragma unroll
                for (int j = 0; j < 4; ++j)
                    bilateral_tap(v[S::VOFF + xf + j], cen[j], m[xf], nk, d[j], pp[j]);
        }
        float res[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) res[j] = bilateral_finish(d[j], pp[j]);
        float *orow = reinterpret_cast<float *>(c.out.data + (int64_t)b * c.out.bstride +
                                                (int64_t)oy * c.out.stride);
        if (x_out + 3 < roi_x1 && ((x_out & 3) == 0) && ((c.out.stride & 15) == 0) &&
            ((reinterpret_cast<uintptr_t>(c.out.data + (int64_t)b * c.out.bstride) & 15) == 0)) {
            *reinterpret_cast<float4 *>(orow + x_out) = make_float4(res[0], res[1], res[2], res[3]);
        } else {
#pragma unroll
            for (int j = 0; j < 4; ++j)
                if (x_out + j < roi_x1) orow[x_out + j] = res[j];
        }
    }
}

template <int RX>
static cudaError_t launch_tiled_rx(const BilateralTiled &p, cudaStream_t stream)
{
    using S = tiled::Shape<RX>;
    const size_t smem = (size_t)(tiled::smem_rows(p.c.ry) * S::SW + (2 * p.c.ry + 1) * 4 * S::MV) *
                        sizeof(float);
    static size_t configured = 0;
    if (smem > 48 * 1024 && smem > configured) {
        cudaError_t e = cudaFuncSetAttribute(bilateral_tiled_kernel<RX>,
                                             cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
        configured = smem;
    }
    dim3 grid((p.c.roi_w + tiled::TW - 1) / tiled::TW, (p.c.roi_h + tiled::TH - 1) / tiled::TH,
              p.c.batch);
    bilateral_tiled_kernel<RX><<<grid, tiled::NT, smem, stream>>>(p);
    return cudaGetLastError();
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

}  // namespace lop

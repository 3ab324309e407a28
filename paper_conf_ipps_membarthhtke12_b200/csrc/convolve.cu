// convolve.cu -- local operators with a filter mask (Gaussian, Sobel, any odd
// mask): PAPER.md L274-L282 (window (2m+1)x(2n+1) centred at [0,0]),
// Listing 5 / Listing 9 (Mask(xf,yf) * Input(xf,yf): correlation, reading c5),
// Tables VIII-IX (Gaussian 3x3 / 5x5; Sobel "same implementation", L847-L849).
//
//  * conv_generic: one thread per output pixel, per-tap boundary resolution,
//    mask in the kernel parameter block.  Any odd window up to 63x63.
//  * conv_tiled (conv_tiled.cu): the HBM-bound hot kernels.
#include <cuda_runtime.h>
#include <stdint.h>

#include "boundary.cuh"
#include "lop_params.h"

namespace lop {

__global__ void __launch_bounds__(256) conv_generic_kernel(const __grid_constant__ ConvGeneric p)
{
    const Common &c = p.c;
    const int ox = c.roi_x0 + blockIdx.x * blockDim.x + threadIdx.x;
    const int oy = c.roi_y0 + blockIdx.y * blockDim.y + threadIdx.y;
    const int b = blockIdx.z;
    if (ox >= c.roi_x0 + c.roi_w || oy >= c.roi_y0 + c.roi_h) return;
    const int ix = ox + c.off_x, iy = oy + c.off_y;
    const int sx = 2 * c.rx + 1;
    char *obase = c.out.data + (int64_t)b * c.out.bstride + (int64_t)oy * c.out.stride;
    if (p.kind == CONV_F32) {
        float acc = 0.0f;
        for (int yf = -c.ry; yf <= c.ry; ++yf) {
            int row;
            const bool row_ok = resolve_row(iy + yf, c.in, c.mode, row);
            const float *rp = row_ok ? row_ptr<float>(c.in, b, row) : nullptr;
            const float *m = p.m.f + (yf + c.ry) * sx + c.rx;
            for (int xf = -c.rx; xf <= c.rx; ++xf) {
                int col;
                float v = c.cval_f;
                if (row_ok && resolve_col(ix + xf, c.in, c.mode, col)) v = __ldg(rp + col);
                acc = __fmaf_rn(m[xf], v, acc);
            }
        }
        reinterpret_cast<float *>(obase)[ox] = acc;
    } else {
        int acc = 0;
        for (int yf = -c.ry; yf <= c.ry; ++yf) {
            int row;
            const bool row_ok = resolve_row(iy + yf, c.in, c.mode, row);
            const uint8_t *rp = row_ok ? row_ptr<uint8_t>(c.in, b, row) : nullptr;
            const int *m = p.m.i + (yf + c.ry) * sx + c.rx;
            for (int xf = -c.rx; xf <= c.rx; ++xf) {
                int col;
                int v = c.cval_i;
                if (row_ok && resolve_col(ix + xf, c.in, c.mode, col)) v = __ldg(rp + col);
                acc += m[xf] * v;
            }
        }
        const int q = quantize_shift(acc, p.shift);
        if (p.kind == CONV_U8_U8)
            reinterpret_cast<uint8_t *>(obase)[ox] = (uint8_t)min(max(q, 0), 255);
        else
            reinterpret_cast<int32_t *>(obase)[ox] = q;
    }
}

cudaError_t launch_conv_generic(const ConvGeneric &p, cudaStream_t stream)
{
    dim3 block(32, 8, 1);
    dim3 grid((p.c.roi_w + 31) / 32, (p.c.roi_h + 7) / 8, p.c.batch);
    conv_generic_kernel<<<grid, block, 0, stream>>>(p);
    return cudaGetLastError();
}

}  // namespace lop

// stage.cuh -- staging of an input footprint into shared memory (SURVEY §8(a)
// a2/a3), shared by the convolution kernels: every staged row whose source row
// exists (in-image, halo, or mapped by the boundary mode) is copied by one
// cp.async.bulk (TMA bulk engine, SASS UBLKCP) of its 16-B aligned in-image
// column span, completing on `bar` (thread 0 arms it with the byte count; a
// count of 0 completes at once); the out-of-image columns and CONSTANT rows
// are filled element by element with the boundary resolved per column
// (visible after the caller's __syncthreads).
#pragma once
#include <stdint.h>

#include "boundary.cuh"

namespace lop {

// rows [iy0, iy0 + srows) x columns [ix0, ix0 + SWE) of frame b -> tile
// (row pitch SWE elements); NT threads participate.
// Only columns [0, ncols) are staged (ncols <= SWE; the rest of each smem row
// is left untouched for callers whose tile extends past the needed range).
template <typename T, int SWE, int NT>
__device__ __forceinline__ void stage_rows(const Common &c, int b, int ix0, int iy0, int srows,
                                           T *tile, uint64_t *bar, int ncols = SWE)
{
    constexpr bool F = sizeof(T) == 4;
    const Geom &g = c.in;
    const char *fbase = g.data + (int64_t)b * g.bstride;
    const T cval = F ? (T)c.cval_f : (T)c.cval_i;
    const bool aligned = ((reinterpret_cast<uintptr_t>(fbase) | (uintptr_t)g.stride |
                           (uintptr_t)(ix0 * (int)sizeof(T))) % 16 == 0);
    constexpr int V16 = 16 / sizeof(T);                            // elements per 16 B
    int xa = max(0, -ix0), xb = min(ncols, g.W - ix0);             // bulk span, smem columns
    xa = (xa + V16 - 1) / V16 * V16;
    xb = xb / V16 * V16;
    const bool bulk = aligned && xb > xa;
    if (threadIdx.x == 0) {
        int nbytes = 0;
        if (bulk)
            for (int r = 0; r < srows; ++r) {
                int row;
                if (resolve_row(iy0 + r, g, c.mode, row)) nbytes += (xb - xa) * (int)sizeof(T);
            }
        asm volatile("mbarrier.arrive.expect_tx.shared.b64 _, [%0], %1;"
                     ::"r"(smem_addr(bar)), "r"(nbytes) : "memory");
    }
    if (bulk) {
        for (int r = threadIdx.x; r < srows; r += NT) {
            int row;
            if (!resolve_row(iy0 + r, g, c.mode, row)) continue;
            const char *src = fbase + (int64_t)row * g.stride + (int64_t)(ix0 + xa) * sizeof(T);
            asm volatile(
                "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                ::"r"(smem_addr(tile + r * SWE + xa)), "l"(src), "r"((xb - xa) * (int)sizeof(T)),
                  "r"(smem_addr(bar))
                : "memory");
        }
    }
    // element-wise part: the columns outside the bulk span of every row ...
    const int side = bulk ? xa + (ncols - xb) : ncols;
    for (int i = threadIdx.x; i < srows * side; i += NT) {
        const int r = i / side, k = i - r * side;
        const int x = !bulk ? k : (k < xa ? k : xb + (k - xa));
        int row, col;
        T v;
        if (resolve_row(iy0 + r, g, c.mode, row) && resolve_col(ix0 + x, g, c.mode, col))
            v = __ldg(row_ptr<T>(g, b, row) + col);
        else
            v = cval;
        tile[r * SWE + x] = v;
    }
    // ... and the bulk span of CONSTANT rows (no source row to copy)
    if (bulk && c.mode == M_CONSTANT) {
        for (int r = 0; r < srows; ++r) {
            int row;
            if (resolve_row(iy0 + r, g, c.mode, row)) continue;
            for (int x = xa + threadIdx.x; x < xb; x += NT) tile[r * SWE + x] = cval;
        }
    }
}

}  // namespace lop

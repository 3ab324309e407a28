// select.cpp -- Algorithm 2 of the paper (§V-C
// L640-L689): the kernel-configuration / tiling heuristic, on B200 terms.
//
// The paper's source-to-source compiler enumerates configurations (threads
// per block) that are multiples of the SIMD width, keeps those within the
// device's resource limits, sorts them by occupancy, and -- when the kernel
// has border handling -- picks among the highest-occupancy ones the tiling
// with the fewest threads executing border-handling code, preferring tall
// (y) tilings; without border handling the highest-occupancy configuration
// with an x-preferred tiling.  Here the occupancy comes from
// cudaOccupancyMaxActiveBlocksPerMultiprocessor (the caller), the border
// threads from the launch geometry: a CTA executes border handling iff its
// tile footprint (tile + window radii) leaves the image -- exactly the CTAs
// that take the per-element staging path in the tiled kernels (boundary
// resolved at staging time, interior CTAs unchecked), i.e. the B200 form of
// the paper's nine-region kernels (Fig. 3, Listing 8).
#include <algorithm>
#include <vector>

#include "lop.h"
#include "select.h"

namespace lop {

// CTAs of a (tw x th)-output tiling of a width x height image whose
// footprint [x0 - rx, x0 + tw - 1 + rx] x [y0 - ry, y0 + th - 1 + ry] leaves
// the image, times the threads per CTA.
int64_t border_threads(int64_t width, int64_t height, int64_t tw, int64_t th, int64_t rx,
                       int64_t ry, int64_t threads)
{
    if (tw <= 0 || th <= 0 || width <= 0 || height <= 0) return 0;
    const int64_t ntx = (width + tw - 1) / tw, nty = (height + th - 1) / th;
    auto border_1d = [](int64_t n, int64_t t, int64_t ext, int64_t r) {
        int64_t b = 0;
        for (int64_t i = 0; i < n; ++i)
            if (i * t - r < 0 || (i + 1) * t - 1 + r > ext - 1) ++b;
        return b;
    };
    const int64_t bx = border_1d(ntx, tw, width, rx), by = border_1d(nty, th, height, ry);
    const int64_t border_ctas = ntx * nty - (ntx - bx) * (nty - by);
    return border_ctas * threads;
}

int alg2_select(const lop_config_candidate *cand, int n, int simd, int width, int height, int rx,
                int ry, int64_t *bh_out)
{
    // lines 1-3: multiples of the SIMD width, within resource limits; sort by
    // descending occupancy, ascending threads (stable: list order breaks ties)
    std::vector<int> C;
    for (int i = 0; i < n; ++i) {
        const int64_t thr = (int64_t)cand[i].block_x * cand[i].block_y;
        if (cand[i].valid && thr > 0 && simd > 0 && thr % simd == 0) C.push_back(i);
    }
    if (C.empty()) return -1;
    std::stable_sort(C.begin(), C.end(), [&](int a, int b) {
        if (cand[a].occupancy != cand[b].occupancy) return cand[a].occupancy > cand[b].occupancy;
        return (int64_t)cand[a].block_x * cand[a].block_y < (int64_t)cand[b].block_x * cand[b].block_y;
    });
    auto bh = [&](int i) {
        const lop_config_candidate &c = cand[i];
        return border_threads(width, height, (int64_t)c.block_x * c.out_x, (int64_t)c.block_y * c.out_y,
                              rx, ry, (int64_t)c.block_x * c.block_y);
    };
    int opt = C[0];                                    // lines 5 / 19
    int64_t bh_opt = bh(opt);                          // line 7
    if (rx > 0 || ry > 0) {                            // line 4: border handling
        const double top = cand[C[0]].occupancy;       // line 8: C0 = highest occupancy
        for (int i : C) {                              // lines 9-17
            if (cand[i].occupancy != top) break;
            const int64_t b = bh(i);
            if (b < bh_opt) { opt = i; bh_opt = b; }
        }
    }
    if (bh_out) *bh_out = bh_opt;
    return opt;
}

}  // namespace lop

extern "C" int32_t lop_alg2_select(const lop_config_candidate *cand, int32_t n, int32_t simd_width,
                                   int32_t width, int32_t height, int32_t rx, int32_t ry,
                                   int64_t *border_threads)
{
    if (!cand || n <= 0) return -1;
    return lop::alg2_select(cand, n, simd_width, width, height, rx, ry, border_threads);
}

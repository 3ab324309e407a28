// select.h -- Algorithm 2 and the tiling helpers the
// launchers use (select.cpp).
#pragma once
#include <stdint.h>

#include "lop.h"

namespace lop {

int64_t border_threads(int64_t width, int64_t height, int64_t tw, int64_t th, int64_t rx,
                       int64_t ry, int64_t threads);
int alg2_select(const lop_config_candidate *cand, int n, int simd, int width, int height, int rx,
                int ry, int64_t *bh_out);

}  // namespace lop

// lop_params.h -- kernel parameter blocks shared by the C-ABI host code
// (lop_api.cpp) and the CUDA kernels (*.cu).  Product code only; the oracle
// (oracle/) shares nothing with this tree.
#pragma once
#include <stdint.h>

namespace lop {

// Device-side view of an Image (lop_image) used for boundary resolution.
// Row y (band-local, may be negative inside the top halo) of frame b starts at
// data + b*bstride + y*stride.
struct Geom {
    const char *data;
    int64_t stride;    // bytes
    int64_t bstride;   // bytes between frames
    int32_t W, H;      // owned columns / rows
    int32_t halo_top, halo_bottom;
    int32_t gy0, GH;   // band origin / global height
};

struct OutGeom {
    char *data;
    int64_t stride, bstride;
    int32_t W, H;
};

// Everything a local-operator launch needs besides the mask.
struct Common {
    Geom in;
    OutGeom out;
    int32_t roi_x0, roi_y0, roi_w, roi_h;  // iteration space (output coords)
    int32_t off_x, off_y;                  // accessor offset
    int32_t mode;                          // lop_boundary
    int32_t rx, ry;                        // window radii (size = 2r+1)
    int32_t batch;
    float cval_f;                          // CONSTANT value (f32 images)
    int32_t cval_i;                        // CONSTANT value (u8 images)
};

constexpr int kMaxRadius = 31;                                // windows up to 63x63
constexpr int kMaxTaps = (2 * kMaxRadius + 1) * (2 * kMaxRadius + 1);  // 3969
constexpr int kTiledMaxRX = 7;                                // tiled kernels: 2*rx+1 <= 15
constexpr int kTiledMaskPitch = 16;                           // floats per mask row in the tiled kernels
constexpr int kTiledMaxTaps = (2 * kMaxRadius + 1) * kTiledMaskPitch;

// Bilateral: weight w = ex2(lc[tap] + nk * (v - centre)^2)
//   lc[tap] = log2 c(xf, yf), nk = -log2(e) / (2 sigma_r^2)
// sep = 1 (closeness from sigma_d, Eq. 1): c(xf,yf) = cy[yf] * 2^lx[xf] and the
// kernels use the per-row folded form (boundary.cuh bilateral_row_*).
struct BilateralGeneric {
    Common c;
    float nk;
    int32_t sep;
    int32_t npoly;                   // sep form: columns xf = -rx .. -rx+npoly-1 use ex2_poly
    int32_t scaled;                  // sep form: scaled-difference exponent (alpha * I)
    int32_t pair;                    // sep form: symmetric pair-sharing summation order
    float alpha, inv_alpha;
    float lx[2 * kMaxRadius + 1];
    float cy[2 * kMaxRadius + 1];
    float lc[kMaxTaps];
};
struct BilateralSep {
    Common c;
    float nk;
    int32_t npoly;                   // leftmost npoly window columns use ex2_poly (FMA pipe)
    int32_t scaled;                  // stage alpha * I; exponent lx - (J - J0)^2
    int32_t pair_rows;               // pair kernel: output rows per warp (0: not the pair kernel)
    float alpha, inv_alpha;          // alpha = sqrt(log2(e) / (2 sigma_r^2))
    float lx[2 * kTiledMaxRX + 1];   // log2 of the x factor (compile-time indexed)
    float cy[2 * kMaxRadius + 1];    // linear y factor
    alignas(8) float lx2[2 * (2 * kTiledMaxRX + 1)];   // (lx, lx) pairs: packed FFMA2 operand
};
struct BilateralTiled {
    Common c;
    float nk;
    int32_t scaled;                  // stage alpha * I; exponent lc - (J - J0)^2
    float alpha, inv_alpha;
    float lc[kTiledMaxTaps];   // row pitch kTiledMaskPitch
};

// Convolution (correlation).  kind: 0 = f32->f32, 1 = u8->u8, 2 = u8->i32.
enum ConvKind { CONV_F32 = 0, CONV_U8_U8 = 1, CONV_U8_I32 = 2 };
struct ConvGeneric {
    Common c;
    int32_t kind;
    int32_t shift;
    union {
        float f[kMaxTaps];     // f32 masks
        int32_t i[kMaxTaps];   // integer masks (u8 images)
    } m;
};

// Separable factorisation of a convolution mask, M = c r^T (conv_tiled.cu).
struct ConvSep {
    Common c;
    int32_t kind;
    int32_t shift;
    float rf[9], cf[9];      // f32 row / column coefficients
    int32_t ri[9], ci[9];    // integer row / column coefficients
    // signed SWAR (u8 -> i32, conv_tiled.cu): lane biases that keep both 16-bit
    // lanes of the row sums / column sums in [0, 65535]; S = V - sw_off
    int32_t sw_bias_h, sw_bias_v, sw_off;
};

// Fused two-stage local operator (conv_chain.cu): out = M2 (*) (M1 (*) I), both
// stages with the same boundary condition; the intermediate image never
// leaves shared memory.  Intermediate of the u8 path is quantised to u8
// exactly like a lop_convolve_execute u8 -> u8 pass.
// Local reduction over a mask domain (Listing 9's convolve(mask, <reduction>, f)
// with the MIN / MAX reductions; reduce.cu): out = min / max of Read(x+xf, y+yf)
// over the taps where the mask is non-zero.  dom[yf + ry] bit (xf + rx) = tap.
enum ReduceOp { RED_SUM = 0, RED_MIN = 1, RED_MAX = 2, RED_SUMSQ = 3 };   // SUMSQ: global only
struct ReduceParams {
    Common c;
    int32_t op;                      // RED_MIN / RED_MAX
    int32_t u8;                      // 1: u8 -> u8, 0: f32 -> f32
    int32_t full;                    // domain is the whole window (separable)
    uint64_t dom[2 * kMaxRadius + 1];
};

// Global operator (global_reduce.cu): SUM / MIN / MAX over a region of all
// frames, deterministic (fixed parts, fixed trees), result in double.
#ifndef LOP_GLOBAL_PARTS
#define LOP_GLOBAL_PARTS 512
#endif
constexpr int kGlobalParts = LOP_GLOBAL_PARTS;               // fixed partition (not per GPU)
constexpr int kGlobalCounter = 1024;                         // + 1 = LOP_GLOBAL_WORK_DOUBLES
static_assert(kGlobalParts <= kGlobalCounter && kGlobalParts % 256 == 0, "global parts");
struct GlobalReduce {
    Common c;                    // c.in: the image; c.roi_*: the region; c.batch
    int32_t op;                  // RED_SUM / RED_MIN / RED_MAX / RED_SUMSQ
    int32_t u8;
    double *work;                // kGlobalParts doubles, arrival counter at [kGlobalCounter]
    double *result;              // 1 double (device)
};

// Two local operators on one input, combined by a point operator (conv_pair.cu):
// out = combine(Ma (*) I, Mb (*) I).  L2: sqrt(a^2 + b^2) (f32), L1: |a| + |b|,
// SUMSQ: a^2 + b^2.  f32 -> f32 or u8 -> i32.
enum PairCombine { PAIR_L2 = 0, PAIR_L1 = 1, PAIR_SUMSQ = 2 };
struct ConvPair {            // both masks exactly separable, same radius <= 2
    ConvSep a, b;            // a.c holds the launch geometry
    int32_t combine;
    int32_t u8;
};
constexpr int kPairMaxR = 15;                                 // generic pair: windows up to 31x31
constexpr int kPairMaxTaps = (2 * kPairMaxR + 1) * (2 * kPairMaxR + 1);
struct ConvPairGeneric {
    Common c;
    int32_t combine;
    int32_t u8;
    union { float ma[kPairMaxTaps]; int32_t ia[kPairMaxTaps]; };
    union { float mb[kPairMaxTaps]; int32_t ib[kPairMaxTaps]; };
};

// Row-streaming plan of the fused chain (conv_chain.cu, set by the launcher):
// warps stream output rows [sy0, sy1) in frames of 32 lanes; the rows above
// and below (where pass 2 reads G outside the image) are band tiles of the
// tile kernel in the same launch.
struct ChainPlan {
    int32_t sy0, sy1;            // streamed output rows
    int32_t T, nseg, nframes;    // rows per warp, row segments, frames across
    int32_t ox_base;             // output column of frame 0, lane 1, element 0
    int32_t stream_ctas;         // CTAs of streaming warps (per image)
    int32_t ntx;                 // band tiles across
    int32_t top_rows, bot_rows;  // band tile rows above / below the streamed rows
};
struct ConvChain {
    ConvSep s1, s2;          // s1.c holds the launch geometry
    int32_t kind;            // 0: f32 -> f32 -> f32; 1: u8 -> u8 -> u8; 2: u8 -> u8 -> i32
    ChainPlan plan;
};

// Local operator over several Accessors with a per-tap function (local.cu;
// SURVEY §8(f) N2, Listing 9).  Accessor k reads its own
// image through its own boundary condition at its own offset; its mask
// occupies m[moff .. moff + (2ry+1)(2rx+1)).  c.rx / c.ry: the largest radii
// (the launch's halo).  op: RED_SUM / RED_MIN / RED_MAX; fn: LOP_TAP_*.
constexpr int kLocalMaxAcc = 4;
constexpr int kLocalMaxR = 15;                                // each mask up to 31 x 31
constexpr int kLocalMaxTaps = 3844;                           // all masks together
struct LocalAcc {
    Geom in;
    int32_t off_x, off_y, mode, rx, ry;
    float cval_f;
    int32_t cval_i;
    int32_t moff;
    int32_t point;               // point-operator prologue Read' = pa * Read + pb (reading c27)
    float pa_f, pb_f;            // f32 images
    int32_t pa_i, pb_i;          // u8 images (exact)
};
constexpr int kLocalSmallR = 7;                               // register-blocked path: radii <= 7
constexpr int kLocalSmallW = 2 * kLocalSmallR + 1;
struct LocalParams {
    Common c;                    // output, ROI, batch, largest radii
    int32_t n, op, fn, u8;
    int32_t small;               // every radius <= kLocalSmallR: masks also in ms (15 x 15 slots)
    int32_t any_point;           // some accessor has a point-operator prologue
    LocalAcc acc[kLocalMaxAcc];
    union {                      // mask k embedded centred in a 15 x 15 slot (zeros outside)
        float f[kLocalMaxAcc][kLocalSmallW * kLocalSmallW];
        int32_t i[kLocalMaxAcc][kLocalSmallW * kLocalSmallW];
    } ms;
    union {
        float f[kLocalMaxTaps];
        int32_t i[kLocalMaxTaps];
    } m;
};

// Laplacian-pyramid REDUCE / EXPAND (pyramid.cu, reading c28).
struct PyrParams {
    Geom in;                     // level read (whole image, no band)
    OutGeom out;                 // level written
    const char *add;             // EXPAND: addend image (may alias out) or nullptr
    int64_t add_stride, add_bstride;
    float sign;                  // EXPAND: out = add + sign * E
    int32_t mode;
    float cval;
    int32_t batch;
};

}  // namespace lop

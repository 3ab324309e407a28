// lop_api.cpp -- the C ABI (include/lop.h): argument validation, mask
// construction, kernel dispatch.  Host C++ only; every pixel of every step of
// the path is computed by the CUDA kernels in *.cu.
#include "lop.h"

#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <memory>
#include <string>

#include "kernels.h"
#include "lop_params.h"

namespace {

thread_local std::string g_error;
thread_local int64_t g_launches = 0;
std::atomic<int32_t> g_variant{LOP_VARIANT_AUTO};

lop_status fail(lop_status st, const char *fmt, ...)
{
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    g_error = buf;
    return st;
}

lop_status cuda_fail(cudaError_t e, const char *what)
{
    return fail(LOP_ERR_CUDA, "%s: %s", what, cudaGetErrorString(e));
}

int elem_size(int32_t dt)
{
    switch (dt) {
    case LOP_U8: return 1;
    case LOP_I32: return 4;
    case LOP_F32: return 4;
    default: return 0;
    }
}

const double kLog2e = 1.4426950408889634073599246810019;
const int kDefaultNpoly = 0;   // MUFU offload: slower on B200, kept for tuning
const int kDefaultScaled = 1;  // scaled-difference exponent: +2.5 % on B200
const int kDefaultPair = 1;    // symmetric pair-sharing kernel

// ---------------------------------------------------------------- validation
lop_status check_image(const lop_image &im, const char *name)
{
    if (!im.data) return fail(LOP_ERR_INVALID, "%s: data is NULL", name);
    const int es = elem_size(im.dtype);
    if (!es) return fail(LOP_ERR_INVALID, "%s: unknown dtype %d", name, im.dtype);
    if (im.width <= 0 || im.height <= 0)
        return fail(LOP_ERR_INVALID, "%s: width/height must be > 0 (got %d x %d)", name, im.width,
                    im.height);
    if (im.stride_bytes < (int64_t)im.width * es || im.stride_bytes % es)
        return fail(LOP_ERR_INVALID, "%s: stride_bytes %lld invalid for width %d", name,
                    (long long)im.stride_bytes, im.width);
    if (im.batch < 1) return fail(LOP_ERR_INVALID, "%s: batch must be >= 1", name);
    if (im.halo_top < 0 || im.halo_bottom < 0)
        return fail(LOP_ERR_INVALID, "%s: negative halo", name);
    const int64_t rows = (int64_t)im.height + im.halo_top + im.halo_bottom;
    if (im.batch > 1 && im.batch_stride_bytes < rows * im.stride_bytes)
        return fail(LOP_ERR_INVALID, "%s: batch_stride_bytes too small", name);
    const int32_t gh = im.global_height ? im.global_height : im.height;
    if (im.global_y0 < 0 || (int64_t)im.global_y0 + im.height > gh)
        return fail(LOP_ERR_INVALID, "%s: band [%d, %d) outside global height %d", name,
                    im.global_y0, im.global_y0 + im.height, gh);
    cudaPointerAttributes attr;
    cudaError_t e = cudaPointerGetAttributes(&attr, im.data);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return fail(LOP_ERR_INVALID, "%s: data is not a CUDA pointer (%s)", name,
                    cudaGetErrorString(e));
    }
    if (attr.type != cudaMemoryTypeDevice && attr.type != cudaMemoryTypeManaged)
        return fail(LOP_ERR_INVALID, "%s: data must be device memory", name);
    int dev = -1;
    cudaGetDevice(&dev);
    if (attr.device != dev)
        return fail(LOP_ERR_INVALID, "%s: data lives on device %d, current device is %d", name,
                    attr.device, dev);
    return LOP_OK;
}

lop::Geom make_geom(const lop_image &im)
{
    lop::Geom g;
    g.data = static_cast<const char *>(im.data);
    g.stride = im.stride_bytes;
    g.bstride = im.batch > 1 ? im.batch_stride_bytes : 0;
    g.W = im.width;
    g.H = im.height;
    g.halo_top = im.halo_top;
    g.halo_bottom = im.halo_bottom;
    g.gy0 = im.global_y0;
    g.GH = im.global_height ? im.global_height : im.height;
    return g;
}

int map_axis_host(int64_t i, int64_t n, int mode)
{
    if (i >= 0 && i < n) return (int)i;
    if (mode == LOP_REPEAT) { int64_t q = i % n; return (int)(q < 0 ? q + n : q); }
    if (mode == LOP_MIRROR) {
        int64_t per = 2 * n, q = i % per;
        if (q < 0) q += per;
        return (int)(q < n ? q : per - 1 - q);
    }
    return i < 0 ? 0 : (int)(n - 1);
}

// Every input row the launch can touch must be physically addressable in the
// band view: same resolution rule as lop::resolve_row (boundary.cuh).
lop_status check_rows(const lop::Geom &g, int mode, int64_t iy_lo, int64_t iy_hi)
{
    for (int64_t iy = iy_lo; iy <= iy_hi; ++iy) {
        if (iy >= 0 && iy < g.H) continue;
        const int64_t gy = iy + g.gy0;
        int64_t row;
        if (gy >= 0 && gy < g.GH) row = iy;
        else if (mode == LOP_CONSTANT) continue;
        else if (mode == LOP_REPEAT && iy >= -g.halo_top && iy < g.H + g.halo_bottom) continue;
        else row = map_axis_host(gy, g.GH, mode) - g.gy0;
        if (row < -g.halo_top || row >= g.H + g.halo_bottom)
            return fail(LOP_ERR_INVALID,
                        "input row %lld (global %lld) resolves to band row %lld outside the "
                        "view [-%d, %d): halo too small for the window",
                        (long long)iy, (long long)gy, (long long)row, g.halo_top,
                        g.H + g.halo_bottom);
    }
    return LOP_OK;
}

// Byte range [lo, hi) of device memory a view spans: rows -halo_top ..
// height + halo_bottom - 1 of every frame.
void view_span(const lop_image &im, int64_t halo_top, int64_t halo_bottom, uintptr_t &lo,
               uintptr_t &hi)
{
    const int64_t es = elem_size(im.dtype);
    const int64_t last_frame = im.batch > 1 ? (int64_t)(im.batch - 1) * im.batch_stride_bytes : 0;
    const uintptr_t base = reinterpret_cast<uintptr_t>(im.data);
    lo = base - (uintptr_t)(halo_top * im.stride_bytes);
    hi = base + (uintptr_t)(last_frame + (im.height + halo_bottom - 1) * im.stride_bytes +
                            (int64_t)im.width * es);
}

// The stencil kernels read input rows other CTAs (warps) may already have
// written: input and output storage must not overlap (include/lop.h).
lop_status check_disjoint(const lop_image &in, const lop_image &out)
{
    uintptr_t a0, a1, b0, b1;
    view_span(in, in.halo_top, in.halo_bottom, a0, a1);
    view_span(out, 0, 0, b0, b1);
    if (a0 < b1 && b0 < a1)
        return fail(LOP_ERR_INVALID,
                    "input and output storage overlap (input bytes [%p, %p), output [%p, %p)): "
                    "local operators cannot run in place", (void *)a0, (void *)a1, (void *)b0,
                    (void *)b1);
    return LOP_OK;
}

struct Prepared {
    lop::Common c;
};

lop_status prepare(const lop_iteration_space *is, const lop_accessor *in, Prepared &pp)
{
    if (!is) return fail(LOP_ERR_INVALID, "iteration space is NULL");
    if (!in || !in->bc) return fail(LOP_ERR_INVALID, "accessor / boundary condition is NULL");
    const lop_boundary_condition &bc = *in->bc;
    lop_status st = check_image(bc.image, "input");
    if (st) return st;
    st = check_image(is->image, "output");
    if (st) return st;
    if (bc.mode < LOP_UNDEFINED || bc.mode > LOP_CONSTANT)
        return fail(LOP_ERR_INVALID, "unknown boundary mode %d", bc.mode);
    if (bc.size_x < 1 || bc.size_y < 1 || !(bc.size_x & 1) || !(bc.size_y & 1))
        return fail(LOP_ERR_INVALID, "window %d x %d must be odd and positive (PAPER.md L274-L282)",
                    bc.size_x, bc.size_y);
    if (bc.size_x > 2 * lop::kMaxRadius + 1 || bc.size_y > 2 * lop::kMaxRadius + 1)
        return fail(LOP_ERR_UNSUPPORTED, "window %d x %d larger than 63 x 63", bc.size_x,
                    bc.size_y);
    const lop_image &ii = bc.image, &oi = is->image;
    if (ii.batch != oi.batch) return fail(LOP_ERR_INVALID, "input/output batch differ");
    if (ii.width != oi.width || ii.height != oi.height)
        return fail(LOP_ERR_INVALID, "input %d x %d and output %d x %d differ (Listing 2 l.8-9)",
                    ii.width, ii.height, oi.width, oi.height);
    st = check_disjoint(ii, oi);
    if (st) return st;
    if (!std::isfinite(bc.constant)) return fail(LOP_ERR_INVALID, "constant is not finite");
    if (ii.dtype == LOP_U8 && bc.mode == LOP_CONSTANT &&
        (bc.constant < 0 || bc.constant > 255 || bc.constant != std::floor(bc.constant)))
        return fail(LOP_ERR_INVALID, "constant %g is not a u8 value", bc.constant);
    lop::Common &c = pp.c;
    std::memset(&c, 0, sizeof c);
    c.in = make_geom(ii);
    c.out.data = static_cast<char *>(oi.data);
    c.out.stride = oi.stride_bytes;
    c.out.bstride = oi.batch > 1 ? oi.batch_stride_bytes : 0;
    c.out.W = oi.width;
    c.out.H = oi.height;
    c.roi_x0 = is->x0;
    c.roi_y0 = is->y0;
    c.roi_w = is->width ? is->width : oi.width - is->x0;
    c.roi_h = is->height ? is->height : oi.height - is->y0;
    if (c.roi_x0 < 0 || c.roi_y0 < 0 || c.roi_w <= 0 || c.roi_h <= 0 ||
        (int64_t)c.roi_x0 + c.roi_w > oi.width || (int64_t)c.roi_y0 + c.roi_h > oi.height)
        return fail(LOP_ERR_INVALID, "iteration space [%d,%d)+%dx%d outside the %d x %d output",
                    is->x0, is->y0, c.roi_w, c.roi_h, oi.width, oi.height);
    c.off_x = in->offset_x;
    c.off_y = in->offset_y;
    c.mode = bc.mode;
    c.rx = bc.size_x / 2;
    c.ry = bc.size_y / 2;
    c.batch = ii.batch;
    c.cval_f = (float)bc.constant;
    c.cval_i = (int32_t)bc.constant;
    return check_rows(c.in, c.mode, (int64_t)c.roi_y0 + c.off_y - c.ry,
                      (int64_t)c.roi_y0 + c.roi_h - 1 + c.off_y + c.ry);
}

// Bilateral kernel choice (the paper's configuration
// exploration, §V-D / Fig. 4): the symmetric pair-sharing kernel
// (84 exps / px at 13x13, but warps stream rows with an R-row warm-up and
// 2 x ceil(R/4) halo lanes) against the unshared separable kernel (168 exps /
// px, no warm-up), from the B200 sweep profiles/r02/sweep_bilateral_pair_vs_sep.jsonl
// (tools/sweep_bilateral.py): pair wins on small launches (latency-bound,
// fewer exps per warp step) and on large ones with windows of 7x7 and up;
// the unshared kernel in between and for 3x3 / 5x5 beyond 768^2 / 512^2.
// Keyed to the WHOLE launch's work -- width x GLOBAL height x frames, never
// the iteration space or the band -- so ROI launches, row-band views (every
// rank of a band split) and pipeline chunks of one image take the same kernel
// as the whole-image call and stay bit-identical to it.  (A batch of frames
// and the same frames launched one by one may differ; both meet the 1e-5
// contract.)
int pair_preferred(const lop::Common &c, int dflt)
{
    if (!dflt) return 0;
    const double px = (double)c.in.W * (double)c.in.GH * (double)c.batch;
    const int r = c.rx;
    static const double lo[8] = {0, 768.0 * 768, 512.0 * 512, 512.0 * 512, 384.0 * 384,
                                 256.0 * 256, 256.0 * 256, 256.0 * 256};   // pair at or below
    static const double hi[8] = {0, 1e300, 1e300, 4096.0 * 4096, 3072.0 * 3072,
                                 3072.0 * 3072, 2048.0 * 2048, 2048.0 * 2048};  // pair at or above
    if (r < 1 || r > 7) return dflt;
    return px <= lo[r] || px >= hi[r] ? 1 : 0;
}

lop_status launched(cudaError_t e, const char *what)
{
    if (e != cudaSuccess) return cuda_fail(e, what);
    ++g_launches;
    return LOP_OK;
}

}  // namespace

namespace lop_detail {
void set_error(const std::string &msg) { g_error = msg; }
}  // namespace lop_detail

extern "C" {

const char *lop_last_error(void) { return g_error.c_str(); }
int32_t lop_version(void) { return LOP_VERSION; }
int64_t lop_launch_count(void) { return g_launches; }
void lop_reset_launch_count(void) { g_launches = 0; }

lop_status lop_set_variant(int32_t v)
{
    if (v < LOP_VARIANT_AUTO || v > LOP_VARIANT_TILED)
        return fail(LOP_ERR_INVALID, "unknown variant %d", v);
    g_variant = v;
    return LOP_OK;
}
int32_t lop_get_variant(void) { return g_variant; }

// ------------------------------------------------------------------ masks
lop_status lop_mask_closeness(float sigma_d, int32_t size_x, int32_t size_y, float *out)
{
    if (!out) return fail(LOP_ERR_INVALID, "out is NULL");
    if (!(sigma_d > 0) || !std::isfinite(sigma_d)) return fail(LOP_ERR_INVALID, "sigma_d must be > 0");
    if (size_x < 1 || size_y < 1 || !(size_x & 1) || !(size_y & 1))
        return fail(LOP_ERR_INVALID, "mask size must be odd");
    const int m = size_x / 2, n = size_y / 2;
    const double c_d = 1.0 / (2.0 * (double)sigma_d * (double)sigma_d);  // Listing 1 l.13
    for (int yf = -n; yf <= n; ++yf)
        for (int xf = -m; xf <= m; ++xf)
            out[(yf + n) * size_x + (xf + m)] = (float)std::exp(-c_d * (double)(xf * xf + yf * yf));
    return LOP_OK;
}

lop_status lop_mask_gaussian(int32_t size, int32_t dtype, void *out, int32_t *shift)
{
    if (!out || !shift) return fail(LOP_ERR_INVALID, "out/shift is NULL");
    if (size < 1 || size > 31 || !(size & 1)) return fail(LOP_ERR_INVALID, "size must be odd in 1..31");
    if (dtype != LOP_I32 && dtype != LOP_F32) return fail(LOP_ERR_INVALID, "dtype must be I32 or F32");
    if (dtype == LOP_I32 && size > 11)   // 255 * 2^(2(size-1)) must fit the int32 sums
        return fail(LOP_ERR_INVALID, "integer Gaussian masks are limited to 11x11");
    int64_t binom[32];
    for (int k = 0; k < size; ++k) {                 // C(size-1, k) via the multiplicative formula
        int64_t v = 1;
        for (int j = 1; j <= k; ++j) v = v * (size - j) / j;
        binom[k] = v;
    }
    const int k = 2 * (size - 1);
    for (int y = 0; y < size; ++y)
        for (int x = 0; x < size; ++x) {
            const int64_t v = binom[y] * binom[x];
            if (dtype == LOP_I32) static_cast<int32_t *>(out)[y * size + x] = (int32_t)v;
            else static_cast<float *>(out)[y * size + x] = (float)std::ldexp((double)v, -k);
        }
    *shift = dtype == LOP_I32 ? k : 0;
    return LOP_OK;
}

lop_status lop_mask_sobel(int32_t dir, int32_t dtype, void *out)
{
    if (!out) return fail(LOP_ERR_INVALID, "out is NULL");
    if (dir != 0 && dir != 1) return fail(LOP_ERR_INVALID, "dir must be 0 (x) or 1 (y)");
    if (dtype != LOP_I32 && dtype != LOP_F32) return fail(LOP_ERR_INVALID, "dtype must be I32 or F32");
    for (int y = -1; y <= 1; ++y)
        for (int x = -1; x <= 1; ++x) {
            const int d = dir == 0 ? x : y, o = dir == 0 ? y : x;   // derivative / smoothing axes
            const int v = d * (2 - o * o);                           // [-1,0,1] x [1,2,1]
            if (dtype == LOP_I32) static_cast<int32_t *>(out)[(y + 1) * 3 + x + 1] = v;
            else static_cast<float *>(out)[(y + 1) * 3 + x + 1] = (float)v;
        }
    return LOP_OK;
}

// -------------------------------------------------------------- bilateral
lop_status lop_bilateral_execute(const lop_iteration_space *is, const lop_accessor *in,
                                 const lop_mask *closeness, float sigma_d, float sigma_r,
                                 void *cuda_stream)
{
    Prepared pp;
    lop_status st = prepare(is, in, pp);
    if (st) return st;
    const lop::Common &c = pp.c;
    if (in->bc->image.dtype != LOP_F32 || is->image.dtype != LOP_F32)
        return fail(LOP_ERR_INVALID, "bilateral filter is Kernel<float>: F32 in/out (Listing 1)");
    if (!(sigma_r > 0) || !std::isfinite(sigma_r)) return fail(LOP_ERR_INVALID, "sigma_r must be > 0");
    const int sx = 2 * c.rx + 1, sy = 2 * c.ry + 1;
    // log2 of the closeness coefficients (Listing 5 l.10 c = CMask(xf, yf))
    std::unique_ptr<float[]> lc(new float[sx * sy]);
    if (closeness) {
        if (closeness->dtype != LOP_F32 || !closeness->coeffs)
            return fail(LOP_ERR_INVALID, "closeness mask must be F32 with coefficients");
        if (closeness->size_x != sx || closeness->size_y != sy)
            return fail(LOP_ERR_INVALID, "closeness mask %d x %d != window %d x %d",
                        closeness->size_x, closeness->size_y, sx, sy);
        const float *cm = static_cast<const float *>(closeness->coeffs);
        for (int i = 0; i < sx * sy; ++i) {
            if (!(cm[i] >= 0) || !std::isfinite(cm[i]))
                return fail(LOP_ERR_INVALID, "closeness coefficient %d = %g must be finite and >= 0",
                            i, (double)cm[i]);
            lc[i] = cm[i] > 0 ? (float)std::log2((double)cm[i]) : -INFINITY;
        }
        if (!(cm[c.ry * sx + c.rx] > 0))
            return fail(LOP_ERR_INVALID, "closeness centre must be > 0 (reading c14)");
    } else {
        if (!(sigma_d > 0) || !std::isfinite(sigma_d))
            return fail(LOP_ERR_INVALID, "sigma_d must be > 0");
        const double c_d = 1.0 / (2.0 * (double)sigma_d * (double)sigma_d);
        for (int yf = -c.ry; yf <= c.ry; ++yf)
            for (int xf = -c.rx; xf <= c.rx; ++xf)  // Eq. (1) in the log2 domain
                lc[(yf + c.ry) * sx + xf + c.rx] = (float)(-c_d * (double)(xf * xf + yf * yf) * kLog2e);
    }
    const float nk = (float)(-kLog2e / (2.0 * (double)sigma_r * (double)sigma_r));
    cudaStream_t stream = static_cast<cudaStream_t>(cuda_stream);
    const int32_t variant = g_variant;
    const bool tiled_ok = c.rx <= lop::kTiledMaxRX;
    if (variant == LOP_VARIANT_TILED && !tiled_ok)
        return fail(LOP_ERR_UNSUPPORTED, "no tiled bilateral instance for window width %d", sx);
    // Closeness from sigma_d (Eq. 1) is separable: c = cy[yf] * 2^lx[xf]
    // (Listing 1 l.21: exp(-c_d xf^2) * exp(-c_d yf^2)).
    float lx[2 * lop::kMaxRadius + 1], cy[2 * lop::kMaxRadius + 1];
    if (!closeness) {
        const double c_d = 1.0 / (2.0 * (double)sigma_d * (double)sigma_d);
        for (int xf = -c.rx; xf <= c.rx; ++xf) lx[xf + c.rx] = (float)(-c_d * (double)(xf * xf) * kLog2e);
        for (int yf = -c.ry; yf <= c.ry; ++yf) cy[yf + c.ry] = (float)std::exp(-c_d * (double)(yf * yf));
    }
    // A user closeness mask (Listing 4 / 5) that factors into x and y factors --
    // the paper's own mask exp(-c (xf^2 + yf^2)) does -- takes the separable
    // kernels (and the pair-sharing one): cy[i] = M[i][m], cx[j] = M[n][j] / M[n][m],
    // accepted when every coefficient is > 0, both factors are exactly
    // symmetric (pair sharing needs c(d) = c(-d) bit for bit) and cy[i] cx[j]
    // reproduces M to 2^-20 relative (reading c21).  LOP_BILATERAL_FACTOR=0 keeps
    // the mask kernels.
    bool sepform = !closeness;
    if (closeness) {
        bool ok = true;
        if (const char *env = std::getenv("LOP_BILATERAL_FACTOR")) ok = std::atoi(env) != 0;
        const float *cm = static_cast<const float *>(closeness->coeffs);
        for (int i = 0; i < sx * sy && ok; ++i) ok = cm[i] > 0;
        if (ok) {
            const double centre = cm[c.ry * sx + c.rx];
            double cxd[2 * lop::kMaxRadius + 1], cyd[2 * lop::kMaxRadius + 1];
            for (int j = 0; j < sx; ++j) cxd[j] = (double)cm[c.ry * sx + j] / centre;
            for (int i = 0; i < sy; ++i) cyd[i] = (double)cm[i * sx + c.rx];
            for (int j = 0; j < sx && ok; ++j) ok = cxd[j] == cxd[sx - 1 - j];
            for (int i = 0; i < sy && ok; ++i) ok = cyd[i] == cyd[sy - 1 - i];
            for (int i = 0; i < sy && ok; ++i)
                for (int j = 0; j < sx && ok; ++j)
                    ok = std::fabs(cyd[i] * cxd[j] - (double)cm[i * sx + j]) <=
                         std::ldexp((double)cm[i * sx + j], -20);
            if (ok) {
                for (int j = 0; j < sx; ++j) lx[j] = (float)std::log2(cxd[j]);
                for (int i = 0; i < sy; ++i) cy[i] = (float)cyd[i];
                sepform = true;
            }
        }
    }
    // window columns whose exp runs on the FMA pipe (ex2_poly) instead of the
    // MUFU: tuned on B200; LOP_BILATERAL_NPOLY overrides
    int npoly = 0;
    if (sepform) {
        npoly = c.rx >= 4 ? kDefaultNpoly : 0;
        if (const char *env = std::getenv("LOP_BILATERAL_NPOLY")) npoly = std::atoi(env);
        npoly = std::max(0, std::min(npoly, lop::bilateral_sep_max_npoly(c.rx)));
    }
    // scaled-difference exponent: LOP_BILATERAL_SCALED overrides
    int scaled = kDefaultScaled;
    if (const char *env = std::getenv("LOP_BILATERAL_SCALED")) scaled = std::atoi(env) != 0;
    if (scaled) npoly = 0;
    // symmetric pair-sharing: square separable windows, scaled
    // exponent, chosen per launch by the measured configuration space
    // (pair_preferred); LOP_BILATERAL_PAIR overrides
    int pair = pair_preferred(c, kDefaultPair);
    if (const char *env = std::getenv("LOP_BILATERAL_PAIR")) pair = std::atoi(env) != 0;
    pair = pair && sepform && scaled && c.rx == c.ry && c.rx >= 1 && c.rx <= lop::kTiledMaxRX;
    const double alpha_d = std::sqrt(kLog2e / (2.0 * (double)sigma_r * (double)sigma_r));
    const float alpha = (float)alpha_d, inv_alpha = (float)(1.0 / alpha_d);
    if (variant != LOP_VARIANT_GENERIC && tiled_ok && sepform) {
        static thread_local lop::BilateralSep p;
        p.c = c;
        p.nk = nk;
        p.npoly = npoly;
        p.scaled = scaled;
        p.alpha = alpha;
        p.inv_alpha = inv_alpha;
        std::memcpy(p.lx, lx, sizeof(float) * sx);
        std::memcpy(p.cy, cy, sizeof(float) * sy);
        for (int k = 0; k < sx; ++k) p.lx2[2 * k] = p.lx2[2 * k + 1] = lx[k];
        p.pair_rows = 0;
        if (pair) return launched(lop::launch_bilateral_pair(p, stream), "bilateral_pair launch");
        return launched(lop::launch_bilateral_sep(p, stream), "bilateral_sep launch");
    }
    if (variant != LOP_VARIANT_GENERIC && tiled_ok) {
        static thread_local lop::BilateralTiled p;
        p.c = c;
        p.nk = nk;
        p.scaled = scaled;
        p.alpha = alpha;
        p.inv_alpha = inv_alpha;
        for (int r = 0; r < sy; ++r)
            for (int k = 0; k < lop::kTiledMaskPitch; ++k)
                p.lc[r * lop::kTiledMaskPitch + k] = k < sx ? lc[r * sx + k] : 0.0f;
        return launched(lop::launch_bilateral_tiled(p, stream), "bilateral_tiled launch");
    }
    static thread_local lop::BilateralGeneric p;
    p.c = c;
    p.nk = nk;
    p.sep = sepform ? 1 : 0;
    p.pair = pair;
    p.npoly = npoly;
    p.scaled = scaled;
    p.alpha = alpha;
    p.inv_alpha = inv_alpha;
    if (!sepform) {
        std::memcpy(p.lc, lc.get(), sizeof(float) * sx * sy);
    } else {
        std::memcpy(p.lx, lx, sizeof(float) * sx);
        std::memcpy(p.cy, cy, sizeof(float) * sy);
    }
    return launched(lop::launch_bilateral_generic(p, stream), "bilateral_generic launch");
}

// ------------------------------------------------------------ convolution
lop_status lop_convolve_execute(const lop_iteration_space *is, const lop_accessor *in,
                                const lop_mask *mask, void *cuda_stream)
{
    Prepared pp;
    lop_status st = prepare(is, in, pp);
    if (st) return st;
    const lop::Common &c = pp.c;
    if (!mask || !mask->coeffs) return fail(LOP_ERR_INVALID, "mask is NULL");
    const int sx = 2 * c.rx + 1, sy = 2 * c.ry + 1;
    if (mask->size_x != sx || mask->size_y != sy)
        return fail(LOP_ERR_INVALID, "mask %d x %d != window %d x %d", mask->size_x, mask->size_y,
                    sx, sy);
    const int32_t idt = in->bc->image.dtype, odt = is->image.dtype;
    static thread_local lop::ConvGeneric p;
    p.c = c;
    p.shift = 0;
    if (idt == LOP_F32 && odt == LOP_F32) {
        if (mask->dtype != LOP_F32) return fail(LOP_ERR_INVALID, "F32 images need an F32 mask");
        if (mask->shift != 0) return fail(LOP_ERR_INVALID, "F32 masks take shift 0");
        p.kind = lop::CONV_F32;
        const float *m = static_cast<const float *>(mask->coeffs);
        for (int i = 0; i < sx * sy; ++i) {
            if (!std::isfinite(m[i])) return fail(LOP_ERR_INVALID, "mask coefficient %d not finite", i);
            p.m.f[i] = m[i];
        }
    } else if (idt == LOP_U8 && (odt == LOP_U8 || odt == LOP_I32)) {
        if (mask->dtype != LOP_I32) return fail(LOP_ERR_INVALID, "U8 images need an I32 mask");
        if (mask->shift < 0 || mask->shift > 30) return fail(LOP_ERR_INVALID, "shift must be in 0..30");
        p.kind = odt == LOP_U8 ? lop::CONV_U8_U8 : lop::CONV_U8_I32;
        p.shift = mask->shift;
        const int32_t *m = static_cast<const int32_t *>(mask->coeffs);
        int64_t l1 = 0;
        for (int i = 0; i < sx * sy; ++i) {
            p.m.i[i] = m[i];
            l1 += m[i] < 0 ? -(int64_t)m[i] : m[i];
        }
        if (l1 * 255 + (1ll << 30) >= (1ll << 31))
            return fail(LOP_ERR_UNSUPPORTED, "integer mask too large: sums may overflow int32");
    } else {
        return fail(LOP_ERR_INVALID, "unsupported dtype combination %d -> %d (F32->F32, U8->U8, U8->I32)",
                    idt, odt);
    }
    cudaStream_t stream = static_cast<cudaStream_t>(cuda_stream);
    const int32_t variant = g_variant;
    const bool tiled_ok = lop::conv_tiled_supported(p);
    if (variant == LOP_VARIANT_TILED && !tiled_ok)
        return fail(LOP_ERR_UNSUPPORTED, "no tiled convolution instance for this mask");
    if (variant != LOP_VARIANT_GENERIC && tiled_ok)
        return launched(lop::launch_conv_tiled(p, stream), "conv_tiled launch");
    return launched(lop::launch_conv_generic(p, stream), "conv_generic launch");
}

// ------------------------------------------------ local MIN / MAX reduction
lop_status lop_reduce_execute(const lop_iteration_space *is, const lop_accessor *in,
                              const lop_mask *domain, int32_t op, void *cuda_stream)
{
    if (op == LOP_REDUCE_SUM) return lop_convolve_execute(is, in, domain, cuda_stream);
    if (op != LOP_REDUCE_MIN && op != LOP_REDUCE_MAX)
        return fail(LOP_ERR_INVALID, "unknown reduction %d (SUM, MIN, MAX)", op);
    Prepared pp;
    lop_status st = prepare(is, in, pp);
    if (st) return st;
    const lop::Common &c = pp.c;
    if (!domain || !domain->coeffs) return fail(LOP_ERR_INVALID, "domain mask is NULL");
    const int sx = 2 * c.rx + 1, sy = 2 * c.ry + 1;
    if (domain->size_x != sx || domain->size_y != sy)
        return fail(LOP_ERR_INVALID, "domain %d x %d != window %d x %d", domain->size_x,
                    domain->size_y, sx, sy);
    const int32_t idt = in->bc->image.dtype, odt = is->image.dtype;
    static thread_local lop::ReduceParams p;
    p.c = c;
    p.op = op == LOP_REDUCE_MIN ? lop::RED_MIN : lop::RED_MAX;
    if (idt == LOP_F32 && odt == LOP_F32) {
        if (domain->dtype != LOP_F32) return fail(LOP_ERR_INVALID, "F32 images need an F32 domain mask");
        p.u8 = 0;
    } else if (idt == LOP_U8 && odt == LOP_U8) {
        if (domain->dtype != LOP_I32) return fail(LOP_ERR_INVALID, "U8 images need an I32 domain mask");
        p.u8 = 1;
    } else {
        return fail(LOP_ERR_INVALID, "unsupported dtype combination %d -> %d (F32->F32, U8->U8)",
                    idt, odt);
    }
    int taps = 0;
    for (int yf = 0; yf < sy; ++yf) {
        uint64_t bits = 0;
        for (int xf = 0; xf < sx; ++xf) {
            const bool on = domain->dtype == LOP_F32
                                ? static_cast<const float *>(domain->coeffs)[yf * sx + xf] != 0.0f
                                : static_cast<const int32_t *>(domain->coeffs)[yf * sx + xf] != 0;
            if (on) { bits |= 1ull << xf; ++taps; }
        }
        p.dom[yf] = bits;
    }
    if (!taps) return fail(LOP_ERR_INVALID, "domain mask has no non-zero coefficient");
    p.full = taps == sx * sy;
    const int32_t variant = g_variant;
    const bool tiled_ok = p.full && c.rx == c.ry && c.rx >= 1 && c.rx <= 4;
    if (variant == LOP_VARIANT_TILED && !tiled_ok)
        return fail(LOP_ERR_UNSUPPORTED, "no tiled reduction instance for this domain");
    return launched(lop::launch_reduce(p, variant != LOP_VARIANT_GENERIC,
                                       static_cast<cudaStream_t>(cuda_stream)),
                    "reduce launch");
}

// ------------------------------------------------------- global operators
lop_status lop_global_reduce_execute(const lop_iteration_space *is, int32_t op, double *d_result,
                                     double *d_work, void *cuda_stream)
{
    static_assert(lop::kGlobalCounter + 1 == LOP_GLOBAL_WORK_DOUBLES, "work size");
    if (!is) return fail(LOP_ERR_INVALID, "iteration space is NULL");
    if (op != LOP_REDUCE_SUM && op != LOP_REDUCE_MIN && op != LOP_REDUCE_MAX && op != LOP_REDUCE_SUMSQ)
        return fail(LOP_ERR_INVALID, "unknown reduction %d (SUM, MIN, MAX, SUMSQ)", op);
    if (!d_result || !d_work) return fail(LOP_ERR_INVALID, "d_result / d_work is NULL");
    lop_status st = check_image(is->image, "image");
    if (st) return st;
    const lop_image &im = is->image;
    if (im.dtype != LOP_F32 && im.dtype != LOP_U8)
        return fail(LOP_ERR_INVALID, "global reductions take F32 or U8 images");
    for (const void *ptr : {static_cast<const void *>(d_result), static_cast<const void *>(d_work)}) {
        cudaPointerAttributes attr;
        if (cudaPointerGetAttributes(&attr, ptr) != cudaSuccess ||
            (attr.type != cudaMemoryTypeDevice && attr.type != cudaMemoryTypeManaged)) {
            cudaGetLastError();
            return fail(LOP_ERR_INVALID, "d_result / d_work must be device memory");
        }
    }
    static thread_local lop::GlobalReduce p;
    std::memset(&p.c, 0, sizeof p.c);
    p.c.in = make_geom(im);
    p.c.roi_x0 = is->x0;
    p.c.roi_y0 = is->y0;
    p.c.roi_w = is->width ? is->width : im.width - is->x0;
    p.c.roi_h = is->height ? is->height : im.height - is->y0;
    if (p.c.roi_x0 < 0 || p.c.roi_y0 < 0 || p.c.roi_w <= 0 || p.c.roi_h <= 0 ||
        (int64_t)p.c.roi_x0 + p.c.roi_w > im.width || (int64_t)p.c.roi_y0 + p.c.roi_h > im.height)
        return fail(LOP_ERR_INVALID, "region [%d,%d)+%dx%d outside the %d x %d image", is->x0,
                    is->y0, p.c.roi_w, p.c.roi_h, im.width, im.height);
    p.c.batch = im.batch;
    p.op = op == LOP_REDUCE_SUM ? lop::RED_SUM : op == LOP_REDUCE_MIN ? lop::RED_MIN
         : op == LOP_REDUCE_MAX ? lop::RED_MAX : lop::RED_SUMSQ;
    p.u8 = im.dtype == LOP_U8;
    p.work = d_work;
    p.result = d_result;
    cudaError_t e = lop::launch_global_reduce(p, static_cast<cudaStream_t>(cuda_stream));
    return launched(e, "global reduce launch");
}

// -------------------------------- two local operators + point-operator epilogue
lop_status lop_convolve2_execute(const lop_iteration_space *is, const lop_accessor *in,
                                 const lop_mask *a, const lop_mask *b, int32_t combine,
                                 void *cuda_stream)
{
    if (combine < LOP_COMBINE_L2 || combine > LOP_COMBINE_SUMSQ)
        return fail(LOP_ERR_INVALID, "unknown combine %d (L2, L1, SUMSQ)", combine);
    Prepared pp;
    lop_status st = prepare(is, in, pp);
    if (st) return st;
    const lop::Common &c = pp.c;
    if (!a || !a->coeffs || !b || !b->coeffs) return fail(LOP_ERR_INVALID, "mask is NULL");
    const int sx = 2 * c.rx + 1, sy = 2 * c.ry + 1;
    if (a->size_x != sx || a->size_y != sy || b->size_x != sx || b->size_y != sy)
        return fail(LOP_ERR_INVALID, "masks must both be the window size %d x %d", sx, sy);
    if (c.rx > lop::kPairMaxR || c.ry > lop::kPairMaxR)
        return fail(LOP_ERR_UNSUPPORTED, "window %d x %d larger than 31 x 31", sx, sy);
    const int32_t idt = in->bc->image.dtype, odt = is->image.dtype;
    int u8 = 0;
    if (idt == LOP_F32 && odt == LOP_F32) {
        if (a->dtype != LOP_F32 || b->dtype != LOP_F32 || a->shift || b->shift)
            return fail(LOP_ERR_INVALID, "F32 images need F32 masks with shift 0");
        u8 = 0;
    } else if (idt == LOP_U8 && odt == LOP_I32) {
        if (a->dtype != LOP_I32 || b->dtype != LOP_I32 || a->shift || b->shift)
            return fail(LOP_ERR_INVALID, "U8 images need I32 masks with shift 0");
        if (combine == LOP_COMBINE_L2)
            return fail(LOP_ERR_INVALID, "LOP_COMBINE_L2 needs F32 images (U8 -> I32 is exact: L1 or SUMSQ)");
        u8 = 1;
        int64_t la = 0, lb = 0;
        for (int i = 0; i < sx * sy; ++i) {
            const int32_t va = static_cast<const int32_t *>(a->coeffs)[i];
            const int32_t vb = static_cast<const int32_t *>(b->coeffs)[i];
            la += va < 0 ? -(int64_t)va : va;
            lb += vb < 0 ? -(int64_t)vb : vb;
        }
        const int64_t ma = 255 * la, mb = 255 * lb;
        if (ma * ma + mb * mb >= (1ll << 31))
            return fail(LOP_ERR_UNSUPPORTED, "integer masks too large: the combined value may overflow int32");
    } else {
        return fail(LOP_ERR_INVALID, "unsupported dtype combination %d -> %d (F32->F32, U8->I32)",
                    idt, odt);
    }
    cudaStream_t stream = static_cast<cudaStream_t>(cuda_stream);
    // tiled: both masks exactly separable (the convolution's own factorisation)
    static thread_local lop::ConvGeneric g;
    static thread_local lop::ConvPair tp;
    bool sep = c.rx == c.ry && c.rx >= 1 && c.rx <= 2 && g_variant != LOP_VARIANT_GENERIC;
    for (int k = 0; k < 2 && sep; ++k) {
        const lop_mask *m = k ? b : a;
        g.c = c;
        g.kind = u8 ? lop::CONV_U8_I32 : lop::CONV_F32;
        g.shift = 0;
        for (int i = 0; i < sx * sy; ++i) {
            if (u8) g.m.i[i] = static_cast<const int32_t *>(m->coeffs)[i];
            else g.m.f[i] = static_cast<const float *>(m->coeffs)[i];
        }
        lop::ConvSep &s = k ? tp.b : tp.a;
        sep = lop::conv_factor(g, s);
        s.c = c;
        s.kind = g.kind;
        s.shift = 0;
    }
    if (sep) {
        tp.combine = combine;
        tp.u8 = u8;
        cudaError_t e = lop::launch_conv_pair(tp, stream);
        if (e != cudaErrorNotSupported) return launched(e, "conv_pair launch");
    }
    if (g_variant == LOP_VARIANT_TILED)
        return fail(LOP_ERR_UNSUPPORTED, "no tiled instance for this mask pair");
    static thread_local lop::ConvPairGeneric gp;
    gp.c = c;
    gp.combine = combine;
    gp.u8 = u8;
    for (int i = 0; i < sx * sy; ++i) {
        if (u8) {
            gp.ia[i] = static_cast<const int32_t *>(a->coeffs)[i];
            gp.ib[i] = static_cast<const int32_t *>(b->coeffs)[i];
        } else {
            gp.ma[i] = static_cast<const float *>(a->coeffs)[i];
            gp.mb[i] = static_cast<const float *>(b->coeffs)[i];
        }
    }
    return launched(lop::launch_conv_pair_generic(gp, stream), "conv_pair_generic launch");
}

// ------------------------------------------------- fused two-stage operator
namespace {
// One stage's mask -> exact separable factors (reusing the convolution path).
lop_status chain_stage(const lop::Common &c, const lop_mask *m, int32_t img_dtype,
                       lop::ConvSep &s, const char *name)
{
    if (!m || !m->coeffs) return fail(LOP_ERR_INVALID, "%s mask is NULL", name);
    if (m->size_x != m->size_y || !(m->size_x & 1))
        return fail(LOP_ERR_UNSUPPORTED, "%s mask must be square and odd", name);
    const int r = m->size_x / 2;
    if (r < 1 || r > 2) return fail(LOP_ERR_UNSUPPORTED, "%s mask must be 3x3 or 5x5", name);
    static thread_local lop::ConvGeneric g;
    g.c = c;
    g.c.rx = g.c.ry = r;
    const int n = m->size_x * m->size_y;
    if (img_dtype == LOP_F32) {
        if (m->dtype != LOP_F32 || m->shift != 0)
            return fail(LOP_ERR_INVALID, "%s mask must be F32 with shift 0", name);
        g.kind = lop::CONV_F32;
        std::memcpy(g.m.f, m->coeffs, sizeof(float) * n);
    } else {
        if (m->dtype != LOP_I32 || m->shift < 0 || m->shift > 30)
            return fail(LOP_ERR_INVALID, "%s mask must be I32 with shift in 0..30", name);
        g.kind = lop::CONV_U8_U8;
        std::memcpy(g.m.i, m->coeffs, sizeof(int32_t) * n);
    }
    g.shift = m->shift;
    if (!lop::conv_factor(g, s))
        return fail(LOP_ERR_UNSUPPORTED, "%s mask is not exactly separable", name);
    s.c = g.c;
    s.kind = g.kind;
    s.shift = g.shift;
    return LOP_OK;
}
}  // namespace

namespace {
// Shared validation of the chain calls: both stages factored, the accessor's
// window = the combined footprint, whole images.
lop_status chain_prepare(const lop_iteration_space *is, const lop_accessor *in,
                         const lop_mask *first, const lop_mask *second, Prepared &pp,
                         lop::ConvChain &p)
{
    if (!first || !second) return fail(LOP_ERR_INVALID, "mask is NULL");
    if (in && in->bc &&
        (in->bc->size_x != first->size_x + second->size_x - 1 ||
         in->bc->size_y != first->size_y + second->size_y - 1))
        return fail(LOP_ERR_INVALID,
                    "boundary condition window %d x %d must be the combined footprint %d x %d",
                    in->bc->size_x, in->bc->size_y, first->size_x + second->size_x - 1,
                    first->size_y + second->size_y - 1);
    lop_status st = prepare(is, in, pp);
    if (st) return st;
    const lop::Common &c = pp.c;
    const lop_image &ii = in->bc->image;
    if (ii.halo_top || ii.halo_bottom || ii.global_y0 ||
        (ii.global_height && ii.global_height != ii.height))
        return fail(LOP_ERR_UNSUPPORTED, "fused chains take whole images (no band views)");
    const int32_t idt = ii.dtype, odt = is->image.dtype;
    if (idt == LOP_F32 && odt == LOP_F32) p.kind = 0;
    else if (idt == LOP_U8 && odt == LOP_U8) p.kind = 1;
    else if (idt == LOP_U8 && odt == LOP_I32) p.kind = 2;
    else return fail(LOP_ERR_INVALID, "unsupported dtype combination %d -> %d", idt, odt);
    st = chain_stage(c, first, idt, p.s1, "first");
    if (st) return st;
    return chain_stage(c, second, idt, p.s2, "second");
}

// Intermediate image of the two-pass route: the whole input extent in the
// input's dtype, rows 16-byte aligned.
int64_t chain_ws_pitch(const lop_image &ii) { return ((int64_t)ii.width * elem_size(ii.dtype) + 15) & ~(int64_t)15; }
int64_t chain_ws_bytes(const lop_image &ii) { return chain_ws_pitch(ii) * ii.height * ii.batch; }
}  // namespace

lop_status lop_convolve_chain_execute(const lop_iteration_space *is, const lop_accessor *in,
                                      const lop_mask *first, const lop_mask *second,
                                      void *cuda_stream)
{
    Prepared pp;
    static thread_local lop::ConvChain p;
    lop_status st = chain_prepare(is, in, first, second, pp, p);
    if (st) return st;
    cudaError_t e = lop::launch_conv_chain(p, static_cast<cudaStream_t>(cuda_stream));
    if (e == cudaErrorNotSupported)
        return fail(LOP_ERR_UNSUPPORTED, "no fused chain instance for this mask pair");
    return launched(e, "conv_chain launch");
}

lop_status lop_convolve_chain_workspace_bytes(const lop_iteration_space *is, const lop_accessor *in,
                                              const lop_mask *first, const lop_mask *second,
                                              int64_t *bytes)
{
    if (!bytes) return fail(LOP_ERR_INVALID, "bytes is NULL");
    Prepared pp;
    static thread_local lop::ConvChain p;
    lop_status st = chain_prepare(is, in, first, second, pp, p);
    if (st) return st;
    *bytes = chain_ws_bytes(in->bc->image);
    return LOP_OK;
}

lop_status lop_convolve_chain_execute_ws(const lop_iteration_space *is, const lop_accessor *in,
                                         const lop_mask *first, const lop_mask *second,
                                         void *d_workspace, int64_t workspace_bytes,
                                         void *cuda_stream)
{
    Prepared pp;
    static thread_local lop::ConvChain p;
    lop_status st = chain_prepare(is, in, first, second, pp, p);
    if (st) return st;
    const lop_image &ii = in->bc->image;
    bool two_pass = d_workspace && workspace_bytes >= chain_ws_bytes(ii);
    if (const char *env = std::getenv("LOP_CHAIN_FUSED")) two_pass = two_pass && std::atoi(env) == 0;
    if (!two_pass) return lop_convolve_chain_execute(is, in, first, second, cuda_stream);
    // Two passes through the workspace (DESIGN.md §6 "Fused chain"): on B200
    // the intermediate of a 4096^2 image (64 MiB f32 / 16 MiB u8) stays in the
    // 126 MB L2 between the passes, and the two HBM-bound separable kernels
    // beat the fused kernel; bit-identical to it by construction (the fused
    // kernel reproduces exactly these two passes).
    lop_image g = ii;                                       // G: whole input extent
    g.data = d_workspace;
    g.stride_bytes = chain_ws_pitch(ii);
    g.batch_stride_bytes = g.stride_bytes * ii.height;
    {
        cudaPointerAttributes attr;
        if (cudaPointerGetAttributes(&attr, d_workspace) != cudaSuccess ||
            (attr.type != cudaMemoryTypeDevice && attr.type != cudaMemoryTypeManaged)) {
            cudaGetLastError();
            return fail(LOP_ERR_INVALID, "workspace must be device memory");
        }
    }
    lop_iteration_space is1{};
    is1.image = g;
    lop_boundary_condition bc1 = *in->bc;
    bc1.size_x = first->size_x;
    bc1.size_y = first->size_y;
    lop_accessor a1{&bc1, 0, 0};
    st = lop_convolve_execute(&is1, &a1, first, cuda_stream);
    if (st) return st;
    lop_boundary_condition bc2 = *in->bc;
    bc2.image = g;
    bc2.size_x = second->size_x;
    bc2.size_y = second->size_y;
    lop_accessor a2{&bc2, in->offset_x, in->offset_y};
    return lop_convolve_execute(is, &a2, second, cuda_stream);
}

// ------------------------------------- local operator over several accessors
lop_status lop_local_execute(const lop_iteration_space *is, const lop_accessor *const *inputs,
                             const lop_mask *const *masks, int32_t n_inputs, int32_t op,
                             int32_t tap_fn, void *cuda_stream)
{
    return lop_local_execute_point(is, inputs, masks, n_inputs, op, tap_fn, nullptr, nullptr,
                                   cuda_stream);
}

lop_status lop_local_execute_point(const lop_iteration_space *is, const lop_accessor *const *inputs,
                                   const lop_mask *const *masks, int32_t n_inputs, int32_t op,
                                   int32_t tap_fn, const double *scale, const double *offset,
                                   void *cuda_stream)
{
    if (!inputs || !masks) return fail(LOP_ERR_INVALID, "inputs / masks is NULL");
    if (n_inputs < 1 || n_inputs > LOP_MAX_ACCESSORS)
        return fail(LOP_ERR_INVALID, "n_inputs %d outside 1..%d", n_inputs, LOP_MAX_ACCESSORS);
    if (op != LOP_REDUCE_SUM && op != LOP_REDUCE_MIN && op != LOP_REDUCE_MAX)
        return fail(LOP_ERR_INVALID, "unknown reduction %d (SUM, MIN, MAX)", op);
    if (tap_fn < LOP_TAP_PRODUCT || tap_fn > LOP_TAP_SQUARE)
        return fail(LOP_ERR_INVALID, "unknown tap function %d", tap_fn);
    static thread_local lop::LocalParams p;
    p.n = n_inputs;
    p.op = op == LOP_REDUCE_SUM ? lop::RED_SUM : (op == LOP_REDUCE_MIN ? lop::RED_MIN : lop::RED_MAX);
    p.fn = tap_fn;
    int taps = 0, rx = 0, ry = 0;
    bool any_tap = false;
    double bound = 0.0;                               // worst-case |out| (integer path)
    p.any_point = 0;
    for (int k = 0; k < n_inputs; ++k) {
        Prepared pp;
        lop_status st = prepare(is, inputs[k], pp);
        if (st) return fail(st, "accessor %d: %s", k, lop_last_error());
        const lop::Common &c = pp.c;
        const int32_t idt = inputs[k]->bc->image.dtype;
        if (k == 0) {
            p.c = c;
            const int32_t odt = is->image.dtype;
            if (idt == LOP_F32 && odt == LOP_F32) p.u8 = 0;
            else if (idt == LOP_U8 && odt == LOP_I32) p.u8 = 1;
            else return fail(LOP_ERR_INVALID, "unsupported dtype combination %d -> %d (F32 -> F32, U8 -> I32)",
                             idt, odt);
        } else if ((idt == LOP_U8) != (p.u8 == 1)) {
            return fail(LOP_ERR_INVALID, "accessor %d: every input must have the same dtype", k);
        }
        if (c.rx > lop::kLocalMaxR || c.ry > lop::kLocalMaxR)
            return fail(LOP_ERR_UNSUPPORTED, "accessor %d: window larger than 31 x 31", k);
        const lop_mask *m = masks[k];
        const int sx = 2 * c.rx + 1, sy = 2 * c.ry + 1;
        if (!m || !m->coeffs) return fail(LOP_ERR_INVALID, "mask %d is NULL", k);
        if (m->size_x != sx || m->size_y != sy)
            return fail(LOP_ERR_INVALID, "mask %d is %d x %d, its accessor's window %d x %d", k,
                        m->size_x, m->size_y, sx, sy);
        if (m->dtype != (p.u8 ? LOP_I32 : LOP_F32) || m->shift != 0)
            return fail(LOP_ERR_INVALID, "mask %d: %s images need %s masks with shift 0", k,
                        p.u8 ? "U8" : "F32", p.u8 ? "I32" : "F32");
        if (taps + sx * sy > lop::kLocalMaxTaps)
            return fail(LOP_ERR_UNSUPPORTED, "masks have more than %d taps in total", lop::kLocalMaxTaps);
        lop::LocalAcc &a = p.acc[k];
        a.in = c.in;
        a.off_x = c.off_x;
        a.off_y = c.off_y;
        a.mode = c.mode;
        a.rx = c.rx;
        a.ry = c.ry;
        a.cval_f = c.cval_f;
        a.cval_i = c.cval_i;
        a.moff = taps;
        // point-operator prologue Read' = pa * Read + pb (reading c27)
        const double pa = scale ? scale[k] : 1.0, pb = offset ? offset[k] : 0.0;
        if (!std::isfinite(pa) || !std::isfinite(pb))
            return fail(LOP_ERR_INVALID, "accessor %d: point operator %g * v + %g not finite", k, pa, pb);
        double lo = 0.0, hi = 255.0;                  // range of the (mapped) reads, u8 path
        if (p.u8) {
            if (pa != std::floor(pa) || pb != std::floor(pb) || std::fabs(pa) > 65536.0 ||
                std::fabs(pb) > 65536.0)
                return fail(LOP_ERR_INVALID,
                            "accessor %d: U8 point operator needs integers |scale|, |offset| <= 2^16", k);
            a.pa_i = (int32_t)pa;
            a.pb_i = (int32_t)pb;
            a.point = a.pa_i != 1 || a.pb_i != 0;
            lo = std::min(pb, 255.0 * pa + pb);
            hi = std::max(pb, 255.0 * pa + pb);
        } else {
            a.pa_f = (float)pa;
            a.pb_f = (float)pb;
            a.point = a.pa_f != 1.0f || a.pb_f != 0.0f;
        }
        p.any_point |= a.point;
        const double vmax = std::max(std::fabs(lo), std::fabs(hi));
        const double gmax = tap_fn == LOP_TAP_SQDIFF ? (hi - lo) * (hi - lo)
                          : tap_fn == LOP_TAP_SQUARE ? vmax * vmax
                          : tap_fn == LOP_TAP_ABSDIFF ? hi - lo : vmax;
        double l1 = 0.0, mx = 0.0;
        for (int i = 0; i < sx * sy; ++i) {
            if (p.u8) {
                const int32_t v = static_cast<const int32_t *>(m->coeffs)[i];
                p.m.i[taps + i] = v;
                any_tap |= v != 0;
                l1 += std::fabs((double)v);
                mx = std::max(mx, std::fabs((double)v));
            } else {
                const float v = static_cast<const float *>(m->coeffs)[i];
                if (!std::isfinite(v)) return fail(LOP_ERR_INVALID, "mask %d coefficient %d not finite", k, i);
                p.m.f[taps + i] = v;
                any_tap |= v != 0.0f;
            }
        }
        bound += op == LOP_REDUCE_SUM ? l1 * gmax : 0.0;
        if (op != LOP_REDUCE_SUM) bound = std::max(bound, mx * gmax);
        taps += sx * sy;
        rx = std::max(rx, c.rx);
        ry = std::max(ry, c.ry);
    }
    if (op != LOP_REDUCE_SUM && !any_tap)
        return fail(LOP_ERR_INVALID, "MIN / MAX need at least one non-zero mask coefficient");
    if (p.u8 && bound >= 2147483647.0)
        return fail(LOP_ERR_UNSUPPORTED, "integer masks too large: the result may overflow int32");
    p.c.rx = rx;                                     // the largest window (L556-L558)
    p.c.ry = ry;
    // small-window path: every mask embedded centred in a 7 x 7 slot
    p.small = rx <= lop::kLocalSmallR && ry <= lop::kLocalSmallR;
    if (const char *env = std::getenv("LOP_LOCAL_SMALL")) p.small = p.small && std::atoi(env) != 0;
    if (p.small) {
        constexpr int SR = lop::kLocalSmallR, SW = lop::kLocalSmallW;
        std::memset(&p.ms, 0, sizeof p.ms);
        for (int k = 0; k < n_inputs; ++k) {
            const lop::LocalAcc &a = p.acc[k];
            const int sx = 2 * a.rx + 1;
            for (int yf = -a.ry; yf <= a.ry; ++yf)
                for (int xf = -a.rx; xf <= a.rx; ++xf) {
                    const int src = a.moff + (yf + a.ry) * sx + xf + a.rx, dst = (yf + SR) * SW + xf + SR;
                    if (p.u8) p.ms.i[k][dst] = p.m.i[src];
                    else p.ms.f[k][dst] = p.m.f[src];
                }
        }
    }
    const bool tiled = g_variant != LOP_VARIANT_GENERIC;
    return launched(lop::launch_local(p, tiled, static_cast<cudaStream_t>(cuda_stream)),
                    "local launch");
}

}  // extern "C"

// ------------------------------------------ multiresolution filter (N4, c28)
namespace {

int pyr_half(int n) { return (n + 1) / 2; }

// Whole, unbanded F32 image (pyramid levels).
lop_status pyr_check_level(const lop_image &im, const char *name)
{
    lop_status st = check_image(im, name);
    if (st) return st;
    if (im.dtype != LOP_F32) return fail(LOP_ERR_INVALID, "%s: pyramid levels are F32 images", name);
    if (im.halo_top || im.halo_bottom || im.global_y0 ||
        (im.global_height && im.global_height != im.height))
        return fail(LOP_ERR_INVALID, "%s: pyramid levels are whole images (no band views)", name);
    return LOP_OK;
}

// Common validation of REDUCE / EXPAND; reduce: the output is the coarse level.
lop_status pyr_prepare(const lop_iteration_space *is, const lop_accessor *in, bool reduce,
                       lop::PyrParams &p)
{
    if (!is) return fail(LOP_ERR_INVALID, "iteration space is NULL");
    if (!in || !in->bc) return fail(LOP_ERR_INVALID, "accessor / boundary condition is NULL");
    const lop_boundary_condition &bc = *in->bc;
    lop_status st = pyr_check_level(bc.image, "input");
    if (st) return st;
    st = pyr_check_level(is->image, "output");
    if (st) return st;
    const lop_image &ii = bc.image, &oi = is->image;
    if (bc.mode < LOP_CLAMP || bc.mode > LOP_CONSTANT)
        return fail(LOP_ERR_INVALID, "pyramid boundary mode %d: CLAMP, REPEAT, MIRROR or CONSTANT", bc.mode);
    if (bc.size_x != 5 || bc.size_y != 5)
        return fail(LOP_ERR_INVALID, "pyramid window must be 5 x 5 (the binomial), got %d x %d", bc.size_x,
                    bc.size_y);
    if (in->offset_x || in->offset_y) return fail(LOP_ERR_INVALID, "pyramid accessors take no offset");
    if (!std::isfinite(bc.constant)) return fail(LOP_ERR_INVALID, "constant is not finite");
    if (is->x0 || is->y0 || (is->width && is->width != oi.width) || (is->height && is->height != oi.height))
        return fail(LOP_ERR_INVALID, "pyramid levels are computed whole (no ROI)");
    if (ii.batch != oi.batch) return fail(LOP_ERR_INVALID, "input/output batch differ");
    const lop_image &fine = reduce ? ii : oi, &coarse = reduce ? oi : ii;
    if (coarse.width != pyr_half(fine.width) || coarse.height != pyr_half(fine.height))
        return fail(LOP_ERR_INVALID, "coarse level %d x %d is not ceil(%d/2) x ceil(%d/2)", coarse.width,
                    coarse.height, fine.width, fine.height);
    st = check_disjoint(ii, oi);
    if (st) return st;
    std::memset(&p, 0, sizeof p);
    p.in = make_geom(ii);
    p.out.data = static_cast<char *>(oi.data);
    p.out.stride = oi.stride_bytes;
    p.out.bstride = oi.batch > 1 ? oi.batch_stride_bytes : 0;
    p.out.W = oi.width;
    p.out.H = oi.height;
    p.mode = bc.mode;
    p.cval = (float)bc.constant;
    p.batch = oi.batch;
    p.sign = 1.0f;
    return LOP_OK;
}

struct PyrLevel {
    int32_t w, h;
    int64_t stride, frame, bytes;     // row pitch, frame bytes, all frames (256-B rounded)
};

PyrLevel pyr_level(int32_t w, int32_t h, int32_t batch)
{
    PyrLevel L;
    L.w = w;
    L.h = h;
    L.stride = ((int64_t)w * 4 + 15) & ~(int64_t)15;
    L.frame = L.stride * h;
    L.bytes = (L.frame * batch + 255) & ~(int64_t)255;
    return L;
}

lop_image pyr_view(void *data, const PyrLevel &L, int32_t batch)
{
    lop_image im;
    std::memset(&im, 0, sizeof im);
    im.data = data;
    im.width = L.w;
    im.height = L.h;
    im.stride_bytes = L.stride;
    im.dtype = LOP_F32;
    im.batch = batch;
    im.batch_stride_bytes = L.frame;
    return im;
}

// Workspace: the Gaussian levels 1 .. L-1, then T0 (band-pass level 0, later
// the filtered levels 1 .. L-1).
int64_t multires_layout(int32_t w, int32_t h, int32_t batch, int32_t levels, PyrLevel *lv,
                        int64_t *goff, int64_t *t0off, int64_t *foff)
{
    lv[0] = pyr_level(w, h, batch);
    for (int l = 1; l < levels; ++l) lv[l] = pyr_level(pyr_half(lv[l - 1].w), pyr_half(lv[l - 1].h), batch);
    int64_t off = 0;
    for (int l = 1; l < levels; ++l) { goff[l] = off; off += lv[l].bytes; }
    *t0off = off;
    int64_t fsum = 0;
    for (int l = 1; l < levels; ++l) { foff[l] = off + fsum; fsum += lv[l].bytes; }
    return off + std::max(levels > 1 ? lv[0].bytes : (int64_t)0, fsum);
}

constexpr int kMaxLevels = 16;

}  // namespace

extern "C" {

lop_status lop_pyramid_reduce_execute(const lop_iteration_space *is, const lop_accessor *in,
                                      void *cuda_stream)
{
    lop::PyrParams p;
    lop_status st = pyr_prepare(is, in, true, p);
    if (st) return st;
    return launched(lop::launch_pyr_reduce(p, static_cast<cudaStream_t>(cuda_stream)), "pyramid reduce launch");
}

lop_status lop_pyramid_expand_execute(const lop_iteration_space *is, const lop_accessor *in,
                                      const lop_image *addend, float sign, void *cuda_stream)
{
    lop::PyrParams p;
    lop_status st = pyr_prepare(is, in, false, p);
    if (st) return st;
    if (!std::isfinite(sign)) return fail(LOP_ERR_INVALID, "sign is not finite");
    p.sign = sign;
    if (addend) {
        st = pyr_check_level(*addend, "addend");
        if (st) return st;
        const lop_image &oi = is->image;
        if (addend->width != oi.width || addend->height != oi.height || addend->batch != oi.batch)
            return fail(LOP_ERR_INVALID, "addend %d x %d x %d differs from the output %d x %d x %d",
                        addend->width, addend->height, addend->batch, oi.width, oi.height, oi.batch);
        const bool same = addend->data == oi.data && addend->stride_bytes == oi.stride_bytes &&
                          (oi.batch == 1 || addend->batch_stride_bytes == oi.batch_stride_bytes);
        if (!same) {
            st = check_disjoint(*addend, oi);
            if (st) return fail(LOP_ERR_INVALID, "addend must be the output itself or disjoint from it");
        }
        st = check_disjoint(in->bc->image, *addend);
        if (st) return st;
        p.add = static_cast<const char *>(addend->data);
        p.add_stride = addend->stride_bytes;
        p.add_bstride = addend->batch > 1 ? addend->batch_stride_bytes : 0;
    }
    return launched(lop::launch_pyr_expand(p, static_cast<cudaStream_t>(cuda_stream)), "pyramid expand launch");
}

lop_status lop_multires_workspace_bytes(int32_t width, int32_t height, int32_t batch, int32_t levels,
                                        int64_t *bytes)
{
    if (!bytes) return fail(LOP_ERR_INVALID, "bytes is NULL");
    if (width <= 0 || height <= 0 || batch <= 0) return fail(LOP_ERR_INVALID, "empty image");
    if (levels < 1 || levels > kMaxLevels) return fail(LOP_ERR_INVALID, "levels %d outside 1..%d", levels, kMaxLevels);
    PyrLevel lv[kMaxLevels];
    int64_t goff[kMaxLevels], foff[kMaxLevels], t0;
    *bytes = multires_layout(width, height, batch, levels, lv, goff, &t0, foff);
    return LOP_OK;
}

lop_status lop_multires_bilateral_execute(const lop_iteration_space *is, const lop_accessor *in,
                                          int32_t levels, float sigma_d, const float *sigma_r,
                                          void *d_workspace, int64_t workspace_bytes,
                                          void *cuda_stream)
{
    if (!is || !in || !in->bc) return fail(LOP_ERR_INVALID, "iteration space / accessor is NULL");
    if (levels < 1 || levels > kMaxLevels) return fail(LOP_ERR_INVALID, "levels %d outside 1..%d", levels, kMaxLevels);
    if (!sigma_r) return fail(LOP_ERR_INVALID, "sigma_r is NULL");
    if (!(sigma_d > 0.0f) || !std::isfinite(sigma_d)) return fail(LOP_ERR_INVALID, "sigma_d must be > 0");
    for (int l = 0; l < levels; ++l)
        if (!std::isfinite(sigma_r[l])) return fail(LOP_ERR_INVALID, "sigma_r[%d] is not finite", l);
    const lop_boundary_condition &bc = *in->bc;
    const lop_image &ii = bc.image, &oi = is->image;
    lop_status st = pyr_check_level(ii, "input");
    if (st) return st;
    st = pyr_check_level(oi, "output");
    if (st) return st;
    if (ii.width != oi.width || ii.height != oi.height || ii.batch != oi.batch)
        return fail(LOP_ERR_INVALID, "input and output differ in size or batch");
    if (bc.mode < LOP_CLAMP || bc.mode > LOP_CONSTANT)
        return fail(LOP_ERR_INVALID, "multiresolution mode %d: CLAMP, REPEAT, MIRROR or CONSTANT", bc.mode);
    if (in->offset_x || in->offset_y) return fail(LOP_ERR_INVALID, "the multiresolution accessor takes no offset");
    if (is->x0 || is->y0 || (is->width && is->width != oi.width) || (is->height && is->height != oi.height))
        return fail(LOP_ERR_INVALID, "the multiresolution filter is computed whole (no ROI)");
    st = check_disjoint(ii, oi);
    if (st) return st;
    PyrLevel lv[kMaxLevels];
    int64_t goff[kMaxLevels], foff[kMaxLevels], t0off;
    const int64_t need = multires_layout(oi.width, oi.height, oi.batch, levels, lv, goff, &t0off, foff);
    if (need > 0 && (!d_workspace || workspace_bytes < need))
        return fail(LOP_ERR_INVALID, "workspace of %lld bytes needed (%lld given)", (long long)need,
                    (long long)workspace_bytes);
    if (reinterpret_cast<uintptr_t>(d_workspace) & 15) return fail(LOP_ERR_INVALID, "workspace not 16-B aligned");
    const cudaStream_t stream = static_cast<cudaStream_t>(cuda_stream);
    char *ws = static_cast<char *>(d_workspace);
    const int32_t B = oi.batch;
    lop_image G[kMaxLevels], F[kMaxLevels];
    G[0] = ii;
    for (int l = 1; l < levels; ++l) G[l] = pyr_view(ws + goff[l], lv[l], B);
    const lop_image T0 = pyr_view(ws + t0off, lv[0], B);

    auto bcond = [&](const lop_image &im, int sx, int sy, double cval) {
        lop_boundary_condition c;
        c.image = im;
        c.mode = bc.mode;
        c.size_x = sx;
        c.size_y = sy;
        c.constant = cval;
        return c;
    };
    auto space = [](const lop_image &im) {
        lop_iteration_space s;
        std::memset(&s, 0, sizeof s);
        s.image = im;
        return s;
    };
    // 1. Gaussian levels
    for (int l = 0; l + 1 < levels; ++l) {
        const lop_boundary_condition c = bcond(G[l], 5, 5, bc.constant);
        const lop_accessor a{&c, 0, 0};
        const lop_iteration_space s = space(G[l + 1]);
        st = lop_pyramid_reduce_execute(&s, &a, cuda_stream);
        if (st) return st;
    }
    // 2. band-pass levels: B_0 -> T0, B_l (l >= 1) in place of G_l
    lop_image Bv[kMaxLevels];
    for (int l = 0; l + 1 < levels; ++l) {
        Bv[l] = l == 0 ? T0 : G[l];
        const lop_boundary_condition c = bcond(G[l + 1], 5, 5, bc.constant);
        const lop_accessor a{&c, 0, 0};
        const lop_iteration_space s = space(Bv[l]);
        st = lop_pyramid_expand_execute(&s, &a, &G[l], -1.0f, cuda_stream);
        if (st) return st;
    }
    Bv[levels - 1] = G[levels - 1];
    // 3. filtered levels: F_0 -> out; F_l (l >= 1) -> T0's sub-buffers, after F_0
    for (int l = 0; l < levels; ++l) {
        const double cval = l == levels - 1 ? bc.constant : 0.0;   // band-pass levels read 0
        lop_image dst = l == 0 ? oi : pyr_view(ws + foff[l], lv[l], B);
        if (sigma_r[l] > 0.0f) {
            const lop_boundary_condition c = bcond(Bv[l], bc.size_x, bc.size_y, cval);
            const lop_accessor a{&c, 0, 0};
            const lop_iteration_space s = space(dst);
            st = lop_bilateral_execute(&s, &a, nullptr, sigma_d, sigma_r[l], cuda_stream);
            if (st) return fail(st, "level %d bilateral: %s", l, lop_last_error());
            F[l] = dst;
        } else if (l == 0) {                                        // unfiltered level 0: copy to out
            for (int b = 0; b < B; ++b) {
                const cudaError_t e = cudaMemcpy2DAsync(
                    static_cast<char *>(oi.data) + (int64_t)b * (B > 1 ? oi.batch_stride_bytes : 0), oi.stride_bytes,
                    static_cast<const char *>(Bv[0].data) + (int64_t)b * (B > 1 ? Bv[0].batch_stride_bytes : 0),
                    Bv[0].stride_bytes, (size_t)oi.width * 4, oi.height, cudaMemcpyDeviceToDevice, stream);
                if (e != cudaSuccess) return cuda_fail(e, "level 0 copy");
            }
            F[0] = oi;
        } else {
            F[l] = Bv[l];
        }
    }
    // 4. reconstruction, coarse to fine, in place on F_l (F_0 = out)
    for (int l = levels - 2; l >= 0; --l) {
        const lop_boundary_condition c = bcond(F[l + 1], 5, 5, bc.constant);
        const lop_accessor a{&c, 0, 0};
        const lop_iteration_space s = space(F[l]);
        st = lop_pyramid_expand_execute(&s, &a, &F[l], 1.0f, cuda_stream);
        if (st) return st;
    }
    return LOP_OK;
}

}  // extern "C"

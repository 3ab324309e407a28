/*
 * lop_oracle.c -- plain, slow, obviously-correct CPU ORACLE for the local
 * operators of Membarth et al., "Generating Device-specific GPU Code for Local
 * Operators in Medical Imaging", IPDPS 2012.
 *
 *   *** TEST INFRASTRUCTURE ONLY. ***
 *   Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 *   --impl reference legs may load this library.  The product path
 *   (paper_conf_ipps_membarthhtke12_b200/) never calls it, shares no code,
 *   header, table or constant with it, and neither side includes the other.
 *
 * Arithmetic: IEEE double throughout (the paper fixes no precision for the
 * reference semantics; the GPU path is f32 and is compared within 1e-5).
 * Integer (u8) operators: exact int64 sums.
 * No blocking, fusion or reordering: every output is the brute-force double
 * loop of Algorithm 1 in its stated order (yf outer,
 * xf inner).  OpenMP only distributes independent output rows over cores.
 *
 * Citations are PAPER.md line numbers ("Lnnn"); readings of ambiguous
 * passages are the ones listed in DESIGN.md section "Readings" (= SURVEY §8(c)).
 *
 * Parity pins: see tests/test_oracle_pins.py.  Every function below is pinned
 * by at least one test against something other than itself (Fig. 2 golden
 * cells, np.pad / scipy.ndimage library routines, the paper's printed mask
 * value 0.018316, closed-form invariants, hand-computed worked examples).
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#ifdef _OPENMP
#include <omp.h>
#endif

/* Boundary handling modes, Table I.  Numbering is part
 * of the test interface only. */
enum { OR_UNDEFINED = 0, OR_CLAMP = 1, OR_REPEAT = 2, OR_MIRROR = 3, OR_CONSTANT = 4 };

int oracle_num_threads(void)
{
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

/*
 * Per-axis index adjustment, PAPER.md L340-L357 ("adjusting the index of the
 * accessed pixel to a pixel that resides within the image"), Table I and
 * Fig. 2 (L359-L432).  Returns the in-image index, or -1 when the access is
 * out of bounds and the mode does not remap (Constant, Undefined).
 *   clamp : last valid pixel within image               (Fig. 2c)
 *   repeat: image repeated at the border (true modulo)   (Fig. 2b, reading c7)
 *   mirror: mirrored at the border, edge pixel repeated  (Fig. 2d edges, reading c6)
 */
int64_t oracle_map_index(int64_t i, int64_t n, int mode)
{
    if (i >= 0 && i < n)
        return i;
    switch (mode) {
    case OR_CLAMP:
        return i < 0 ? 0 : n - 1;
    case OR_REPEAT: {
        int64_t q = i % n;
        if (q < 0) q += n;
        return q;
    }
    case OR_MIRROR: {
        int64_t period = 2 * n;
        int64_t q = i % period;
        if (q < 0) q += period;
        return q < n ? q : period - 1 - q;
    }
    default: /* OR_CONSTANT, OR_UNDEFINED */
        return -1;
    }
}

/*
 * Read(x', y') of the virtually expanded image:
 * in range -> the pixel; out of range -> Constant: the user constant
 * (Table I; reading c8: if either axis is out of bounds), Clamp/Repeat/
 * Mirror: the pixel at the per-axis adjusted indices; Undefined: not
 * specified (L295) -> *undef is set and the value must not be used.
 */
static double read_f32(const float *img, int64_t W, int64_t H, int64_t stride,
                       int64_t x, int64_t y, int mode, double cval, int *undef)
{
    if (x >= 0 && x < W && y >= 0 && y < H)
        return (double)img[y * stride + x];
    if (mode == OR_CONSTANT)
        return cval;
    if (mode == OR_UNDEFINED) {
        *undef = 1;
        return 0.0;
    }
    int64_t mx = oracle_map_index(x, W, mode);
    int64_t my = oracle_map_index(y, H, mode);
    return (double)img[my * stride + mx];
}

static int64_t read_u8(const uint8_t *img, int64_t W, int64_t H, int64_t stride,
                       int64_t x, int64_t y, int mode, int64_t cval, int *undef)
{
    if (x >= 0 && x < W && y >= 0 && y < H)
        return (int64_t)img[y * stride + x];
    if (mode == OR_CONSTANT)
        return cval;
    if (mode == OR_UNDEFINED) {
        *undef = 1;
        return 0;
    }
    int64_t mx = oracle_map_index(x, W, mode);
    int64_t my = oracle_map_index(y, H, mode);
    return (int64_t)img[my * stride + mx];
}

/* The same Read() applied to one output of a 4x4 (or any) test image, exported
 * so the Fig. 2 golden cells can be checked cell by cell. */
double oracle_read_f32(const float *img, int64_t W, int64_t H, int64_t stride,
                       int64_t x, int64_t y, int mode, double cval, int *undef)
{
    *undef = 0;
    return read_f32(img, W, H, stride, x, y, mode, cval, undef);
}

/*
 * Closeness, Eq. (1) (reading c2):
 *   closeness((x,y),(x',y')) = exp(-1/2 * (||(x,y)-(x',y')|| / sigma_d)^2)
 * Mask layout (reading c4): row-major, yf outer, first element (-m,-n);
 * Listing 4 (L364-L372) stores it as Mask<float> CMask(4*sigma_d+1, ...).
 */
void oracle_closeness_mask(double sigma_d, int mw, int mh, double *mask)
{
    int m = mw / 2, n = mh / 2;
    for (int yf = -n; yf <= n; ++yf)
        for (int xf = -m; xf <= m; ++xf) {
            double dist = sqrt((double)(xf * xf + yf * yf));
            mask[(yf + n) * mw + (xf + m)] = exp(-0.5 * (dist / sigma_d) * (dist / sigma_d));
        }
}

/* Binomial Gaussian masks (reading c11): outer product of row n of Pascal's
 * triangle with itself; returns the normalising shift k (sum = 2^k). */
int oracle_gaussian_mask_int(int size, int32_t *mask)
{
    int64_t row[64];
    if (size < 1 || size > 63 || (size % 2) == 0)
        return -1;
    row[0] = 1;
    for (int i = 1; i < size; ++i) {          /* Pascal: row_i from row_{i-1} */
        row[i] = 0;
        for (int j = i; j >= 1; --j)
            row[j] = row[j] + row[j - 1];
    }
    for (int y = 0; y < size; ++y)
        for (int x = 0; x < size; ++x)
            mask[y * size + x] = (int32_t)(row[y] * row[x]);
    return 2 * (size - 1);
}

/* Sobel 3x3 (reading c12): dir 0 = x-gradient [[-1,0,1],[-2,0,2],[-1,0,1]]
 * (correlation, reading c5); dir 1 = its transpose (y-gradient). */
void oracle_sobel_mask_int(int dir, int32_t *mask)
{
    static const int32_t smooth[3] = {1, 2, 1};
    static const int32_t deriv[3] = {-1, 0, 1};
    for (int y = 0; y < 3; ++y)
        for (int x = 0; x < 3; ++x)
            mask[y * 3 + x] = dir == 0 ? smooth[y] * deriv[x] : deriv[y] * smooth[x];
}

/* ------------------------------------------------------------------ */
/* Local operator: convolution with a filter mask (PAPER.md L274-L282:  */
/* window (2m+1)x(2n+1), mask centred at [0,0]; Listing 5 / Listing 9  */
/* multiply Mask(xf,yf) by Input(xf,yf): correlation, reading c5).     */
/* ------------------------------------------------------------------ */

static double conv_px_f32(const float *img, int64_t W, int64_t H, int64_t stride,
                          const double *mask, int mw, int mh, int mode, double cval,
                          int64_t x, int64_t y, uint8_t *valid)
{
    int m = mw / 2, n = mh / 2, undef = 0;
    double acc = 0.0;
    for (int yf = -n; yf <= n; ++yf)
        for (int xf = -m; xf <= m; ++xf)
            acc += mask[(yf + n) * mw + (xf + m)] *
                   read_f32(img, W, H, stride, x + xf, y + yf, mode, cval, &undef);
    *valid = (uint8_t)!undef;
    return acc;
}

void oracle_convolve_f32(const float *img, int64_t W, int64_t H, int64_t stride,
                         const double *mask, int mw, int mh, int mode, double cval,
                         int64_t y0, int64_t y1, double *out, uint8_t *valid)
{
#pragma omp parallel for schedule(dynamic, 1)
    for (int64_t y = y0; y < y1; ++y)
        for (int64_t x = 0; x < W; ++x) {
            int64_t o = (y - y0) * W + x;
            out[o] = conv_px_f32(img, W, H, stride, mask, mw, mh, mode, cval, x, y, &valid[o]);
        }
}

void oracle_convolve_f32_points(const float *img, int64_t W, int64_t H, int64_t stride,
                                const double *mask, int mw, int mh, int mode, double cval,
                                const int64_t *xs, const int64_t *ys, int64_t npts,
                                double *out, uint8_t *valid)
{
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < npts; ++i)
        out[i] = conv_px_f32(img, W, H, stride, mask, mw, mh, mode, cval, xs[i], ys[i], &valid[i]);
}

/* Integer path: exact sum S = sum M(xf,yf) * Read(x+xf, y+yf). */
static int64_t conv_px_u8(const uint8_t *img, int64_t W, int64_t H, int64_t stride,
                          const int32_t *mask, int mw, int mh, int mode, int64_t cval,
                          int64_t x, int64_t y, uint8_t *valid)
{
    int m = mw / 2, n = mh / 2, undef = 0;
    int64_t acc = 0;
    for (int yf = -n; yf <= n; ++yf)
        for (int xf = -m; xf <= m; ++xf)
            acc += (int64_t)mask[(yf + n) * mw + (xf + m)] *
                   read_u8(img, W, H, stride, x + xf, y + yf, mode, cval, &undef);
    *valid = (uint8_t)!undef;
    return acc;
}

void oracle_convolve_u8_sum(const uint8_t *img, int64_t W, int64_t H, int64_t stride,
                            const int32_t *mask, int mw, int mh, int mode, int64_t cval,
                            int64_t y0, int64_t y1, int64_t *out, uint8_t *valid)
{
#pragma omp parallel for schedule(dynamic, 1)
    for (int64_t y = y0; y < y1; ++y)
        for (int64_t x = 0; x < W; ++x) {
            int64_t o = (y - y0) * W + x;
            out[o] = conv_px_u8(img, W, H, stride, mask, mw, mh, mode, cval, x, y, &valid[o]);
        }
}

void oracle_convolve_u8_sum_points(const uint8_t *img, int64_t W, int64_t H, int64_t stride,
                                   const int32_t *mask, int mw, int mh, int mode, int64_t cval,
                                   const int64_t *xs, const int64_t *ys, int64_t npts,
                                   int64_t *out, uint8_t *valid)
{
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < npts; ++i)
        out[i] = conv_px_u8(img, W, H, stride, mask, mw, mh, mode, cval, xs[i], ys[i], &valid[i]);
}

/* ------------------------------------------------------------------ */
/* Local reduction over a mask domain: Listing 9's                      */
/*   output() = convolve(cMask, <reduction>, [&] () { ... })            */
/* with the MIN / MAX reductions (grey-value       */
/* erosion / dilation; the SUM form is the convolution above).  The     */
/* domain is the set of taps whose mask coefficient is non-zero; taps   */
/* are visited yf outer, xf inner, each read through Read() with the    */
/* boundary mode.  op: 1 = min, 2 = max.                                */
/* ------------------------------------------------------------------ */
static double reduce_px_f32(const float *img, int64_t W, int64_t H, int64_t stride,
                            const int32_t *dom, int mw, int mh, int op, int mode, double cval,
                            int64_t x, int64_t y, uint8_t *valid)
{
    int m = mw / 2, n = mh / 2, undef = 0, first = 1;
    double acc = 0.0;
    for (int yf = -n; yf <= n; ++yf)
        for (int xf = -m; xf <= m; ++xf) {
            if (!dom[(yf + n) * mw + (xf + m)])
                continue;
            double v = read_f32(img, W, H, stride, x + xf, y + yf, mode, cval, &undef);
            if (first || (op == 1 ? v < acc : v > acc))
                acc = v;
            first = 0;
        }
    *valid = (uint8_t)!undef;
    return acc;
}

static int64_t reduce_px_u8(const uint8_t *img, int64_t W, int64_t H, int64_t stride,
                            const int32_t *dom, int mw, int mh, int op, int mode, int64_t cval,
                            int64_t x, int64_t y, uint8_t *valid)
{
    int m = mw / 2, n = mh / 2, undef = 0, first = 1;
    int64_t acc = 0;
    for (int yf = -n; yf <= n; ++yf)
        for (int xf = -m; xf <= m; ++xf) {
            if (!dom[(yf + n) * mw + (xf + m)])
                continue;
            int64_t v = read_u8(img, W, H, stride, x + xf, y + yf, mode, cval, &undef);
            if (first || (op == 1 ? v < acc : v > acc))
                acc = v;
            first = 0;
        }
    *valid = (uint8_t)!undef;
    return acc;
}

void oracle_reduce_f32(const float *img, int64_t W, int64_t H, int64_t stride,
                       const int32_t *dom, int mw, int mh, int op, int mode, double cval,
                       int64_t y0, int64_t y1, double *out, uint8_t *valid)
{
#pragma omp parallel for schedule(dynamic, 1)
    for (int64_t y = y0; y < y1; ++y)
        for (int64_t x = 0; x < W; ++x) {
            int64_t o = (y - y0) * W + x;
            out[o] = reduce_px_f32(img, W, H, stride, dom, mw, mh, op, mode, cval, x, y, &valid[o]);
        }
}

void oracle_reduce_u8(const uint8_t *img, int64_t W, int64_t H, int64_t stride,
                      const int32_t *dom, int mw, int mh, int op, int mode, int64_t cval,
                      int64_t y0, int64_t y1, int64_t *out, uint8_t *valid)
{
#pragma omp parallel for schedule(dynamic, 1)
    for (int64_t y = y0; y < y1; ++y)
        for (int64_t x = 0; x < W; ++x) {
            int64_t o = (y - y0) * W + x;
            out[o] = reduce_px_u8(img, W, H, stride, dom, mw, mh, op, mode, cval, x, y, &valid[o]);
        }
}

/* Output quantisation of the integer sum (reading c12): rounding half-up by
 * (S + 2^(k-1)) >> k (arithmetic shift = floor), then for u8 outputs
 * saturation to [0, 255]; i32 outputs keep the shifted value. */
int64_t oracle_quantize(int64_t S, int shift, int to_u8)
{
    int64_t v = S;
    if (shift > 0) {
        int64_t num = S + ((int64_t)1 << (shift - 1));
        /* floor division by 2^shift, valid for negative numerators too */
        int64_t d = (int64_t)1 << shift;
        v = num >= 0 ? num / d : -((-num + d - 1) / d);
    }
    if (to_u8) {
        if (v < 0) v = 0;
        if (v > 255) v = 255;
    }
    return v;
}

/* ------------------------------------------------------------------ */
/* Bilateral filter, Algorithm 1, Eq. (1)-(2)     */
/* (L187-L193), Listings 1 and 5 (L204-L265, L379-L416).                */
/* ------------------------------------------------------------------ */

static double bilateral_px(const float *img, int64_t W, int64_t H, int64_t stride,
                           const double *cmask, int mw, int mh, double sigma_d,
                           double sigma_r, int mode, double cval, int64_t x, int64_t y,
                           uint8_t *valid)
{
    int m = mw / 2, n = mh / 2, undef = 0;
    double center = (double)img[y * stride + x];   /* input[x, y]: always in range */
    double p = 0.0, k = 0.0;                        /* Alg. 1 line 5 */
    for (int yf = -n; yf <= n; ++yf)                /* Alg. 1 line 6 */
        for (int xf = -m; xf <= m; ++xf) {          /* Alg. 1 line 7 */
            double v = read_f32(img, W, H, stride, x + xf, y + yf, mode, cval, &undef);
            double c;                               /* Alg. 1 line 8 */
            if (cmask) {
                c = cmask[(yf + n) * mw + (xf + m)];   /* Listing 5 l.10: CMask(xf,yf) */
            } else {
                double dist = sqrt((double)(xf * xf + yf * yf));
                c = exp(-0.5 * (dist / sigma_d) * (dist / sigma_d));   /* Eq. (1) */
            }
            double dp = fabs(v - center);
            double s = exp(-0.5 * (dp / sigma_r) * (dp / sigma_r)); /* Eq. (2), Alg. 1 line 9 */
            k = k + c * s;                          /* Alg. 1 line 10 */
            p = p + c * s * v;                      /* Alg. 1 line 11 */
        }
    *valid = (uint8_t)!undef;
    return p / k;                                   /* Alg. 1 line 14 */
}

void oracle_bilateral_f32(const float *img, int64_t W, int64_t H, int64_t stride,
                          const double *cmask, int mw, int mh, double sigma_d,
                          double sigma_r, int mode, double cval, int64_t y0, int64_t y1,
                          double *out, uint8_t *valid)
{
#pragma omp parallel for schedule(dynamic, 1)
    for (int64_t y = y0; y < y1; ++y)
        for (int64_t x = 0; x < W; ++x) {
            int64_t o = (y - y0) * W + x;
            out[o] = bilateral_px(img, W, H, stride, cmask, mw, mh, sigma_d, sigma_r, mode,
                                  cval, x, y, &valid[o]);
        }
}

void oracle_bilateral_f32_points(const float *img, int64_t W, int64_t H, int64_t stride,
                                 const double *cmask, int mw, int mh, double sigma_d,
                                 double sigma_r, int mode, double cval,
                                 const int64_t *xs, const int64_t *ys, int64_t npts,
                                 double *out, uint8_t *valid)
{
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < npts; ++i)
        out[i] = bilateral_px(img, W, H, stride, cmask, mw, mh, sigma_d, sigma_r, mode, cval,
                              xs[i], ys[i], &valid[i]);
}

/* ------------------------------------------------------------------ */
/* Local operator over several Accessors.            */
/* "In case multiple Accessors are used within one */
/* kernel, the largest window size specified is taken"; L160-L162 and */
/* L315-L318: an Accessor reads its input through its own               */
/* BoundaryCondition (mode, window) at an offset; Listing 9 (L961-L964):*/
/*   output() = convolve(cMask, SUM, [&] () {                           */
/*                  return cMask() * Input(cMask); });                  */
/* -- a reduction over the mask's taps of a per-tap function.  Here K   */
/* accessors k, each with its own mask M_k (size mw_k x mh_k, odd),     */
/* offset (ox_k, oy_k), mode and constant; f from a fixed set           */
/* (reading c22):                                                       */
/*   fn 0 PRODUCT  f = M * v             (Listing 9's cMask()*Input())  */
/*   fn 1 ABSDIFF  f = M * |v - c|       c = Read_k(x + ox_k, y + oy_k) */
/*   fn 2 SQDIFF   f = M * (v - c)^2         (the accessor's own centre) */
/*   fn 3 SQUARE   f = M * v^2                                          */
/* and the reduction op 0 SUM (over all taps), 1 MIN, 2 MAX (over the    */
/* taps with M != 0, reading c18):                                       */
/*   out(x, y) = op_{k, yf, xf} f(M_k(xf, yf),                          */
/*                  Read_k(x + ox_k + xf, y + oy_k + yf), c_k)           */
/* Point-operator prologue (reading c27): every read */
/* of accessor k is Read'_k = pa_k * Read_k + pb_k (centre included).    */
/* Undefined mode: the output is valid iff no read of any accessor      */
/* (its whole window, centre included) leaves its image (reading c9).   */
/* f32 images: double arithmetic; u8 images: exact int64.               */
/* ------------------------------------------------------------------ */
static double tap_fn_f64(int fn, double M, double v, double c)
{
    switch (fn) {
    case 1: return M * fabs(v - c);
    case 2: return M * (v - c) * (v - c);
    case 3: return M * v * v;
    default: return M * v;
    }
}

static int64_t tap_fn_i64(int fn, int64_t M, int64_t v, int64_t c)
{
    switch (fn) {
    case 1: return M * (v > c ? v - c : c - v);
    case 2: return M * (v - c) * (v - c);
    case 3: return M * v * v;
    default: return M * v;
    }
}

static double local_px_f32(int K, const float *const *imgs, const int64_t *strides, int64_t W,
                           int64_t H, const double *const *masks, const int *mws, const int *mhs,
                           const int *oxs, const int *oys, const int *modes, const double *cvals,
                           const double *pa, const double *pb, int op, int fn, int64_t x,
                           int64_t y, uint8_t *valid)
{
    int undef = 0, first = 1;
    double acc = 0.0;
    for (int k = 0; k < K; ++k) {
        const int m = mws[k] / 2, n = mhs[k] / 2;
        const int64_t cx = x + oxs[k], cy = y + oys[k];
        const double c = pa[k] * read_f32(imgs[k], W, H, strides[k], cx, cy, modes[k], cvals[k],
                                          &undef) + pb[k];
        for (int yf = -n; yf <= n; ++yf)
            for (int xf = -m; xf <= m; ++xf) {
                const double M = masks[k][(yf + n) * mws[k] + (xf + m)];
                const double v = pa[k] * read_f32(imgs[k], W, H, strides[k], cx + xf, cy + yf,
                                                  modes[k], cvals[k], &undef) + pb[k];
                if (op == 0) {
                    acc += tap_fn_f64(fn, M, v, c);
                } else if (M != 0.0) {
                    const double f = tap_fn_f64(fn, M, v, c);
                    if (first || (op == 1 ? f < acc : f > acc)) acc = f;
                    first = 0;
                }
            }
    }
    *valid = (uint8_t)!undef;
    return acc;
}

static int64_t local_px_u8(int K, const uint8_t *const *imgs, const int64_t *strides, int64_t W,
                           int64_t H, const int32_t *const *masks, const int *mws, const int *mhs,
                           const int *oxs, const int *oys, const int *modes, const int64_t *cvals,
                           const int64_t *pa, const int64_t *pb, int op, int fn, int64_t x,
                           int64_t y, uint8_t *valid)
{
    int undef = 0, first = 1;
    int64_t acc = 0;
    for (int k = 0; k < K; ++k) {
        const int m = mws[k] / 2, n = mhs[k] / 2;
        const int64_t cx = x + oxs[k], cy = y + oys[k];
        const int64_t c = pa[k] * read_u8(imgs[k], W, H, strides[k], cx, cy, modes[k], cvals[k],
                                          &undef) + pb[k];
        for (int yf = -n; yf <= n; ++yf)
            for (int xf = -m; xf <= m; ++xf) {
                const int64_t M = masks[k][(yf + n) * mws[k] + (xf + m)];
                const int64_t v = pa[k] * read_u8(imgs[k], W, H, strides[k], cx + xf, cy + yf,
                                                  modes[k], cvals[k], &undef) + pb[k];
                if (op == 0) {
                    acc += tap_fn_i64(fn, M, v, c);
                } else if (M != 0) {
                    const int64_t f = tap_fn_i64(fn, M, v, c);
                    if (first || (op == 1 ? f < acc : f > acc)) acc = f;
                    first = 0;
                }
            }
    }
    *valid = (uint8_t)!undef;
    return acc;
}

void oracle_local_f32(int K, const float *const *imgs, const int64_t *strides, int64_t W,
                      int64_t H, const double *const *masks, const int *mws, const int *mhs,
                      const int *oxs, const int *oys, const int *modes, const double *cvals,
                      const double *pa, const double *pb, int op, int fn, int64_t y0, int64_t y1,
                      double *out, uint8_t *valid)
{
#pragma omp parallel for schedule(dynamic, 1)
    for (int64_t y = y0; y < y1; ++y)
        for (int64_t x = 0; x < W; ++x) {
            int64_t o = (y - y0) * W + x;
            out[o] = local_px_f32(K, imgs, strides, W, H, masks, mws, mhs, oxs, oys, modes, cvals,
                                  pa, pb, op, fn, x, y, &valid[o]);
        }
}

void oracle_local_u8(int K, const uint8_t *const *imgs, const int64_t *strides, int64_t W,
                     int64_t H, const int32_t *const *masks, const int *mws, const int *mhs,
                     const int *oxs, const int *oys, const int *modes, const int64_t *cvals,
                     const int64_t *pa, const int64_t *pb, int op, int fn, int64_t y0, int64_t y1,
                     int64_t *out, uint8_t *valid)
{
#pragma omp parallel for schedule(dynamic, 1)
    for (int64_t y = y0; y < y1; ++y)
        for (int64_t x = 0; x < W; ++x) {
            int64_t o = (y - y0) * W + x;
            out[o] = local_px_u8(K, imgs, strides, W, H, masks, mws, mhs, oxs, oys, modes, cvals,
                                 pa, pb, op, fn, x, y, &valid[o]);
        }
}

/* ------------------------------------------------------------------ */
/* Multiresolution filter: PAPER.md L309-L314 -- "a */
/* multiresolution filter (see [7]) ... the image gets upsampled       */
/* multiple times", with Mirror at the borders -- read as a Laplacian  */
/* pyramid whose band-pass levels are filtered by the bilateral filter */
/* (reading c28).  Images here are double (the pyramid's intermediate  */
/* levels are not f32 data in the oracle).                             */
/*   w = [1 4 6 4 1] / 16 (the binomial of the paper's Gaussian)       */
/*   REDUCE: G'(x, y) = sum_{j=-2..2} sum_{i=-2..2} w(i) w(j)          */
/*                      Read_G(2x + i, 2y + j),                        */
/*           G' of size ceil(W/2) x ceil(H/2)                          */
/*   EXPAND: E(x, y) = sum_{j=-2..2} sum_{i=-2..2} 4 w(i) w(j)         */
/*                     Read_G'((x - i) / 2, (y - j) / 2)               */
/*           over the taps with x - i and y - j even; Read applies the */
/*           boundary mode at the level being read.                    */
/* Modes: Clamp / Repeat / Mirror / Constant (Undefined has no pyramid */
/* meaning: its reads would leave every border output unspecified).   */
/* ------------------------------------------------------------------ */

static double read_f64(const double *img, int64_t W, int64_t H, int64_t x, int64_t y, int mode,
                       double cval)
{
    if (x >= 0 && x < W && y >= 0 && y < H)
        return img[y * W + x];
    if (mode == OR_CONSTANT)
        return cval;
    return img[oracle_map_index(y, H, mode) * W + oracle_map_index(x, W, mode)];
}

static const double PYR_W[5] = {1.0 / 16, 4.0 / 16, 6.0 / 16, 4.0 / 16, 1.0 / 16};

void oracle_pyr_reduce_f64(const double *g, int64_t W, int64_t H, int mode, double cval,
                           double *out)
{
    const int64_t Wc = (W + 1) / 2, Hc = (H + 1) / 2;
#pragma omp parallel for schedule(dynamic, 1)
    for (int64_t y = 0; y < Hc; ++y)
        for (int64_t x = 0; x < Wc; ++x) {
            double acc = 0.0;
            for (int j = -2; j <= 2; ++j)
                for (int i = -2; i <= 2; ++i)
                    acc += PYR_W[i + 2] * PYR_W[j + 2] *
                           read_f64(g, W, H, 2 * x + i, 2 * y + j, mode, cval);
            out[y * Wc + x] = acc;
        }
}

/* floor((v) / 2) for the even v the caller passes (exact for negatives) */
static int64_t half_even(int64_t v) { return v >= 0 ? v / 2 : -((-v) / 2); }

void oracle_pyr_expand_f64(const double *gc, int64_t Wc, int64_t Hc, int64_t W, int64_t H,
                           int mode, double cval, double *out)
{
#pragma omp parallel for schedule(dynamic, 1)
    for (int64_t y = 0; y < H; ++y)
        for (int64_t x = 0; x < W; ++x) {
            double acc = 0.0;
            for (int j = -2; j <= 2; ++j) {
                if ((y - j) % 2 != 0) continue;
                for (int i = -2; i <= 2; ++i) {
                    if ((x - i) % 2 != 0) continue;
                    acc += 4.0 * PYR_W[i + 2] * PYR_W[j + 2] *
                           read_f64(gc, Wc, Hc, half_even(x - i), half_even(y - j), mode, cval);
                }
            }
            out[y * W + x] = acc;
        }
}

/* Bilateral filter of a double image: Alg. 1 exactly as bilateral_px     */
/* (closeness from Eq. (1), similarity Eq. (2)), for the pyramid levels.  */
void oracle_bilateral_f64(const double *img, int64_t W, int64_t H, int mw, int mh,
                          double sigma_d, double sigma_r, int mode, double cval, double *out)
{
    const int m = mw / 2, n = mh / 2;
#pragma omp parallel for schedule(dynamic, 1)
    for (int64_t y = 0; y < H; ++y)
        for (int64_t x = 0; x < W; ++x) {
            const double center = img[y * W + x];
            double p = 0.0, k = 0.0;
            for (int yf = -n; yf <= n; ++yf)
                for (int xf = -m; xf <= m; ++xf) {
                    const double v = read_f64(img, W, H, x + xf, y + yf, mode, cval);
                    const double dist = sqrt((double)(xf * xf + yf * yf));
                    const double c = exp(-0.5 * (dist / sigma_d) * (dist / sigma_d));
                    const double dp = fabs(v - center);
                    const double s = exp(-0.5 * (dp / sigma_r) * (dp / sigma_r));
                    k = k + c * s;
                    p = p + c * s * v;
                }
            out[y * W + x] = p / k;
        }
}

/*
 * lop.h -- C ABI of the B200-native local-operator library ("lop").
 *
 * The calls mirror the problem statement of Membarth, Hannig, Teich, Koerner,
 * Eckert, "Generating Device-specific GPU Code for Local Operators in Medical
 * Imaging", IPDPS 2012 (cited as PAPER.md line numbers "Lnnn"):
 *
 *   Image             lop_image               (§II; Listing 2 l.8-9)
 *   IterationSpace    lop_iteration_space     (§II; Listing 2 l.15)
 *   BoundaryCondition lop_boundary_condition  (§III-A; Listing 3)
 *   Accessor          lop_accessor            (§II; L315-L318)
 *   Mask              lop_mask                (§III-B; Listing 4)
 *   Kernel::execute   lop_bilateral_execute / lop_convolve_execute
 *                                             (Listing 2 l.21-24; Listing 5)
 *
 * Conventions (all entry points):
 *   - Ownership: the caller owns every host and device buffer.  The library
 *     never allocates on the execute path; mask coefficients are copied into
 *     the kernel's parameter block at the call, so the caller may free them on
 *     return (no __constant__ symbol, no global device state).
 *     The host pipeline (lop_pipeline_*) owns the device staging buffers it
 *     allocates in lop_pipeline_create and frees in lop_pipeline_destroy.
 *   - Asynchrony: execute calls enqueue work on `cuda_stream` (a cudaStream_t,
 *     NULL = legacy default stream) and return without synchronising.
 *   - Errors: every function returns a lop_status.  Invalid arguments return
 *     LOP_ERR_INVALID before anything is launched; launch failures return
 *     LOP_ERR_CUDA.  lop_last_error() returns a thread-local message for the
 *     last non-OK status of the calling thread.  No C++ exception crosses
 *     this ABI.
 *   - Layout: images are row-major; row y of frame b starts at
 *     (char*)data + b*batch_stride_bytes + y*stride_bytes.  Rows must be
 *     addressable for y in [-halo_top, height + halo_bottom).
 *   - Index types: coordinates are int32, byte offsets int64 (a 32768^2 f32
 *     image is 4 GiB).
 *   - No in-place operation: a local operator reads input pixels that other
 *     threads may already have written, so the byte range of the input view
 *     (all frames, halo rows included) must not intersect that of the output
 *     view; overlapping views return LOP_ERR_INVALID before any launch (the
 *     check is on address ranges, so interleaved layouts are rejected too).
 */
#ifndef LOP_H
#define LOP_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define LOP_VERSION 100 /* 1.0.0 */

typedef enum {
    LOP_OK = 0,
    LOP_ERR_INVALID = -1,     /* argument validation failed; nothing launched */
    LOP_ERR_UNSUPPORTED = -2, /* valid request outside what this build supports */
    LOP_ERR_CUDA = -3         /* CUDA runtime error (message has cudaGetErrorString) */
} lop_status;

/* Pixel types (Image<T>, L150-L154).  Bilateral: F32 -> F32 (Kernel<float>,
 * Listing 1).  Convolution: F32 -> F32, U8 -> U8, U8 -> I32 (reading c12). */
typedef enum { LOP_U8 = 0, LOP_I32 = 1, LOP_F32 = 2 } lop_dtype;

/* Boundary handling modes, Table I (L290-L299), Fig. 2 (L359-L432):
 *   UNDEFINED  out-of-bounds reads are not specified: outputs whose window
 *              leaves the image are unspecified, but the library stays
 *              memory-safe (it never reads outside the image);
 *   CLAMP      last valid pixel within the image;
 *   REPEAT     image repeated periodically (true modulo, any distance);
 *   MIRROR     mirrored at the border with the edge pixel repeated
 *              (c b a | a b c d | d c b), periodic with period 2N;
 *   CONSTANT   user-defined constant (lop_boundary_condition.constant) if
 *              either coordinate is out of bounds.
 * Index adjustment is per axis (L340-L357). */
typedef enum {
    LOP_UNDEFINED = 0,
    LOP_CLAMP = 1,
    LOP_REPEAT = 2,
    LOP_MIRROR = 3,
    LOP_CONSTANT = 4
} lop_boundary;

/* Image<T> (L150-L154): non-owning view of device memory.
 * A single image has batch = 1, halo_top = halo_bottom = 0, global_y0 = 0,
 * global_height = height (0 is accepted as "= height").
 * Frame sequences (config C4): batch = F frames, batch_stride_bytes apart.
 * Row bands (config C5): the view owns global rows
 *   [global_y0, global_y0 + height) of a global_height-row image and may read
 *   halo_top rows above / halo_bottom rows below it (filled by the caller,
 *   e.g. by the NCCL halo exchange).  Boundary modes always use the global
 *   image extent (reading c10).  A halo row that lies outside the global image
 *   is read as stored (this is how a REPEAT ring halo is supplied). */
typedef struct {
    void *data;                 /* device pointer to pixel (0, 0) of the first owned row */
    int32_t width, height;      /* owned columns / rows */
    int64_t stride_bytes;       /* row pitch, >= width * elem_size */
    int32_t dtype;              /* lop_dtype */
    int32_t batch;              /* frames, >= 1 */
    int64_t batch_stride_bytes; /* distance between frames (ignored if batch == 1) */
    int32_t halo_top, halo_bottom;
    int32_t global_y0, global_height;
} lop_image;

/* BoundaryCondition<T>(image, size_x, size_y, mode[, constant]) (Listing 3,
 * L331-L338; L329-L330).  size_x/size_y: the window of the local operator,
 * odd (L274-L282). constant: used by LOP_CONSTANT; for U8 images it must be
 * an integer in [0, 255]. */
typedef struct {
    lop_image image;
    int32_t mode;               /* lop_boundary */
    int32_t size_x, size_y;
    double constant;
} lop_boundary_condition;

/* Accessor<T> (L160-L162, L315-L318): a view of an input through a
 * BoundaryCondition; allocates nothing.  Input(xf, yf) of output (x, y) reads
 * input pixel (x + offset_x + xf, y + offset_y + yf). */
typedef struct {
    const lop_boundary_condition *bc;
    int32_t offset_x, offset_y;
} lop_accessor;

/* Mask<T>(size_x, size_y) (Listing 4): HOST pointer to
 * size_y * size_x coefficients, row-major, yf outer, first element at
 * (xf, yf) = (-m, -n) (reading c4).  dtype F32 (float coefficients) or I32
 * (integer coefficients for U8 images).  shift: for integer masks, the output
 * is (S + 2^(shift-1)) >> shift (reading c12); 0 for float masks. */
typedef struct {
    int32_t size_x, size_y;
    int32_t dtype;              /* LOP_F32 or LOP_I32 */
    const void *coeffs;         /* host memory, copied at the call */
    int32_t shift;
} lop_mask;

/* IterationSpace<T> (L155-L157): rectangular region of interest of the output
 * image; every point is one output pixel (1:1 work items, L168-L171).
 * width/height 0 = the whole output image. */
typedef struct {
    lop_image image;
    int32_t x0, y0, width, height;
} lop_iteration_space;

/* Bilateral filter (Alg. 1, Eq. 1-2, Listing 5):
 *   out(x,y) = sum c(xf,yf) s(I(x+xf,y+yf) - I(x,y)) I(x+xf,y+yf)
 *            / sum c(xf,yf) s(I(x+xf,y+yf) - I(x,y))
 *   s(d) = exp(-d^2 / (2 sigma_r^2)),
 *   c = closeness mask (coefficients > 0 required, centre > 0) or, if
 *       closeness == NULL, c = exp(-(xf^2 + yf^2) / (2 sigma_d^2)) over the
 *       BoundaryCondition's size_x x size_y window (Eq. 1).
 * Input and output: LOP_F32, same width/height/batch.
 * Window: odd, up to 63 x 63 (13 x 13 is the paper's 4*sigma_d+1 for
 * sigma_d = 3).  sigma_r > 0, sigma_d > 0 when closeness == NULL. */
lop_status lop_bilateral_execute(const lop_iteration_space *is, const lop_accessor *in,
                                 const lop_mask *closeness, float sigma_d, float sigma_r,
                                 void *cuda_stream);

/* Local operator with a filter mask (L274-L282, Listing 5 / Listing 9):
 *   S(x,y) = sum_{yf,xf} M(xf,yf) * Read(x+xf, y+yf)   (correlation, reading c5)
 * F32 -> F32 with an F32 mask: out = S.
 * U8 -> U8 with an I32 mask: out = clamp((S + 2^(k-1)) >> k, 0, 255), k = shift.
 * U8 -> I32 with an I32 mask: out = (S + 2^(k-1)) >> k (k = 0: out = S).
 * Window: odd, up to 63 x 63; mask size must equal the BoundaryCondition's. */
lop_status lop_convolve_execute(const lop_iteration_space *is, const lop_accessor *in,
                                const lop_mask *mask, void *cuda_stream);

/* Fused two-stage local operator (PAPER.md L107-L122 on
 * combining operators): out = second (*) (first (*) I), both stages with the
 * accessor's BoundaryCondition, computed in one pass without the intermediate
 * image leaving on-chip memory.  Bit-identical to two lop_convolve_execute
 * calls (the first with an intermediate of the input's type: F32, or U8
 * rounded and saturated with first->shift).
 * Masks: square 3x3 or 5x5, exactly separable (Gaussian, Sobel, box ...);
 * the BoundaryCondition window must be the combined footprint
 * (first->size + second->size - 1, the paper's "largest window" rule L556-L558).
 * dtypes: F32 -> F32, U8 -> U8, U8 -> I32.  Whole images only (no band views). */
lop_status lop_convolve_chain_execute(const lop_iteration_space *is, const lop_accessor *in,
                                      const lop_mask *first, const lop_mask *second,
                                      void *cuda_stream);
/* The same chain with a caller-owned device workspace of at least
 * lop_convolve_chain_workspace_bytes() bytes (the intermediate image, whole
 * input extent, input dtype, 16-B aligned rows): the library then runs the
 * route measured faster on B200 -- two lop_convolve_execute passes through the
 * workspace, whose intermediate stays in L2 (DESIGN.md §6 "Fused chain") --
 * with a result bit-identical to lop_convolve_chain_execute.  A NULL or too
 * small workspace runs the fused kernel.  Two kernel launches. */
lop_status lop_convolve_chain_workspace_bytes(const lop_iteration_space *is, const lop_accessor *in,
                                              const lop_mask *first, const lop_mask *second,
                                              int64_t *bytes);
lop_status lop_convolve_chain_execute_ws(const lop_iteration_space *is, const lop_accessor *in,
                                         const lop_mask *first, const lop_mask *second,
                                         void *d_workspace, int64_t workspace_bytes,
                                         void *cuda_stream);

/* Local reduction over a mask domain -- Listing 9's
 * convolve(mask, <reduction>, f) (L956-L967) with the MIN / MAX reductions
 * (grey-value erosion / dilation with a structuring element):
 *   out(x,y) = min (or max) of Read(x+xf, y+yf) over the taps with M(xf,yf) != 0
 * LOP_REDUCE_SUM is the paper's SUM form and equals lop_convolve_execute
 * (the mask's values are then the weights).
 * Images: F32 -> F32 (mask F32) or U8 -> U8 (mask I32); only whether a
 * coefficient is zero matters for MIN / MAX, and at least one must be non-zero
 * (LOP_ERR_INVALID otherwise).  Window: odd, up to 63 x 63, equal to the
 * BoundaryCondition's; boundary modes as for every local operator (Table I).
 * Exact: every output is an input value or the constant. */
typedef enum {
    LOP_REDUCE_SUM = 0,
    LOP_REDUCE_MIN = 1,
    LOP_REDUCE_MAX = 2,
    LOP_REDUCE_SUMSQ = 3        /* global operators only (lop_global_reduce_execute) */
} lop_reduce_op;
lop_status lop_reduce_execute(const lop_iteration_space *is, const lop_accessor *in,
                              const lop_mask *domain, int32_t op, void *cuda_stream);

/* Two local operators on one input combined by a point operator, in one pass
 * (PAPER.md L107-L122 -- point operators after local ones):
 *   A = Ma (*) I,  B = Mb (*) I   (correlation, as lop_convolve_execute)
 *   out = sqrt(A^2 + B^2)  (LOP_COMBINE_L2, F32 only; e.g. the Sobel gradient
 *         magnitude with Ma = Sobel-x, Mb = Sobel-y, Table IX)
 *       = |A| + |B|        (LOP_COMBINE_L1)
 *       = A^2 + B^2        (LOP_COMBINE_SUMSQ)
 * F32 -> F32 (F32 masks; the epilogue in IEEE f32: A*A, B*B, +, sqrt, each
 * rounded) or U8 -> I32 (I32 masks, shift 0; exact integers).  Both masks
 * have the BoundaryCondition's size (odd, up to 31 x 31).  When both are
 * exactly separable and 3x3 or 5x5, A and B are bit-identical to
 * lop_convolve_execute's results, so out equals the epilogue applied to two
 * separate passes, without A and B making a round trip through HBM. */
typedef enum { LOP_COMBINE_L2 = 0, LOP_COMBINE_L1 = 1, LOP_COMBINE_SUMSQ = 2 } lop_combine;
lop_status lop_convolve2_execute(const lop_iteration_space *is, const lop_accessor *in,
                                 const lop_mask *a, const lop_mask *b, int32_t combine,
                                 void *cuda_stream);

/* Global operator (one output for all pixels, "e.g. the
 * sum of all pixels"): SUM, MIN, MAX or SUMSQ of the pixels of the
 * region (x0, y0, width, height) of is->image (here the INPUT; width/height 0
 * = to the image edge), over all frames of a batch.  The result is one double
 * written to device memory d_result; d_work is a device scratch array of
 * LOP_GLOBAL_WORK_DOUBLES doubles owned by the caller, ZERO-initialised before
 * its first use (its last element is an arrival counter that every call leaves
 * at zero again; calls sharing one d_work must be ordered on one stream).
 * SUMSQ merges two pixels a, b into a^2 + b^2 ("operations
 * that merge/reduce two pixels"; reading c26): the sum of squares, which with
 * SUM gives a region's mean and variance.
 * F32 (sums accumulated in double; an f32 value's square is exact in double) or
 * U8 (exact integer sums).  Deterministic:
 * fixed partition and fixed reduction trees, so the same input gives the same
 * bits on every run.  Asynchronous on cuda_stream (one kernel launch). */
#define LOP_GLOBAL_WORK_DOUBLES 1025
lop_status lop_global_reduce_execute(const lop_iteration_space *is, int32_t op, double *d_result,
                                     double *d_work, void *cuda_stream);

/* Local operator over several Accessors with a per-tap function
 * (SURVEY §8(f) N2): PAPER.md L556-L558 ("In case multiple Accessors are used
 * within one kernel, the largest window size specified is taken") and
 * Listing 9 (L961-L964) `convolve(cMask, SUM, [&] () { return cMask() *
 * Input(cMask); })`, with the per-tap function chosen from a fixed set
 * (reading c22):
 *   out(x, y) = op over k = 0..n_inputs-1, yf, xf of
 *               f(M_k(xf, yf), Read_k(x + ox_k + xf, y + oy_k + yf), c_k)
 *   c_k = Read_k(x + ox_k, y + oy_k)           (accessor k's window centre)
 *   f:  LOP_TAP_PRODUCT  M * v            (Listing 9's cMask() * Input(cMask))
 *       LOP_TAP_ABSDIFF  M * |v - c_k|
 *       LOP_TAP_SQDIFF   M * (v - c_k)^2
 *       LOP_TAP_SQUARE   M * v^2
 *   op: LOP_REDUCE_SUM over all taps; LOP_REDUCE_MIN / _MAX over the taps
 *       with M_k != 0 (reading c18).
 * inputs[k]: an Accessor (its own image, BoundaryCondition -- mode, window,
 * constant -- and offset); masks[k]: its mask, of its BoundaryCondition's
 * window size (odd, up to 31 x 31 each, 3844 taps in total).  The launch's
 * halo is the largest window (L556-L558).  All images share the output's
 * width / height / batch.
 * dtypes: every input F32 with F32 masks -> F32 output (SUM accumulated in
 * f32 in a fixed order: per accessor one FMA chain over its taps, window rows
 * top to bottom, taps left to right; accessors in order); or every input U8 with I32
 * masks -> I32 output (exact integers; the worst-case magnitude must fit
 * int32, else LOP_ERR_UNSUPPORTED).
 * Kernel configuration: Algorithm 2 on B200 terms --
 * see lop_alg2_select. */
typedef enum {
    LOP_TAP_PRODUCT = 0,
    LOP_TAP_ABSDIFF = 1,
    LOP_TAP_SQDIFF = 2,
    LOP_TAP_SQUARE = 3
} lop_tap_fn;
#define LOP_MAX_ACCESSORS 4
lop_status lop_local_execute(const lop_iteration_space *is, const lop_accessor *const *inputs,
                             const lop_mask *const *masks, int32_t n_inputs, int32_t op,
                             int32_t tap_fn, void *cuda_stream);
/* The same local operator with a point-operator prologue per accessor
 * (point operators precede local ones in an image
 * pipeline; reading c27): every read of accessor k -- the window taps, its
 * centre c_k and, in LOP_CONSTANT mode, the boundary constant -- is replaced by
 *   Read'_k = scale[k] * Read_k + offset[k]
 * before the tap function (window/level, inversion, gain) without the mapped
 * image making a round trip through HBM.  scale / offset: n_inputs host
 * doubles each (NULL = 1 / 0 for every accessor).  F32 inputs: scale and
 * offset are rounded to f32 and applied as one f32 FMA when the footprint is
 * staged; U8 inputs: integers with |scale|, |offset| <= 2^16 (exact int32
 * arithmetic; LOP_ERR_INVALID otherwise), and the result's worst case must
 * fit int32 (LOP_ERR_UNSUPPORTED otherwise).  lop_local_execute is this call
 * with scale = offset = NULL. */
lop_status lop_local_execute_point(const lop_iteration_space *is, const lop_accessor *const *inputs,
                                   const lop_mask *const *masks, int32_t n_inputs, int32_t op,
                                   int32_t tap_fn, const double *scale, const double *offset,
                                   void *cuda_stream);

/* ---- Multiresolution filter ----
 * "a multiresolution filter (see [7]) is applied to an
 * image: the image gets upsampled multiple times", Mirror at the borders
 * avoiding artifacts.  Reading c28: a Laplacian pyramid with the
 * binomial w = [1 4 6 4 1] / 16 whose levels are bilateral-filtered.
 * Pyramid levels are whole F32 images (no ROI, no band views), batch allowed
 * (all frames at once); modes CLAMP / REPEAT / MIRROR / CONSTANT (UNDEFINED
 * is rejected: every border output of a pyramid level would be unspecified).
 *
 * REDUCE: is->image (the coarse level, ceil(W/2) x ceil(H/2), same batch)
 *   G'(x, y) = sum_{i,j=-2..2} w(i) w(j) Read(2x + i, 2y + j)
 * of the accessor's image (W x H) with its BoundaryCondition (mode,
 * constant; window 5 x 5; offset 0).  One kernel launch. */
lop_status lop_pyramid_reduce_execute(const lop_iteration_space *is, const lop_accessor *in,
                                      void *cuda_stream);
/* EXPAND: is->image (the fine level, W x H) receives
 *   out(x, y) = addend(x, y) + sign * E(x, y),
 *   E(x, y) = sum 4 w(i) w(j) Read((x - i) / 2, (y - j) / 2) over the i, j in
 *             -2..2 with x - i and y - j even,
 * Read: the accessor's image, the coarse level (ceil(W/2) x ceil(H/2)), with
 * its BoundaryCondition (window 5 x 5, offset 0).  addend: NULL (out = sign
 * E) or an F32 image of the output's size; it may be the output itself (in
 * place: each output reads only its own addend pixel) but must not partially
 * overlap it.  sign -1 gives a band-pass level G - EXPAND(G'), +1 the
 * reconstruction step.  One kernel launch. */
lop_status lop_pyramid_expand_execute(const lop_iteration_space *is, const lop_accessor *in,
                                      const lop_image *addend, float sign, void *cuda_stream);
/* The whole filter, reading c28:
 *   G_0 = input, G_{l+1} = REDUCE(G_l)            (l < levels - 1)
 *   B_l = G_l - EXPAND(G_{l+1}), B_{levels-1} = G_{levels-1}
 *   F_l = bilateral(B_l; sigma_d, sigma_r[l]) (window = the BoundaryCondition's
 *         size, closeness Eq. 1), or F_l = B_l when sigma_r[l] <= 0
 *   R_{levels-1} = F_{levels-1}, R_l = F_l + EXPAND(R_{l+1}); out = R_0.
 * in: the F32 input through its BoundaryCondition (mode for every level; in
 * CONSTANT mode the Gaussian levels read the constant and the band-pass
 * levels 0); is->image: the F32 output, same size and batch, whole image.
 * levels: 1 .. 16 (1 = the bilateral filter itself); sigma_r: `levels` host
 * floats.  d_workspace: device memory of at least
 * lop_multires_workspace_bytes() bytes (16-B aligned), owned by the caller.
 * At most 4 * levels kernel launches on cuda_stream, nothing synchronised; if a
 * launch fails part of the sequence may already be enqueued (the status says
 * which level failed) and the output is unspecified. */
lop_status lop_multires_workspace_bytes(int32_t width, int32_t height, int32_t batch,
                                        int32_t levels, int64_t *bytes);
lop_status lop_multires_bilateral_execute(const lop_iteration_space *is, const lop_accessor *in,
                                          int32_t levels, float sigma_d, const float *sigma_r,
                                          void *d_workspace, int64_t workspace_bytes,
                                          void *cuda_stream);

/* Algorithm 2, the kernel-configuration heuristic, as a
 * pure host function (no CUDA call; the library feeds it cudaOccupancy*
 * figures).  cand[i] describes configuration i: threads per CTA, its tiling
 * (block_x x block_y threads, each thread computing out_x x out_y outputs),
 * whether it fits the device's resource limits (valid) and its occupancy
 * (resident threads per SM / max threads per SM).  Lines 1-3: drop
 * configurations whose thread count is not a multiple of simd_width or that
 * are not valid; sort by descending occupancy, then ascending threads.
 * Lines 4-17 (border handling, rx | ry > 0): among the configurations with
 * the highest occupancy, take the one with the fewest threads in CTAs whose
 * footprint (tile + window radii rx, ry) leaves the width x height image
 * (ties keep the earlier one); the caller lists each thread count's tiling
 * with y preferred (block_x = simd_width).  Lines 18-20 (no border
 * handling): the first configuration (the caller lists x-preferred tilings).
 * Returns the index chosen, -1 if none is valid; *border_threads (optional)
 * receives its border-handling thread count. */
typedef struct {
    int32_t block_x, block_y;   /* threads */
    int32_t out_x, out_y;       /* outputs per thread */
    int32_t valid;              /* within the device's resource limits */
    double occupancy;           /* 0..1 */
} lop_config_candidate;
int32_t lop_alg2_select(const lop_config_candidate *cand, int32_t n, int32_t simd_width,
                        int32_t width, int32_t height, int32_t rx, int32_t ry,
                        int64_t *border_threads);

/* Mask builders (host only).
 * lop_mask_closeness: Eq. (1), float coefficients (Listing 4's mask[]).
 * lop_mask_gaussian:  binomial size x size (size odd; 1..11 for LOP_I32, 1..31
 *                     for LOP_F32); LOP_I32 writes integers and
 *                     *shift = 2*(size-1); LOP_F32 writes
 *                     the normalised floats and *shift = 0 (reading c11).
 * lop_mask_sobel:     3x3 Sobel, dir 0 = d/dx [[-1,0,1],[-2,0,2],[-1,0,1]],
 *                     dir 1 = d/dy (transpose); dtype LOP_I32 or LOP_F32. */
lop_status lop_mask_closeness(float sigma_d, int32_t size_x, int32_t size_y, float *out);
lop_status lop_mask_gaussian(int32_t size, int32_t dtype, void *out, int32_t *shift);
lop_status lop_mask_sobel(int32_t dir, int32_t dtype, void *out);

/* Kernel selection (process-wide; for tests and the tuning sweep):
 *   LOP_VARIANT_AUTO    tiled shared-memory kernels where a template instance
 *                       exists, generic otherwise (default);
 *   LOP_VARIANT_GENERIC one-thread-per-pixel kernel with per-tap remapping;
 *   LOP_VARIANT_TILED   force the tiled kernel (LOP_ERR_UNSUPPORTED if none). */
typedef enum { LOP_VARIANT_AUTO = 0, LOP_VARIANT_GENERIC = 1, LOP_VARIANT_TILED = 2 } lop_variant;
lop_status lop_set_variant(int32_t variant);
int32_t lop_get_variant(void);

/* Number of kernel launches issued by this thread since the last reset
 * (bench.py's "gpu_launches" evidence). */
int64_t lop_launch_count(void);
void lop_reset_launch_count(void);

/* Thread-local message for the last non-OK status ("" if none). */
const char *lop_last_error(void);
int32_t lop_version(void);

/* ---- Host pipeline (Listing 2 flow: IN = host_in; execute(); getData()) ----
 * End-to-end execution from pageable or pinned HOST buffers: the image is cut
 * into row chunks of `chunk_rows` rows; chunk i+1 is copied host->device while
 * chunk i is filtered and chunk i-1 copied device->host, on separate streams
 * of `device`.  Halo rows for the window are uploaded with each chunk.  The
 * pipeline allocates its device staging buffers once at create time (sized
 * for width x height x max window 63) and frees them at destroy.
 * The call returns after the result is in host_out (synchronous). */
typedef struct lop_pipeline lop_pipeline;

lop_status lop_pipeline_create(int32_t device, int32_t width, int32_t height,
                               int32_t chunk_rows, lop_pipeline **out);
lop_status lop_pipeline_bilateral(lop_pipeline *p, const float *host_in, int64_t in_stride_bytes,
                                  float *host_out, int64_t out_stride_bytes, int32_t mode,
                                  double constant, int32_t size_x, int32_t size_y,
                                  const lop_mask *closeness, float sigma_d, float sigma_r);
/* A sequence of nframes images (an angiography run, L102-L104; BASELINE config
 * 4): frame f at host_in + f * in_frame_stride_bytes, its result at host_out +
 * f * out_frame_stride_bytes.  The frames stream through the chunk ring back
 * to back -- frame f+1 uploads while frame f is filtered and downloaded --
 * so only the first upload and the last download are not overlapped.  Each
 * frame is filtered exactly as by lop_pipeline_bilateral. */
lop_status lop_pipeline_bilateral_frames(lop_pipeline *p, const float *host_in,
                                         int64_t in_stride_bytes, int64_t in_frame_stride_bytes,
                                         float *host_out, int64_t out_stride_bytes,
                                         int64_t out_frame_stride_bytes, int32_t nframes,
                                         int32_t mode, double constant, int32_t size_x,
                                         int32_t size_y, const lop_mask *closeness, float sigma_d,
                                         float sigma_r);
lop_status lop_pipeline_convolve(lop_pipeline *p, const void *host_in, int32_t in_dtype,
                                 int64_t in_stride_bytes, void *host_out, int32_t out_dtype,
                                 int64_t out_stride_bytes, int32_t mode, double constant,
                                 const lop_mask *mask);
/* Host->device and device->host bytes moved by the last pipeline call
 * (image rows + window halo rows re-uploaded at chunk seams; all frames). */
lop_status lop_pipeline_bytes(const lop_pipeline *p, int64_t *h2d, int64_t *d2h);
lop_status lop_pipeline_destroy(lop_pipeline *p);

#ifdef __cplusplus
}
#endif
#endif /* LOP_H */

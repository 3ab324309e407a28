// pipeline.cpp -- host pipeline for end-to-end execution from host buffers
// (the paper's Listing 2 flow, L201-L253: IN = host_in; BF.execute();
// host_out = OUT.getData()), overlapped on B200:
//   stream h2d : chunk k+1 host -> device (rows + window halo)
//   stream comp: chunk k filtered by the same kernels as lop_*_execute
//   stream d2h : chunk k-1 device -> host
// A ring of device staging buffers, ordered with events.  The chunk views are
// row bands of the global image (lop_image.global_y0/global_height), so the
// boundary handling is exactly that of the whole-image call; REPEAT halo rows
// outside the image are uploaded as ring rows.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstring>
#include <string>
#include <vector>
#include <chrono>
#include <cstdio>
#include <cstdlib>

#include "lop.h"

namespace lop_detail {
void set_error(const std::string &msg);   // lop_api.cpp
}

// staging buffers per direction: by default one per chunk of the schedule
// (HBM is not the constraint: 2 x 64 MiB for a 4096^2 f32 image), so no
// upload ever waits for a buffer to be released; LOP_PIPELINE_BUFS caps the
// ring (a ring of >= 2 still decouples the H2D and D2H engines).
constexpr int kBufs = 64;

struct lop_pipeline {
    int device = 0;
    int W = 0, H = 0, chunk = 0, nbufs = 0;
    size_t in_bytes = 0, out_bytes = 0;     // per staging buffer
    void *d_in[kBufs] = {};
    void *d_out[kBufs] = {};
    cudaStream_t s_h2d = nullptr, s_comp = nullptr, s_d2h = nullptr;
    cudaEvent_t up_done[kBufs] = {}, comp_done[kBufs] = {}, down_done[kBufs] = {};
    int64_t h2d_bytes = 0, d2h_bytes = 0;   // of the last run
};

namespace {

constexpr int kMaxHalo = 31;   // largest window radius (63 x 63)

lop_status perr(cudaError_t e, const char *what)
{
    lop_detail::set_error(std::string(what) + ": " + cudaGetErrorString(e));
    return LOP_ERR_CUDA;
}

lop_status pfail(lop_status st, const char *msg)
{
    lop_detail::set_error(std::string("pipeline: ") + msg);
    return st;
}

int esize(int32_t dt) { return dt == LOP_U8 ? 1 : 4; }

struct DevGuard {
    int prev = -1;
    explicit DevGuard(int dev) { cudaGetDevice(&prev); cudaSetDevice(dev); }
    ~DevGuard() { if (prev >= 0) cudaSetDevice(prev); }
};

// Row block copy: one linear DMA when both pitches equal the row width.
cudaError_t copy_rows(void *dst, int64_t dpitch, const void *src, int64_t spitch, int64_t width,
                      int64_t rows, cudaMemcpyKind kind, cudaStream_t s)
{
    if (dpitch == width && spitch == width)
        return cudaMemcpyAsync(dst, src, (size_t)(width * rows), kind, s);
    return cudaMemcpy2DAsync(dst, dpitch, src, spitch, width, rows, kind, s);
}

int64_t wrap_row(int64_t gy, int64_t H)
{
    int64_t q = gy % H;
    return q < 0 ? q + H : q;
}

// Enqueue the upload of chunk [y0, y1) with `ry` halo rows into buffer `buf`;
// returns the band view.
lop_status upload_chunk(lop_pipeline *p, int buf, const char *host, int64_t hstride, int es,
                        int32_t dtype, int y0, int y1, int ry, int mode, lop_image *view)
{
    const int64_t dstride = (int64_t)p->W * es;
    const int lo_in = std::max(0, y0 - ry), hi_in = std::min(p->H, y1 + ry);
    int halo_top = y0 - lo_in, halo_bot = hi_in - y1;
    if (mode == LOP_REPEAT) { halo_top = ry; halo_bot = ry; }   // ring rows always present
    char *base = static_cast<char *>(p->d_in[buf]);
    char *own0 = base + (int64_t)halo_top * dstride;         // row y0
    cudaError_t e;
    if (mode == LOP_REPEAT) {
        for (int gy = y0 - ry; gy < y1 + ry; ++gy) {
            if (gy >= lo_in && gy < hi_in) continue;
            const int64_t src = wrap_row(gy, p->H);
            e = cudaMemcpyAsync(own0 + (int64_t)(gy - y0) * dstride, host + src * hstride, dstride,
                                cudaMemcpyHostToDevice, p->s_h2d);
            p->h2d_bytes += dstride;
            if (e != cudaSuccess) return perr(e, "pipeline ring row upload");
        }
    }
    e = copy_rows(own0 + (int64_t)(lo_in - y0) * dstride, dstride, host + (int64_t)lo_in * hstride,
                  hstride, dstride, hi_in - lo_in, cudaMemcpyHostToDevice, p->s_h2d);
    if (e != cudaSuccess) return perr(e, "pipeline upload");
    p->h2d_bytes += (int64_t)(hi_in - lo_in) * dstride;
    std::memset(view, 0, sizeof *view);
    view->data = own0;
    view->width = p->W;
    view->height = y1 - y0;
    view->stride_bytes = dstride;
    view->dtype = dtype;
    view->batch = 1;
    view->halo_top = halo_top;
    view->halo_bottom = halo_bot;
    view->global_y0 = y0;
    view->global_height = p->H;
    return LOP_OK;
}

// Row cuts of the pipeline: chunks ramp up (c/8, c/4, c/2) at the start and
// down again at the end, so that only a small first upload and a small last
// download are not overlapped with the other direction.
std::vector<int> chunk_schedule(int H, int c)
{
    std::vector<int> sizes;
    int rest = H;
    std::vector<int> ramp;
    for (int d = 8; d >= 2; d /= 2)
        if (c / d >= 16) ramp.push_back(c / d);
    int ramp_rows = 0;
    for (int r : ramp) ramp_rows += 2 * r;
    if (ramp_rows + c > H) ramp.clear();
    for (int r : ramp) { sizes.push_back(r); rest -= r; }
    std::vector<int> tail(ramp.rbegin(), ramp.rend());
    int tail_rows = 0;
    for (int r : tail) tail_rows += r;
    rest -= tail_rows;
    while (rest > 0) { sizes.push_back(std::min(c, rest)); rest -= c; }
    for (int r : tail) sizes.push_back(r);
    std::vector<int> cuts(1, 0);
    for (int sz : sizes) cuts.push_back(cuts.back() + sz);
    return cuts;
}

// nframes images (frame f at host_in + f * in_fstride, host_out + f * out_fstride)
// stream through the same ring back to back: the chunks of frame f+1 upload
// while frame f computes and downloads, with no drain between frames.
template <typename Exec>
lop_status run(lop_pipeline *p, const void *host_in, int32_t in_dtype, int64_t in_stride,
               void *host_out, int32_t out_dtype, int64_t out_stride, int mode, double constant,
               int size_x, int size_y, Exec exec, int nframes = 1, int64_t in_fstride = 0,
               int64_t out_fstride = 0)
{
    if (!p || !host_in || !host_out) return pfail(LOP_ERR_INVALID, "NULL pipeline or host buffer");
    const int ry = size_y / 2;
    if (ry > kMaxHalo || size_x / 2 > kMaxHalo)
        return pfail(LOP_ERR_UNSUPPORTED, "window larger than 63 x 63");
    const int ies = esize(in_dtype), oes = esize(out_dtype);
    if (in_stride < (int64_t)p->W * ies || out_stride < (int64_t)p->W * oes)
        return pfail(LOP_ERR_INVALID, "host row stride smaller than the row");
    DevGuard guard(p->device);
    p->h2d_bytes = p->d2h_bytes = 0;
    static const bool trace = std::getenv("LOP_PIPELINE_TRACE") != nullptr;
    const auto t_start = std::chrono::steady_clock::now();
    if (nframes < 1) return pfail(LOP_ERR_INVALID, "nframes must be >= 1");
    const std::vector<int> cuts = chunk_schedule(p->H, p->chunk);
    const int nchunks = (int)cuts.size() - 1;
    const int ntotal = nchunks * nframes;
    // trace mode: per-chunk timeline (upload start/end, compute end, download end)
    std::vector<cudaEvent_t> tev;
    auto tmark = [&](cudaStream_t s) {
        if (!trace) return;
        cudaEvent_t ev;
        cudaEventCreate(&ev);
        cudaEventRecord(ev, s);
        tev.push_back(ev);
    };
    for (int kk = 0; kk < ntotal; ++kk) {
        const int f = kk / nchunks, k = kk - f * nchunks;       // frame, chunk within the frame
        const char *hin = static_cast<const char *>(host_in) + (int64_t)f * in_fstride;
        char *hout = static_cast<char *>(host_out) + (int64_t)f * out_fstride;
        const int buf = kk % p->nbufs;
        const int y0 = cuts[k], y1 = cuts[k + 1];
        cudaError_t e;
        if (kk >= p->nbufs) {
            e = cudaStreamWaitEvent(p->s_h2d, p->comp_done[buf], 0);
            if (e != cudaSuccess) return perr(e, "wait");
        }
        lop_image in_view;
        tmark(p->s_h2d);
        lop_status st = upload_chunk(p, buf, hin, in_stride, ies, in_dtype, y0, y1, ry, mode, &in_view);
        if (st) return st;
        tmark(p->s_h2d);
        cudaEventRecord(p->up_done[buf], p->s_h2d);
        cudaStreamWaitEvent(p->s_comp, p->up_done[buf], 0);
        if (kk >= p->nbufs) cudaStreamWaitEvent(p->s_comp, p->down_done[buf], 0);
        lop_image out_view;
        std::memset(&out_view, 0, sizeof out_view);
        out_view.data = p->d_out[buf];
        out_view.width = p->W;
        out_view.height = y1 - y0;
        out_view.stride_bytes = (int64_t)p->W * oes;
        out_view.dtype = out_dtype;
        out_view.batch = 1;
        out_view.global_y0 = y0;
        out_view.global_height = p->H;
        lop_boundary_condition bc;
        std::memset(&bc, 0, sizeof bc);
        bc.image = in_view;
        bc.mode = mode;
        bc.size_x = size_x;
        bc.size_y = size_y;
        bc.constant = constant;
        lop_accessor acc = {&bc, 0, 0};
        lop_iteration_space is;
        std::memset(&is, 0, sizeof is);
        is.image = out_view;
        tmark(p->s_comp);
        st = exec(&is, &acc, p->s_comp);
        if (st) return st;
        tmark(p->s_comp);
        cudaEventRecord(p->comp_done[buf], p->s_comp);
        cudaStreamWaitEvent(p->s_d2h, p->comp_done[buf], 0);
        e = copy_rows(hout + (int64_t)y0 * out_stride, out_stride, p->d_out[buf],
                      (int64_t)p->W * oes, (int64_t)p->W * oes, y1 - y0, cudaMemcpyDeviceToHost,
                      p->s_d2h);
        if (e != cudaSuccess) return perr(e, "pipeline download");
        p->d2h_bytes += (int64_t)(y1 - y0) * p->W * oes;
        tmark(p->s_d2h);
        cudaEventRecord(p->down_done[buf], p->s_d2h);
    }
    if (trace) {
        const double t_enq = std::chrono::duration<double, std::milli>(
                                 std::chrono::steady_clock::now() - t_start).count();
        cudaStreamSynchronize(p->s_d2h);
        const double t_all = std::chrono::duration<double, std::milli>(
                                 std::chrono::steady_clock::now() - t_start).count();
        std::fprintf(stderr, "lop_pipeline: %d chunks x %d frames, enqueue %.3f ms, total %.3f ms\n",
                     nchunks, nframes, t_enq, t_all);
        // per chunk: rows, upload [start, end], compute [start, end], download end (ms from the first mark)
        for (int k = 0; k < ntotal && (size_t)(5 * k + 4) < tev.size(); ++k) {
            float t[5];
            for (int i = 0; i < 5; ++i) cudaEventElapsedTime(&t[i], tev[0], tev[5 * k + i]);
            std::fprintf(stderr, "  chunk %2d rows %4d  up %.3f-%.3f  comp %.3f-%.3f  down-end %.3f\n", k,
                         cuts[k % nchunks + 1] - cuts[k % nchunks], t[0], t[1], t[2], t[3], t[4]);
        }
        for (cudaEvent_t ev : tev) cudaEventDestroy(ev);
    }
    cudaError_t e = cudaStreamSynchronize(p->s_d2h);
    if (e != cudaSuccess) return perr(e, "pipeline sync");
    e = cudaStreamSynchronize(p->s_comp);
    if (e != cudaSuccess) return perr(e, "pipeline sync");
    return LOP_OK;
}

}  // namespace

extern "C" {

lop_status lop_pipeline_create(int32_t device, int32_t width, int32_t height, int32_t chunk_rows,
                               lop_pipeline **out)
{
    if (!out || width <= 0 || height <= 0)
        return pfail(LOP_ERR_INVALID, "out is NULL or width/height <= 0");
    *out = nullptr;
    if (chunk_rows <= 0) chunk_rows = 512;
    chunk_rows = std::min(chunk_rows, height);
    DevGuard guard(device);
    lop_pipeline *p = new lop_pipeline;
    p->device = device;
    p->W = width;
    p->H = height;
    p->chunk = chunk_rows;
    p->in_bytes = (size_t)(chunk_rows + 2 * kMaxHalo) * width * 4;
    p->out_bytes = (size_t)chunk_rows * width * 4;
    p->nbufs = std::min(kBufs, (int)chunk_schedule(height, chunk_rows).size() - 1);
    if (const char *env = std::getenv("LOP_PIPELINE_BUFS")) p->nbufs = std::max(2, std::min(kBufs, std::atoi(env)));
    cudaError_t e = cudaSuccess;
    for (int i = 0; i < p->nbufs && e == cudaSuccess; ++i) {
        e = cudaMalloc(&p->d_in[i], p->in_bytes);
        if (e == cudaSuccess) e = cudaMalloc(&p->d_out[i], p->out_bytes);
        if (e == cudaSuccess) e = cudaEventCreateWithFlags(&p->up_done[i], cudaEventDisableTiming);
        if (e == cudaSuccess) e = cudaEventCreateWithFlags(&p->comp_done[i], cudaEventDisableTiming);
        if (e == cudaSuccess) e = cudaEventCreateWithFlags(&p->down_done[i], cudaEventDisableTiming);
    }
    if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&p->s_h2d, cudaStreamNonBlocking);
    if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&p->s_comp, cudaStreamNonBlocking);
    if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&p->s_d2h, cudaStreamNonBlocking);
    if (e != cudaSuccess) {
        lop_pipeline_destroy(p);
        return perr(e, "pipeline create");
    }
    *out = p;
    return LOP_OK;
}

lop_status lop_pipeline_bilateral(lop_pipeline *p, const float *host_in, int64_t in_stride_bytes,
                                  float *host_out, int64_t out_stride_bytes, int32_t mode,
                                  double constant, int32_t size_x, int32_t size_y,
                                  const lop_mask *closeness, float sigma_d, float sigma_r)
{
    return run(p, host_in, LOP_F32, in_stride_bytes, host_out, LOP_F32, out_stride_bytes, mode,
               constant, size_x, size_y,
               [&](const lop_iteration_space *is, const lop_accessor *acc, cudaStream_t s) {
                   return lop_bilateral_execute(is, acc, closeness, sigma_d, sigma_r, s);
               });
}

lop_status lop_pipeline_bilateral_frames(lop_pipeline *p, const float *host_in,
                                         int64_t in_stride_bytes, int64_t in_frame_stride_bytes,
                                         float *host_out, int64_t out_stride_bytes,
                                         int64_t out_frame_stride_bytes, int32_t nframes,
                                         int32_t mode, double constant, int32_t size_x,
                                         int32_t size_y, const lop_mask *closeness, float sigma_d,
                                         float sigma_r)
{
    return run(p, host_in, LOP_F32, in_stride_bytes, host_out, LOP_F32, out_stride_bytes, mode,
               constant, size_x, size_y,
               [&](const lop_iteration_space *is, const lop_accessor *acc, cudaStream_t s) {
                   return lop_bilateral_execute(is, acc, closeness, sigma_d, sigma_r, s);
               },
               nframes, in_frame_stride_bytes, out_frame_stride_bytes);
}

lop_status lop_pipeline_convolve(lop_pipeline *p, const void *host_in, int32_t in_dtype,
                                 int64_t in_stride_bytes, void *host_out, int32_t out_dtype,
                                 int64_t out_stride_bytes, int32_t mode, double constant,
                                 const lop_mask *mask)
{
    if (!mask) return pfail(LOP_ERR_INVALID, "mask is NULL");
    return run(p, host_in, in_dtype, in_stride_bytes, host_out, out_dtype, out_stride_bytes, mode,
               constant, mask->size_x, mask->size_y,
               [&](const lop_iteration_space *is, const lop_accessor *acc, cudaStream_t s) {
                   return lop_convolve_execute(is, acc, mask, s);
               });
}

lop_status lop_pipeline_bytes(const lop_pipeline *p, int64_t *h2d, int64_t *d2h)
{
    if (!p || !h2d || !d2h) return pfail(LOP_ERR_INVALID, "NULL argument");
    *h2d = p->h2d_bytes;
    *d2h = p->d2h_bytes;
    return LOP_OK;
}

lop_status lop_pipeline_destroy(lop_pipeline *p)
{
    if (!p) return LOP_OK;
    DevGuard guard(p->device);
    if (p->s_h2d) cudaStreamSynchronize(p->s_h2d);
    if (p->s_comp) cudaStreamSynchronize(p->s_comp);
    if (p->s_d2h) cudaStreamSynchronize(p->s_d2h);
    for (int i = 0; i < kBufs; ++i) {
        if (p->d_in[i]) cudaFree(p->d_in[i]);
        if (p->d_out[i]) cudaFree(p->d_out[i]);
        if (p->up_done[i]) cudaEventDestroy(p->up_done[i]);
        if (p->comp_done[i]) cudaEventDestroy(p->comp_done[i]);
        if (p->down_done[i]) cudaEventDestroy(p->down_done[i]);
    }
    if (p->s_h2d) cudaStreamDestroy(p->s_h2d);
    if (p->s_comp) cudaStreamDestroy(p->s_comp);
    if (p->s_d2h) cudaStreamDestroy(p->s_d2h);
    delete p;
    return LOP_OK;
}

}  // extern "C"

/*
 * bilateral_c.c -- the C ABI used from plain C (no Python, no torch): the
 * paper's Listing 2 host flow against include/lop.h.
 *
 *   Image<float> IN(w,h), OUT(w,h); IN = host_in;           -> cudaMalloc + cudaMemcpy
 *   BoundaryCondition BcIn(IN, 13, 13, CLAMP); Accessor AccIn -> lop_boundary_condition/accessor
 *   IterationSpace IsOut(OUT); BilateralFilter BF(...);       -> lop_iteration_space
 *   BF.execute(); host_out = OUT.getData();                  -> lop_bilateral_execute + memcpy
 *
 * Also runs the same filter through the host pipeline (lop_pipeline_*) and
 * checks that both results are identical.  Exit code 0 on success.
 * Build: nvcc -I include examples/bilateral_c.c -o examples/bilateral_c \
 *            -L paper_conf_ipps_membarthhtke12_b200 -llop -Xlinker -rpath=...
 */
#include <cuda_runtime.h>
#include <math.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include "lop.h"

#define CHECK(x)                                                                  \
    do {                                                                          \
        lop_status st_ = (x);                                                     \
        if (st_ != LOP_OK) {                                                      \
            fprintf(stderr, "%s failed (%d): %s\n", #x, (int)st_, lop_last_error()); \
            return 1;                                                             \
        }                                                                         \
    } while (0)

int main(void)
{
    const int W = 640, H = 480, sigma_d = 3;   /* Listing 2 l.1 uses 1024^2, sigma_d = 3 */
    const float sigma_r = 0.1f;
    const size_t n = (size_t)W * H;
    float *host_in = (float *)malloc(n * sizeof(float));
    float *host_out = (float *)malloc(n * sizeof(float));
    float *host_out2 = (float *)malloc(n * sizeof(float));
    for (size_t i = 0; i < n; ++i)        /* smooth pattern + edges */
        host_in[i] = 0.5f + 0.4f * sinf(0.01f * (float)(i % W)) * ((i / W) % 64 < 32 ? 1.f : -1.f);

    float *d_in = NULL, *d_out = NULL;
    if (cudaMalloc((void **)&d_in, n * 4) != cudaSuccess ||
        cudaMalloc((void **)&d_out, n * 4) != cudaSuccess) {
        fprintf(stderr, "cudaMalloc failed\n");
        return 1;
    }
    cudaMemcpy(d_in, host_in, n * 4, cudaMemcpyHostToDevice);        /* IN = host_in */

    lop_image in_img, out_img;
    memset(&in_img, 0, sizeof in_img);
    in_img.data = d_in;
    in_img.width = W;
    in_img.height = H;
    in_img.stride_bytes = (int64_t)W * 4;
    in_img.dtype = LOP_F32;
    in_img.batch = 1;
    out_img = in_img;
    out_img.data = d_out;

    lop_boundary_condition bc;                                      /* Listing 3 */
    memset(&bc, 0, sizeof bc);
    bc.image = in_img;
    bc.mode = LOP_CLAMP;
    bc.size_x = bc.size_y = 4 * sigma_d + 1;
    lop_accessor acc = {&bc, 0, 0};
    lop_iteration_space is;
    memset(&is, 0, sizeof is);
    is.image = out_img;                                              /* whole image */

    /* Listing 4: a precomputed closeness Mask */
    float mask[13 * 13];
    CHECK(lop_mask_closeness((float)sigma_d, 13, 13, mask));
    if (fabsf(mask[0] - 0.018316f) > 5e-7f) {
        fprintf(stderr, "mask[0] = %f, Listing 4 prints 0.018316\n", mask[0]);
        return 1;
    }
    lop_mask cm = {13, 13, LOP_F32, mask, 0};

    CHECK(lop_bilateral_execute(&is, &acc, &cm, (float)sigma_d, sigma_r, NULL));   /* execute() */
    if (cudaDeviceSynchronize() != cudaSuccess) return 1;
    cudaMemcpy(host_out, d_out, n * 4, cudaMemcpyDeviceToHost);     /* getData() */

    /* invalid arguments come back as LOP_ERR_INVALID with a message, nothing launched */
    bc.size_x = 12;
    if (lop_bilateral_execute(&is, &acc, NULL, 3.f, 0.1f, NULL) != LOP_ERR_INVALID) return 1;
    bc.size_x = 13;

    /* the same through the host pipeline (host buffers in, host buffers out) */
    lop_pipeline *p = NULL;
    CHECK(lop_pipeline_create(0, W, H, 128, &p));
    CHECK(lop_pipeline_bilateral(p, host_in, (int64_t)W * 4, host_out2, (int64_t)W * 4, LOP_CLAMP,
                                 0.0, 13, 13, &cm, (float)sigma_d, sigma_r));
    int64_t h2d = 0, d2h = 0;
    CHECK(lop_pipeline_bytes(p, &h2d, &d2h));
    CHECK(lop_pipeline_destroy(p));
    if (memcmp(host_out, host_out2, n * 4) != 0) {
        fprintf(stderr, "pipeline result differs from the device call\n");
        return 1;
    }
    double mean = 0;
    for (size_t i = 0; i < n; ++i) mean += host_out[i];
    printf("bilateral_c ok: %dx%d, mean %.6f, pipeline moved %lld B up / %lld B down, %lld launches\n",
           W, H, mean / (double)n, (long long)h2d, (long long)d2h, (long long)lop_launch_count());
    cudaFree(d_in);
    cudaFree(d_out);
    free(host_in);
    free(host_out);
    free(host_out2);
    return 0;
}

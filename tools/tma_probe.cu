// tma_probe.cu -- standalone probe of cp.async.bulk.tensor.3d (FLOAT64, tiled,
// no swizzle) behaviour for a given box origin: does an x origin that is not
// 16-byte aligned / negative work?  Usage: tma_probe <x> <y> <z> <boxx> <boxy>
// Prints the first loaded values or the CUDA error.  Development tool.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cudaTypedefs.h>

#include <cstdio>
#include <cstdlib>

__device__ __forceinline__ unsigned s32(const void *p) { return (unsigned)__cvta_generic_to_shared(p); }

__global__ void probe(const __grid_constant__ CUtensorMap m, int x, int y, int z, int bytes, double *out, int n) {
    extern __shared__ __align__(128) unsigned char sm[];
    double *buf = (double *)sm;
    unsigned long long *bar = (unsigned long long *)(sm + ((bytes + 127) / 128) * 128);
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(s32(bar)));
        asm volatile("fence.mbarrier_init.release.cluster;");
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(s32(bar)), "r"(bytes));
        asm volatile(
            "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], "
            "[%5];" ::"r"(s32(buf)),
            "l"((unsigned long long)&m), "r"(x), "r"(y), "r"(z), "r"(s32(bar))
            : "memory");
        asm volatile(
            "{\n.reg .pred P;\nW:\nmbarrier.try_wait.parity.shared::cta.b64 P, [%0], 0;\n@!P bra W;\n}" ::"r"(s32(bar)));
        for (int i = 0; i < n; i++) out[i] = buf[i];
    }
}

int main(int argc, char **argv) {
    int x = atoi(argv[1]), y = atoi(argv[2]), z = atoi(argv[3]), bx = atoi(argv[4]), by = atoi(argv[5]);
    const int nx = 70, ny = 34, nz = 20;
    double *d;
    cudaMalloc(&d, sizeof(double) * nx * ny * nz);
    double *h = (double *)malloc(sizeof(double) * nx * ny * nz);
    for (int i = 0; i < nx * ny * nz; i++) h[i] = i;
    cudaMemcpy(d, h, sizeof(double) * nx * ny * nz, cudaMemcpyHostToDevice);
    void *fn;
    cudaDriverEntryPointQueryResult q;
    cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q);
    CUtensorMap m;
    cuuint64_t gd[3] = {nx, ny, nz}, gs[2] = {nx * 8, nx * ny * 8};
    cuuint32_t box[3] = {(cuuint32_t)bx, (cuuint32_t)by, 1}, es[3] = {1, 1, 1};
    CUresult r = ((PFN_cuTensorMapEncodeTiled_v12000)fn)(&m, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 3, d, gd, gs, box, es,
                                                        CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                                                        CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                                                        CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r) {
        printf("encode error %d\n", r);
        return 1;
    }
    double *out;
    cudaMalloc(&out, 8 * 4);
    int bytes = bx * by * 8;
    int smem = ((bytes + 127) / 128) * 128 + 16;
    cudaFuncSetAttribute(probe, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    probe<<<1, 32, smem>>>(m, x, y, z, bytes, out, 4);
    cudaError_t e = cudaDeviceSynchronize();
    double ho[4] = {0};
    cudaMemcpy(ho, out, 32, cudaMemcpyDeviceToHost);
    printf("x=%d y=%d z=%d box=%dx%d: %s  first=[%g %g %g %g] expect first=%d\n", x, y, z, bx, by,
           cudaGetErrorString(e), ho[0], ho[1], ho[2], ho[3], (z * ny + y) * nx + x);
    return 0;
}

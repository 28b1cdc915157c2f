// tmem_probe.cu -- measure tcgen05.ld / tcgen05.st (TMEM <-> registers)
// throughput per SM on this B200: the number that decides whether a retimed
// accumulator ring can live in TMEM instead of the register file (DESIGN.md
// §10 item 1; the guides disagree: 16 TB/s/SM vs 64 B/clk).
//
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tmem_probe tools/tmem_probe.cu
// One CTA per SM, W warps; every warp owns 32 lanes (its quadrant, warp % 4)
// x 32 columns per round; each iteration stores 32 columns (32x32b.x32: 4 KB
// per warp) and loads them back.  Prints bytes/clk/SM for st-only, ld-only,
// and st+ld, plus single-warp load latency.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

template <int MODE>  // 0 st only, 1 ld only, 2 st + ld
__global__ void __launch_bounds__(256, 1) probe(int iters, unsigned long long *cycles, uint32_t *sink) {
    __shared__ uint32_t taddr_s;
    const int w = threadIdx.x / 32;
    if (w == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(&taddr_s)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    const uint32_t base = taddr_s;
    const uint32_t ta = base + ((uint32_t(32 * (w % 4))) << 16) + uint32_t((w / 4) * 128);
    uint32_t r[32];
#pragma unroll
    for (int i = 0; i < 32; i++) r[i] = threadIdx.x * 7 + i;
    __syncthreads();
    const unsigned long long t0 = clock64();
    for (int it = 0; it < iters; it++) {
        const uint32_t a = ta + uint32_t((it & 3) * 32);
        if (MODE != 1) {
            asm volatile(
                "tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,"
                "%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32};" ::"r"(a),
                "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]), "r"(r[8]),
                "r"(r[9]), "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]), "r"(r[15]), "r"(r[16]),
                "r"(r[17]), "r"(r[18]), "r"(r[19]), "r"(r[20]), "r"(r[21]), "r"(r[22]), "r"(r[23]), "r"(r[24]),
                "r"(r[25]), "r"(r[26]), "r"(r[27]), "r"(r[28]), "r"(r[29]), "r"(r[30]), "r"(r[31]));
            asm volatile("tcgen05.wait::st.sync.aligned;");
        }
        if (MODE != 0) {
            asm volatile(
                "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,"
                "%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
                : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
                  "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]),
                  "=r"(r[15]), "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]),
                  "=r"(r[22]), "=r"(r[23]), "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]),
                  "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
                : "r"(a));
            asm volatile("tcgen05.wait::ld.sync.aligned;");
            r[it & 31] += 1;  // a dependence on the loaded values
        }
    }
    const unsigned long long t1 = clock64();
    uint32_t s = 0;
#pragma unroll
    for (int i = 0; i < 32; i++) s += r[i];
    if (s == 0xdeadbeef) sink[0] = s;
    if (threadIdx.x == 0) cycles[blockIdx.x] = t1 - t0;
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    if (w == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(base));
}

template <int MODE>
double run(int sms, int warps, int iters) {
    unsigned long long *cyc;
    uint32_t *sink;
    cudaMalloc(&cyc, sizeof(unsigned long long) * sms);
    cudaMalloc(&sink, 4);
    // 160 KB of (unused) dynamic shared memory: one CTA per SM, so one TMEM owner
    cudaFuncSetAttribute(probe<MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, 160 * 1024);
    probe<MODE><<<sms, warps * 32, 160 * 1024>>>(iters, cyc, sink);  // warm
    probe<MODE><<<sms, warps * 32, 160 * 1024>>>(iters, cyc, sink);
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) {
        printf("error: %s\n", cudaGetErrorString(e));
        return -1;
    }
    unsigned long long h[1024];
    cudaMemcpy(h, cyc, sizeof(unsigned long long) * sms, cudaMemcpyDeviceToHost);
    double mx = 0;
    for (int i = 0; i < sms; i++) mx = h[i] > mx ? h[i] : mx;
    cudaFree(cyc);
    cudaFree(sink);
    const double ops = (MODE == 2 ? 2.0 : 1.0) * iters * warps * 4096.0;  // bytes moved per SM
    return ops / mx;  // bytes per clock per SM
}

int main() {
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const int iters = 4096;
    for (int warps : {1, 4, 8}) {
        printf("{\"warps\": %d, \"st_B_per_clk_per_SM\": %.1f, \"ld_B_per_clk_per_SM\": %.1f, "
               "\"st_ld_B_per_clk_per_SM\": %.1f}\n",
               warps, run<0>(sms, warps, iters), run<1>(sms, warps, iters), run<2>(sms, warps, iters));
    }
    // single-warp round trip latency: st + wait + ld + wait per iteration
    {
        unsigned long long *cyc;
        uint32_t *sink;
        cudaMalloc(&cyc, 8);
        cudaMalloc(&sink, 4);
        probe<1><<<1, 32>>>(iters, cyc, sink);
        probe<1><<<1, 32>>>(iters, cyc, sink);
        cudaDeviceSynchronize();
        unsigned long long h;
        cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
        printf("{\"ld_x32_plus_wait_cycles_single_warp\": %.1f}\n", double(h) / iters);
    }
    return 0;
}

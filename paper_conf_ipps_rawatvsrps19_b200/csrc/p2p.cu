// p2p.cu -- flag kernels of the peer-memory z-slab halo (dist p2p path,
// SURVEY 8(e) "B200-native alternative", NEXT-4).
//
// Each rank owns a word per z-neighbour in its own HBM; the neighbour writes
// it over NVLink (st.release.sys) after the launch that stored its boundary
// planes into this rank's ghost planes; this rank's stream waits on it
// (ld.acquire.sys) before the launch that reads those ghosts.  One counter
// orders both hazards of the ping-pong buffers (see dist.cpp).  A wait that
// does not complete within SDAG_P2P_TIMEOUT_S (default 60 s) traps instead of
// hanging the device.
#include <cstdio>
#include <cstdlib>

#include "plan.hpp"

namespace sdag {
namespace dev {

__device__ __forceinline__ uint32_t ld_acquire_sys(const uint32_t *p) {
    uint32_t v;
    asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_sys(uint32_t *p, uint32_t v) {
    asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ uint64_t globaltimer() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

__global__ void sdag_p2p_wait(const uint32_t *flags, uint32_t need0, uint32_t need1, int has0, int has1,
                              uint64_t timeout_ns) {
    const uint64_t t0 = globaltimer();
    for (;;) {
        const bool ok0 = !has0 || int32_t(ld_acquire_sys(flags) - need0) >= 0;
        const bool ok1 = !has1 || int32_t(ld_acquire_sys(flags + 1) - need1) >= 0;
        if (ok0 && ok1) return;
        if (globaltimer() - t0 > timeout_ns) {
            printf("sdag p2p halo: timed out waiting for neighbour flags (have %u %u, need %u %u)\n",
                   ld_acquire_sys(flags), ld_acquire_sys(flags + 1), need0, need1);
            __trap();
        }
        __nanosleep(256);
    }
}

__global__ void sdag_p2p_signal(uint32_t *f0, uint32_t *f1, uint32_t v) {
    asm volatile("fence.sc.sys;" ::: "memory");
    if (f0) st_release_sys(f0, v);
    if (f1) st_release_sys(f1, v);
}

}  // namespace dev

void p2p_preload() {
    // With lazy module loading (CUDA 12 default) the first launch of a kernel
    // loads it, which can wait for kernels already running: a flag wait
    // spinning on another stream would then deadlock.  Load the two flag
    // kernels up front (callers do the same for their sweep kernels).
    cudaFuncAttributes fa;
    check_cuda(cudaFuncGetAttributes(&fa, dev::sdag_p2p_wait), "cudaFuncGetAttributes");
    check_cuda(cudaFuncGetAttributes(&fa, dev::sdag_p2p_signal), "cudaFuncGetAttributes");
}

void p2p_wait(const uint32_t *flags, const uint32_t need[2], const int has[2], cudaStream_t stream) {
    if (!has[0] && !has[1]) return;
    static const uint64_t timeout_ns = [] {
        const char *e = std::getenv("SDAG_P2P_TIMEOUT_S");
        const double s = e ? std::atof(e) : 60.0;
        return uint64_t((s > 0 ? s : 60.0) * 1e9);
    }();
    dev::sdag_p2p_wait<<<1, 1, 0, stream>>>(flags, need[0], need[1], has[0], has[1], timeout_ns);
    check_cuda(cudaGetLastError(), "p2p wait launch");
    count_launch();
}

void p2p_signal(uint32_t *f0, uint32_t *f1, uint32_t v, cudaStream_t stream) {
    if (!f0 && !f1) return;
    dev::sdag_p2p_signal<<<1, 1, 0, stream>>>(f0, f1, v);
    check_cuda(cudaGetLastError(), "p2p signal launch");
    count_launch();
}

}  // namespace sdag

// Instantiations for ExpCNS hypterm: the retimed/folded kernel first, the
// generic skeleton (z-taps through L1/L2) as fallback variants.
// Order = heuristic preference, from tools/perf_sweep.py on B200 at 320^3.
#include "kdesc.cuh"
namespace sdag {
void add_kernels_hypterm(std::vector<KernelDesc> &v) {
    SDAG_HYP_PAIR(v, "hypterm", 64, 8, 2, 0);  // 0.793-0.796 ms at 320^3 (pf1: 0.826)
    // cropped per-array boxes: 0.799 ms (32x16: 0.874), no gain -- DESIGN 6.4
    SDAG_HYPC_PAIR(v, "hypterm", 64, 8, 2, 1);
    // round 2, measured and removed: thread 0 issuing TMA without blocking on the
    // slot (mbarrier.test_wait at three points of the plane, blocking only for the
    // plane needed next) 0.876 ms (pf2) / 0.873 (pf1) vs 0.794 -- DESIGN 6.4
    SDAG_HYP_PAIR(v, "hypterm", 16, 16, 2, 1);
    SDAG_HYP_PAIR(v, "hypterm", 64, 8, 1, 2);
    SDAG_HYP_PAIR(v, "hypterm", 32, 16, 1, 3);
    // round 2, measured and removed (ms at 320^3 vs 0.779 for 64x8 pf2): 32x16 pf2
    // 0.850 (less y-halo fill, fewer warps/SM), 32x8 pf3 1.046
    SDAG_HYP_PAIR(v, "hypterm", 32, 8, 2, 4);
    // 12 warps/SM (64x12 or 32x24 tiles, 384 threads, pf1 to fit the ring) caps
    // the thread at 168 registers: 896 B of spill stores per thread, into the
    // shared/L1 data pipe that already binds this kernel -- not registered
    // round 2, measured and removed: plane loop unrolled 2 / 4 / 8 (the 8-slot
    // output ring rotated by register renaming instead of ~90 moves per plane):
    // 0.781-0.787 / 1.27 (spills) / 1.40 (spills) ms vs 0.778 -- the moves are
    // not on the critical path (DESIGN 6.4)
    SDAG_PAIR(v, Hypterm, "hypterm", 32, 8, 1, 1, 2, 10);
}
}  // namespace sdag

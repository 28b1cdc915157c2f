// Instantiations for the 25-point radius-4 Laplacian: the star kernel (register
// z-queue, 128-bit smem reads) first, the generic skeleton as fallback variants.
// Order = heuristic preference, from tools/perf_sweep.py on B200 at 512^3
// (DESIGN.md 6.4 has the numbers; star2 = half queue in smem, L = late head,
// S = split accumulators: measured slower, kept as comparison variants).
#include "kdesc.cuh"
namespace sdag {
void add_kernels_lap25(std::vector<KernelDesc> &v) {
    SDAG_STAR_UNR(v, Lap25Star, "lap25", 32, 32, 4, 3, 1, 2, 0);   // 80.9% of HBM roofline
    SDAG_STAR_UNR(v, Lap25Star, "lap25", 32, 32, 4, 3, 1, 3, 1);   // 80.3%
    SDAG_STAR_ROT(v, Lap25Star, "lap25", 32, 32, 4, 3, 1, 2);      // 79.9%, no queue moves
    SDAG_STAR_ROT(v, Lap25Star, "lap25", 32, 16, 2, 3, 3, 3);      // 79.9%, 12 warps/SM
    SDAG_STAR_UNR(v, Lap25Star, "lap25", 32, 24, 3, 3, 1, 3, 4);   // 78.8%
    SDAG_STAR_PAIR(v, Lap25Star, "lap25", 32, 32, 4, 3, 5);        // 77.2%, queue shifted every plane
    SDAG_STAR_PAIR(v, Lap25Star, "lap25", 64, 16, 4, 3, 6);
    SDAG_STAR_PAIR(v, Lap25Star, "lap25", 32, 32, 4, 4, 7);
    SDAG_STAR_MB(v, Lap25Star, "lap25", 32, 24, 3, 2, 3, 8);
    SDAG_PAIR(v, Lap25, "lap25", 64, 16, 1, 4, 1, 10);              // generic skeleton
    SDAG_STAR2_PAIR(v, Lap25Star, "lap25", 32, 32, 4, 3, 1, 40);
    SDAG_STAR_LATE(v, Lap25Star, "lap25", 32, 32, 4, 3, 1, 2, 41);
    SDAG_STAR_SPLIT(v, Lap25Star, "lap25", 32, 32, 4, 3, 1, 2, 42);
    // round 2, measured and removed (ms at 512^3, two runs): prefetch depth of the
    // default unroll-2 kernel pf2 0.420, pf4 0.3945-0.3963 (= pf3's 0.3947-0.3950),
    // pf5 / pf6 0.559-0.563 (the 10-11 slot ring leaves room for one CTA per SM),
    // pf4 with unroll 3 0.399 -- the ring is deep enough at pf3 (DESIGN 6.4);
    // tile shapes with unroll 2 (less halo fill per point): 64x32 0.404, 32x64
    // 0.401, 64x16 0.397, 32x48 0.481 (6 warps/SM) vs 32x32's 0.3944
    // code differencing, profiling only: never chosen unless forced
    SDAG_STAR_DIFF(v, Lap25Star, "lap25", 32, 32, 4, 3, 2, 1000);
    SDAG_STAR_DIFF(v, Lap25Star, "lap25", 32, 32, 4, 3, 3, 1001);
}
}  // namespace sdag

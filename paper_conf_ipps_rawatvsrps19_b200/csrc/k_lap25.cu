// Instantiations for the 25-point radius-4 Laplacian: the star kernel (register
// z-queue, 128-bit smem reads) first, the generic skeleton as fallback variants.
// Order = heuristic preference, from tools/perf_sweep.py on B200 at 512^3
// (star2 = half queue in smem, more warps: measured slower).
#include "kdesc.cuh"
namespace sdag {
void add_kernels_lap25(std::vector<KernelDesc> &v) {
    SDAG_STAR_PAIR(v, Lap25Star, "lap25", 32, 32, 4, 3, 0);
    SDAG_STAR_PAIR(v, Lap25Star, "lap25", 64, 16, 4, 3, 1);
    SDAG_STAR_PAIR(v, Lap25Star, "lap25", 32, 32, 4, 4, 2);
    SDAG_STAR_PAIR(v, Lap25Star, "lap25", 64, 32, 4, 3, 3);
    SDAG_STAR_MB(v, Lap25Star, "lap25", 32, 24, 3, 2, 3, 4);
    SDAG_STAR2_PAIR(v, Lap25Star, "lap25", 32, 32, 4, 3, 1, 5);
    SDAG_PAIR(v, Lap25, "lap25", 64, 16, 1, 4, 1, 10);
    // code differencing, profiling only: never chosen unless forced
    SDAG_STAR_DIFF(v, Lap25Star, "lap25", 32, 32, 4, 3, 2, 1000);
    SDAG_STAR_DIFF(v, Lap25Star, "lap25", 32, 32, 4, 3, 3, 1001);
}
}  // namespace sdag

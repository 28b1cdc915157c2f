// Instantiations for the 25-point radius-4 Laplacian: the star kernel (register
// z-queue, 128-bit smem reads) first, the generic skeleton as fallback variants.
// Order = heuristic preference, from tools/perf_sweep.py on B200 at 512^3.
#include "kdesc.cuh"
namespace sdag {
void add_kernels_lap25(std::vector<KernelDesc> &v) {
    SDAG_STAR_PAIR(v, Lap25Star, "lap25", 32, 32, 4, 3, 0);
    SDAG_STAR_PAIR(v, Lap25Star, "lap25", 64, 16, 4, 3, 1);
    SDAG_STARQ(v, Lap25Star, "lap25", 32, 32, 4, 3, 2);
    SDAG_STAR_PAIR(v, Lap25Star, "lap25", 32, 32, 4, 4, 3);
    SDAG_STAR_PAIR(v, Lap25Star, "lap25", 32, 32, 2, 3, 4);
    SDAG_STAR_PAIR(v, Lap25Star, "lap25", 64, 32, 4, 3, 5);
    SDAG_STAR_PAIR(v, Lap25Star, "lap25", 72, 24, 4, 3, 6);
    SDAG_PAIR(v, Lap25, "lap25", 64, 16, 1, 4, 1, 10);
}
}  // namespace sdag

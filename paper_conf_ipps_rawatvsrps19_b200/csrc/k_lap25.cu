// Instantiations for the 25-point radius-4 Laplacian: the star kernel (register
// z-queue, 128-bit smem reads) first, the generic skeleton as fallback variants.
#include "kdesc.cuh"
namespace sdag {
void add_kernels_lap25(std::vector<KernelDesc> &v) {
    SDAG_STAR_PAIR(v, Lap25Star, "lap25", 72, 24, 4, 3, 0);  // 504^2 interior -> 7 x 21 = 147 tiles
    SDAG_STAR_PAIR(v, Lap25Star, "lap25", 64, 32, 4, 3, 1);
    SDAG_STAR_PAIR(v, Lap25Star, "lap25", 72, 24, 4, 4, 2);
    SDAG_STAR_PAIR(v, Lap25Star, "lap25", 64, 16, 4, 3, 3);
    SDAG_STAR_PAIR(v, Lap25Star, "lap25", 32, 32, 4, 3, 4);
    SDAG_PAIR(v, Lap25, "lap25", 64, 16, 1, 4, 1, 10);
    SDAG_PAIR(v, Lap25, "lap25", 32, 16, 1, 4, 1, 11);
}
}  // namespace sdag

// Instantiations of the sweep skeleton for the 25-point radius-4 Laplacian.
#include "kdesc.cuh"
namespace sdag {
void add_kernels_lap25(std::vector<KernelDesc> &v) {
    SDAG_PAIR(v, Lap25, "lap25", 64, 16, 1, 4, 1, 0);
    SDAG_PAIR(v, Lap25, "lap25", 32, 16, 1, 4, 1, 1);
    SDAG_PAIR(v, Lap25, "lap25", 64, 8, 1, 2, 1, 2);
}
}  // namespace sdag

// Instantiations of the sweep skeleton for the 27-point smoother.
#include "kdesc.cuh"
namespace sdag {
void add_kernels_smooth27(std::vector<KernelDesc> &v) {
    SDAG_PAIR(v, Smooth27, "smooth27", 64, 16, 1, 4, 2, 0);
    SDAG_PAIR(v, Smooth27, "smooth27", 32, 16, 1, 2, 2, 1);
    SDAG_PAIR(v, Smooth27, "smooth27", 64, 8, 1, 2, 2, 2);
}
}  // namespace sdag

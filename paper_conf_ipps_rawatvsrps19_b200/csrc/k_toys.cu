// Instantiations for the bookkeeping toys: shift (|offset| <= 4) and j1d3pt.
#include "kdesc.cuh"
namespace sdag {
void add_kernels_toys(std::vector<KernelDesc> &v) {
    SDAG_PAIR(v, Shift4, "shift", 32, 8, 1, 1, 1, 0);
    SDAG_PAIR(v, J1d3pt, "j1d3pt", 64, 1, 1, 1, 1, 0);
}
}  // namespace sdag

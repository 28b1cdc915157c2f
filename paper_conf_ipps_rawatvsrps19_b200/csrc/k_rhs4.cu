// Instantiations of the sweep skeleton for SW4 rhs4center (2-wide x patches
// were measured slower: stride-2 smem access and register pressure).
#include "kdesc.cuh"
namespace sdag {
void add_kernels_rhs4(std::vector<KernelDesc> &v) {
    SDAG_PAIR(v, Rhs4, "rhs4center", 16, 16, 1, 1, 1, 0);
    SDAG_PAIR(v, Rhs4, "rhs4center", 32, 8, 1, 1, 1, 1);
    SDAG_PAIR(v, Rhs4, "rhs4center", 16, 16, 1, 2, 1, 2);
}
}  // namespace sdag

// Instantiations of the sweep skeleton for ExpCNS hypterm.
#include "kdesc.cuh"
namespace sdag {
void add_kernels_hypterm(std::vector<KernelDesc> &v) {
    SDAG_PAIR(v, Hypterm, "hypterm", 32, 8, 1, 1, 2, 0);
    SDAG_PAIR(v, Hypterm, "hypterm", 16, 16, 1, 1, 2, 1);
    SDAG_PAIR(v, Hypterm, "hypterm", 32, 16, 1, 2, 1, 2);
}
}  // namespace sdag

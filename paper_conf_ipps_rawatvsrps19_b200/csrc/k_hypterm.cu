// Instantiations for ExpCNS hypterm: the retimed/folded kernel first, the
// generic skeleton (z-taps through L1/L2) as fallback variants.
#include "kdesc.cuh"
namespace sdag {
void add_kernels_hypterm(std::vector<KernelDesc> &v) {
    SDAG_HYP_PAIR(v, "hypterm", 32, 8, 2, 0);
    SDAG_HYP_PAIR(v, "hypterm", 32, 16, 1, 1);
    SDAG_HYP_PAIR(v, "hypterm", 64, 8, 1, 2);
    SDAG_HYP_PAIR(v, "hypterm", 16, 16, 2, 3);
    SDAG_PAIR(v, Hypterm, "hypterm", 32, 8, 1, 1, 2, 10);
    SDAG_PAIR(v, Hypterm, "hypterm", 16, 16, 1, 1, 2, 11);
}
}  // namespace sdag

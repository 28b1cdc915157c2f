// Instantiations of the sweep skeleton for SW4 rhs4center: maxfuse and the
// paper's trivial fission (Fig 3: one kernel per uacc component, mux1..muz4
// replicated).  2-wide x patches were measured slower (stride-2 smem access).
#include "kdesc.cuh"
namespace sdag {
void add_kernels_rhs4(std::vector<KernelDesc> &v) {
    SDAG_PAIR(v, Rhs4, "rhs4center", 16, 16, 1, 1, 1, 0);
    SDAG_PAIR(v, Rhs4, "rhs4center", 32, 8, 1, 1, 1, 1);
    SDAG_PAIR(v, Rhs4, "rhs4center", 16, 16, 1, 2, 1, 2);
    SDAG_FISSION_PAIR(v, Rhs4, "rhs4center", 16, 16, 1, 1, 1, 3);
    SDAG_FISSION_PAIR(v, Rhs4, "rhs4center", 32, 16, 1, 2, 1, 4);
    SDAG_FISSION_PAIR(v, Rhs4, "rhs4center", 16, 16, 1, 1, 2, 5);
}
}  // namespace sdag

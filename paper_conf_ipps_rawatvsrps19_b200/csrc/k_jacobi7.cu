// Instantiations of the sweep skeleton for Listing 1's 7-point Jacobi (K1).
#include "kdesc.cuh"
namespace sdag {
void add_kernels_jacobi7(std::vector<KernelDesc> &v) {
    SDAG_PAIR(v, Jacobi7, "jacobi7", 64, 16, 1, 4, 2, 0);
    SDAG_PAIR(v, Jacobi7, "jacobi7", 32, 16, 1, 2, 2, 1);
    SDAG_PAIR(v, Jacobi7, "jacobi7", 64, 8, 1, 2, 2, 2);
}
}  // namespace sdag

// Instantiations for Listing 1's 7-point Jacobi (K1): the retimed cross kernel
// (box27.cuh FORM 1), the star kernel, and the generic skeleton.
#include "kdesc.cuh"
namespace sdag {
void add_kernels_jacobi7(std::vector<KernelDesc> &v) {
    SDAG_STAR_PAIR(v, Jacobi7Star, "jacobi7", 64, 16, 2, 3, 0);
    SDAG_CROSS_PAIR(v, "jacobi7", 64, 8, 2, 3, 1);
    SDAG_CROSS_PAIR(v, "jacobi7", 64, 16, 4, 6, 2);
    SDAG_CROSS_PAIR(v, "jacobi7", 64, 8, 2, 6, 3);
    SDAG_CROSS_PAIR(v, "jacobi7", 64, 32, 4, 4, 4);
    SDAG_CROSS_PAIR(v, "jacobi7", 64, 64, 8, 3, 5);
    SDAG_STAR_PAIR(v, Jacobi7Star, "jacobi7", 64, 16, 2, 6, 6);
    SDAG_PAIR(v, Jacobi7, "jacobi7", 64, 16, 1, 4, 2, 10);
}
}  // namespace sdag

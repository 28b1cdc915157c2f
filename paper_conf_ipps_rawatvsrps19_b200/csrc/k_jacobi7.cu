// Instantiations for Listing 1's 7-point Jacobi (K1): the star kernel first,
// the generic skeleton as fallback variants.
#include "kdesc.cuh"
namespace sdag {
void add_kernels_jacobi7(std::vector<KernelDesc> &v) {
    SDAG_STAR_PAIR(v, Jacobi7Star, "jacobi7", 64, 16, 2, 3, 0);
    SDAG_STAR_PAIR(v, Jacobi7Star, "jacobi7", 32, 16, 4, 3, 1);
    SDAG_STAR_PAIR(v, Jacobi7Star, "jacobi7", 64, 32, 4, 3, 2);
    SDAG_STARQ(v, Jacobi7Star, "jacobi7", 64, 16, 2, 3, 3);
    SDAG_PAIR(v, Jacobi7, "jacobi7", 64, 16, 1, 4, 2, 10);
    SDAG_PAIR(v, Jacobi7, "jacobi7", 32, 16, 1, 2, 2, 11);
}
}  // namespace sdag

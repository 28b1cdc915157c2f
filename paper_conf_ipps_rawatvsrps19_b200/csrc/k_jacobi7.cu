// Instantiations for Listing 1's 7-point Jacobi (K1): the retimed cross kernel
// (box27.cuh FORM 1), the star kernel, and the generic skeleton.
#include "kdesc.cuh"
namespace sdag {
void add_kernels_jacobi7(std::vector<KernelDesc> &v) {
    // prefetch depth 6 (8-slot ring, 2 CTAs/SM) ahead of depth 3 (3 CTAs/SM):
    // batched 128 x 64^3 0.1058-0.1061 ms vs 0.1072-0.1078 (round 2, two runs
    // each); one 64^3 problem unchanged (~9 us, latency).  Measured and not
    // registered: pf3/pf4 at 4 CTAs/SM 0.1087-0.1104, pf4 at 3 CTAs/SM 0.1083-0.1088,
    // unroll 2 0.1089, 64x8 0.111, 64x32 0.116, 64x16 with 4-row patches 0.1094
    SDAG_STAR_PAIR(v, Jacobi7Star, "jacobi7", 64, 16, 2, 6, 0);
    SDAG_STAR_PAIR(v, Jacobi7Star, "jacobi7", 64, 16, 2, 3, 6);
    SDAG_CROSS_PAIR(v, "jacobi7", 64, 8, 2, 3, 1);
    SDAG_CROSS_PAIR(v, "jacobi7", 64, 16, 4, 6, 2);
    SDAG_CROSS_PAIR(v, "jacobi7", 64, 8, 2, 6, 3);
    SDAG_CROSS_PAIR(v, "jacobi7", 64, 32, 4, 4, 4);
    SDAG_CROSS_PAIR(v, "jacobi7", 64, 64, 8, 3, 5);
    SDAG_PAIR(v, Jacobi7, "jacobi7", 64, 16, 1, 4, 2, 10);
    // temporal fusion for apply_iterated (NEXT-1; the paper's 7pt-smoother,
    // Table II): two sweeps per launch, overlapped tiles.  The cross stencil's
    // y-neighbour rows need only the patch's own (aligned) pair, so the
    // even-aligned layout wins here (tools/table2_sweep.py, 1024^3 T=12:
    // 2.03 ms/sweep vs 2.19 odd-aligned vs 3.04 unfused)
    v.push_back(make_fuse2_desc<64, 16, 2, 2, 2, 2, false, 1>("jacobi7", 20));
    v.back().fhint = 1.29;  // f(2) measured at 1024^3 (tools/table2_sweep.py --all)
    v.push_back(make_fuse2_desc<64, 16, 2, 2, 2, 2, true, 1>("jacobi7", 21));
    v.push_back(make_fuse2_desc<32, 16, 2, 2, 3, 2, true, 1>("jacobi7", 22));
    v.push_back(make_fuse2_desc<128, 16, 4, 2, 1, 2, true, 1>("jacobi7", 23));
    // fusion degrees 3 and 4 (fuseN.cuh): the paper's Table II / Fig 4 sweep
    v.push_back(make_fuseN_desc<3, 64, 32, 2, 2, 1, 2, false, 1>("jacobi7", 40));
    v.back().fhint = 1.96;  // f(3): 0.65 per sweep, the cusp (f(2)/2 = 0.64)
    v.push_back(make_fuseN_desc<3, 64, 32, 2, 2, 1, 2, true, 1>("jacobi7", 41));
    v.push_back(make_fuseN_desc<3, 128, 16, 2, 2, 1, 2, false, 1>("jacobi7", 42));
    v.push_back(make_fuseN_desc<4, 64, 32, 2, 2, 1, 2, false, 1>("jacobi7", 43));
    v.back().fhint = 3.17;  // f(4): 0.79 per sweep
    v.push_back(make_fuseN_desc<4, 64, 16, 2, 2, 2, 2, false, 1>("jacobi7", 44));
}
}  // namespace sdag

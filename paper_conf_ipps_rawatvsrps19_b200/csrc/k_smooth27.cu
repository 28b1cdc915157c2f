// Instantiations for the 27-point smoother: the retimed/folded box kernel
// first, the generic skeleton as fallback variants.
// Order = heuristic preference, from tools/perf_sweep.py on B200 at 512^3.
#include "kdesc.cuh"
namespace sdag {
void add_kernels_smooth27(std::vector<KernelDesc> &v) {
    SDAG_BOX_PAIR(v, "smooth27", 128, 16, 4, 2, 0);
    // FORM 2 (generated DAGs in box form, jit.cu): weights by tap class
    // (preferred over every generated candidate of such a plan: negative priorities)
    v.push_back(make_box27_desc<128, 16, 4, 2, true, 2>("(box27)", -40));
    v.push_back(make_box27_desc<128, 16, 4, 2, false, 2>("(box27)", 60));
    v.push_back(make_box27_desc<64, 32, 4, 3, true, 2>("(box27)", -39));
    v.push_back(make_fuse2_desc<64, 16, 2, 2, 2, 2, true, 2>("(box27)", -40));  // temporal fusion, FORM 2
    v.back().fhint = 1.69;
    SDAG_BOX_PAIR(v, "smooth27", 64, 32, 4, 3, 1);
    SDAG_BOX_PAIR(v, "smooth27", 64, 16, 4, 3, 2);
    SDAG_BOX_PAIR(v, "smooth27", 128, 16, 4, 3, 3);
    SDAG_BOX_PAIR(v, "smooth27", 128, 32, 4, 2, 4);
    SDAG_PAIR(v, Smooth27, "smooth27", 64, 16, 1, 4, 2, 10);
    // temporal fusion (2 sweeps per launch) for apply_iterated; order from
    // tools/fusion_sweep.py at 1024^3, T=12: odd-aligned 62x14 2.27 ms/sweep,
    // even-aligned 62x14 2.51, unfused 2.77
    v.push_back(make_fuse2_desc<64, 16, 2, 2, 2, 2, true>("smooth27", 20));  // mb2: 2 CTAs/SM need <= 128 registers
    v.back().fhint = 1.69;  // f(2) measured at 1024^3 (tools/table2_sweep.py --all)
    v.push_back(make_fuse2_desc<32, 16, 2, 2, 3, 2, true>("smooth27", 21));
    v.push_back(make_fuse2_desc<64, 16, 2, 2, 2>("smooth27", 22));
    v.push_back(make_fuse2_desc<32, 16, 2, 2, 3>("smooth27", 23));
    v.push_back(make_fuse2_desc<128, 16, 4, 2, 1, 2, true>("smooth27", 24));
    v.push_back(make_fuse2_desc<128, 16, 4, 2>("smooth27", 25));
    v.push_back(make_fuse2_desc<64, 32, 2, 2>("smooth27", 26));
    v.push_back(make_fuse2_desc<128, 16, 2, 2>("smooth27", 27));
    v.push_back(make_fuse2_desc<64, 16, 2, 2, 2, 4, true>("smooth27", 28));
    v.push_back(make_fuse2_desc<64, 16, 2, 2, 1, 4>("smooth27", 29));  // 4-wide patch: bank-conflicted, kept for comparison
    // round 2, measured and removed (tools/fusion_sweep.py, 1024^3, T = 12, ms per
    // sweep vs 2.39 for fuse2o 62x14 u2x2 mb2): 2x4 patches 62x14 mb3 2.94 (168 regs,
    // spills), 62x22 mb2 3.05, 62x30 2.63 (224 regs, 8 warps/SM); 2x2 with 3 CTAs/SM
    // (80 regs, spills) 3.82
    // fusion degrees 3 and 4 (fuseN.cuh): the paper's Table II / Fig 4 sweep
    v.push_back(make_fuseN_desc<3, 64, 32, 2, 2, 1, 2, false, 0>("smooth27", 40));
    v.back().fhint = 3.12;  // f(3): 1.04 per sweep -- past the cusp (shared-memory bound folds)
    v.push_back(make_fuseN_desc<3, 64, 32, 2, 2, 1, 2, true, 0>("smooth27", 41));
    v.push_back(make_fuseN_desc<3, 128, 16, 2, 2, 1, 2, false, 0>("smooth27", 42));
    v.push_back(make_fuseN_desc<4, 64, 32, 2, 2, 1, 2, false, 0>("smooth27", 43));
    v.back().fhint = 4.96;  // f(4): 1.24 per sweep
    v.push_back(make_fuseN_desc<4, 64, 16, 2, 2, 2, 2, false, 0>("smooth27", 44));
}
}  // namespace sdag

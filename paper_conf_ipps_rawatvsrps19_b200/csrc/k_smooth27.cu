// Instantiations for the 27-point smoother: the retimed/folded box kernel
// first, the generic skeleton as fallback variants.
// Order = heuristic preference, from tools/perf_sweep.py on B200 at 512^3.
#include "kdesc.cuh"
namespace sdag {
void add_kernels_smooth27(std::vector<KernelDesc> &v) {
    SDAG_BOX_PAIR(v, "smooth27", 128, 16, 4, 2, 0);
    SDAG_BOX_PAIR(v, "smooth27", 64, 32, 4, 3, 1);
    SDAG_BOX_PAIR(v, "smooth27", 64, 16, 4, 3, 2);
    SDAG_BOX_PAIR(v, "smooth27", 128, 16, 4, 3, 3);
    SDAG_BOX_PAIR(v, "smooth27", 128, 32, 4, 2, 4);
    SDAG_PAIR(v, Smooth27, "smooth27", 64, 16, 1, 4, 2, 10);
    // temporal fusion (2 sweeps per launch) for apply_iterated; order from
    // tools/fusion_sweep.py at 1024^3, T=12: odd-aligned 62x14 2.27 ms/sweep,
    // even-aligned 62x14 2.51, unfused 2.77
    v.push_back(make_fuse2_desc<64, 16, 2, 2, 2, 2, true>("smooth27", 20));  // mb2: 2 CTAs/SM need <= 128 registers
    v.push_back(make_fuse2_desc<32, 16, 2, 2, 3, 2, true>("smooth27", 21));
    v.push_back(make_fuse2_desc<64, 16, 2, 2, 2>("smooth27", 22));
    v.push_back(make_fuse2_desc<32, 16, 2, 2, 3>("smooth27", 23));
    v.push_back(make_fuse2_desc<128, 16, 4, 2, 1, 2, true>("smooth27", 24));
    v.push_back(make_fuse2_desc<128, 16, 4, 2>("smooth27", 25));
    v.push_back(make_fuse2_desc<64, 32, 2, 2>("smooth27", 26));
    v.push_back(make_fuse2_desc<128, 16, 2, 2>("smooth27", 27));
    v.push_back(make_fuse2_desc<64, 16, 2, 2, 2, 4, true>("smooth27", 28));
    v.push_back(make_fuse2_desc<64, 16, 2, 2, 1, 4>("smooth27", 29));  // 4-wide patch: bank-conflicted, kept for comparison
}
}  // namespace sdag

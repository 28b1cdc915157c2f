// Instantiations of the sweep skeleton for SW4 rhs4center: maxfuse and the
// paper's trivial fission (Fig 3: one kernel per uacc component, mux1..muz4
// replicated).  2-wide x patches were measured slower (stride-2 smem access).
#include "kdesc.cuh"
namespace sdag {
void add_kernels_rhs4(std::vector<KernelDesc> &v) {
    // specialised kernel (rhs4.cuh): 2 x UY patches from 128-bit pair loads, derivative fields
    // (2 x 2 / 2 x 4 patches spill at 255 registers and run 3x slower; not registered)
    SDAG_RHS4_PAIR(v, "rhs4center", 32, 16, 1, 1, -10);
    // round 2, measured and removed: two output planes per step sharing the z-tap
    // loads of planes k-2..k+3 (7-plane ring, 226 KB of smem): correct (bitwise on
    // the exact cases) but 1.264-1.276 ms -- ncu: 67.6 LDS.128 per point (the
    // compiler re-loads what the per-plane order was meant to share, at 254
    // registers) and ~50 SYNCS + 49 YIELD per point spinning on the 2-plane refill
    // (DESIGN 6.4)
    // cooperative derivative fields + retimed z (rhs4f.cuh)
    SDAG_RHS4F_PAIR(v, "rhs4center", 32, 16, 1, -3);
    SDAG_RHS4F_PAIR(v, "rhs4center", 32, 8, 1, -2);
    SDAG_RHS4G_PAIR(v, "rhs4center", 32, 16, -1);  // double-buffered fields, one barrier per plane
    // round 2, measured and removed: the r4g CTA barrier split into mbarriers
    // ("fields stored" / "fields read", warps skew by up to a phase) 1.488 ms vs
    // 1.437 -- lock-step phases are not what holds the field kernels back (DESIGN 6.4)
    SDAG_RHS4_PAIR(v, "rhs4center", 16, 16, 1, 1, -9);
    SDAG_RHS4_PAIR(v, "rhs4center", 64, 8, 1, 1, -8);
    SDAG_RHS4_PAIR(v, "rhs4center", 32, 8, 1, 1, -7);
    SDAG_RHS4_PAIR(v, "rhs4center", 32, 16, 1, 2, -6);
    SDAG_RHS4_PAIR(v, "rhs4center", 16, 32, 1, 1, -5);
    SDAG_PAIR(v, Rhs4, "rhs4center", 16, 16, 1, 1, 1, 0);
    SDAG_PAIR(v, Rhs4, "rhs4center", 32, 8, 1, 1, 1, 1);
    SDAG_PAIR(v, Rhs4, "rhs4center", 16, 16, 1, 2, 1, 2);
    SDAG_FISSION_PAIR(v, Rhs4, "rhs4center", 16, 16, 1, 1, 1, 3);
    SDAG_FISSION_PAIR(v, Rhs4, "rhs4center", 32, 16, 1, 2, 1, 4);
    SDAG_FISSION_PAIR(v, Rhs4, "rhs4center", 16, 16, 1, 1, 2, 5);
}
}  // namespace sdag

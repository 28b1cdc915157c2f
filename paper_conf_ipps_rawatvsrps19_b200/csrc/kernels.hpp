// kernels.hpp -- host-side table of the compiled sm_100a sweep kernels.
#pragma once

#include <string>
#include <utility>
#include <vector>

namespace sdag {

struct KernelDesc {
    std::string dag;      // registry DAG this kernel evaluates
    std::string variant;  // "tma_64x16_u1x4_pf2", ...
    const void *fn = nullptr;
    bool fission = false;                 // trivial fission: one launch per output
    std::vector<const void *> fission_fns;  // fission kernel for output m
    int threads = 0, smem = 0;
    int tx = 0, ty = 0, ux = 0, uy = 0, pf = 0;
    bool tma = false;
    int nin = 0, nout = 0, nio = 0, n1d = 0;
    int rz = 0, ry = 0, rx = 0, rzr = 0;  // body radius and shared-memory ring z-window
    int prio = 0;                         // heuristic preference (lower first)
    const void *fn_mirror = nullptr;      // same kernel, also storing into SweepArgs::peer (dist p2p halo)
    int tsteps = 1;                       // sweeps fused per launch (temporal fusion, NEXT-1)
    double fhint = 0.0;                   // measured f(x): launch cost / one sweep (0 = generic estimate)
    std::vector<std::pair<int, int>> inbox;  // per staged input: TMA box (x, y) if cropped (else tx+2rx, ty+2ry)
    void *cufn = nullptr;                 // CUfunction of an NVRTC-compiled kernel (jit.cu); fn is then null
};

// all kernels, in heuristic preference order per DAG
const std::vector<KernelDesc> &kernel_table();

}  // namespace sdag

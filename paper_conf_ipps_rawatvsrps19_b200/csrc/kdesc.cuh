// kdesc.cuh -- builds a KernelDesc for one instantiation of the sweep skeleton.
#pragma once

#include <cstdio>
#include <utility>

#include "bodies.cuh"
#include "kernels.hpp"
#include "box27.cuh"
#include "fuse2.cuh"
#include "fuseN.cuh"
#include "hyp.cuh"
#include "rhs4.cuh"
#include "rhs4f.cuh"
#include "star.cuh"
#include "sweep.cuh"

namespace sdag {

template <class B, int TX, int TY, int UX, int UY, int PF, bool TMA>
KernelDesc make_desc(const char *dag, int prio) {
    using G = dev::Geo<B, TX, TY, UX, UY, PF>;
    KernelDesc d;
    d.dag = dag;
    char buf[96];
    std::snprintf(buf, sizeof buf, "%s_%dx%d_u%dx%d_pf%d", TMA ? "tma" : "lsu", TX, TY, UX, UY, PF);
    d.variant = buf;
    d.fn = reinterpret_cast<const void *>(&dev::sdag_sweep<B, TX, TY, UX, UY, PF, TMA>);
    d.threads = G::THREADS;
    d.smem = G::SMEM;
    d.tx = TX;
    d.ty = TY;
    d.ux = UX;
    d.uy = UY;
    d.pf = PF;
    d.tma = TMA;
    d.nin = B::NIN;
    d.nout = B::NOUT;
    d.nio = B::NIO;
    d.n1d = B::N1D;
    d.rz = B::RZ;
    d.ry = B::RY;
    d.rx = B::RX;
    d.rzr = dev::ring_rz<B>();
    d.prio = prio;
    return d;
}

// star-stencil kernel (star.cuh): 2-wide x patch, UY-tall y patch, register z-queue
template <class B, int TX, int TY, int UY, int PF, bool TMA, int QMODE = 0, int MINB = 1, int UNR = 1>
KernelDesc make_star_desc(const char *dag, int prio) {
    using G = dev::StarGeo<B, TX, TY, UY, PF>;
    KernelDesc d;
    d.dag = dag;
    char buf[96];
    char unr[16] = "";
    if (UNR > 1) std::snprintf(unr, sizeof unr, "_z%d", UNR);
    std::snprintf(buf, sizeof buf, "star%s_%s_%dx%d_u2x%d_pf%d%s%s",
                  QMODE == 1 ? "q" : (QMODE == 2 ? "DIFFmem" : (QMODE == 3 ? "DIFFnost" : (QMODE == 4 ? "L" : (QMODE == 5 ? "S" : (QMODE == 6 ? "R" : ""))))), TMA ? "tma" : "lsu", TX,
                  TY, UY, PF, MINB > 1 ? (MINB == 2 ? "_mb2" : (MINB == 3 ? "_mb3" : "_mb4")) : "", unr);
    d.variant = buf;
    d.fn = reinterpret_cast<const void *>(&dev::sdag_star<B, TX, TY, UY, PF, TMA, QMODE, MINB, UNR>);
    if constexpr (QMODE == 0)  // the dist p2p path's fused-store twin
        d.fn_mirror = reinterpret_cast<const void *>(&dev::sdag_star<B, TX, TY, UY, PF, TMA, QMODE, MINB, UNR, true>);
    d.threads = G::THREADS;
    d.smem = G::SMEM;
    d.tx = TX;
    d.ty = TY;
    d.ux = 2;
    d.uy = UY;
    d.pf = PF;
    d.tma = TMA;
    d.nin = 1;
    d.nout = 1;
    d.rz = B::R;
    d.ry = B::R;
    d.rx = G::ML;  // TMA box margin in x (R rounded up to even)
    d.rzr = B::R;
    d.prio = prio;
    return d;
}

// 27-point box kernel (box27.cuh): retimed, folded in-plane partial sums
template <int TX, int TY, int UY, int PF, bool TMA, int FORM = 0>
KernelDesc make_box27_desc(const char *dag, int prio) {
    using G = dev::BoxGeo<TX, TY, UY, PF>;
    KernelDesc d;
    d.dag = dag;
    char buf[96];
    std::snprintf(buf, sizeof buf, "%s_%s_%dx%d_u2x%d_pf%d", FORM == 1 ? "cross" : (FORM == 2 ? "jitbox" : "box"),
                  TMA ? "tma" : "lsu", TX, TY, UY, PF);
    d.variant = buf;
    d.fn = reinterpret_cast<const void *>(&dev::sdag_box27<TX, TY, UY, PF, TMA, FORM>);
    d.fn_mirror = reinterpret_cast<const void *>(&dev::sdag_box27<TX, TY, UY, PF, TMA, FORM, true>);
    d.threads = G::THREADS;
    d.smem = G::SMEM;
    d.tx = TX;
    d.ty = TY;
    d.ux = 2;
    d.uy = UY;
    d.pf = PF;
    d.tma = TMA;
    d.nin = 1;
    d.nout = 1;
    d.rz = 1;
    d.ry = 1;
    d.rx = G::ML;
    d.rzr = 0;  // each plane is read once
    d.prio = prio;
    return d;
}

#define SDAG_CROSS_PAIR(v, DAG, TX, TY, UY, PF, PRIO)                               \
    do {                                                                            \
        v.push_back(make_box27_desc<TX, TY, UY, PF, true, 1>(DAG, PRIO));           \
        v.push_back(make_box27_desc<TX, TY, UY, PF, false, 1>(DAG, PRIO + 100));    \
    } while (0)

#define SDAG_BOX_PAIR(v, DAG, TX, TY, UY, PF, PRIO)                                 \
    do {                                                                            \
        v.push_back(make_box27_desc<TX, TY, UY, PF, true>(DAG, PRIO));              \
        v.push_back(make_box27_desc<TX, TY, UY, PF, false>(DAG, PRIO + 100));       \
    } while (0)

// hypterm kernel (hyp.cuh): retimed z, folded fluxes, x-pairs
template <int TX, int TY, int PF, bool TMA>
KernelDesc make_hyp_desc(const char *dag, int prio) {
    using G = dev::HypGeo<TX, TY, PF>;
    KernelDesc d;
    d.dag = dag;
    char buf[96];
    std::snprintf(buf, sizeof buf, "hyp_%s_%dx%d_u2x1_pf%d", TMA ? "tma" : "lsu", TX, TY, PF);
    d.variant = buf;
    d.fn = reinterpret_cast<const void *>(&dev::sdag_hyp<TX, TY, PF, TMA>);
    d.threads = G::THREADS;
    d.smem = G::SMEM;
    d.tx = TX;
    d.ty = TY;
    d.ux = 2;
    d.uy = 1;
    d.pf = PF;
    d.tma = TMA;
    d.nin = 8;
    d.nout = 5;
    d.rz = 4;
    d.ry = 4;
    d.rx = G::ML;
    d.rzr = 4;  // z-halo planes streamed per chunk
    d.prio = prio;
    return d;
}

// hypterm with cropped per-array boxes (hyp.cuh, sdag_hypc)
template <int TX, int TY, int PF, bool TMA>
KernelDesc make_hypc_desc(const char *dag, int prio) {
    using G = dev::HypcGeo<TX, TY, PF>;
    KernelDesc d;
    d.dag = dag;
    d.tx = TX;
    d.ty = TY;
    d.ux = 2;
    d.uy = 1;
    d.pf = PF;
    d.tma = TMA;
    d.nin = 8;
    d.nout = 5;
    d.rz = 4;
    d.ry = 4;
    d.rx = 4;
    d.rzr = 4;  // z-halo planes streamed per chunk
    d.prio = prio;
    char buf[96];
    std::snprintf(buf, sizeof buf, "hypc_%s_%dx%d_u2x1_pf%d", TMA ? "tma" : "lsu", TX, TY, PF);
    d.variant = buf;
    d.fn = reinterpret_cast<const void *>(&dev::sdag_hypc<TX, TY, PF, TMA>);
    d.threads = G::THREADS;
    d.smem = G::SMEM;
    for (int q = 0; q < G::NA; q++) d.inbox.emplace_back(G::px(q), G::py(q));
    return d;
}

#define SDAG_HYPC_PAIR(v, DAG, TX, TY, PF, PRIO)                                  \
    do {                                                                          \
        v.push_back(make_hypc_desc<TX, TY, PF, true>(DAG, PRIO));                 \
        v.push_back(make_hypc_desc<TX, TY, PF, false>(DAG, PRIO + 100));          \
    } while (0)

#define SDAG_HYP_PAIR(v, DAG, TX, TY, PF, PRIO)                                   \
    do {                                                                          \
        v.push_back(make_hyp_desc<TX, TY, PF, true>(DAG, PRIO));                  \
        v.push_back(make_hyp_desc<TX, TY, PF, false>(DAG, PRIO + 100));           \
    } while (0)

// rhs4center kernel (rhs4.cuh): 2 x UY patches, derivative fields, 5-plane TMA ring
template <int TX, int TY, int UY, int PF, bool TMA>
KernelDesc make_rhs4_desc(const char *dag, int prio) {
    using G = dev::R4Geo<TX, TY, UY, PF>;
    KernelDesc d;
    d.dag = dag;
    char buf[96];
    std::snprintf(buf, sizeof buf, "r4_%s_%dx%d_u2x%d_pf%d", TMA ? "tma" : "lsu", TX, TY, UY, PF);
    d.variant = buf;
    d.fn = reinterpret_cast<const void *>(&dev::sdag_rhs4<TX, TY, UY, PF, TMA>);
    d.threads = G::THREADS;
    d.smem = G::SMEM;
    d.tx = TX;
    d.ty = TY;
    d.ux = 2;
    d.uy = UY;
    d.pf = PF;
    d.tma = TMA;
    d.nin = 5;
    d.nout = 3;
    d.nio = 3;
    d.n1d = 3;
    d.rz = 2;
    d.ry = 2;
    d.rx = 2;
    d.rzr = 2;
    d.prio = prio;
    return d;
}

// rhs4center with cooperative derivative fields (rhs4f.cuh)
template <int TX, int TY, int PF, bool TMA, int FB = 1>
KernelDesc make_rhs4f_desc(const char *dag, int prio) {
    using G = dev::R4fGeo<TX, TY, PF, FB>;
    KernelDesc d = make_rhs4_desc<TX, TY, 1, PF, TMA>(dag, prio);
    char buf[96];
    std::snprintf(buf, sizeof buf, "r4%s_%s_%dx%d_u2x1_pf%d", FB == 2 ? "g" : "f", TMA ? "tma" : "lsu", TX, TY, PF);
    d.variant = buf;
    d.fn = reinterpret_cast<const void *>(&dev::sdag_rhs4f<TX, TY, PF, TMA, FB>);
    d.threads = G::THREADS;
    d.smem = G::SMEM;
    return d;
}

#define SDAG_RHS4F_PAIR(v, DAG, TX, TY, PF, PRIO)                                  \
    do {                                                                           \
        v.push_back(make_rhs4f_desc<TX, TY, PF, true>(DAG, PRIO));                 \
        v.push_back(make_rhs4f_desc<TX, TY, PF, false>(DAG, PRIO + 100));          \
    } while (0)
#define SDAG_RHS4G_PAIR(v, DAG, TX, TY, PRIO)                                      \
    do {                                                                           \
        v.push_back(make_rhs4f_desc<TX, TY, 0, true, 2>(DAG, PRIO));               \
        v.push_back(make_rhs4f_desc<TX, TY, 0, false, 2>(DAG, PRIO + 100));        \
    } while (0)

#define SDAG_RHS4_PAIR(v, DAG, TX, TY, UY, PF, PRIO)                               \
    do {                                                                           \
        v.push_back(make_rhs4_desc<TX, TY, UY, PF, true>(DAG, PRIO));              \
        v.push_back(make_rhs4_desc<TX, TY, UY, PF, false>(DAG, PRIO + 100));       \
    } while (0)

// register-capped variant: __launch_bounds__(threads, MINB), TMA only
#define SDAG_STAR_MB(v, BODY, DAG, TX, TY, UY, PF, MB, PRIO) \
    v.push_back(make_star_desc<dev::BODY, TX, TY, UY, PF, true, 0, MB>(DAG, PRIO))

// star2: z-taps k+1..k+R from the ring, k-1..k-R in a register queue
template <class B, int TX, int TY, int UY, int PF, bool TMA, int MINB = 1>
KernelDesc make_star2_desc(const char *dag, int prio) {
    KernelDesc d = make_star_desc<B, TX, TY, UY, PF, TMA, 0, MINB>(dag, prio);
    d.variant = "star2" + d.variant.substr(4);
    d.fn = reinterpret_cast<const void *>(&dev::sdag_star2<B, TX, TY, UY, PF, TMA, MINB>);
    return d;
}
#define SDAG_STAR2_PAIR(v, BODY, DAG, TX, TY, UY, PF, MB, PRIO)                            \
    do {                                                                                   \
        v.push_back(make_star2_desc<dev::BODY, TX, TY, UY, PF, true, MB>(DAG, PRIO));      \
        v.push_back(make_star2_desc<dev::BODY, TX, TY, UY, PF, false, MB>(DAG, PRIO + 100)); \
    } while (0)

// code-differencing variants: QMODE 2 = no arithmetic, 3 = no stores (profiling only)
// plane-loop unroll UNR (queue shifted once per UNR planes), TMA + LSU twin
#define SDAG_STAR_UNR(v, BODY, DAG, TX, TY, UY, PF, MB, UNR, PRIO)                                \
    do {                                                                                          \
        v.push_back(make_star_desc<dev::BODY, TX, TY, UY, PF, true, 0, MB, UNR>(DAG, PRIO));       \
        v.push_back(make_star_desc<dev::BODY, TX, TY, UY, PF, false, 0, MB, UNR>(DAG, PRIO + 100)); \
    } while (0)

// late-head variant (QMODE 4, TMA only)
#define SDAG_STAR_LATE(v, BODY, DAG, TX, TY, UY, PF, MB, UNR, PRIO) \
    v.push_back(make_star_desc<dev::BODY, TX, TY, UY, PF, true, 4, MB, UNR>(DAG, PRIO))

// split-accumulator variant (QMODE 5) + LSU twin
#define SDAG_STAR_SPLIT(v, BODY, DAG, TX, TY, UY, PF, MB, UNR, PRIO)                                \
    do {                                                                                            \
        v.push_back(make_star_desc<dev::BODY, TX, TY, UY, PF, true, 5, MB, UNR>(DAG, PRIO));         \
        v.push_back(make_star_desc<dev::BODY, TX, TY, UY, PF, false, 5, MB, UNR>(DAG, PRIO + 100));  \
    } while (0)

// rotating-queue variant (QMODE 6, plane loop unrolled by 2R+1) + LSU twin
#define SDAG_STAR_ROT(v, BODY, DAG, TX, TY, UY, PF, MB, PRIO)                                              \
    do {                                                                                                   \
        v.push_back(make_star_desc<dev::BODY, TX, TY, UY, PF, true, 6, MB, 2 * dev::BODY::R + 1>(DAG, PRIO)); \
        v.push_back(                                                                                       \
            make_star_desc<dev::BODY, TX, TY, UY, PF, false, 6, MB, 2 * dev::BODY::R + 1>(DAG, PRIO + 100));  \
    } while (0)

#define SDAG_STAR_DIFF(v, BODY, DAG, TX, TY, UY, PF, QM, PRIO) \
    v.push_back(make_star_desc<dev::BODY, TX, TY, UY, PF, true, QM, 1>(DAG, PRIO))

// two fused sweeps of the 27-point smoother (fuse2.cuh), TMA only
template <int GX, int GY, int UY, int PF, int MINB = 1, int UX = 2, bool ODD = false, int FORM = 0>
KernelDesc make_fuse2_desc(const char *dag, int prio) {
    using G = dev::Fuse2Geo<GX, GY, UY, PF, UX, ODD>;
    KernelDesc d;
    d.dag = dag;
    char buf[96];
    const char *tag = ODD ? "fuse2o" : "fuse2";
    if (MINB > 1)
        std::snprintf(buf, sizeof buf, "%s_tma_%dx%d_u%dx%d_pf%d_mb%d", tag, GX - 2, GY - 2, UX, UY, PF, MINB);
    else
        std::snprintf(buf, sizeof buf, "%s_tma_%dx%d_u%dx%d_pf%d", tag, GX - 2, GY - 2, UX, UY, PF);
    d.variant = buf;
    d.fn = reinterpret_cast<const void *>(&dev::sdag_box27x2<GX, GY, UY, PF, MINB, UX, ODD, FORM>);
    d.fn_mirror = reinterpret_cast<const void *>(&dev::sdag_box27x2<GX, GY, UY, PF, MINB, UX, ODD, FORM, true>);
    d.threads = G::THREADS;
    d.smem = G::SMEM;
    d.tx = GX - 2;
    d.ty = GY - 2;
    d.ux = UX;
    d.uy = UY;
    d.pf = PF;
    d.tma = true;
    d.nin = 1;
    d.nout = 1;
    d.rz = 1;
    d.ry = 2;  // TMA box (GY+2) = ty + 2*ry
    d.rx = ODD ? 4 : 3;  // TMA box PX = tx + 2*rx, origin tile - rx (even)
    d.rzr = 2;
    d.prio = prio;
    d.tsteps = 2;
    return d;
}

// NT >= 2 fused sweeps (fuseN.cuh), TMA only
template <int NT, int GX, int GY, int UY, int PF, int MINB, int UX, bool ODD, int FORM>
KernelDesc make_fuseN_desc(const char *dag, int prio) {
    using G = dev::FuseNGeo<NT, GX, GY, UY, PF, UX, ODD>;
    constexpr int H = NT - 1;
    KernelDesc d;
    d.dag = dag;
    char buf[96];
    std::snprintf(buf, sizeof buf, "fuse%d%s_tma_%dx%d_u%dx%d_pf%d_mb%d", NT, ODD ? "o" : "", GX - 2 * H, GY - 2 * H,
                  UX, UY, PF, MINB);
    d.variant = buf;
    d.fn = reinterpret_cast<const void *>(&dev::sdag_boxfuse<NT, GX, GY, UY, PF, MINB, UX, ODD, FORM>);
    d.fn_mirror = reinterpret_cast<const void *>(&dev::sdag_boxfuse<NT, GX, GY, UY, PF, MINB, UX, ODD, FORM, true>);
    d.threads = G::THREADS;
    d.smem = G::SMEM;
    d.tx = GX - 2 * H;
    d.ty = GY - 2 * H;
    d.ux = UX;
    d.uy = UY;
    d.pf = PF;
    d.tma = true;
    d.nin = 1;
    d.nout = 1;
    d.rz = 1;
    d.ry = NT;          // TMA box (GY + 2) = ty + 2 * ry
    d.rx = H + G::ML;   // TMA box PX = tx + 2 * rx, origin tile - rx (even)
    d.rzr = 1;
    d.prio = prio;
    d.tsteps = NT;
    return d;
}

// phase-unrolled queue (QMODE 1), TMA only
#define SDAG_STARQ(v, BODY, DAG, TX, TY, UY, PF, PRIO) \
    v.push_back(make_star_desc<dev::BODY, TX, TY, UY, PF, true, 1>(DAG, PRIO))

#define SDAG_STAR_PAIR(v, BODY, DAG, TX, TY, UY, PF, PRIO)                                \
    do {                                                                                   \
        v.push_back(make_star_desc<dev::BODY, TX, TY, UY, PF, true>(DAG, PRIO));           \
        v.push_back(make_star_desc<dev::BODY, TX, TY, UY, PF, false>(DAG, PRIO + 100));    \
    } while (0)

// trivial-fission variant of the generic skeleton: NOUT kernels, kernel m
// evaluating OnlyOut<B, m> (named "fis_...")
template <class B, int TX, int TY, int UX, int UY, int PF, bool TMA, int... M>
KernelDesc make_fission_desc(const char *dag, int prio, std::integer_sequence<int, M...>) {
    KernelDesc d = make_desc<B, TX, TY, UX, UY, PF, TMA>(dag, prio);
    d.variant = "fis_" + d.variant;
    d.fission = true;
    d.fission_fns = {reinterpret_cast<const void *>(&dev::sdag_sweep<dev::OnlyOut<B, M>, TX, TY, UX, UY, PF, TMA>)...};
    d.fn = d.fission_fns[0];
    return d;
}

#define SDAG_FISSION_PAIR(v, BODY, DAG, TX, TY, UX, UY, PF, PRIO)                                                \
    do {                                                                                                       \
        v.push_back(make_fission_desc<dev::BODY, TX, TY, UX, UY, PF, true>(                                   \
            DAG, PRIO, std::make_integer_sequence<int, dev::BODY::NOUT>{}));                                   \
        v.push_back(make_fission_desc<dev::BODY, TX, TY, UX, UY, PF, false>(                                  \
            DAG, PRIO + 100, std::make_integer_sequence<int, dev::BODY::NOUT>{}));                             \
    } while (0)

// a TMA variant and its LSU twin (same geometry) for unaligned grids
#define SDAG_PAIR(v, BODY, DAG, TX, TY, UX, UY, PF, PRIO)                          \
    do {                                                                           \
        v.push_back(make_desc<dev::BODY, TX, TY, UX, UY, PF, true>(DAG, PRIO));    \
        v.push_back(make_desc<dev::BODY, TX, TY, UX, UY, PF, false>(DAG, PRIO + 100)); \
    } while (0)

}  // namespace sdag

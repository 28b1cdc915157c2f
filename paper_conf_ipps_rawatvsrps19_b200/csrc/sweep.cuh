// sweep.cuh -- a4/a5: the sm_100a z-streaming sweep skeleton.
//
// Design: serial streaming along z (the paper's
// section III-A2: an order-k stencil needs at most 2k+1 planes
// resident) combined with concurrent streaming (every CTA streams
// a z-chunk, so a 512^2 plane with 64x16 tiles still fills 148 SMs) and
// prefetching -- but re-designed for Blackwell:
//
//  * each CTA owns an xy output tile TX x TY and a z-chunk; the input boxes
//    (TX+2RX) x (TY+2RY) of every staged array, one z-plane at a time, are
//    moved HBM/L2 -> shared memory by the Tensor Memory Accelerator
//    (cp.async.bulk.tensor.3d, one elected thread) into a ring of
//    NS = 2RZ+1+PF plane slots, each guarded by an mbarrier with
//    expect_tx -- the paper's compute/shift/load phases with a register
//    prefetch become a PF-deep asynchronous copy pipeline with no register
//    staging and no "shift" copies (the ring index rotates instead);
//  * an LSU fallback (cp.async 8-byte + commit/wait groups) serves grids
//    TMA cannot describe (nx odd or pointer not 16-byte aligned);
//  * every thread evaluates a UY x UX patch of output points per plane
//    (blocked unrolling) straight from the ring; the body functor
//    addresses neighbours with compile-time offsets so overlapping taps of
//    the patch are loaded once (register-level reuse);
//  * only interior points are stored (Listing 2 guards), with
//    streaming stores (st.global.cs) so outputs do not evict the halo planes
//    neighbouring CTAs still read from L2.
//
// The body functor B supplies: NIN (staged 3D inputs), NOUT (3D outputs),
// NIO (inout arrays read at offset 0 from global), N1D, per-axis staging
// radius RZ/RY/RX and
//     template <class G> static void eval(const G &g, double (&o)[NOUT]);
// with g.at(arr, dz, dy, dx), g.io(m), g.s1(arr, off), g.s(n).
#pragma once

#ifdef __CUDACC_RTC__
// NVRTC (jit.cu, NEXT-4): no host headers; the few types the skeleton needs
typedef unsigned int uint32_t;
typedef int int32_t;
typedef unsigned long long uint64_t;
typedef long long int64_t;
typedef unsigned long long uintptr_t;
struct alignas(64) CUtensorMap {
    unsigned long long opaque[16];
};
#else
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>
#endif

namespace sdag {
namespace dev {

constexpr int MAXIN = 8, MAXOUT = 5, MAXIO = 3, MAX1D = 3, MAXS = 8;

// Kernel parameters (passed __grid_constant__: the CUtensorMaps must live in
// parameter space for cp.async.bulk.tensor).
struct SweepArgs {
    CUtensorMap tmap[MAXIN];      // staged inputs, TMA variants (3D: x, y, batch*nz)
    const double *in[MAXIN];      // staged inputs, LSU variants
    double *out[MAXOUT];          // outputs (inout arrays included, in place)
    const double *io[MAXIO];      // inout arrays, read at offset 0
    const double *a1d[MAX1D];     // 1D coefficient arrays
    double s[MAXS];               // scalars, formal order
    int64_t nx, ny, nz;           // per-problem extents
    int64_t a1d_bstride[MAX1D];   // batch stride of each 1D array (0 = shared)
    int32_t lo[3], hi[3];         // output point range per axis (z, y, x)
    int32_t tiles_x, tiles_y, nchunk, zchunk;
    int32_t xmin;                 // first interior x (lo[2] may be rounded down to even as tile origin)
    int32_t zr_lo, zr_hi;         // multi-sweep kernels: planes [zr_lo, zr_hi) are global interior (others ring)
    // peer-memory halo (dist p2p path): output plane k in [peer_klo[s], peer_khi[s])
    // is also stored into z-neighbour s's buffer at element offset
    // (o - out[0]) + peer_off[s] (s = 0 lower, 1 upper; null = none)
    double *peer[2];
    int64_t peer_off[2];
    int32_t peer_klo[2], peer_khi[2];
};

// Store-side fusion of the z-slab halo exchange: a
// kernel that writes output plane k also writes it, over NVLink P2P, into the
// ghost band of the neighbour that reads it next sweep.
// true iff output plane k goes to a neighbour too (uniform per plane: test it
// once, outside the store loop, so the common path carries no per-store checks)
__device__ __forceinline__ bool mirror_plane(const SweepArgs &a, int k) {
    return (a.peer[0] && k >= a.peer_klo[0] && k < a.peer_khi[0]) ||
           (a.peer[1] && k >= a.peer_klo[1] && k < a.peer_khi[1]);
}
__device__ __forceinline__ void mirror2(const SweepArgs &a, int k, const double *o, double x, double y) {
#pragma unroll
    for (int s = 0; s < 2; s++)
        if (a.peer[s] && k >= a.peer_klo[s] && k < a.peer_khi[s])
            __stcs(reinterpret_cast<double2 *>(a.peer[s] + (o - a.out[0]) + a.peer_off[s]), make_double2(x, y));
}
__device__ __forceinline__ void mirror1(const SweepArgs &a, int k, const double *o, double v) {
#pragma unroll
    for (int s = 0; s < 2; s++)
        if (a.peer[s] && k >= a.peer_klo[s] && k < a.peer_khi[s]) __stcs(a.peer[s] + (o - a.out[0]) + a.peer_off[s], v);
}

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}

__device__ __forceinline__ void mbar_expect_tx(uint64_t *bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred P;\n"
        "SDAG_WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1;\n\t"
        "@!P bra SDAG_WAIT_%=;\n}" ::"r"(smem_u32(bar)),
        "r"(parity)
        : "memory");
}

// non-blocking probe of the phase (mbarrier.test_wait): lets a warp start the
// barrier check, do independent work, and only spin if the phase is not done
__device__ __forceinline__ bool mbar_test(uint64_t *bar, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred P;\n\t"
        "mbarrier.test_wait.parity.shared::cta.b64 P, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, P;\n}"
        : "=r"(ok)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
    return ok != 0;
}

__device__ __forceinline__ void tma_load_3d(void *dst, const CUtensorMap *map, uint64_t *bar, int x, int y, int z) {
    asm volatile(
        "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];" ::
            "r"(smem_u32(dst)),
        "l"(reinterpret_cast<uint64_t>(map)), "r"(x), "r"(y), "r"(z), "r"(smem_u32(bar))
        : "memory");
}

__device__ __forceinline__ void cp_async8(void *dst, const void *src, bool valid) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;" ::"r"(smem_u32(dst)), "l"(src), "r"(valid ? 8 : 0)
                 : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() {
    asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}

__device__ __forceinline__ void st_stream(double *p, double v) { __stcs(p, v); }

// z-window of the shared-memory ring: B::RZR if set (>= 0), else B::RZ.
template <class B>
__host__ __device__ constexpr int ring_rz() {
    return B::RZR >= 0 ? B::RZR : B::RZ;
}

// Geometry of one kernel instantiation, shared by host (smem sizing, grid)
// and device.
template <class B, int TX, int TY, int UX, int UY, int PF>
struct Geo {
    // RZ = z-window held in the shared-memory ring (B::RZR); taps beyond it
    // (bodies with RZR < RZ) are served by ld.global.nc through L1/L2.
    static constexpr int RZ = ring_rz<B>(), RY = B::RY, RX = B::RX, NIN = B::NIN;
    static constexpr int PX = TX + 2 * RX;  // ring row pitch (elements); TX even => PX even (16-B TMA rows)
    static constexpr int PY = TY + 2 * RY;
    static constexpr int PLANE = PX * PY;
    static constexpr int PLANE_AL = ((PLANE * 8 + 127) / 128) * 128 / 8;  // 128-B aligned array planes
    static constexpr int SLOT = NIN * PLANE_AL;                          // elements per ring slot
    static constexpr int NS = 2 * RZ + 1 + PF;                           // ring depth
    static constexpr int THREADS = (TX / UX) * (TY / UY);
    static constexpr int SMEM = NS * SLOT * 8 + NS * 8;                  // ring + mbarriers
    static_assert(TX % UX == 0 && TY % UY == 0, "tile must be a multiple of the patch");
    static_assert(TX % 2 == 0, "TMA rows must be 16-byte multiples");
    static_assert(PX <= 256 && PY <= 256, "TMA box dims <= 256");
    static_assert(NIN >= 1 && NIN <= MAXIN, "staged inputs");
};

// Neighbour accessor handed to the body for one patch point.
template <class B, int PX, int NIN, int SLOT_ELEMS>
struct Tap {
    const double *ring;  // smem ring base
    const int *soff;     // soff[dz + RZ] = element offset of that plane's slot
    int base;            // element offset of this point inside an array plane
    const SweepArgs *a;
    int64_t gidx;        // global linear index of the point
    int64_t b;           // problem index
    int gk, gj, gi;      // per-problem coordinates
    static constexpr int PLANE_AL = SLOT_ELEMS / NIN;

    __device__ __forceinline__ double at(int arr, int dz, int dy, int dx) const {
        constexpr int RZR = ring_rz<B>();
        if (dz < -RZR || dz > RZR)  // outside the ring window: L1/L2 path
            return __ldg(a->in[arr] + gidx + (int64_t(dz) * a->ny + dy) * a->nx + dx);
        return ring[soff[dz + RZR] + arr * PLANE_AL + base + dy * PX + dx];
    }
    // an input assigned to global memory (#assign gmem): not staged
    __device__ __forceinline__ double gm(int arr, int dz, int dy, int dx) const {
        return __ldg(a->in[arr] + gidx + (int64_t(dz) * a->ny + dy) * a->nx + dx);
    }
    __device__ __forceinline__ double io(int m) const { return a->io[m][gidx]; }
    __device__ __forceinline__ double s(int n) const { return a->s[n]; }
    __device__ __forceinline__ double s1(int arr, int off) const {
        const int ax = B::axis1d(arr);
        const int c = ax == 0 ? gk : (ax == 1 ? gj : gi);
        return __ldg(a->a1d[arr] + b * a->a1d_bstride[arr] + c + off);
    }
};

template <class B, int TX, int TY, int UX, int UY, int PF, bool USE_TMA>
__global__ void __launch_bounds__(Geo<B, TX, TY, UX, UY, PF>::THREADS)
    sdag_sweep(const __grid_constant__ SweepArgs a) {
    using G = Geo<B, TX, TY, UX, UY, PF>;
    constexpr int RZ = G::RZ, RY = G::RY, RX = G::RX, NIN = G::NIN;
    constexpr int PX = G::PX, NS = G::NS, SLOT = G::SLOT;
    constexpr int NTX = TX / UX;

    extern __shared__ __align__(128) unsigned char smem_raw[];
    double *ring = reinterpret_cast<double *>(smem_raw);
    uint64_t *bars = reinterpret_cast<uint64_t *>(smem_raw + NS * SLOT * 8);

    // ---- work unit: xy tile, z-chunk, problem ----
    const int tile_x = blockIdx.x, tile_y = blockIdx.y;
    const int chunk = blockIdx.z % a.nchunk;
    const int64_t prob = blockIdx.z / a.nchunk;
    const int x0 = a.lo[2] + tile_x * TX, y0 = a.lo[1] + tile_y * TY;
    const int kb = a.lo[0] + chunk * a.zchunk;
    const int ke = min(a.hi[0], kb + a.zchunk);
    if (kb >= ke) return;
    const int p0 = kb - RZ;          // first plane of the chunk's window
    const int plast = ke - 1 + RZ;   // last plane needed
    const int64_t zbase = prob * a.nz;

    const int t = threadIdx.x;
    const int lx = t % NTX, ly = t / NTX;

    // ---- plane loader ----
    auto issue = [&](int p) {
        const int slot = (p - p0) % NS;
        double *dst = ring + slot * SLOT;
        if constexpr (USE_TMA) {
            if (t == 0) {
                uint64_t *bar = &bars[slot];
                mbar_expect_tx(bar, uint32_t(NIN * G::PX * G::PY * 8));
#pragma unroll
                for (int q = 0; q < NIN; q++)
                    tma_load_3d(dst + q * G::PLANE_AL, &a.tmap[q], bar, x0 - RX, y0 - RY, int(zbase + p));
            }
        } else {
            const int64_t pl = (zbase + p) * a.ny * a.nx;
            for (int e = t; e < NIN * G::PLANE; e += G::THREADS) {
                const int q = e / G::PLANE, r = e % G::PLANE;
                const int yy = r / PX, xx = r % PX;
                const int gx = x0 - RX + xx, gy = y0 - RY + yy;
                const bool ok = gx >= 0 && gx < a.nx && gy >= 0 && gy < a.ny && p >= 0 && p < a.nz;
                const double *src = a.in[q] + (ok ? pl + int64_t(gy) * a.nx + gx : 0);
                cp_async8(dst + q * G::PLANE_AL + r, src, ok);
            }
        }
    };

    if constexpr (USE_TMA) {
        if (t == 0) {
            for (int s = 0; s < NS; s++) mbar_init(&bars[s], 1);
            asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        }
        __syncthreads();
    }

    // prologue: planes p0 .. p0 + 2RZ + PF - 1
    for (int p = p0; p < p0 + 2 * RZ + PF; p++) {
        if (p <= plast) issue(p);
        if constexpr (!USE_TMA) cp_async_commit();
    }

    int soff[2 * RZ + 1];

    // the first window also needs planes kb-RZ .. kb+RZ-1 (the loop waits only
    // for the newest plane of each window)
    if constexpr (USE_TMA) {
        for (int p = p0; p < kb + RZ && p <= plast; p++) mbar_wait(&bars[(p - p0) % NS], ((p - p0) / NS) & 1);
    }

    for (int k = kb; k < ke; k++) {
        // prefetch plane k+RZ+PF into the slot of plane k-RZ-1 (freed by the
        // barrier that ended the previous iteration)
        {
            const int p = k + RZ + PF;
            if (p <= plast) issue(p);
            if constexpr (!USE_TMA) cp_async_commit();
        }
        // wait for plane k+RZ
        if constexpr (USE_TMA) {
            const int p = k + RZ;
            mbar_wait(&bars[(p - p0) % NS], ((p - p0) / NS) & 1);
        } else {
            cp_async_wait<PF>();
            __syncthreads();
        }
#pragma unroll
        for (int d = 0; d < 2 * RZ + 1; d++) soff[d] = ((k - RZ + d - p0) % NS) * SLOT;

        // evaluate the thread's UY x UX patch
#pragma unroll
        for (int py = 0; py < UY; py++) {
#pragma unroll
            for (int px = 0; px < UX; px++) {
                const int ty = ly * UY + py, tx = lx * UX + px;
                const int gj = y0 + ty, gi = x0 + tx;
                const bool inside = gj < a.hi[1] && gi < a.hi[2] && gi >= a.xmin;
                Tap<B, PX, NIN, SLOT> g;
                g.ring = ring;
                g.soff = soff;
                g.base = (ty + RY) * PX + (tx + RX);
                g.a = &a;
                g.b = prob;
                g.gk = k;
                g.gj = gj;
                g.gi = gi;
                g.gidx = ((zbase + k) * a.ny + gj) * a.nx + gi;
                if (inside) {
                    double o[B::NOUT];
                    B::eval(g, o);
#pragma unroll
                    for (int m = 0; m < B::NOUT; m++) st_stream(a.out[m] + g.gidx, o[m]);
                }
            }
        }
        __syncthreads();  // plane k-RZ may be overwritten from the next iteration on
    }
}

// ---------------------------------------------------------------------------
// z-queue variant of the skeleton (NEXT-4 code generation, the star kernel's
// register queue made generic): the body's on-axis z-taps (dy = dx = 0, the
// stream dimension) come from a per-thread register queue of the
// last 2*RZQ+1 planes of each staged array, filled once per plane from the
// shared-memory ring; only off-axis taps read the ring, which therefore spans
// RZQ + RZR + 1 + PF planes (RZR = max |dz| of the off-axis taps) instead of
// 2RZ + 1 + PF.  Body interface as above plus RZQ (= RZ) -- same eval().
// ---------------------------------------------------------------------------

template <class B, int TX, int TY, int UX, int UY, int PF>
struct GeoQ {
    static constexpr int RZQ = B::RZ, RZR = B::RZR < 0 ? B::RZ : B::RZR, RY = B::RY, RX = B::RX, NIN = B::NIN;
    static constexpr int PX = TX + 2 * RX, PY = TY + 2 * RY, PLANE = PX * PY;
    static constexpr int PLANE_AL = ((PLANE * 8 + 127) / 128) * 128 / 8;
    static constexpr int SLOT = NIN * PLANE_AL;
    static constexpr int NS = RZQ + RZR + 1 + PF;
    static constexpr int NQ = 2 * RZQ + 1;
    static constexpr int THREADS = (TX / UX) * (TY / UY);
    static constexpr int SMEM = NS * SLOT * 8 + NS * 8;
    static_assert(TX % UX == 0 && TY % UY == 0, "tile must be a multiple of the patch");
    static_assert(TX % 2 == 0, "TMA rows must be 16-byte multiples");
    static_assert(PX <= 256 && PY <= 256, "TMA box dims <= 256");
};

template <class B, int PX, int NIN, int SLOT_ELEMS, int RZQ, int RZR, int NQ>
struct TapQ {
    const double *ring;
    const int *soff;    // soff[dz + RZR] = slot offset of plane k + dz, |dz| <= RZR
    const double *qv;   // this point's queue: qv[arr * NQ + dz + RZQ]
    int base;
    const SweepArgs *a;
    int64_t gidx, b;
    int gk, gj, gi;
    static constexpr int PLANE_AL = SLOT_ELEMS / NIN;

    __device__ __forceinline__ double at(int arr, int dz, int dy, int dx) const {
        if (dy == 0 && dx == 0) return qv[arr * NQ + dz + RZQ];
        return ring[soff[dz + RZR] + arr * PLANE_AL + base + dy * PX + dx];
    }
    __device__ __forceinline__ double gm(int arr, int dz, int dy, int dx) const {
        return __ldg(a->in[arr] + gidx + (int64_t(dz) * a->ny + dy) * a->nx + dx);
    }
    __device__ __forceinline__ double io(int m) const { return a->io[m][gidx]; }
    __device__ __forceinline__ double s(int n) const { return a->s[n]; }
    __device__ __forceinline__ double s1(int arr, int off) const {
        const int ax = B::axis1d(arr);
        const int c = ax == 0 ? gk : (ax == 1 ? gj : gi);
        return __ldg(a->a1d[arr] + b * a->a1d_bstride[arr] + c + off);
    }
};

template <class B, int TX, int TY, int UX, int UY, int PF, bool USE_TMA>
__global__ void __launch_bounds__(GeoQ<B, TX, TY, UX, UY, PF>::THREADS)
    sdag_sweepq(const __grid_constant__ SweepArgs a) {
    using G = GeoQ<B, TX, TY, UX, UY, PF>;
    constexpr int RZQ = G::RZQ, RZR = G::RZR, RY = G::RY, RX = G::RX, NIN = G::NIN;
    constexpr int PX = G::PX, NS = G::NS, SLOT = G::SLOT, NQ = G::NQ;
    constexpr int NTX = TX / UX;

    extern __shared__ __align__(128) unsigned char smem_raw[];
    double *ring = reinterpret_cast<double *>(smem_raw);
    uint64_t *bars = reinterpret_cast<uint64_t *>(smem_raw + NS * SLOT * 8);

    const int tile_x = blockIdx.x, tile_y = blockIdx.y;
    const int chunk = blockIdx.z % a.nchunk;
    const int64_t prob = blockIdx.z / a.nchunk;
    const int x0 = a.lo[2] + tile_x * TX, y0 = a.lo[1] + tile_y * TY;
    const int kb = a.lo[0] + chunk * a.zchunk;
    const int ke = min(a.hi[0], kb + a.zchunk);
    if (kb >= ke) return;
    const int p0 = kb - RZQ;
    const int plast = ke - 1 + RZQ;
    const int64_t zbase = prob * a.nz;

    const int t = threadIdx.x;
    const int lx = t % NTX, ly = t / NTX;

    auto issue = [&](int p) {
        const int slot = unsigned(p - p0) % NS;
        double *dst = ring + slot * SLOT;
        if constexpr (USE_TMA) {
            if (t == 0) {
                uint64_t *bar = &bars[slot];
                mbar_expect_tx(bar, uint32_t(NIN * G::PX * G::PY * 8));
#pragma unroll
                for (int q = 0; q < NIN; q++)
                    tma_load_3d(dst + q * G::PLANE_AL, &a.tmap[q], bar, x0 - RX, y0 - RY, int(zbase + p));
            }
        } else {
            const int64_t pl = (zbase + p) * a.ny * a.nx;
            for (int e = t; e < NIN * G::PLANE; e += G::THREADS) {
                const int q = e / G::PLANE, r = e % G::PLANE;
                const int yy = r / PX, xx = r % PX;
                const int gx = x0 - RX + xx, gy = y0 - RY + yy;
                const bool ok = gx >= 0 && gx < a.nx && gy >= 0 && gy < a.ny && p >= 0 && p < a.nz;
                const double *src = a.in[q] + (ok ? pl + int64_t(gy) * a.nx + gx : 0);
                cp_async8(dst + q * G::PLANE_AL + r, src, ok);
            }
        }
    };

    if constexpr (USE_TMA) {
        if (t == 0) {
            for (int s = 0; s < NS; s++) mbar_init(&bars[s], 1);
            asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        }
        __syncthreads();
    }
    for (int p = p0; p < p0 + PF; p++) {
        if (p <= plast) issue(p);
        if constexpr (!USE_TMA) cp_async_commit();
    }

    // queue[py][px][arr * NQ + i] = array arr at plane p - 2RZQ + i (own point)
    double qv[UY][UX][NIN * NQ];
#pragma unroll
    for (int py = 0; py < UY; py++)
#pragma unroll
        for (int px = 0; px < UX; px++)
#pragma unroll
            for (int e = 0; e < NIN * NQ; e++) qv[py][px][e] = 0.0;

    int soff[2 * RZR + 1];
    for (int p = p0; p <= plast; p++) {
        {
            const int pn = p + PF;
            if (pn <= plast) issue(pn);
            if constexpr (!USE_TMA) cp_async_commit();
        }
        if constexpr (USE_TMA) {
            mbar_wait(&bars[unsigned(p - p0) % NS], (unsigned(p - p0) / NS) & 1);
        } else {
            cp_async_wait<PF>();
            __syncthreads();
        }
        const int k = p - RZQ;  // output plane of this step
        // queue: shift, then the own values of the newest plane p
        const double *pl = ring + (unsigned(p - p0) % NS) * SLOT;
#pragma unroll
        for (int py = 0; py < UY; py++)
#pragma unroll
            for (int px = 0; px < UX; px++) {
                const int ty = ly * UY + py, tx = lx * UX + px;
#pragma unroll
                for (int q = 0; q < NIN; q++) {
#pragma unroll
                    for (int i = 0; i < NQ - 1; i++) qv[py][px][q * NQ + i] = qv[py][px][q * NQ + i + 1];
                    qv[py][px][q * NQ + NQ - 1] = pl[q * G::PLANE_AL + (ty + RY) * PX + (tx + RX)];
                }
            }
        if (k >= kb) {
#pragma unroll
            for (int d = 0; d < 2 * RZR + 1; d++) soff[d] = (unsigned(k - RZR + d - p0) % NS) * SLOT;
#pragma unroll
            for (int py = 0; py < UY; py++) {
#pragma unroll
                for (int px = 0; px < UX; px++) {
                    const int ty = ly * UY + py, tx = lx * UX + px;
                    const int gj = y0 + ty, gi = x0 + tx;
                    const bool inside = gj < a.hi[1] && gi < a.hi[2] && gi >= a.xmin;
                    TapQ<B, PX, NIN, SLOT, RZQ, RZR, NQ> g;
                    g.ring = ring;
                    g.soff = soff;
                    g.qv = qv[py][px];
                    g.base = (ty + RY) * PX + (tx + RX);
                    g.a = &a;
                    g.b = prob;
                    g.gk = k;
                    g.gj = gj;
                    g.gi = gi;
                    g.gidx = ((zbase + k) * a.ny + gj) * a.nx + gi;
                    if (inside) {
                        double o[B::NOUT];
                        B::eval(g, o);
#pragma unroll
                        for (int m = 0; m < B::NOUT; m++) st_stream(a.out[m] + g.gidx, o[m]);
                    }
                }
            }
        }
        __syncthreads();  // plane p - RZQ - RZR may be overwritten from the next step on
    }
}

}  // namespace dev
}  // namespace sdag

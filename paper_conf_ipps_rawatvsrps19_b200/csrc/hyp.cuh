// hyp.cuh -- sm_100a z-streaming kernel for ExpCNS hypterm
// (Table I: k=4, 358 flops, 13 IO arrays; formula reading
// SURVEY A.4 / specs/hypterm.sdag).
//
// B200 design.  hypterm moves 108 B/point from HBM but needs 48 x-taps, 48
// y-taps and 48 z-taps of raw fields per point; staging 9 planes of 8 arrays
// in shared memory does not fit, and serving z-taps from L1/L2 (the generic
// skeleton) is latency-bound.  Here every input plane is read exactly once,
// as it streams past:
//  * computation folding: per point and axis a the five flux
//    quantities F_{m,a} (cons_a; cons_m*V_a [+ q_4 if a == m]; (cons_4 + q_4)
//    V_a written as cons_4*V_a + q_4*V_a) are formed once per tap point;
//  * retiming of the z-derivative: plane p contributes
//    -dxinv2*C_r*F_z(p) to output p-r and +dxinv2*C_r*F_z(p) to output p+r,
//    accumulated in a per-thread register ring of 8 pending outputs x 5
//    fluxes; output p-4 is complete when plane p has been added;
//  * x-derivatives from 10-wide aligned windows shared by a 2-point x-pair
//    (128-bit LDS), y-derivatives from 128-bit loads of the 8 tap rows.
// Planes of all 8 arrays arrive by TMA (one mbarrier per slot, expect_tx of
// 8 boxes) into a ring of 1+PF slots with full/empty barriers.
//
// Arithmetic is re-associated relative to the spec; parity by the scaled
// error gate (reading R13).
#pragma once

#include "sweep.cuh"

namespace sdag {
namespace dev {

struct HyptermBody {
    static constexpr int R = 4, NIN = 8, NOUT = 5, NIO = 0, N1D = 0, RZ = 4, RY = 4, RX = 4, RZR = 0;
    __host__ __device__ static constexpr int axis1d(int) { return 2; }
};

template <int TX, int TY, int PF>
struct HypGeo {
    static constexpr int R = 4, ML = 4, NA = 8;
    static constexpr int NTX = TX / 2, THREADS = NTX * TY, NWARPS = (THREADS + 31) / 32;
    static constexpr int PX = TX + 2 * ML, PY = TY + 2 * R, PLANE = PX * PY;
    static constexpr int PLANE_AL = ((PLANE * 8 + 127) / 128) * 128 / 8;
    static constexpr int SLOT = NA * PLANE_AL;
    static constexpr int NS = 1 + PF;
    static constexpr int SMEM = NS * SLOT * 8 + 2 * NS * 8;
    static_assert(TX % 2 == 0, "tile");
    static_assert(PX <= 256 && PY <= 256, "TMA box");
};

template <int TX, int TY, int PF, bool USE_TMA>
__global__ void __launch_bounds__(HypGeo<TX, TY, PF>::THREADS, 1)
    sdag_hyp(const __grid_constant__ SweepArgs a) {
    using G = HypGeo<TX, TY, PF>;
    constexpr int PX = G::PX, NS = G::NS, PAL = G::PLANE_AL, SLOT = G::SLOT, ML = G::ML, R = 4;
    enum { C1 = 0, C2, C3, C4, Q1, Q2, Q3, Q4 };

    extern __shared__ __align__(128) unsigned char smem_raw[];
    double *ring = reinterpret_cast<double *>(smem_raw);
    uint64_t *full = reinterpret_cast<uint64_t *>(smem_raw + NS * SLOT * 8);
    uint64_t *empty = full + NS;

    const int tile_x = blockIdx.x, tile_y = blockIdx.y;
    const int chunk = blockIdx.z % a.nchunk;
    const int64_t prob = blockIdx.z / a.nchunk;
    const int x0 = a.lo[2] + tile_x * TX, y0 = a.lo[1] + tile_y * TY;
    const int kb = a.lo[0] + chunk * a.zchunk;
    const int ke = min(a.hi[0], kb + a.zchunk);
    if (kb >= ke) return;
    const int p0 = kb - R, plast = ke - 1 + R;
    const int64_t zbase = prob * a.nz;

    const int t = threadIdx.x;
    const int lx = t % G::NTX, ly = t / G::NTX;
    const int cx = 2 * lx, cy = ly;

    auto issue = [&](int p) {
        const int slot = (p - p0) % NS;
        double *dst = ring + slot * SLOT;
        if constexpr (USE_TMA) {
            if (t == 0) {
                const int prev = p - NS;
                if (prev >= p0) mbar_wait(&empty[slot], ((prev - p0) / NS) & 1);
                mbar_expect_tx(&full[slot], uint32_t(G::NA * G::PLANE * 8));
#pragma unroll
                for (int q = 0; q < G::NA; q++)
                    tma_load_3d(dst + q * PAL, &a.tmap[q], &full[slot], x0 - ML, y0 - R, int(zbase + p));
            }
        } else {
            const int64_t pl = (zbase + p) * a.ny * a.nx;
            for (int e = t; e < G::NA * G::PLANE; e += G::THREADS) {
                const int q = e / G::PLANE, rr = e % G::PLANE;
                const int yy = rr / PX, xx = rr % PX;
                const int gx = x0 - ML + xx, gy = y0 - R + yy;
                const bool ok = gx >= 0 && gx < a.nx && gy >= 0 && gy < a.ny && p >= 0 && p < a.nz;
                cp_async8(dst + q * PAL + rr, a.in[q] + (ok ? pl + int64_t(gy) * a.nx + gx : 0), ok);
            }
        }
    };

    if constexpr (USE_TMA) {
        if (t == 0) {
            for (int s = 0; s < NS; s++) {
                mbar_init(&full[s], 1);
                mbar_init(&empty[s], G::NWARPS);
            }
            asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        }
        __syncthreads();
    }
    for (int p = p0; p < p0 + PF; p++) {
        if (p <= plast) issue(p);
        if constexpr (!USE_TMA) cp_async_commit();
    }

    const double dx0 = a.s[0], dx1 = a.s[1], dx2 = a.s[2];
    const double C[5] = {0.0, a.s[3], a.s[4], a.s[5], a.s[6]};
    double wx[5], wy[5], wz[5];  // dxinv_a * C_r
#pragma unroll
    for (int r = 1; r <= R; r++) {
        wx[r] = dx0 * C[r];
        wy[r] = dx1 * C[r];
        wz[r] = dx2 * C[r];
    }

    const int gi = x0 + cx, gj = y0 + cy;
    const bool ok0 = gi >= a.xmin && gi < a.hi[2];
    const bool ok1 = gi + 1 >= a.xmin && gi + 1 < a.hi[2];
    const bool rowok = gj < a.hi[1];
    const bool vec = ok0 && ok1 && (a.nx % 2 == 0);

    // acc[j][m][px]: pending outputs p-4+j (j = 0..7) for flux m at the 2 points
    double acc[8][5][2];
#pragma unroll
    for (int j = 0; j < 8; j++)
#pragma unroll
        for (int m = 0; m < 5; m++) acc[j][m][0] = acc[j][m][1] = 0.0;

    // the plane loop, compiled twice: tiles entirely inside the interior (16-B
    // aligned outputs) store without per-row / per-point conditions
    auto run = [&](auto full_tag) {
    constexpr bool FULL = decltype(full_tag)::value;
    for (int p = p0; p <= plast; p++) {
        {
            const int pn = p + PF;
            if (pn <= plast) issue(pn);
            if constexpr (!USE_TMA) cp_async_commit();
        }
        if constexpr (USE_TMA) {
            mbar_wait(&full[(p - p0) % NS], ((p - p0) / NS) & 1);
        } else {
            cp_async_wait<PF>();
            __syncthreads();
        }
        const double *sl = ring + ((p - p0) % NS) * SLOT;
        auto rowp = [&](int arr, int dy) { return sl + arr * PAL + (cy + R + dy) * PX; };
        auto pair = [&](int arr, int dy) {  // the 2 centre-column values of row dy
            return *reinterpret_cast<const double2 *>(rowp(arr, dy) + cx + ML);
        };

        // ---- z: fold the 5 flux quantities of this plane and scatter them ----
        {
            const double2 c1 = pair(C1, 0), c2 = pair(C2, 0), c3 = pair(C3, 0), c4 = pair(C4, 0);
            const double2 q3 = pair(Q3, 0), q4 = pair(Q4, 0);
            double F[5][2];
            F[0][0] = c3.x, F[0][1] = c3.y;
            F[1][0] = c1.x * q3.x, F[1][1] = c1.y * q3.y;
            F[2][0] = c2.x * q3.x, F[2][1] = c2.y * q3.y;
            F[3][0] = fma(c3.x, q3.x, q4.x), F[3][1] = fma(c3.y, q3.y, q4.y);
            F[4][0] = fma(c4.x, q3.x, q4.x * q3.x), F[4][1] = fma(c4.y, q3.y, q4.y * q3.y);
#pragma unroll
            for (int m = 0; m < 5; m++)
#pragma unroll
                for (int px = 0; px < 2; px++) {
#pragma unroll
                    for (int r = 1; r <= R; r++) {
                        acc[4 - r][m][px] = fma(-wz[r], F[m][px], acc[4 - r][m][px]);  // output p-r
                        if (r < 4) acc[4 + r][m][px] = fma(wz[r], F[m][px], acc[4 + r][m][px]);
                    }
                }
            // ---- output p-4 is complete ----
            const int k = p - R;
            if (k >= kb && (FULL || rowok)) {
                const int64_t off = ((zbase + k) * a.ny + gj) * a.nx + gi;
#pragma unroll
                for (int m = 0; m < 5; m++) {
                    double *o = a.out[m] + off;
                    if (FULL || (vec && (reinterpret_cast<uintptr_t>(a.out[m]) & 15) == 0)) {
                        __stcs(reinterpret_cast<double2 *>(o), make_double2(acc[0][m][0], acc[0][m][1]));
                    } else {
                        if (ok0) __stcs(o, acc[0][m][0]);
                        if (ok1) __stcs(o + 1, acc[0][m][1]);
                    }
                }
            }
            // ---- rotate: slot j <- j+1, slot 7 <- output p+4 (first contribution) ----
#pragma unroll
            for (int j = 0; j < 7; j++)
#pragma unroll
                for (int m = 0; m < 5; m++) {
                    acc[j][m][0] = acc[j + 1][m][0];
                    acc[j][m][1] = acc[j + 1][m][1];
                }
#pragma unroll
            for (int m = 0; m < 5; m++) {
                acc[7][m][0] = wz[4] * F[m][0];
                acc[7][m][1] = wz[4] * F[m][1];
            }
        }
        // ---- x and y derivatives of output p (now ring slot 3) ----
        if (p >= kb && p < ke) {
            {  // x: windows [cx-4, cx+6) of row 0; index 4+px+dx
                double u1[10], p4[10];
                const double *ru = rowp(Q1, 0) + cx, *rp4 = rowp(Q4, 0) + cx;
#pragma unroll
                for (int c = 0; c < 5; c++) {
                    const double2 v = *reinterpret_cast<const double2 *>(ru + 2 * c);
                    u1[2 * c] = v.x, u1[2 * c + 1] = v.y;
                    const double2 w = *reinterpret_cast<const double2 *>(rp4 + 2 * c);
                    p4[2 * c] = w.x, p4[2 * c + 1] = w.y;
                }
#pragma unroll
                for (int m = 0; m < 5; m++) {
                    double f[10];
                    const int arr = (m == 0) ? C1 : (m == 4 ? C4 : m - 1);  // cons_1 for mass along x
                    const double *rc = rowp(arr, 0) + cx;
#pragma unroll
                    for (int c = 0; c < 5; c++) {
                        const double2 v = *reinterpret_cast<const double2 *>(rc + 2 * c);
                        f[2 * c] = v.x, f[2 * c + 1] = v.y;
                    }
#pragma unroll
                    for (int c = 0; c < 10; c++) {
                        if (m == 1) f[c] = fma(f[c], u1[c], p4[c]);                 // cons_1*u + p
                        else if (m == 2 || m == 3) f[c] = f[c] * u1[c];             // cons_m*u
                        else if (m == 4) f[c] = fma(f[c], u1[c], p4[c] * u1[c]);    // (cons_4 + p)*u
                    }
#pragma unroll
                    for (int px = 0; px < 2; px++)
#pragma unroll
                        for (int r = 1; r <= R; r++)
                            acc[3][m][px] = fma(-wx[r], f[4 + px + r] - f[4 + px - r], acc[3][m][px]);
                }
            }
            {  // y: tap rows +-r, 2-wide pairs
#pragma unroll
                for (int r = 1; r <= R; r++) {
                    double fp[5][2], fm[5][2];
#pragma unroll
                    for (int s = 0; s < 2; s++) {
                        const int dy = s == 0 ? r : -r;
                        const double2 c1 = pair(C1, dy), c2 = pair(C2, dy), c3 = pair(C3, dy), c4 = pair(C4, dy);
                        const double2 v = pair(Q2, dy), pr = pair(Q4, dy);
                        double(&f)[5][2] = s == 0 ? fp : fm;
                        f[0][0] = c2.x, f[0][1] = c2.y;
                        f[1][0] = c1.x * v.x, f[1][1] = c1.y * v.y;
                        f[2][0] = fma(c2.x, v.x, pr.x), f[2][1] = fma(c2.y, v.y, pr.y);
                        f[3][0] = c3.x * v.x, f[3][1] = c3.y * v.y;
                        f[4][0] = fma(c4.x, v.x, pr.x * v.x), f[4][1] = fma(c4.y, v.y, pr.y * v.y);
                    }
#pragma unroll
                    for (int m = 0; m < 5; m++)
#pragma unroll
                        for (int px = 0; px < 2; px++)
                            acc[3][m][px] = fma(-wy[r], fp[m][px] - fm[m][px], acc[3][m][px]);
                }
            }
        }
        if constexpr (USE_TMA) {  // all reads of this plane's slot are done
            __syncwarp();
            if ((t & 31) == 0)
                asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&empty[(p - p0) % NS]))
                             : "memory");
        }
        if constexpr (!USE_TMA) __syncthreads();
    }
    };
    bool tile_full = x0 >= a.xmin && x0 + TX <= a.hi[2] && y0 + TY <= a.hi[1] && (a.nx % 2 == 0);
#pragma unroll
    for (int m = 0; m < 5; m++) tile_full = tile_full && (reinterpret_cast<uintptr_t>(a.out[m]) & 15) == 0;
    if (tile_full)
        run(std::integral_constant<bool, true>{});
    else
        run(std::integral_constant<bool, false>{});
}

// ---------------------------------------------------------------------------
// hypc: the same retimed/folded sweep with each array's staged box cropped to
// the taps it has.  Per the formula the x-fluxes read cons_1..4,
// q_1, q_4; the y-fluxes cons_1..4, q_2, q_4; the z-fluxes only the centre
// column.  So q_1 needs no y-halo, q_2 no x-halo and q_3 no halo at all: the
// TMA fill shrinks from 8 full (TX+8)x(TY+8) boxes to 5 full + 3 cropped ones
// (-15 % shared-memory writes and L2->SM bytes at 64x8).  The centre pairs the
// z-fold loads are reused by the x-windows (one LDS.128 less per array).
// Shared memory is the bound of this kernel (DESIGN 6.4).
template <int TX, int TY, int PF>
struct HypcGeo {
    static constexpr int R = 4, NA = 8;
    static constexpr int NTX = TX / 2, THREADS = NTX * TY, NWARPS = (THREADS + 31) / 32;
    // arrays C1 C2 C3 C4 Q1 Q2 Q3 Q4 (formal order)
    __host__ __device__ static constexpr int mx(int q) { return (q == 5 || q == 6) ? 0 : R; }
    __host__ __device__ static constexpr int my(int q) { return (q == 4 || q == 6) ? 0 : R; }
    __host__ __device__ static constexpr int px(int q) { return TX + 2 * mx(q); }
    __host__ __device__ static constexpr int py(int q) { return TY + 2 * my(q); }
    __host__ __device__ static constexpr int al(int q) { return ((px(q) * py(q) * 8 + 127) / 128) * 128 / 8; }
    __host__ __device__ static constexpr int off(int q) {
        int o = 0;
        for (int i = 0; i < q; i++) o += al(i);
        return o;
    }
    __host__ __device__ static constexpr int bytes() {
        int b = 0;
        for (int i = 0; i < NA; i++) b += px(i) * py(i) * 8;
        return b;
    }
    static constexpr int SLOT = off(NA);
    static constexpr int NS = 1 + PF;
    static constexpr int SMEM = NS * SLOT * 8 + 2 * NS * 8;
    static_assert(TX % 2 == 0, "tile");
    static_assert(TX + 2 * R <= 256 && TY + 2 * R <= 256, "TMA box");
};

template <int TX, int TY, int PF, bool USE_TMA>
__global__ void __launch_bounds__(HypcGeo<TX, TY, PF>::THREADS, 1)
    sdag_hypc(const __grid_constant__ SweepArgs a) {
    using G = HypcGeo<TX, TY, PF>;
    constexpr int NS = G::NS, SLOT = G::SLOT, R = 4;
    enum { C1 = 0, C2, C3, C4, Q1, Q2, Q3, Q4 };

    extern __shared__ __align__(128) unsigned char smem_raw[];
    double *ring = reinterpret_cast<double *>(smem_raw);
    uint64_t *full = reinterpret_cast<uint64_t *>(smem_raw + NS * SLOT * 8);
    uint64_t *empty = full + NS;

    const int tile_x = blockIdx.x, tile_y = blockIdx.y;
    const int chunk = blockIdx.z % a.nchunk;
    const int64_t prob = blockIdx.z / a.nchunk;
    const int x0 = a.lo[2] + tile_x * TX, y0 = a.lo[1] + tile_y * TY;
    const int kb = a.lo[0] + chunk * a.zchunk;
    const int ke = min(a.hi[0], kb + a.zchunk);
    if (kb >= ke) return;
    const int p0 = kb - R, plast = ke - 1 + R;
    const int64_t zbase = prob * a.nz;

    const int t = threadIdx.x;
    const int lx = t % G::NTX, ly = t / G::NTX;
    const int cx = 2 * lx, cy = ly;

    auto issue = [&](int p) {
        const int slot = (p - p0) % NS;
        double *dst = ring + slot * SLOT;
        if constexpr (USE_TMA) {
            if (t == 0) {
                const int prev = p - NS;
                if (prev >= p0) mbar_wait(&empty[slot], ((prev - p0) / NS) & 1);
                mbar_expect_tx(&full[slot], uint32_t(G::bytes()));
#pragma unroll
                for (int q = 0; q < G::NA; q++)
                    tma_load_3d(dst + G::off(q), &a.tmap[q], &full[slot], x0 - G::mx(q), y0 - G::my(q),
                                int(zbase + p));
            }
        } else {
            const int64_t pl = (zbase + p) * a.ny * a.nx;
#pragma unroll
            for (int q = 0; q < G::NA; q++) {
                const int PXq = G::px(q), NE = G::px(q) * G::py(q);
                for (int e = t; e < NE; e += G::THREADS) {
                    const int yy = e / PXq, xx = e % PXq;
                    const int gx = x0 - G::mx(q) + xx, gy = y0 - G::my(q) + yy;
                    const bool ok = gx >= 0 && gx < a.nx && gy >= 0 && gy < a.ny && p >= 0 && p < a.nz;
                    cp_async8(dst + G::off(q) + e, a.in[q] + (ok ? pl + int64_t(gy) * a.nx + gx : 0), ok);
                }
            }
        }
    };

    if constexpr (USE_TMA) {
        if (t == 0) {
            for (int s = 0; s < NS; s++) {
                mbar_init(&full[s], 1);
                mbar_init(&empty[s], G::NWARPS);
            }
            asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        }
        __syncthreads();
    }
    for (int p = p0; p < p0 + PF; p++) {
        if (p <= plast) issue(p);
        if constexpr (!USE_TMA) cp_async_commit();
    }

    const double dx0 = a.s[0], dx1 = a.s[1], dx2 = a.s[2];
    const double C[5] = {0.0, a.s[3], a.s[4], a.s[5], a.s[6]};
    double wx[5], wy[5], wz[5];  // dxinv_a * C_r
#pragma unroll
    for (int r = 1; r <= R; r++) {
        wx[r] = dx0 * C[r];
        wy[r] = dx1 * C[r];
        wz[r] = dx2 * C[r];
    }

    const int gi = x0 + cx, gj = y0 + cy;
    const bool ok0 = gi >= a.xmin && gi < a.hi[2];
    const bool ok1 = gi + 1 >= a.xmin && gi + 1 < a.hi[2];
    const bool rowok = gj < a.hi[1];
    const bool vec = ok0 && ok1 && (a.nx % 2 == 0);

    // acc[j][m][px]: pending outputs p-4+j (j = 0..7) for flux m at the 2 points
    double acc[8][5][2];
#pragma unroll
    for (int j = 0; j < 8; j++)
#pragma unroll
        for (int m = 0; m < 5; m++) acc[j][m][0] = acc[j][m][1] = 0.0;

    for (int p = p0; p <= plast; p++) {
        {
            const int pn = p + PF;
            if (pn <= plast) issue(pn);
            if constexpr (!USE_TMA) cp_async_commit();
        }
        if constexpr (USE_TMA) {
            mbar_wait(&full[(p - p0) % NS], ((p - p0) / NS) & 1);
        } else {
            cp_async_wait<PF>();
            __syncthreads();
        }
        const double *sl = ring + ((p - p0) % NS) * SLOT;
        // pointer to (cx + dx, cy + dy) of array q in this slot
        auto at = [&](int q, int dy, int dx) {
            return sl + G::off(q) + (cy + G::my(q) + dy) * G::px(q) + (cx + G::mx(q) + dx);
        };
        auto pair = [&](int q, int dy) { return *reinterpret_cast<const double2 *>(at(q, dy, 0)); };

        const double2 c1 = pair(C1, 0), c2 = pair(C2, 0), c3 = pair(C3, 0), c4 = pair(C4, 0);
        const double2 q1 = pair(Q1, 0), q3 = pair(Q3, 0), q4 = pair(Q4, 0);
        // ---- z: fold the 5 flux quantities of this plane and scatter them ----
        {
            double F[5][2];
            F[0][0] = c3.x, F[0][1] = c3.y;
            F[1][0] = c1.x * q3.x, F[1][1] = c1.y * q3.y;
            F[2][0] = c2.x * q3.x, F[2][1] = c2.y * q3.y;
            F[3][0] = fma(c3.x, q3.x, q4.x), F[3][1] = fma(c3.y, q3.y, q4.y);
            F[4][0] = fma(c4.x, q3.x, q4.x * q3.x), F[4][1] = fma(c4.y, q3.y, q4.y * q3.y);
#pragma unroll
            for (int m = 0; m < 5; m++)
#pragma unroll
                for (int px = 0; px < 2; px++) {
#pragma unroll
                    for (int r = 1; r <= R; r++) {
                        acc[4 - r][m][px] = fma(-wz[r], F[m][px], acc[4 - r][m][px]);  // output p-r
                        if (r < 4) acc[4 + r][m][px] = fma(wz[r], F[m][px], acc[4 + r][m][px]);
                    }
                }
            const int k = p - R;
            if (k >= kb && rowok) {
                const int64_t off = ((zbase + k) * a.ny + gj) * a.nx + gi;
#pragma unroll
                for (int m = 0; m < 5; m++) {
                    double *o = a.out[m] + off;
                    if (vec && (reinterpret_cast<uintptr_t>(a.out[m]) & 15) == 0) {
                        __stcs(reinterpret_cast<double2 *>(o), make_double2(acc[0][m][0], acc[0][m][1]));
                    } else {
                        if (ok0) __stcs(o, acc[0][m][0]);
                        if (ok1) __stcs(o + 1, acc[0][m][1]);
                    }
                }
            }
#pragma unroll
            for (int j = 0; j < 7; j++)
#pragma unroll
                for (int m = 0; m < 5; m++) {
                    acc[j][m][0] = acc[j + 1][m][0];
                    acc[j][m][1] = acc[j + 1][m][1];
                }
#pragma unroll
            for (int m = 0; m < 5; m++) {
                acc[7][m][0] = wz[4] * F[m][0];
                acc[7][m][1] = wz[4] * F[m][1];
            }
        }
        // ---- x and y derivatives of output p (now ring slot 3) ----
        if (p >= kb && p < ke) {
            {  // x: windows [cx-4, cx+6) of row 0; index 4+px+dx; centre pair reused
                auto window = [&](int q, double2 ctr, double (&f)[10]) {
#pragma unroll
                    for (int c = 0; c < 5; c++) {
                        const double2 v = c == 2 ? ctr : *reinterpret_cast<const double2 *>(at(q, 0, 2 * c - 4));
                        f[2 * c] = v.x, f[2 * c + 1] = v.y;
                    }
                };
                double u1[10], p4[10];
                window(Q1, q1, u1);
                window(Q4, q4, p4);
#pragma unroll
                for (int m = 0; m < 5; m++) {
                    double f[10];
                    if (m <= 1) window(C1, c1, f);
                    else if (m == 2) window(C2, c2, f);
                    else if (m == 3) window(C3, c3, f);
                    else window(C4, c4, f);
#pragma unroll
                    for (int c = 0; c < 10; c++) {
                        if (m == 1) f[c] = fma(f[c], u1[c], p4[c]);                 // cons_1*u + p
                        else if (m == 2 || m == 3) f[c] = f[c] * u1[c];             // cons_m*u
                        else if (m == 4) f[c] = fma(f[c], u1[c], p4[c] * u1[c]);    // (cons_4 + p)*u
                    }
#pragma unroll
                    for (int px = 0; px < 2; px++)
#pragma unroll
                        for (int r = 1; r <= R; r++)
                            acc[3][m][px] = fma(-wx[r], f[4 + px + r] - f[4 + px - r], acc[3][m][px]);
                }
            }
            {  // y: tap rows +-r, 2-wide pairs
#pragma unroll
                for (int r = 1; r <= R; r++) {
                    double fp[5][2], fm[5][2];
#pragma unroll
                    for (int s = 0; s < 2; s++) {
                        const int dy = s == 0 ? r : -r;
                        const double2 e1 = pair(C1, dy), e2 = pair(C2, dy), e3 = pair(C3, dy), e4 = pair(C4, dy);
                        const double2 v = pair(Q2, dy), pr = pair(Q4, dy);
                        double(&f)[5][2] = s == 0 ? fp : fm;
                        f[0][0] = e2.x, f[0][1] = e2.y;
                        f[1][0] = e1.x * v.x, f[1][1] = e1.y * v.y;
                        f[2][0] = fma(e2.x, v.x, pr.x), f[2][1] = fma(e2.y, v.y, pr.y);
                        f[3][0] = e3.x * v.x, f[3][1] = e3.y * v.y;
                        f[4][0] = fma(e4.x, v.x, pr.x * v.x), f[4][1] = fma(e4.y, v.y, pr.y * v.y);
                    }
#pragma unroll
                    for (int m = 0; m < 5; m++)
#pragma unroll
                        for (int px = 0; px < 2; px++)
                            acc[3][m][px] = fma(-wy[r], fp[m][px] - fm[m][px], acc[3][m][px]);
                }
            }
        }
        if constexpr (USE_TMA) {  // all reads of this plane's slot are done
            __syncwarp();
            if ((t & 31) == 0)
                asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&empty[(p - p0) % NS]))
                             : "memory");
        }
        if constexpr (!USE_TMA) __syncthreads();
    }
}

}  // namespace dev
}  // namespace sdag

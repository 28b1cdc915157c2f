// rhs4.cuh -- sm_100a z-streaming kernel for SW4 rhs4center
// (Table I: k=2, 666 flops, 8 IO arrays; temporaries of Fig 3,
// P:1347-1370; formula reading SURVEY A.5 / specs/rhs4center.sdag).
//
// B200 design.  rhs4center is FP64-bound (OI 7.4 > ridge 5.8), but the
// generic skeleton is shared-memory bound before it gets there: one point
// reads 161 distinct taps (26 of mu/la, 39 of the u stars, 96 corner taps of
// the mixed derivatives) ~= 10 smem wavefronts, ~10 SM clocks per point against
// ~6 for its FP64 work.  This kernel
//  * evaluates a 2 x UY patch per thread from 128-bit loads of aligned x-pairs
//    (a row window [x-2, x+4) is three LDS.128), so the patch shares its taps:
//    ~45 double2 loads per point instead of 161 scalar ones;
//  * factors every mixed term D_a[c * D_b u] (the spec's inner/outer
//    4-point first differences) into a derivative *field*
//    D_b u evaluated once per tap position of the patch and then
//    differentiated -- e.g. D_x[la * D_y u1] needs D_y u1 on the 6 columns of
//    the row window, each computed once, not 4 times per point (computation
//    folding);
//  * streams z through a TMA ring of 5+PF planes of the 5 staged arrays
//    (u0, u1, u2, mu, la; the z-window is +-2) with full/empty mbarriers as
//    the star/box/hyp kernels.
// Arithmetic is re-associated relative to the spec (and the mu/la products
// are shared between taps); parity by the scaled error gate (reading R13).
#pragma once

#include "sweep.cuh"

namespace sdag {
namespace dev {

template <int TX, int TY, int UY, int PF>
struct R4Geo {
    static constexpr int R = 2, NA = 5;
    static constexpr int NTX = TX / 2, NTY = TY / UY, THREADS = NTX * NTY, NWARPS = (THREADS + 31) / 32;
    static constexpr int PX = TX + 4, PY = TY + 4, PLANE = PX * PY;
    static constexpr int PLANE_AL = ((PLANE * 8 + 127) / 128) * 128 / 8;
    static constexpr int SLOT = NA * PLANE_AL;
    static constexpr int NS = 5 + PF;
    static constexpr int IOQ = 2 * 3 * UY * THREADS;  // double2 staging of uacc (2 planes)
    static constexpr int NSTR = PX + PY + NS;          // strx/stry windows of the tile, strz per ring slot
    static constexpr int SMEM = NS * SLOT * 8 + 2 * NS * 8 + IOQ * 16 + NSTR * 8;
    static_assert(TX % 2 == 0 && TY % UY == 0, "tile");
    static_assert(PX <= 256 && PY <= 256, "TMA box");
};

// 4-point first difference (inner form of the spec): g(-2) - g(+2) + 8*(g(+1) - g(-1))
__device__ __forceinline__ double d4(double m2, double m1, double p1, double p2) {
    return (m2 - p2) + 8.0 * (p1 - m1);
}
// weight of offset d in D[g] = g(-2) - 8 g(-1) + 8 g(+1) - g(+2)
__host__ __device__ constexpr double w4(int d) {
    return d == -2 ? 1.0 : (d == -1 ? -8.0 : (d == 1 ? 8.0 : (d == 2 ? -1.0 : 0.0)));
}

// compiler scheduling fence between evaluation phases: keeps the loads of a
// phase from being hoisted into the previous one (register pressure)
#define SDAG_PHASE()

__device__ __forceinline__ double2 lds2(const double *p) { return *reinterpret_cast<const double2 *>(p); }

// the four SW4 coefficient combinations of c_s(-2..2) along one axis (mux1..mux4)
struct Coef4 {
    double c1, c2, c3, c4;
    __device__ __forceinline__ Coef4(double m2, double m1, double m0, double p1, double p2, double tf) {
        c1 = m1 - tf * (m0 + m2);
        c2 = m2 + p1 + 3.0 * (m0 + m1);
        c3 = m1 + p2 + 3.0 * (p1 + m0);
        c4 = p1 - tf * (m0 + p2);
    }
};
// sum_m K_m * (u(s_m) - u(0)), s = (-2, -1, +1, +2)
__device__ __forceinline__ double ksum(const Coef4 &K, double um2, double um1, double u0, double up1, double up2) {
    return K.c1 * (um2 - u0) + K.c2 * (um1 - u0) + K.c3 * (up1 - u0) + K.c4 * (up2 - u0);
}
__device__ __forceinline__ Coef4 k2ml(const Coef4 &m, const Coef4 &l) {  // 2*mu + la
    Coef4 r = m;
    r.c1 = fma(2.0, m.c1, l.c1);
    r.c2 = fma(2.0, m.c2, l.c2);
    r.c3 = fma(2.0, m.c3, l.c3);
    r.c4 = fma(2.0, m.c4, l.c4);
    return r;
}

template <int TX, int TY, int UY, int PF, bool USE_TMA>
__global__ void __launch_bounds__(R4Geo<TX, TY, UY, PF>::THREADS, 1)
    sdag_rhs4(const __grid_constant__ SweepArgs a) {
    using G = R4Geo<TX, TY, UY, PF>;
    constexpr int PX = G::PX, NS = G::NS, PAL = G::PLANE_AL, SLOT = G::SLOT;
    constexpr int NR = UY + 4;  // rows of the patch's y-window
    enum { U0 = 0, U1, U2, MU, LA };

    extern __shared__ __align__(128) unsigned char smem_raw[];
    double *ring = reinterpret_cast<double *>(smem_raw);
    uint64_t *full = reinterpret_cast<uint64_t *>(smem_raw + NS * SLOT * 8);
    uint64_t *empty = full + NS;
    double2 *ioq = reinterpret_cast<double2 *>(smem_raw + NS * SLOT * 8 + 2 * NS * 8);
    double *strs = reinterpret_cast<double *>(ioq + G::IOQ);  // [PX] strx window, [PY] stry window, [NS] strz
    double *szs = strs + PX + G::PY;

    const int tile_x = blockIdx.x, tile_y = blockIdx.y;
    const int chunk = blockIdx.z % a.nchunk;
    const int64_t prob = blockIdx.z / a.nchunk;
    const int x0 = a.lo[2] + tile_x * TX, y0 = a.lo[1] + tile_y * TY;
    const int kb = a.lo[0] + chunk * a.zchunk;
    const int ke = min(a.hi[0], kb + a.zchunk);
    if (kb >= ke) return;
    const int p0 = kb - 2, plast = ke + 1;
    const int64_t zbase = prob * a.nz;
    const int nx = int(a.nx), ny = int(a.ny);

    const int t = threadIdx.x;
    const int lx = t % G::NTX, ly = t / G::NTX;
    const int cx = 2 * lx, cy = UY * ly;  // tile-local patch origin; box column of patch col 0 is cx + 2

    auto issue = [&](int p) {
        const int slot = unsigned(p - p0) % NS;
        double *dst = ring + slot * SLOT;
        if constexpr (USE_TMA) {
            if (t == 0) {
                const int prev = p - NS;
                if (prev >= p0) mbar_wait(&empty[slot], (unsigned(prev - p0) / NS) & 1);
                mbar_expect_tx(&full[slot], uint32_t(G::NA * G::PLANE * 8));
#pragma unroll
                for (int q = 0; q < G::NA; q++)
                    tma_load_3d(dst + q * PAL, &a.tmap[q], &full[slot], x0 - 2, y0 - 2, int(zbase + p));
                // strz[p] rides on the same barrier (second arrival, when the copy lands)
                cp_async8(&szs[slot], a.a1d[2] + prob * a.a1d_bstride[2] + p, true);
                asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(smem_u32(&full[slot]))
                             : "memory");
            }
        } else {
            const int64_t pl = (zbase + p) * a.ny * a.nx;
            for (int e = t; e < G::NA * G::PLANE; e += G::THREADS) {
                const int q = e / G::PLANE, rr = e % G::PLANE;
                const int yy = rr / PX, xx = rr % PX;
                const int gx = x0 - 2 + xx, gy = y0 - 2 + yy;
                const bool ok = gx >= 0 && gx < nx && gy >= 0 && gy < ny && p >= 0 && p < a.nz;
                cp_async8(dst + q * PAL + rr, a.in[q] + (ok ? pl + int64_t(gy) * a.nx + gx : 0), ok);
            }
            if (t == 0) cp_async8(&szs[slot], a.a1d[2] + prob * a.a1d_bstride[2] + p, true);
        }
    };

    if constexpr (USE_TMA) {
        if (t == 0) {
            for (int s = 0; s < NS; s++) {
                mbar_init(&full[s], 2);  // TMA expect_tx arrival + strz cp.async arrival
                mbar_init(&empty[s], G::NWARPS);
            }
            asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        }
        __syncthreads();
    }
    for (int p = p0; p < p0 + 4 + PF; p++) {
        if (p <= plast) issue(p);
        if constexpr (!USE_TMA) cp_async_commit();
    }
    if constexpr (USE_TMA) {
        for (int p = p0; p < kb + 2 && p <= plast; p++) mbar_wait(&full[unsigned(p - p0) % NS], (unsigned(p - p0) / NS) & 1);
    }

    const double tf = a.s[0], i6 = a.s[1], i144 = a.s[2], cof = a.s[3], a1 = a.s[4];
    const double *strx = a.a1d[0] + prob * a.a1d_bstride[0];
    const double *stry = a.a1d[1] + prob * a.a1d_bstride[1];
    const int gi0 = x0 + cx, gj0 = y0 + cy;  // global x, y of the patch origin
    for (int e = t; e < PX + G::PY; e += G::THREADS)
        strs[e] = e < PX ? __ldg(strx + min(max(x0 - 2 + e, 0), nx - 1))
                         : __ldg(stry + min(max(y0 - 2 + (e - PX), 0), ny - 1));
    __syncthreads();
    // strx at window column c of the patch, stry at window row r (shared memory:
    // loop-invariant, kept out of the register file)
    auto sx = [&](int c) { return strs[cx + c]; };
    auto sy = [&](int r) { return strs[PX + cy + r]; };
    bool okx[2];
#pragma unroll
    for (int px = 0; px < 2; px++) okx[px] = gi0 + px >= a.xmin && gi0 + px < a.hi[2];

    // uacc (inout, read at offset 0 from global) of the next plane is copied
    // global -> shared by cp.async (no registers held, no stall) one plane
    // ahead, so its DRAM latency hides behind a plane of arithmetic
    auto load_io = [&](int k) {
        double2 *q = ioq + (k & 1) * (3 * UY * G::THREADS);
#pragma unroll
        for (int py = 0; py < UY; py++) {
            const bool rowok = gj0 + py < a.hi[1] && k < ke;
            const int64_t off = ((zbase + k) * a.ny + gj0 + py) * a.nx + gi0;
#pragma unroll
            for (int c = 0; c < 3; c++) {
                double *dst = reinterpret_cast<double *>(q + (c * UY + py) * G::THREADS + t);
                const double *src = a.io[c] + off;
                if (rowok && okx[0] && okx[1] && ((reinterpret_cast<uintptr_t>(src) & 15) == 0)) {
                    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
                } else {
                    cp_async8(dst, rowok && okx[0] ? src : a.io[c], rowok && okx[0]);
                    cp_async8(dst + 1, rowok && okx[1] ? src + 1 : a.io[c], rowok && okx[1]);
                }
            }
        }
        cp_async_commit();
    };
    load_io(kb);
    for (int k = kb; k < ke; k++) {
        load_io(k + 1);
        {
            const int pn = k + 2 + PF;
            if (pn <= plast) issue(pn);
            if constexpr (!USE_TMA) cp_async_commit();
        }
        if constexpr (USE_TMA) {
            mbar_wait(&full[unsigned(k + 2 - p0) % NS], (unsigned(k + 2 - p0) / NS) & 1);
        } else {
            cp_async_wait<PF>();
            __syncthreads();
        }
        const double *S[5];
#pragma unroll
        for (int d = 0; d < 5; d++) S[d] = ring + (unsigned(k - 2 + d - p0) % NS) * SLOT;
        double sz[5];
#pragma unroll
        for (int d = 0; d < 5; d++) sz[d] = szs[unsigned(k - 2 + d - p0) % NS];

        // address of (array, plane dz, window row r in [0, NR), box column bc)
        auto at = [&](int arr, int dz, int r, int bc) { return S[dz + 2] + arr * PAL + (cy + r) * PX + bc; };
        auto row6 = [&](int arr, int dz, int r, double (&v)[6]) {
            const double *q = at(arr, dz, r, cx);
            const double2 A = lds2(q), B = lds2(q + 2), C = lds2(q + 4);
            v[0] = A.x, v[1] = A.y, v[2] = B.x, v[3] = B.y, v[4] = C.x, v[5] = C.y;
        };
        auto pair = [&](int arr, int dz, int r) { return lds2(at(arr, dz, r, cx + 2)); };

        double sd[3][UY][2], mx[3][UY][2];  // i6-part and i144-part of r_c
#pragma unroll
        for (int c = 0; c < 3; c++)
#pragma unroll
            for (int py = 0; py < UY; py++) sd[c][py][0] = sd[c][py][1] = mx[c][py][0] = mx[c][py][1] = 0.0;

        // ---- x: second-derivative terms along x, and the xz mixed terms ----
#pragma unroll
        for (int py = 0; py < UY; py++) {
            const int r = py + 2;
            double m[6], l[6], v0[6], v1[6], v2[6];
            row6(MU, 0, r, m);
            row6(LA, 0, r, l);
            row6(U0, 0, r, v0);
            row6(U1, 0, r, v1);
            row6(U2, 0, r, v2);
            double ms[6], ls[6];
#pragma unroll
            for (int c = 0; c < 6; c++) ms[c] = m[c] * sx(c), ls[c] = l[c] * sx(c);
#pragma unroll
            for (int px = 0; px < 2; px++) {
                const int c = px + 2;
                const Coef4 M(ms[c - 2], ms[c - 1], ms[c], ms[c + 1], ms[c + 2], tf);
                const Coef4 L(ls[c - 2], ls[c - 1], ls[c], ls[c + 1], ls[c + 2], tf);
                const Coef4 K = k2ml(M, L);
                sd[0][py][px] = fma(sx(c), ksum(K, v0[c - 2], v0[c - 1], v0[c], v0[c + 1], v0[c + 2]), sd[0][py][px]);
                sd[1][py][px] = fma(sx(c), ksum(M, v1[c - 2], v1[c - 1], v1[c], v1[c + 1], v1[c + 2]), sd[1][py][px]);
                sd[2][py][px] = fma(sx(c), ksum(M, v2[c - 2], v2[c - 1], v2[c], v2[c + 1], v2[c + 2]), sd[2][py][px]);
            }
        }
        SDAG_PHASE();
#pragma unroll
        for (int py = 0; py < UY; py++) {
            const int r = py + 2;
            double m[6], l[6];
            row6(MU, 0, r, m);
            row6(LA, 0, r, l);
            // xz: r_x += sx sz (D_x[la D_z u2] + D_z[mu D_x u2]); r_z += sx sz (D_x[mu D_z u0] + D_z[la D_x u0])
            double z2[6], z0[6], ax[2] = {0.0, 0.0}, az[2] = {0.0, 0.0};
#pragma unroll
            for (int c = 0; c < 6; c++) z2[c] = z0[c] = 0.0;
#pragma unroll
            for (int dz = -2; dz <= 2; dz++) {
                if (dz == 0) continue;
                double w2[6], w0[6];
                row6(U2, dz, r, w2);
                row6(U0, dz, r, w0);
#pragma unroll
                for (int c = 0; c < 6; c++) {
                    z2[c] = fma(w4(dz), w2[c], z2[c]);
                    z0[c] = fma(w4(dz), w0[c], z0[c]);
                }
                const double2 mz = pair(MU, dz, r), lz = pair(LA, dz, r);
                ax[0] = fma(w4(dz) * mz.x, d4(w2[0], w2[1], w2[3], w2[4]), ax[0]);
                ax[1] = fma(w4(dz) * mz.y, d4(w2[1], w2[2], w2[4], w2[5]), ax[1]);
                az[0] = fma(w4(dz) * lz.x, d4(w0[0], w0[1], w0[3], w0[4]), az[0]);
                az[1] = fma(w4(dz) * lz.y, d4(w0[1], w0[2], w0[4], w0[5]), az[1]);
            }
            double g2[6], g0[6];
#pragma unroll
            for (int c = 0; c < 6; c++) g2[c] = l[c] * z2[c], g0[c] = m[c] * z0[c];
#pragma unroll
            for (int px = 0; px < 2; px++) {
                const double f = sx(px + 2) * sz[2];
                mx[0][py][px] = fma(f, d4(g2[px], g2[px + 1], g2[px + 3], g2[px + 4]) + ax[px], mx[0][py][px]);
                mx[2][py][px] = fma(f, d4(g0[px], g0[px + 1], g0[px + 3], g0[px + 4]) + az[px], mx[2][py][px]);
            }
        }

        SDAG_PHASE();
        // ---- xy mixed terms ----
        {
            // Y-fields D_y u1, D_y u0 on the 6 columns of each patch row;
            // accX: D_y[mu D_x u1] (r_x), D_y[la D_x u0] (r_y) at the patch points
            double Y1[UY][6], Y0[UY][6], bx[UY][2], by[UY][2];
#pragma unroll
            for (int py = 0; py < UY; py++) {
#pragma unroll
                for (int c = 0; c < 6; c++) Y1[py][c] = Y0[py][c] = 0.0;
                bx[py][0] = bx[py][1] = by[py][0] = by[py][1] = 0.0;
            }
#pragma unroll
            for (int r = 0; r < NR; r++) {
                double v0[6], v1[6];
                row6(U0, 0, r, v0);
                row6(U1, 0, r, v1);
                const double2 mr = pair(MU, 0, r), lr = pair(LA, 0, r);
                const double gm0 = mr.x * d4(v1[0], v1[1], v1[3], v1[4]);
                const double gm1 = mr.y * d4(v1[1], v1[2], v1[4], v1[5]);
                const double gl0 = lr.x * d4(v0[0], v0[1], v0[3], v0[4]);
                const double gl1 = lr.y * d4(v0[1], v0[2], v0[4], v0[5]);
#pragma unroll
                for (int py = 0; py < UY; py++) {
                    const int d = r - (py + 2);
                    if (d < -2 || d > 2 || d == 0) continue;
#pragma unroll
                    for (int c = 0; c < 6; c++) {
                        Y1[py][c] = fma(w4(d), v1[c], Y1[py][c]);
                        Y0[py][c] = fma(w4(d), v0[c], Y0[py][c]);
                    }
                    bx[py][0] = fma(w4(d), gm0, bx[py][0]);
                    bx[py][1] = fma(w4(d), gm1, bx[py][1]);
                    by[py][0] = fma(w4(d), gl0, by[py][0]);
                    by[py][1] = fma(w4(d), gl1, by[py][1]);
                }
            }
#pragma unroll
            for (int py = 0; py < UY; py++) {
                const int r = py + 2;
                double m[6], l[6];
                row6(MU, 0, r, m);
                row6(LA, 0, r, l);
                double g1[6], g0[6];
#pragma unroll
                for (int c = 0; c < 6; c++) g1[c] = l[c] * Y1[py][c], g0[c] = m[c] * Y0[py][c];
                const double syc = sy(r);
#pragma unroll
                for (int px = 0; px < 2; px++) {
                    const double f = sx(px + 2) * syc;
                    mx[0][py][px] = fma(f, d4(g1[px], g1[px + 1], g1[px + 3], g1[px + 4]) + bx[py][px], mx[0][py][px]);
                    mx[1][py][px] = fma(f, d4(g0[px], g0[px + 1], g0[px + 3], g0[px + 4]) + by[py][px], mx[1][py][px]);
                }
            }
        }
        SDAG_PHASE();
        // ---- second derivatives along y (str_y at the tap rows) ----
#pragma unroll
        for (int py = 0; py < UY; py++) {
            double2 mr[5], lr[5], q0[5], q1[5], q2[5];
#pragma unroll
            for (int q = 0; q < 5; q++) {
                mr[q] = pair(MU, 0, py + q);
                lr[q] = pair(LA, 0, py + q);
                q0[q] = pair(U0, 0, py + q);
                q1[q] = pair(U1, 0, py + q);
                q2[q] = pair(U2, 0, py + q);
            }
            const double syc = sy(py + 2);
#pragma unroll
            for (int px = 0; px < 2; px++) {
                auto X = [&](const double2 &v) { return px ? v.y : v.x; };
                double ms[5], ls[5];
#pragma unroll
                for (int q = 0; q < 5; q++) ms[q] = X(mr[q]) * sy(py + q), ls[q] = X(lr[q]) * sy(py + q);
                const Coef4 M(ms[0], ms[1], ms[2], ms[3], ms[4], tf);
                const Coef4 L(ls[0], ls[1], ls[2], ls[3], ls[4], tf);
                const Coef4 K = k2ml(M, L);
                sd[0][py][px] = fma(syc, ksum(M, X(q0[0]), X(q0[1]), X(q0[2]), X(q0[3]), X(q0[4])), sd[0][py][px]);
                sd[1][py][px] = fma(syc, ksum(K, X(q1[0]), X(q1[1]), X(q1[2]), X(q1[3]), X(q1[4])), sd[1][py][px]);
                sd[2][py][px] = fma(syc, ksum(M, X(q2[0]), X(q2[1]), X(q2[2]), X(q2[3]), X(q2[4])), sd[2][py][px]);
            }
        }
        SDAG_PHASE();

        // ---- z: second-derivative terms along z, and the yz mixed terms ----
        {
            // Z-fields D_z u2, D_z u1 on the patch columns of every window row;
            // cz: D_z[mu D_y u2] (r_y), D_z[la D_y u1] (r_z) at the patch points
            double2 Z2[NR], Z1[NR];
            double cyv[UY][2], czv[UY][2];
#pragma unroll
            for (int r = 0; r < NR; r++) Z2[r] = Z1[r] = make_double2(0.0, 0.0);
#pragma unroll
            for (int py = 0; py < UY; py++) cyv[py][0] = cyv[py][1] = czv[py][0] = czv[py][1] = 0.0;
#pragma unroll
            for (int dz = -2; dz <= 2; dz++) {
                if (dz == 0) continue;
                double2 v2[NR], v1[NR];
#pragma unroll
                for (int r = 0; r < NR; r++) {
                    v2[r] = pair(U2, dz, r);
                    v1[r] = pair(U1, dz, r);
                    Z2[r].x = fma(w4(dz), v2[r].x, Z2[r].x);
                    Z2[r].y = fma(w4(dz), v2[r].y, Z2[r].y);
                    Z1[r].x = fma(w4(dz), v1[r].x, Z1[r].x);
                    Z1[r].y = fma(w4(dz), v1[r].y, Z1[r].y);
                }
#pragma unroll
                for (int py = 0; py < UY; py++) {
                    const double2 mz = pair(MU, dz, py + 2), lz = pair(LA, dz, py + 2);
                    cyv[py][0] = fma(w4(dz) * mz.x, d4(v2[py].x, v2[py + 1].x, v2[py + 3].x, v2[py + 4].x), cyv[py][0]);
                    cyv[py][1] = fma(w4(dz) * mz.y, d4(v2[py].y, v2[py + 1].y, v2[py + 3].y, v2[py + 4].y), cyv[py][1]);
                    czv[py][0] = fma(w4(dz) * lz.x, d4(v1[py].x, v1[py + 1].x, v1[py + 3].x, v1[py + 4].x), czv[py][0]);
                    czv[py][1] = fma(w4(dz) * lz.y, d4(v1[py].y, v1[py + 1].y, v1[py + 3].y, v1[py + 4].y), czv[py][1]);
                }
            }
            double2 gl[NR], gm[NR];  // la D_z u2, mu D_z u1 on the window rows
#pragma unroll
            for (int r = 0; r < NR; r++) {
                const double2 lc = pair(LA, 0, r), mc = pair(MU, 0, r);
                gl[r] = make_double2(lc.x * Z2[r].x, lc.y * Z2[r].y);
                gm[r] = make_double2(mc.x * Z1[r].x, mc.y * Z1[r].y);
            }
#pragma unroll
            for (int py = 0; py < UY; py++) {
                const double f = sy(py + 2) * sz[2];
#pragma unroll
                for (int px = 0; px < 2; px++) {
                    auto X = [&](const double2 &v) { return px ? v.y : v.x; };
                    const double dyl = d4(X(gl[py]), X(gl[py + 1]), X(gl[py + 3]), X(gl[py + 4]));
                    const double dym = d4(X(gm[py]), X(gm[py + 1]), X(gm[py + 3]), X(gm[py + 4]));
                    mx[1][py][px] = fma(f, dyl + cyv[py][px], mx[1][py][px]);
                    mx[2][py][px] = fma(f, dym + czv[py][px], mx[2][py][px]);
                }
            }
        }
        SDAG_PHASE();
        // ---- second derivatives along z (str_z at the tap planes) ----
        {
#pragma unroll
            for (int py = 0; py < UY; py++) {
                double2 mz[5], lz[5], q0[5], q1[5], q2[5];
#pragma unroll
                for (int dz = -2; dz <= 2; dz++) {
                    mz[dz + 2] = pair(MU, dz, py + 2);
                    lz[dz + 2] = pair(LA, dz, py + 2);
                    q0[dz + 2] = pair(U0, dz, py + 2);
                    q1[dz + 2] = pair(U1, dz, py + 2);
                    q2[dz + 2] = pair(U2, dz, py + 2);
                }
#pragma unroll
                for (int px = 0; px < 2; px++) {
                    auto X = [&](const double2 &v) { return px ? v.y : v.x; };
                    double ms[5], ls[5];
#pragma unroll
                    for (int q = 0; q < 5; q++) ms[q] = X(mz[q]) * sz[q], ls[q] = X(lz[q]) * sz[q];
                    const Coef4 M(ms[0], ms[1], ms[2], ms[3], ms[4], tf);
                    const Coef4 L(ls[0], ls[1], ls[2], ls[3], ls[4], tf);
                    const Coef4 K = k2ml(M, L);
                    sd[0][py][px] = fma(sz[2], ksum(M, X(q0[0]), X(q0[1]), X(q0[2]), X(q0[3]), X(q0[4])), sd[0][py][px]);
                    sd[1][py][px] = fma(sz[2], ksum(M, X(q1[0]), X(q1[1]), X(q1[2]), X(q1[3]), X(q1[4])), sd[1][py][px]);
                    sd[2][py][px] = fma(sz[2], ksum(K, X(q2[0]), X(q2[1]), X(q2[2]), X(q2[3]), X(q2[4])), sd[2][py][px]);
                }
            }
        }

        // ---- uacc_c = a1*uacc_c + cof*(i6*sd_c + i144*mx_c) ----
        cp_async_wait<1>();  // this plane's uacc (the next plane's copy may still be in flight)
#pragma unroll
        for (int py = 0; py < UY; py++) {
            const int gj = gj0 + py;
            if (gj >= a.hi[1]) continue;
            const int64_t off = ((zbase + k) * a.ny + gj) * a.nx + gi0;
#pragma unroll
            for (int c = 0; c < 3; c++) {
                const double2 ioc = ioq[(k & 1) * (3 * UY * G::THREADS) + (c * UY + py) * G::THREADS + t];
                double o[2];
#pragma unroll
                for (int px = 0; px < 2; px++) {
                    const double rc = fma(i6, sd[c][py][px], i144 * mx[c][py][px]);
                    o[px] = fma(a1, px ? ioc.y : ioc.x, cof * rc);
                }
                double *dst = a.out[c] + off;
                if (okx[0] && okx[1] && ((reinterpret_cast<uintptr_t>(dst) & 15) == 0)) {
                    __stcs(reinterpret_cast<double2 *>(dst), make_double2(o[0], o[1]));
                } else {
                    if (okx[0]) __stcs(dst, o[0]);
                    if (okx[1]) __stcs(dst + 1, o[1]);
                }
            }
        }

        if constexpr (USE_TMA) {  // all reads of plane k-2's slot are done
            __syncwarp();
            if ((t & 31) == 0)
                asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&empty[unsigned(k - 2 - p0) % NS]))
                             : "memory");
        }
        if constexpr (!USE_TMA) __syncthreads();
    }
}

}  // namespace dev
}  // namespace sdag

// rhs4f.cuh -- sm_100a kernel for SW4 rhs4center with cooperative derivative
// fields (Table I: k=2, 666 flops, 8 IO arrays; formula reading
// SURVEY A.5 / specs/rhs4center.sdag; temporaries of Fig 3).
//
// Why a second rhs4 kernel.  rhs4.cuh evaluates every mixed term
// D_a[c * D_b u] per thread from the raw fields: the inner differences of a
// tap point are recomputed by every output that reads it, ~410 FP64
// instructions and ~60 128-bit shared loads per point (ncu, round 1: FP64
// pipe 63 %, LSU 76 %).  Here the nine inner "fields" of the mixed terms
// (computation folding)
//     P1 = mu D_x u1   P2 = la D_x u0   P3 = mu D_x u2
//     P4 = la D_y u1   P5 = mu D_y u0   P6 = mu D_y u2
//     P7 = la D_z u2   P8 = mu D_z u0   P9 = mu D_z u1
// are formed ONCE per point and plane:
//   * the fields differentiated in-plane (outer D_x of P4 P5 P7 P8, outer D_y
//     of P1 P2 P7 P9) go to shared memory, on the tile plus the 2-point halo
//     their outer difference reads (halo points are computed by the CTA too:
//     32 x-halo and 64 y-halo pairs per 32 x 16 tile, spread over all warps);
//   * the fields differentiated along z (P3, P6, str_x P2 + str_y P4) are
//     retimed: plane k's value is added, with its D_z weight, to
//     the pending outputs k-2, k-1, k+1, k+2 held in registers; output k-2 is
//     complete -- and stored -- once plane k has contributed.
// The second-derivative terms (mu/la coefficient combinations) stay per
// output as in rhs4.cuh.  Per CTA-plane: phase A (fields of the tile and
// halo, second derivatives, retimed z contributions; reads the TMA ring) ->
// CTA barrier -> phase B (outer x/y differences from the field planes) ->
// store of output k-2.  A second barrier before phase A's field stores
// protects the previous plane's phase-B reads (one field buffer).
// The ring holds 5 + PF planes of (u0, u1, u2, mu, la) as in rhs4.cuh; the
// loop runs over k = kb-2 .. ke+1: the two steps before and after the chunk
// only form the retimed z fields (their outputs belong to other chunks).
//
// Arithmetic is re-associated relative to the spec; parity by the scaled
// error gate (reading R13) and bitwise on integer inputs (tests/test_gpu_exact.py).
#pragma once

#include "rhs4.cuh"

namespace sdag {
namespace dev {

// FB = 2: double-buffered field planes (phase A of plane k+1 may store while
// slow warps still read plane k's), one CTA barrier per plane; FB = 1: one
// buffer and a second barrier.  The halo pair tasks go to the first warps,
// all 32 lanes busy (no divergent lanes in the other warps).
template <int TX, int TY, int PF, int FB = 1>
struct R4fGeo {
    static constexpr int R = 2, NA = 5;
    static constexpr int NTX = TX / 2, THREADS = NTX * TY, NWARPS = (THREADS + 31) / 32;
    static constexpr int PX = TX + 4, PY = TY + 4, PLANE = PX * PY;
    static constexpr int PLANE_AL = ((PLANE * 8 + 127) / 128) * 128 / 8;
    static constexpr int SLOT = NA * PLANE_AL;
    static constexpr int NS = 5 + PF;
    // field planes: XF (P4, P5, P8) on x in [-2, TX+2) x y in [0, TY);
    // YF (P1, P2, P9) on x in [0, TX) x y in [-2, TY+2); P7 on the box (PX x PY)
    static constexpr int XFW = TX + 4, XFN = XFW * TY, YFW = TX, YFN = YFW * (TY + 4);
    static constexpr int FIELDS = 3 * XFN + 3 * YFN + PLANE;
    static constexpr int NXH = 2 * TY, NYH = 4 * NTX, NHALO = NXH + NYH;  // halo pair tasks
    static constexpr int NSTR = PX + PY + NS;
    static constexpr int SMEM = NS * SLOT * 8 + FB * FIELDS * 8 + 2 * NS * 8 + NSTR * 8;
    static_assert(TX % 2 == 0 && NTX % 8 == 0, "tile: 8-lane groups stay inside one row");
    static_assert(NHALO <= THREADS, "one halo task per thread at most");
    static_assert(PX <= 256 && PY <= 256, "TMA box");
};

template <int TX, int TY, int PF, bool USE_TMA, int FB = 1>
__global__ void __launch_bounds__(R4fGeo<TX, TY, PF, FB>::THREADS, 1)
    sdag_rhs4f(const __grid_constant__ SweepArgs a) {
    using G = R4fGeo<TX, TY, PF, FB>;
    constexpr int PX = G::PX, NS = G::NS, PAL = G::PLANE_AL, SLOT = G::SLOT;
    constexpr int XFW = G::XFW, XFN = G::XFN, YFW = G::YFW, YFN = G::YFN;
    enum { U0 = 0, U1, U2, MU, LA };

    extern __shared__ __align__(128) unsigned char smem_raw[];
    double *ring = reinterpret_cast<double *>(smem_raw);
    double *fld = ring + NS * SLOT;
    uint64_t *full = reinterpret_cast<uint64_t *>(fld + FB * G::FIELDS);
    uint64_t *empty = full + NS;
    double *strs = reinterpret_cast<double *>(empty + NS);  // [PX] strx, [PY] stry, [NS] strz per slot
    double *szs = strs + PX + G::PY;

    const int tile_x = blockIdx.x, tile_y = blockIdx.y;
    const int chunk = blockIdx.z % a.nchunk;
    const int64_t prob = blockIdx.z / a.nchunk;
    const int x0 = a.lo[2] + tile_x * TX, y0 = a.lo[1] + tile_y * TY;
    const int kb = a.lo[0] + chunk * a.zchunk;
    const int ke = min(a.hi[0], kb + a.zchunk);
    if (kb >= ke) return;
    const int p0 = kb - 2, plast = ke + 1;  // planes read by the steps k = kb-2 .. ke+1
    const int64_t zbase = prob * a.nz;
    const int nx = int(a.nx), ny = int(a.ny);

    const int t = threadIdx.x, lane = t & 31, warp = t >> 5;
    const int lx = t % G::NTX, ly = t / G::NTX;
    const int cx = 2 * lx, cy = ly;  // own pair: tile (cx, cy); box col cx + 2, box row cy + 2

    auto slot_of = [&](int p) { return unsigned(p - p0) % NS; };
    auto issue = [&](int p) {
        const int slot = slot_of(p);
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
                const bool ok = gx >= 0 && gx < nx && gy >= 0 && gy < ny;
                cp_async8(dst + q * PAL + rr, a.in[q] + (ok ? pl + int64_t(gy) * a.nx + gx : 0), ok);
            }
            if (t == 0) cp_async8(&szs[slot], a.a1d[2] + prob * a.a1d_bstride[2] + p, true);
        }
    };

    if constexpr (USE_TMA) {
        if (t == 0) {
            for (int s = 0; s < NS; s++) {
                mbar_init(&full[s], 2);  // TMA expect_tx + strz cp.async arrival
                mbar_init(&empty[s], G::NWARPS);
            }
            asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        }
        __syncthreads();
    }
    int pnext = p0, waited = p0 - 1;

    const double tf = a.s[0], i6 = a.s[1], i144 = a.s[2], cof = a.s[3], a1 = a.s[4];
    const double *strx = a.a1d[0] + prob * a.a1d_bstride[0];
    const double *stry = a.a1d[1] + prob * a.a1d_bstride[1];
    for (int e = t; e < PX + G::PY; e += G::THREADS)
        strs[e] = e < PX ? __ldg(strx + min(max(x0 - 2 + e, 0), nx - 1))
                         : __ldg(stry + min(max(y0 - 2 + (e - PX), 0), ny - 1));
    __syncthreads();
    auto sx = [&](int bc) { return strs[bc]; };       // strx at box column bc
    auto sy = [&](int br) { return strs[PX + br]; };  // stry at box row br
    const int gi0 = x0 + cx, gj0 = y0 + cy;
    bool okx[2];
#pragma unroll
    for (int px = 0; px < 2; px++) okx[px] = gi0 + px >= a.xmin && gi0 + px < a.hi[2];
    const bool rowok = gj0 < a.hi[1];
    const double sxo[2] = {sx(cx + 2), sx(cx + 3)}, syo = sy(cy + 2);  // str at the own points

    // pending outputs j = k-2 .. k+2 (slot j - k + 2), per component and point
    double acc[5][3][2];
#pragma unroll
    for (int s = 0; s < 5; s++)
#pragma unroll
        for (int c = 0; c < 3; c++) acc[s][c][0] = acc[s][c][1] = 0.0;

    for (int k = kb - 2; k <= ke + 1; k++) {
        const bool main = k >= kb && k < ke;
        const int j_out = k - 2;  // the output completed by this step
        const bool store = j_out >= kb && j_out < ke && rowok;
        // ---- keep the ring PF planes ahead of the newest plane this step reads ----
        const int need = min(k + 2, plast);
        while (pnext <= min(need + PF, plast)) {
            issue(pnext++);
            if constexpr (!USE_TMA) cp_async_commit();
        }
        // uacc of output k-2 (inout, read at offset 0): loads issued now, consumed
        // at the end of the step, so their DRAM latency hides behind the step
        double2 io[3];
        if (store) {
            const int64_t off = ((zbase + j_out) * a.ny + gj0) * a.nx + gi0;
#pragma unroll
            for (int c = 0; c < 3; c++) {
                const double *src = a.io[c] + off;
                if (okx[0] && okx[1] && ((reinterpret_cast<uintptr_t>(src) & 15) == 0)) {
                    io[c] = __ldcs(reinterpret_cast<const double2 *>(src));
                } else {
                    io[c].x = okx[0] ? __ldcs(src) : 0.0;
                    io[c].y = okx[1] ? __ldcs(src + 1) : 0.0;
                }
            }
        }
        if constexpr (USE_TMA) {
            for (; waited < need; waited++) mbar_wait(&full[slot_of(waited + 1)], (unsigned(waited + 1 - p0) / NS) & 1);
        } else {
            cp_async_wait<0>();
            __syncthreads();
        }
        double szv[5];  // strz at planes k-2..k+2 (read before plane k-2's slot is released)
#pragma unroll
        for (int d = 0; d < 5; d++) szv[d] = szs[slot_of(min(max(k - 2 + d, p0), plast))];

        const double *S[5];
#pragma unroll
        for (int d = 0; d < 5; d++) S[d] = ring + slot_of(min(max(k - 2 + d, p0), plast)) * SLOT;
        auto at = [&](int arr, int dz, int br, int bc) { return S[dz + 2] + arr * PAL + br * PX + bc; };
        auto pair = [&](int arr, int dz, int br, int bc) { return lds2(at(arr, dz, br, bc)); };
        auto row6 = [&](int arr, int dz, int br, int bc, double (&v)[6]) {
            const double *q = at(arr, dz, br, bc);
            const double2 A = lds2(q), B = lds2(q + 2), C = lds2(q + 4);
            v[0] = A.x, v[1] = A.y, v[2] = B.x, v[3] = B.y, v[4] = C.x, v[5] = C.y;
        };
        const int R0 = cy + 2, C0 = cx + 2;  // own pair in box coordinates
        double *XF = fld + (FB == 2 ? (k & 1) * G::FIELDS : 0);  // P4, P5, P8
        double *YF = XF + 3 * XFN;                               // P1, P2, P9
        double *F7 = YF + 3 * YFN;                               // P7 (box layout)

        // ============ phase A: own-pair fields, second derivatives, retimed z ============
        double Q[3][2];      // retimed z fields of plane k: str_x P3, str_y P6, str_x P2 + str_y P4
        double X4[2], X5[2], X7[2], X8[2];  // own values of the x-outer fields (phase B windows)
        double sd[3][2] = {{0.0, 0.0}, {0.0, 0.0}, {0.0, 0.0}};
        double yv1[2], yv9[2], yv7[2], yv2[2];  // own values stored for y-outer
        {
            // x: row windows of plane k
            double u0w[6], u1w[6], u2w[6];
            row6(U0, 0, R0, cx, u0w);
            row6(U1, 0, R0, cx, u1w);
            row6(U2, 0, R0, cx, u2w);
            const double2 mo = pair(MU, 0, R0, C0), lo = pair(LA, 0, R0, C0);
            const double m0[2] = {mo.x, mo.y}, l0[2] = {lo.x, lo.y};
            double D0x[2], D1x[2], D2x[2];
#pragma unroll
            for (int px = 0; px < 2; px++) {
                D0x[px] = d4(u0w[px], u0w[px + 1], u0w[px + 3], u0w[px + 4]);
                D1x[px] = d4(u1w[px], u1w[px + 1], u1w[px + 3], u1w[px + 4]);
                D2x[px] = d4(u2w[px], u2w[px + 1], u2w[px + 3], u2w[px + 4]);
            }
            // y: tap rows R0-2, R0-1, R0+1, R0+2 of the own columns
            double D0y[2], D1y[2], D2y[2];
            {
                const double2 a2 = pair(U0, 0, R0 - 2, C0), a1_ = pair(U0, 0, R0 - 1, C0), b1 = pair(U0, 0, R0 + 1, C0),
                              b2 = pair(U0, 0, R0 + 2, C0);
                D0y[0] = d4(a2.x, a1_.x, b1.x, b2.x), D0y[1] = d4(a2.y, a1_.y, b1.y, b2.y);
                const double2 c2 = pair(U1, 0, R0 - 2, C0), c1 = pair(U1, 0, R0 - 1, C0), e1 = pair(U1, 0, R0 + 1, C0),
                              e2 = pair(U1, 0, R0 + 2, C0);
                D1y[0] = d4(c2.x, c1.x, e1.x, e2.x), D1y[1] = d4(c2.y, c1.y, e1.y, e2.y);
                const double2 f2 = pair(U2, 0, R0 - 2, C0), f1 = pair(U2, 0, R0 - 1, C0), g1 = pair(U2, 0, R0 + 1, C0),
                              g2 = pair(U2, 0, R0 + 2, C0);
                D2y[0] = d4(f2.x, f1.x, g1.x, g2.x), D2y[1] = d4(f2.y, f1.y, g1.y, g2.y);
                if (main) {  // y second derivatives (the u rows are in registers now)
                    const double2 q0[5] = {a2, a1_, pair(U0, 0, R0, C0), b1, b2};
                    const double2 q1[5] = {c2, c1, pair(U1, 0, R0, C0), e1, e2};
                    const double2 q2[5] = {f2, f1, pair(U2, 0, R0, C0), g1, g2};
                    double2 mr[5], lr[5];
#pragma unroll
                    for (int q = 0; q < 5; q++) mr[q] = pair(MU, 0, R0 - 2 + q, C0), lr[q] = pair(LA, 0, R0 - 2 + q, C0);
#pragma unroll
                    for (int px = 0; px < 2; px++) {
                        auto X = [&](const double2 &v) { return px ? v.y : v.x; };
                        double ms[5], ls[5];
#pragma unroll
                        for (int q = 0; q < 5; q++) ms[q] = X(mr[q]) * sy(R0 - 2 + q), ls[q] = X(lr[q]) * sy(R0 - 2 + q);
                        const Coef4 M(ms[0], ms[1], ms[2], ms[3], ms[4], tf);
                        const Coef4 L(ls[0], ls[1], ls[2], ls[3], ls[4], tf);
                        const Coef4 K = k2ml(M, L);
                        sd[0][px] = fma(syo, ksum(M, X(q0[0]), X(q0[1]), X(q0[2]), X(q0[3]), X(q0[4])), sd[0][px]);
                        sd[1][px] = fma(syo, ksum(K, X(q1[0]), X(q1[1]), X(q1[2]), X(q1[3]), X(q1[4])), sd[1][px]);
                        sd[2][px] = fma(syo, ksum(M, X(q2[0]), X(q2[1]), X(q2[2]), X(q2[3]), X(q2[4])), sd[2][px]);
                    }
                }
            }
            // retimed z fields and the own x-outer / y-outer field values
#pragma unroll
            for (int px = 0; px < 2; px++) {
                const double P2 = l0[px] * D0x[px], P3 = m0[px] * D2x[px], P4 = l0[px] * D1y[px], P6 = m0[px] * D2y[px];
                Q[0][px] = sxo[px] * P3;
                Q[1][px] = syo * P6;
                Q[2][px] = fma(sxo[px], P2, syo * P4);
                X4[px] = P4;
                X5[px] = m0[px] * D0y[px];
                yv1[px] = m0[px] * D1x[px];  // P1
                yv2[px] = P2;
            }
            if (main) {
                // x second derivatives (mu, la windows; u windows above)
                double mw[6], lw[6];
                row6(MU, 0, R0, cx, mw);
                row6(LA, 0, R0, cx, lw);
                double ms[6], ls[6];
#pragma unroll
                for (int c = 0; c < 6; c++) ms[c] = mw[c] * sx(cx + c), ls[c] = lw[c] * sx(cx + c);
#pragma unroll
                for (int px = 0; px < 2; px++) {
                    const int c = px + 2;
                    const Coef4 M(ms[c - 2], ms[c - 1], ms[c], ms[c + 1], ms[c + 2], tf);
                    const Coef4 L(ls[c - 2], ls[c - 1], ls[c], ls[c + 1], ls[c + 2], tf);
                    const Coef4 K = k2ml(M, L);
                    sd[0][px] = fma(sxo[px], ksum(K, u0w[c - 2], u0w[c - 1], u0w[c], u0w[c + 1], u0w[c + 2]), sd[0][px]);
                    sd[1][px] = fma(sxo[px], ksum(M, u1w[c - 2], u1w[c - 1], u1w[c], u1w[c + 1], u1w[c + 2]), sd[1][px]);
                    sd[2][px] = fma(sxo[px], ksum(M, u2w[c - 2], u2w[c - 1], u2w[c], u2w[c + 1], u2w[c + 2]), sd[2][px]);
                }
                // z: inner fields P7, P8, P9 and the z second derivatives
                double2 z0[5], z1[5], z2[5], zm[5], zl[5];
#pragma unroll
                for (int d = 0; d < 5; d++) {
                    z0[d] = pair(U0, d - 2, R0, C0), z1[d] = pair(U1, d - 2, R0, C0), z2[d] = pair(U2, d - 2, R0, C0);
                    zm[d] = pair(MU, d - 2, R0, C0), zl[d] = pair(LA, d - 2, R0, C0);
                }
                const double(&sz)[5] = szv;
#pragma unroll
                for (int px = 0; px < 2; px++) {
                    auto X = [&](const double2 &v) { return px ? v.y : v.x; };
                    X7[px] = l0[px] * d4(X(z2[0]), X(z2[1]), X(z2[3]), X(z2[4]));
                    X8[px] = m0[px] * d4(X(z0[0]), X(z0[1]), X(z0[3]), X(z0[4]));
                    yv9[px] = m0[px] * d4(X(z1[0]), X(z1[1]), X(z1[3]), X(z1[4]));
                    yv7[px] = X7[px];
                    double ms[5], ls[5];
#pragma unroll
                    for (int q = 0; q < 5; q++) ms[q] = X(zm[q]) * sz[q], ls[q] = X(zl[q]) * sz[q];
                    const Coef4 M(ms[0], ms[1], ms[2], ms[3], ms[4], tf);
                    const Coef4 L(ls[0], ls[1], ls[2], ls[3], ls[4], tf);
                    const Coef4 K = k2ml(M, L);
                    sd[0][px] = fma(sz[2], ksum(M, X(z0[0]), X(z0[1]), X(z0[2]), X(z0[3]), X(z0[4])), sd[0][px]);
                    sd[1][px] = fma(sz[2], ksum(M, X(z1[0]), X(z1[1]), X(z1[2]), X(z1[3]), X(z1[4])), sd[1][px]);
                    sd[2][px] = fma(sz[2], ksum(K, X(z2[0]), X(z2[1]), X(z2[2]), X(z2[3]), X(z2[4])), sd[2][px]);
                }
            }
        }
        // halo pair fields of plane k (main steps): x-halo (P4 P5 P8 P7), y-halo (P1 P2 P9 P7)
        double h[4][2];
        int hkind = 0, hb_r = 0, hb_c = 0;  // 1 = x-halo, 2 = y-halo; box row / col of the pair
        if (main && t < G::NHALO) {
            const int task = t;
            if (task < G::NXH) {
                hkind = 1;
                hb_r = task / 2 + 2;  // lanes alternate left / right halo pair: conflict-free LDS.128
                hb_c = (task & 1) ? TX + 2 : 0;
                const double2 mo = pair(MU, 0, hb_r, hb_c), lo = pair(LA, 0, hb_r, hb_c);
                const double2 a2 = pair(U1, 0, hb_r - 2, hb_c), a1_ = pair(U1, 0, hb_r - 1, hb_c),
                              b1 = pair(U1, 0, hb_r + 1, hb_c), b2 = pair(U1, 0, hb_r + 2, hb_c);
                const double2 c2 = pair(U0, 0, hb_r - 2, hb_c), c1 = pair(U0, 0, hb_r - 1, hb_c),
                              e1 = pair(U0, 0, hb_r + 1, hb_c), e2 = pair(U0, 0, hb_r + 2, hb_c);
                const double2 f2 = pair(U0, -2, hb_r, hb_c), f1 = pair(U0, -1, hb_r, hb_c),
                              g1 = pair(U0, 1, hb_r, hb_c), g2 = pair(U0, 2, hb_r, hb_c);
                const double2 v2 = pair(U2, -2, hb_r, hb_c), v1 = pair(U2, -1, hb_r, hb_c),
                              w1 = pair(U2, 1, hb_r, hb_c), w2 = pair(U2, 2, hb_r, hb_c);
                h[0][0] = lo.x * d4(a2.x, a1_.x, b1.x, b2.x), h[0][1] = lo.y * d4(a2.y, a1_.y, b1.y, b2.y);  // P4
                h[1][0] = mo.x * d4(c2.x, c1.x, e1.x, e2.x), h[1][1] = mo.y * d4(c2.y, c1.y, e1.y, e2.y);    // P5
                h[2][0] = mo.x * d4(f2.x, f1.x, g1.x, g2.x), h[2][1] = mo.y * d4(f2.y, f1.y, g1.y, g2.y);    // P8
                h[3][0] = lo.x * d4(v2.x, v1.x, w1.x, w2.x), h[3][1] = lo.y * d4(v2.y, v1.y, w1.y, w2.y);    // P7
            } else if (task < G::NHALO) {
                hkind = 2;
                const int yt = task - G::NXH, rs = yt / G::NTX, pxi = yt % G::NTX;
                hb_r = rs < 2 ? rs : TY + rs;  // box rows 0, 1, TY+2, TY+3
                hb_c = 2 * pxi + 2;
                double w1[6], w0[6];
                row6(U1, 0, hb_r, hb_c - 2, w1);
                row6(U0, 0, hb_r, hb_c - 2, w0);
                const double2 mo = pair(MU, 0, hb_r, hb_c), lo = pair(LA, 0, hb_r, hb_c);
                const double2 f2 = pair(U1, -2, hb_r, hb_c), f1 = pair(U1, -1, hb_r, hb_c),
                              g1 = pair(U1, 1, hb_r, hb_c), g2 = pair(U1, 2, hb_r, hb_c);
                const double2 v2 = pair(U2, -2, hb_r, hb_c), v1 = pair(U2, -1, hb_r, hb_c),
                              ww1 = pair(U2, 1, hb_r, hb_c), ww2 = pair(U2, 2, hb_r, hb_c);
#pragma unroll
                for (int px = 0; px < 2; px++) {
                    h[0][px] = (px ? mo.y : mo.x) * d4(w1[px], w1[px + 1], w1[px + 3], w1[px + 4]);  // P1
                    h[1][px] = (px ? lo.y : lo.x) * d4(w0[px], w0[px + 1], w0[px + 3], w0[px + 4]);  // P2
                }
                h[2][0] = mo.x * d4(f2.x, f1.x, g1.x, g2.x), h[2][1] = mo.y * d4(f2.y, f1.y, g1.y, g2.y);        // P9
                h[3][0] = lo.x * d4(v2.x, v1.x, ww1.x, ww2.x), h[3][1] = lo.y * d4(v2.y, v1.y, ww1.y, ww2.y);  // P7
            }
        }
        // the ring slot of plane k-2 is no longer read (phase B reads the field planes only)
        if constexpr (USE_TMA) {
            if (k - 2 >= p0) {
                __syncwarp();
                if (lane == 0)
                    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&empty[slot_of(k - 2)]))
                                 : "memory");
            }
        }

        // ---- retimed z contributions of plane k to outputs k-2, k-1, k+1, k+2 ----
        {
            // D_z[g](j) = sum_d w4(d) g(j + d): g(k) enters output j = k-2+s with w4(2-s)
            const double w[5] = {-1.0, 8.0, 0.0, -8.0, 1.0};
#pragma unroll
            for (int s = 0; s < 5; s++) {
                if (s == 2) continue;
                const int j = k - 2 + s;
                if (j < kb || j >= ke) continue;
                const double f = i144 * w[s] * szv[s];
#pragma unroll
                for (int c = 0; c < 3; c++)
#pragma unroll
                    for (int px = 0; px < 2; px++) acc[s][c][px] = fma(f, Q[c][px], acc[s][c][px]);
            }
        }

        if (main) {
            if constexpr (FB == 1) __syncthreads();  // (2) every warp finished phase B of the previous plane
            // store the own fields and the halo fields of plane k
            *reinterpret_cast<double2 *>(XF + 0 * XFN + cy * XFW + C0) = make_double2(X4[0], X4[1]);
            *reinterpret_cast<double2 *>(XF + 1 * XFN + cy * XFW + C0) = make_double2(X5[0], X5[1]);
            *reinterpret_cast<double2 *>(XF + 2 * XFN + cy * XFW + C0) = make_double2(X8[0], X8[1]);
            *reinterpret_cast<double2 *>(YF + 0 * YFN + R0 * YFW + cx) = make_double2(yv1[0], yv1[1]);
            *reinterpret_cast<double2 *>(YF + 1 * YFN + R0 * YFW + cx) = make_double2(yv2[0], yv2[1]);
            *reinterpret_cast<double2 *>(YF + 2 * YFN + R0 * YFW + cx) = make_double2(yv9[0], yv9[1]);
            *reinterpret_cast<double2 *>(F7 + R0 * PX + C0) = make_double2(yv7[0], yv7[1]);
            if (hkind == 1) {
                const int yr = hb_r - 2;
                *reinterpret_cast<double2 *>(XF + 0 * XFN + yr * XFW + hb_c) = make_double2(h[0][0], h[0][1]);
                *reinterpret_cast<double2 *>(XF + 1 * XFN + yr * XFW + hb_c) = make_double2(h[1][0], h[1][1]);
                *reinterpret_cast<double2 *>(XF + 2 * XFN + yr * XFW + hb_c) = make_double2(h[2][0], h[2][1]);
                *reinterpret_cast<double2 *>(F7 + hb_r * PX + hb_c) = make_double2(h[3][0], h[3][1]);
            } else if (hkind == 2) {
                const int xc = hb_c - 2;
                *reinterpret_cast<double2 *>(YF + 0 * YFN + hb_r * YFW + xc) = make_double2(h[0][0], h[0][1]);
                *reinterpret_cast<double2 *>(YF + 1 * YFN + hb_r * YFW + xc) = make_double2(h[1][0], h[1][1]);
                *reinterpret_cast<double2 *>(YF + 2 * YFN + hb_r * YFW + xc) = make_double2(h[2][0], h[2][1]);
                *reinterpret_cast<double2 *>(F7 + hb_r * PX + hb_c) = make_double2(h[3][0], h[3][1]);
            }
            __syncthreads();  // (1) the field planes of plane k are complete
            // every warp released plane k-2's slot before the barrier: refill it
            // now (plane k+3+PF), a full phase B + phase A ahead of its use
            while (pnext <= min(k + 3 + PF, plast)) {
                issue(pnext++);
                if constexpr (!USE_TMA) cp_async_commit();
            }

            // ============ phase B: outer x / y differences of the field planes ============
            auto xwin = [&](const double *base, const double (&own)[2], double (&o)[2]) {
                const double2 L = lds2(base + cx), Rr = lds2(base + cx + 4);
                o[0] = d4(L.x, L.y, own[1], Rr.x);
                o[1] = d4(L.y, own[0], Rr.x, Rr.y);
            };
            auto ycol = [&](const double *base, int stride, double (&o)[2]) {  // rows R0-2..R0+2 of a field
                const double2 r2 = lds2(base + (R0 - 2) * stride), r1 = lds2(base + (R0 - 1) * stride),
                              s1 = lds2(base + (R0 + 1) * stride), s2 = lds2(base + (R0 + 2) * stride);
                o[0] = d4(r2.x, r1.x, s1.x, s2.x);
                o[1] = d4(r2.y, r1.y, s1.y, s2.y);
            };
            double dx4[2], dx5[2], dx7[2], dx8[2], dy1[2], dy2[2], dy7[2], dy9[2];
            xwin(XF + 0 * XFN + cy * XFW, X4, dx4);
            xwin(XF + 1 * XFN + cy * XFW, X5, dx5);
            xwin(XF + 2 * XFN + cy * XFW, X8, dx8);
            xwin(F7 + R0 * PX, X7, dx7);
            ycol(YF + 0 * YFN + cx, YFW, dy1);
            ycol(YF + 1 * YFN + cx, YFW, dy2);
            ycol(YF + 2 * YFN + cx, YFW, dy9);
            ycol(F7 + C0, PX, dy7);
            const double szk = szv[2];
#pragma unroll
            for (int px = 0; px < 2; px++) {
                const double fxy = sxo[px] * syo, fxz = sxo[px] * szk, fyz = syo * szk;
                const double mxx = fma(fxy, dx4[px] + dy1[px], fxz * dx7[px]);
                const double mxy = fma(fxy, dy2[px] + dx5[px], fyz * dy7[px]);
                const double mxz = fma(fxz, dx8[px], fyz * dy9[px]);
                acc[2][0][px] += fma(i6, sd[0][px], i144 * mxx);
                acc[2][1][px] += fma(i6, sd[1][px], i144 * mxy);
                acc[2][2][px] += fma(i6, sd[2][px], i144 * mxz);
            }
        }

        // ---- output k-2 is complete: uacc = a1 uacc + cof r ----
        {
            if (store) {
                const int64_t off = ((zbase + j_out) * a.ny + gj0) * a.nx + gi0;
#pragma unroll
                for (int c = 0; c < 3; c++) {
                    double *dst = a.out[c] + off;
                    const double o0 = fma(a1, io[c].x, cof * acc[0][c][0]), o1 = fma(a1, io[c].y, cof * acc[0][c][1]);
                    if (okx[0] && okx[1] && ((reinterpret_cast<uintptr_t>(dst) & 15) == 0)) {
                        __stcs(reinterpret_cast<double2 *>(dst), make_double2(o0, o1));
                    } else {
                        if (okx[0]) __stcs(dst, o0);
                        if (okx[1]) __stcs(dst + 1, o1);
                    }
                }
            }
#pragma unroll
            for (int s = 0; s < 4; s++)
#pragma unroll
                for (int c = 0; c < 3; c++) acc[s][c][0] = acc[s + 1][c][0], acc[s][c][1] = acc[s + 1][c][1];
#pragma unroll
            for (int c = 0; c < 3; c++) acc[4][c][0] = acc[4][c][1] = 0.0;
        }
        if constexpr (!USE_TMA) __syncthreads();
    }
}

}  // namespace dev
}  // namespace sdag

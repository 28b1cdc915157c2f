// fuse2.cuh -- temporal fusion of two sweeps of the 27-point smoother (and of
// Listing 1's 7-point Jacobi, FORM 1)
// (NEXT-1: the paper's fusion for arbitrary time iterations, with
// overlapped tiling, Fig 1b).
//
// One launch maps buffer t to buffer t+2 without writing the intermediate
// sweep to HBM, halving the traffic per sweep of the iterated stencil.  Per CTA
// a GX x GY "region" of sweep-1 points is computed (the GX-2 x GY-2 output tile
// plus a 1-point halo recomputed redundantly, as in overlapped tiling), plane by
// plane with the retimed/folded box27 formulation (box27.cuh); each finished
// sweep-1 plane goes to a double-buffered shared-memory plane, from which the
// same formulation produces sweep 2 for the tile.  Input planes stream by TMA
// (full/empty mbarriers) exactly as in box27; sweep-1 output k-1 is final when
// input plane k arrives, sweep-2 output k-2 when sweep-1 plane k-1 is final.
//
// Global ring (reading R1): sweep-1 values at ring points (x, y or z on the
// global boundary) stay equal to the input, exactly as a separate sweep would
// leave them.
#pragma once

#include "box27.cuh"

namespace sdag {
namespace dev {

// ODD = false: the box starts 2 columns left of the region (ML = 2), a patch
//   starts at an even smem column and its 3-point row window [c-1, c+UX] is read
//   as UX/2 + 2 aligned pairs, two of them half used;
// ODD = true: the box starts 3 columns left (ML = 3, tile origin even, box
//   origin still 16-B aligned), a patch starts at an odd smem column, and its
//   window [c-1, c+UX] is exactly UX/2 + 1 aligned pairs -- a third fewer
//   shared-memory reads per fold for UX = 2 (the fused kernel is bound by them).
template <bool V>
struct BoolTag {
    static constexpr bool value = V;
};

template <int GX, int GY, int UY, int PF, int UX = 2, bool ODD = false>
struct Fuse2Geo {
    static constexpr int ML = ODD ? 3 : 2;       // box x margin (region - ML): 16-B alignment of the box origin
    static constexpr int NTX = GX / UX, NTY = GY / UY, THREADS = NTX * NTY, NWARPS = (THREADS + 31) / 32;
    static constexpr int PX = GX + (ODD ? 6 : 4), PY = GY + 2, PLANE = PX * PY;  // input box / S1 plane layout
    static constexpr int PLANE_AL = ((PLANE * 8 + 127) / 128) * 128 / 8;
    static constexpr int NS = 1 + PF;
    static constexpr int SMEM = (NS + 2) * PLANE_AL * 8 + 2 * NS * 8;
    static constexpr int NW = ODD ? UX + 2 : UX + 4;  // row window in smem columns (16-B aligned start)
    static constexpr int W0 = ODD ? ML - 1 : 0;       // window start relative to the patch's smem column - ML
    static_assert((UX == 2 || UX == 4) && GX % UX == 0 && GY % UY == 0, "region");
    static_assert(PX <= 256 && PY <= 256, "TMA box");
};

// UX = 2 or 4 output columns per thread: the row window of a UX-wide patch is
// UX+4 doubles read with (UX+4)/2 128-bit loads, so UX = 4 cuts the fold's
// shared-memory reads per point from 1.5 to 1 LDS.128 per row.
// FORM 0: the 27-point smoother (scalars w0..w3, nu); FORM 2: a generated
//   box-form DAG, B = w0 A + w1 faces + w2 edges + w3 corners (box27.cuh);
// FORM 1: Listing 1's 7-point Jacobi (scalars h2inv, a, b), the paper's
//   7pt-smoother of Table I / Table II, in box27's retimed FORM 1:
//   T_k = s1_k - 6 s0_k + s0_{k-1}, B[k] = a A[k] - (b h2inv)(T_k + s0_{k+1}).
template <int GX, int GY, int UY, int PF, int MINB = 1, int UX = 2, bool ODD = false, int FORM = 0,
          bool MIR = false>
__global__ void __launch_bounds__(Fuse2Geo<GX, GY, UY, PF, UX, ODD>::THREADS, MINB)
    sdag_box27x2(const __grid_constant__ SweepArgs a) {
    using G = Fuse2Geo<GX, GY, UY, PF, UX, ODD>;
    constexpr int PX = G::PX, NS = G::NS, PAL = G::PLANE_AL, ML = G::ML, NW = G::NW, W0 = G::W0;
    constexpr int TX = GX - 2, TY = GY - 2;  // output tile

    extern __shared__ __align__(128) unsigned char smem_raw[];
    double *ring = reinterpret_cast<double *>(smem_raw);
    double *s1buf = ring + NS * PAL;  // 2 sweep-1 planes, same layout as the input box
    uint64_t *full = reinterpret_cast<uint64_t *>(smem_raw + (NS + 2) * PAL * 8);
    uint64_t *empty = full + NS;

    const int tile_x = blockIdx.x, tile_y = blockIdx.y;
    const int chunk = blockIdx.z % a.nchunk;
    const int64_t prob = blockIdx.z / a.nchunk;
    const int ox = a.lo[2] + tile_x * TX, oy = a.lo[1] + tile_y * TY;  // output tile origin
    const int rx0 = ox - 1, ry0 = oy - 1;                              // region origin
    const int kb = a.lo[0] + chunk * a.zchunk;
    const int ke = min(a.hi[0], kb + a.zchunk);
    if (kb >= ke) return;
    const int p0 = kb - 2, plast = ke + 1;  // input planes streamed
    const int64_t zbase = prob * a.nz;
    const int ny = int(a.ny), nx = int(a.nx);

    const int t = threadIdx.x;
    const int lx = t % G::NTX, ly = t / G::NTX;
    const int cx = UX * lx, cy = UY * ly;  // patch origin in region coordinates

    auto issue = [&](int p) {
        const int slot = unsigned(p - p0) % NS;
        if (t == 0) {
            const int prev = p - NS;
            if (prev >= p0) mbar_wait(&empty[slot], (unsigned(prev - p0) / NS) & 1);
            mbar_expect_tx(&full[slot], uint32_t(G::PLANE * 8));
            tma_load_3d(ring + slot * PAL, &a.tmap[0], &full[slot], rx0 - ML, ry0 - 1, int(zbase + p));
        }
    };
    if (t == 0) {
        for (int s = 0; s < NS; s++) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], G::NWARPS);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    for (int p = p0; p < p0 + PF; p++)
        if (p <= plast) issue(p);

    const double w0 = a.s[0], w1 = a.s[1], w2 = a.s[2], w3 = a.s[3], nu = a.s[4];
    const double ja = a.s[1], jc = a.s[2] * a.s[0];  // FORM 1: a, c = b*h2inv

    // region point (cy+py, cx+px) -> global (ry0+cy+py, rx0+cx+px); x/y ring flags
    bool ringxy[UY][UX];
#pragma unroll
    for (int py = 0; py < UY; py++)
#pragma unroll
        for (int px = 0; px < UX; px++) {
            const int gy = ry0 + cy + py, gx = rx0 + cx + px;
            ringxy[py][px] = gy <= 0 || gy >= ny - 1 || gx <= 0 || gx >= nx - 1;
        }
    // outputs: tile points strictly inside the region and inside the interior
    const int gi = rx0 + cx;
    bool outm[UX];
#pragma unroll
    for (int px = 0; px < UX; px++)
        outm[px] = cx + px >= 1 && cx + px <= TX && gi + px >= a.xmin && gi + px < a.hi[2];
    const bool vec_ok = (a.nx % 2 == 0) && ((reinterpret_cast<uintptr_t>(a.out[0]) & 15) == 0) && (gi % 2 == 0);

    double T1[UY][UX], U1[UY][UX], A1[UY][UX];  // sweep-1 retimed state
    double T2[UY][UX], U2[UY][UX], A2[UY][UX];  // sweep-2 retimed state
#pragma unroll
    for (int py = 0; py < UY; py++)
#pragma unroll
        for (int px = 0; px < UX; px++) T1[py][px] = U1[py][px] = A1[py][px] = T2[py][px] = U2[py][px] = A2[py][px] = 0.0;

    // in-plane partial sums -> (c, u) of one plane at the patch points
    auto fold = [&](const double *pl, double (&cc)[UY][UX], double (&uu)[UY][UX], double (&s0v)[UY][UX]) {
        double w[UY + 2][NW];
#pragma unroll
        for (int r = 0; r < UY + 2; r++) {
            const double *rp = pl + (cy + r) * PX + cx + W0;
#pragma unroll
            for (int c = 0; c < NW / 2; c++) {
                const double2 v = *reinterpret_cast<const double2 *>(rp + 2 * c);
                w[r][2 * c] = v.x;
                w[r][2 * c + 1] = v.y;
            }
        }
#pragma unroll
        for (int py = 0; py < UY; py++)
#pragma unroll
            for (int px = 0; px < UX; px++) {
                const int c = ML - W0 + px;  // the patch point's column in the window
                const double s0 = w[py + 1][c];
                const double s1 = (w[py + 1][c - 1] + w[py + 1][c + 1]) + (w[py][c] + w[py + 2][c]);
                if constexpr (FORM == 0 || FORM == 2) {
                    const double s2 = (w[py][c - 1] + w[py][c + 1]) + (w[py + 2][c - 1] + w[py + 2][c + 1]);
                    cc[py][px] = fma(w2, s2, fma(w1, s1, w0 * s0));
                    uu[py][px] = fma(w3, s2, fma(w2, s1, w1 * s0));
                } else {
                    cc[py][px] = s1;  // in-plane face sum
                    uu[py][px] = 0.0;
                }
                s0v[py][px] = s0;
            }
    };

    // (measured, r02, ms per sweep at 1024^3: unrolling this loop by 2 so the
    // retimed state changes roles instead of moving, 2.39 -> 2.46; skipping the
    // per-point ring select in tiles away from the global ring, -> 2.48)
    // the plane loop, compiled twice: CTAs whose region touches the global x/y
    // ring keep the per-point ring select of sweep 1, all others have none
    // (ncu r02: the select and its recomputed predicates were ~4 instructions
    // per point-sweep of 45)
    auto run = [&](auto ring_tag) {
        constexpr bool RING = decltype(ring_tag)::value;
#pragma unroll 2
        for (int p = p0; p <= plast; p++) {
            if (p + PF <= plast) issue(p + PF);
            mbar_wait(&full[unsigned(p - p0) % NS], (unsigned(p - p0) / NS) & 1);
            // ---- sweep 1: input plane p completes sweep-1 plane j = p-1 on the region ----
            double cc[UY][UX], uu[UY][UX], s0[UY][UX];
            fold(ring + (unsigned(p - p0) % NS) * PAL, cc, uu, s0);
            __syncwarp();
            if ((t & 31) == 0)
                asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&empty[unsigned(p - p0) % NS]))
                             : "memory");
            const int j = p - 1;
            const bool zring = j < a.zr_lo || j >= a.zr_hi;
            double *s1 = s1buf + (j & 1) * PAL;
            double v[UY][UX], keep[UY][UX];
    #pragma unroll
            for (int py = 0; py < UY; py++)
    #pragma unroll
                for (int px = 0; px < UX; px++) {
                    keep[py][px] = A1[py][px];  // the input value: what a ring point keeps
                    if constexpr (FORM == 0 || FORM == 2) {
                        v[py][px] = FORM == 0 ? fma(nu, T1[py][px] + uu[py][px], A1[py][px]) : T1[py][px] + uu[py][px];
                        T1[py][px] = U1[py][px] + cc[py][px];
                        U1[py][px] = uu[py][px];
                    } else {
                        v[py][px] = ja * A1[py][px] - jc * (T1[py][px] + s0[py][px]);
                        T1[py][px] = fma(-6.0, s0[py][px], cc[py][px] + A1[py][px]);
                    }
                    if constexpr (RING)
                        if (ringxy[py][px]) v[py][px] = keep[py][px];  // x/y ring: not updated by sweep 1
                    A1[py][px] = s0[py][px];
                }
            // the sweep-1 plane into shared memory; a global z-ring plane keeps its
            // input (a CTA-uniform branch between two store sequences, no per-point select)
            auto store = [&](const double(&w)[UY][UX]) {
    #pragma unroll
                for (int py = 0; py < UY; py++)
    #pragma unroll
                    for (int px = 0; px < UX; px += 2) {
                        double *q = s1 + (cy + py + 1) * PX + cx + ML + px;
                        if constexpr (ODD) {
                            // two 8-byte stores at a 16-byte lane stride are 2-way bank
                            // conflicted (ncu r02: 50 % excess wavefronts on these four
                            // STS.64, 15 % of the kernel's).  Measured and reverted (r02):
                            // aligned STS.128 pairs completed by a shuffle of the next
                            // lane's value cut the conflicts 137 M -> 46 M per launch but
                            // ran 4.51 -> 5.00 ms per launch: the store side is not the
                            // bound, the fold's dependency chains are (issue 58 %).
                            q[0] = w[py][px];
                            q[1] = w[py][px + 1];
                        } else {
                            *reinterpret_cast<double2 *>(q) = make_double2(w[py][px], w[py][px + 1]);
                        }
                    }
            };
            if (zring)
                store(keep);
            else
                store(v);
            // (measured, r02: handing the plane from row block to row block with
            // per-warp counters -- lane-0 spin on ld.acquire, st.release -- instead
            // of this barrier ran 2.2 -> 4.1 ms per sweep; running sweep 2 one plane
            // behind through four slots and per-slot mbarriers (hardware-suspended
            // waits, no CTA barrier) 2.22 -> 2.45)
            __syncthreads();  // sweep-1 plane j is complete in shared memory
            if (j < kb - 1) continue;  // sweep-2 state starts at sweep-1 plane kb-1
            // ---- sweep 2: sweep-1 plane j completes output plane k = j-1 on the tile ----
            fold(s1, cc, uu, s0);
            const int k = j - 1;
            double *o = a.out[0] + ((zbase + k) * a.ny + (ry0 + cy)) * a.nx + gi;
            const bool mp = MIR && mirror_plane(a, k);
    #pragma unroll
            for (int py = 0; py < UY; py++) {
                double res[UX];
    #pragma unroll
                for (int px = 0; px < UX; px++) {
                    if constexpr (FORM == 0 || FORM == 2) {
                        res[px] = FORM == 0 ? fma(nu, T2[py][px] + uu[py][px], A2[py][px]) : T2[py][px] + uu[py][px];
                        T2[py][px] = U2[py][px] + cc[py][px];
                        U2[py][px] = uu[py][px];
                    } else {
                        res[px] = ja * A2[py][px] - jc * (T2[py][px] + s0[py][px]);
                        T2[py][px] = fma(-6.0, s0[py][px], cc[py][px] + A2[py][px]);
                    }
                    A2[py][px] = s0[py][px];
                }
                const int ry = cy + py, gj = ry0 + ry;
                if (k >= kb && ry >= 1 && ry <= TY && gj < a.hi[1]) {
    #pragma unroll
                    for (int px = 0; px < UX; px += 2) {
                        if (vec_ok && outm[px] && outm[px + 1]) {
                            __stcs(reinterpret_cast<double2 *>(o + px), make_double2(res[px], res[px + 1]));
                            if constexpr (MIR) if (mp) mirror2(a, k, o + px, res[px], res[px + 1]);
                        } else {
                            if (outm[px]) __stcs(o + px, res[px]);
                            if (outm[px + 1]) __stcs(o + px + 1, res[px + 1]);
                            if (MIR && mp && outm[px]) mirror1(a, k, o + px, res[px]);
                            if (MIR && mp && outm[px + 1]) mirror1(a, k, o + px + 1, res[px + 1]);
                        }
                    }
                }
                o += a.nx;
            }
        }
    };
    const bool tile_ring = ry0 <= 0 || ry0 + GY - 1 >= ny - 1 || rx0 <= 0 || rx0 + GX - 1 >= nx - 1;
    if (tile_ring)
        run(BoolTag<true>{});
    else
        run(BoolTag<false>{});
}

}  // namespace dev
}  // namespace sdag

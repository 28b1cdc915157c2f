// fuse2.cuh -- temporal fusion of two sweeps of the 27-point smoother
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

template <int GX, int GY, int UY, int PF>
struct Fuse2Geo {
    static constexpr int ML = 2;                 // box x margin (region - 2): 16-B alignment
    static constexpr int NTX = GX / 2, NTY = GY / UY, THREADS = NTX * NTY, NWARPS = (THREADS + 31) / 32;
    static constexpr int PX = GX + 4, PY = GY + 2, PLANE = PX * PY;  // input box / S1 plane layout
    static constexpr int PLANE_AL = ((PLANE * 8 + 127) / 128) * 128 / 8;
    static constexpr int NS = 1 + PF;
    static constexpr int SMEM = (NS + 2) * PLANE_AL * 8 + 2 * NS * 8;
    static_assert(GX % 2 == 0 && GY % UY == 0, "region");
    static_assert(PX <= 256 && PY <= 256, "TMA box");
};

template <int GX, int GY, int UY, int PF, int MINB = 1>
__global__ void __launch_bounds__(Fuse2Geo<GX, GY, UY, PF>::THREADS, MINB)
    sdag_box27x2(const __grid_constant__ SweepArgs a) {
    using G = Fuse2Geo<GX, GY, UY, PF>;
    constexpr int PX = G::PX, NS = G::NS, PAL = G::PLANE_AL, ML = G::ML;
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
    const int nz = int(a.nz), ny = int(a.ny), nx = int(a.nx);

    const int t = threadIdx.x;
    const int lx = t % G::NTX, ly = t / G::NTX;
    const int cx = 2 * lx, cy = UY * ly;  // patch origin in region coordinates

    auto issue = [&](int p) {
        const int slot = (p - p0) % NS;
        if (t == 0) {
            const int prev = p - NS;
            if (prev >= p0) mbar_wait(&empty[slot], ((prev - p0) / NS) & 1);
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

    // region point (cy+py, cx+px) -> global (ry0+cy+py, rx0+cx+px); x/y ring flags
    bool ringxy[UY][2];
#pragma unroll
    for (int py = 0; py < UY; py++)
#pragma unroll
        for (int px = 0; px < 2; px++) {
            const int gy = ry0 + cy + py, gx = rx0 + cx + px;
            ringxy[py][px] = gy <= 0 || gy >= ny - 1 || gx <= 0 || gx >= nx - 1;
        }
    // outputs: tile points strictly inside the region and inside the interior
    const int gi = rx0 + cx;
    const bool out0 = cx >= 1 && cx <= TX && gi >= a.xmin && gi < a.hi[2];
    const bool out1 = cx + 1 >= 1 && cx + 1 <= TX && gi + 1 >= a.xmin && gi + 1 < a.hi[2];

    double T1[UY][2], U1[UY][2], A1[UY][2];  // sweep-1 retimed state
    double T2[UY][2], U2[UY][2], A2[UY][2];  // sweep-2 retimed state
#pragma unroll
    for (int py = 0; py < UY; py++)
#pragma unroll
        for (int px = 0; px < 2; px++) T1[py][px] = U1[py][px] = A1[py][px] = T2[py][px] = U2[py][px] = A2[py][px] = 0.0;

    // in-plane partial sums -> (c, u) of one plane at the patch points
    auto fold = [&](const double *pl, double (&cc)[UY][2], double (&uu)[UY][2], double (&s0v)[UY][2]) {
        double w[UY + 2][6];
#pragma unroll
        for (int r = 0; r < UY + 2; r++) {
            const double *rp = pl + (cy + r) * PX + cx;
#pragma unroll
            for (int c = 0; c < 3; c++) {
                const double2 v = *reinterpret_cast<const double2 *>(rp + 2 * c);
                w[r][2 * c] = v.x;
                w[r][2 * c + 1] = v.y;
            }
        }
#pragma unroll
        for (int py = 0; py < UY; py++)
#pragma unroll
            for (int px = 0; px < 2; px++) {
                const int c = ML + px;
                const double s0 = w[py + 1][c];
                const double s1 = (w[py + 1][c - 1] + w[py + 1][c + 1]) + (w[py][c] + w[py + 2][c]);
                const double s2 = (w[py][c - 1] + w[py][c + 1]) + (w[py + 2][c - 1] + w[py + 2][c + 1]);
                cc[py][px] = fma(w2, s2, fma(w1, s1, w0 * s0));
                uu[py][px] = fma(w3, s2, fma(w2, s1, w1 * s0));
                s0v[py][px] = s0;
            }
    };

    for (int p = p0; p <= plast; p++) {
        if (p + PF <= plast) issue(p + PF);
        mbar_wait(&full[(p - p0) % NS], ((p - p0) / NS) & 1);
        // ---- sweep 1: input plane p completes sweep-1 plane j = p-1 on the region ----
        double cc[UY][2], uu[UY][2], s0[UY][2];
        fold(ring + ((p - p0) % NS) * PAL, cc, uu, s0);
        __syncwarp();
        if ((t & 31) == 0)
            asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&empty[(p - p0) % NS])) : "memory");
        const int j = p - 1;
        const bool zring = j <= 0 || j >= nz - 1;
        double *s1 = s1buf + (j & 1) * PAL;
#pragma unroll
        for (int py = 0; py < UY; py++) {
            double v[2];
#pragma unroll
            for (int px = 0; px < 2; px++) {
                v[px] = fma(nu, T1[py][px] + uu[py][px], A1[py][px]);
                if (zring || ringxy[py][px]) v[px] = A1[py][px];  // ring: not updated by sweep 1
                T1[py][px] = U1[py][px] + cc[py][px];
                U1[py][px] = uu[py][px];
                A1[py][px] = s0[py][px];
            }
            *reinterpret_cast<double2 *>(s1 + (cy + py + 1) * PX + cx + ML) = make_double2(v[0], v[1]);
        }
        __syncthreads();  // sweep-1 plane j is complete in shared memory
        if (j < kb - 1) continue;  // sweep-2 state starts at sweep-1 plane kb-1
        // ---- sweep 2: sweep-1 plane j completes output plane k = j-1 on the tile ----
        fold(s1, cc, uu, s0);
        const int k = j - 1;
        double *o = a.out[0] + ((zbase + k) * a.ny + (ry0 + cy)) * a.nx + gi;
#pragma unroll
        for (int py = 0; py < UY; py++) {
            double res[2];
#pragma unroll
            for (int px = 0; px < 2; px++) {
                res[px] = fma(nu, T2[py][px] + uu[py][px], A2[py][px]);
                T2[py][px] = U2[py][px] + cc[py][px];
                U2[py][px] = uu[py][px];
                A2[py][px] = s0[py][px];
            }
            const int ry = cy + py, gj = ry0 + ry;
            if (k >= kb && ry >= 1 && ry <= TY && gj < a.hi[1]) {
                if (out0) __stcs(o, res[0]);
                if (out1) __stcs(o + 1, res[1]);
            }
            o += a.nx;
        }
    }
}

}  // namespace dev
}  // namespace sdag

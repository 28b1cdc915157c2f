// box27.cuh -- sm_100a z-streaming kernel for the 27-point smoother
// (Table I 27pt-smoother; formula reading SURVEY A.3).
//
// Retiming + computation folding on B200:
// per plane j and point, form the in-plane partial sums
//     s0 = A,  s1 = 4 face neighbours,  s2 = 4 corner neighbours
// and fold them into the two quantities the 3D stencil needs,
//     c_j = w0 s0 + w1 s1 + w2 s2     (plane j as the centre plane)
//     u_j = w1 s0 + w2 s1 + w3 s2     (plane j as the plane above/below)
// so that   B[k] = A[k] + nu * (u_{k-1} + c_k + u_{k+1}).
// Each plane is read once (as it streams past), output k is finished when
// plane k+1 arrives, and the per-point state carried along z is three doubles
// (u_{k-1}+c_k, u_k, A_k) instead of a 3-plane window.  ~15 FP64 ops/point
// instead of 32; ~4.5 doubles of shared-memory reads/point (2x4 patch,
// 128-bit LDS).  Planes arrive by TMA into a ring of 1+PF slots with
// full/empty mbarriers (see star.cuh).
//
// The arithmetic is re-associated relative to the spec; parity by the scaled
// error gate (reading R13) -- and bit-exact on the integer-weight pins.
#pragma once

#include "sweep.cuh"

namespace sdag {
namespace dev {

struct Smooth27Box {
    static constexpr int R = 1, NIN = 1, NOUT = 1, NIO = 0, N1D = 0, RZ = 1, RY = 1, RX = 1, RZR = 1;
    __host__ __device__ static constexpr int axis1d(int) { return 2; }
};

template <int TX, int TY, int UY, int PF>
struct BoxGeo {
    static constexpr int R = 1, ML = 2;  // even left margin: 16-B aligned windows
    static constexpr int NTX = TX / 2, NTY = TY / UY, THREADS = NTX * NTY, NWARPS = (THREADS + 31) / 32;
    static constexpr int PX = TX + 2 * ML, PY = TY + 2 * R, PLANE = PX * PY;
    static constexpr int PLANE_AL = ((PLANE * 8 + 127) / 128) * 128 / 8;
    static constexpr int NS = 1 + PF;
    static constexpr int SMEM = NS * PLANE_AL * 8 + 2 * NS * 8;
    static_assert(TX % 2 == 0 && TY % UY == 0, "tile");
    static_assert(PX <= 256 && PY <= 256, "TMA box");
};

// FORM 0: the 27-point smoother (scalars w0..w3, nu).
// FORM 2: any linear 27-point box stencil whose weights depend only on the tap
//   class (centre, face, edge, corner): B = w0 A + w1 faces + w2 edges + w3
//   corners, w0..w3 in s[0..3] (generated DAGs in box form, jit.cu; the
//   weights are evaluated from the DAG's scalars at launch).
// FORM 1: Listing 1's 7-point Jacobi (scalars h2inv, a, b) in the same
//   retimed form: T_k = s1_k - 6 s0_k + s0_{k-1} is formed when plane k
//   streams past and B[k] = a A[k] - (b h2inv)(T_k + s0_{k+1}) when plane k+1
//   does (2 doubles of z-state per point).
template <int TX, int TY, int UY, int PF, bool USE_TMA, int FORM = 0, bool MIR = false>
__global__ void __launch_bounds__(BoxGeo<TX, TY, UY, PF>::THREADS)
    sdag_box27(const __grid_constant__ SweepArgs a) {
    using G = BoxGeo<TX, TY, UY, PF>;
    constexpr int PX = G::PX, NS = G::NS, PAL = G::PLANE_AL, ML = G::ML;

    extern __shared__ __align__(128) unsigned char smem_raw[];
    double *ring = reinterpret_cast<double *>(smem_raw);
    uint64_t *full = reinterpret_cast<uint64_t *>(smem_raw + NS * PAL * 8);
    uint64_t *empty = full + NS;

    const int tile_x = blockIdx.x, tile_y = blockIdx.y;
    const int chunk = blockIdx.z % a.nchunk;
    const int64_t prob = blockIdx.z / a.nchunk;
    const int x0 = a.lo[2] + tile_x * TX, y0 = a.lo[1] + tile_y * TY;
    const int kb = a.lo[0] + chunk * a.zchunk;
    const int ke = min(a.hi[0], kb + a.zchunk);
    if (kb >= ke) return;
    const int p0 = kb - 1, plast = ke;
    const int64_t zbase = prob * a.nz;

    const int t = threadIdx.x;
    const int lx = t % G::NTX, ly = t / G::NTX;
    const int cx = 2 * lx, cy = UY * ly;

    auto issue = [&](int p) {
        const int slot = (p - p0) % NS;
        double *dst = ring + slot * PAL;
        if constexpr (USE_TMA) {
            if (t == 0) {
                const int prev = p - NS;
                if (prev >= p0) mbar_wait(&empty[slot], ((prev - p0) / NS) & 1);
                mbar_expect_tx(&full[slot], uint32_t(G::PLANE * 8));
                tma_load_3d(dst, &a.tmap[0], &full[slot], x0 - ML, y0 - 1, int(zbase + p));
            }
        } else {
            const int64_t pl = (zbase + p) * a.ny * a.nx;
            for (int e = t; e < G::PLANE; e += G::THREADS) {
                const int yy = e / PX, xx = e % PX;
                const int gx = x0 - ML + xx, gy = y0 - 1 + yy;
                const bool ok = gx >= 0 && gx < a.nx && gy >= 0 && gy < a.ny && p >= 0 && p < a.nz;
                cp_async8(dst + e, a.in[0] + (ok ? pl + int64_t(gy) * a.nx + gx : 0), ok);
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

    const double w0 = a.s[0], w1 = a.s[1], w2 = a.s[2], w3 = a.s[3], nu = a.s[4];
    const double ja = a.s[1], jc = a.s[2] * a.s[0];  // FORM 1: a, c = b*h2inv
    const int gi = x0 + cx;
    const bool ok0 = gi >= a.xmin && gi < a.hi[2];
    const bool ok1 = gi + 1 >= a.xmin && gi + 1 < a.hi[2];
    const bool vec = ok0 && ok1 && (a.nx % 2 == 0) && ((reinterpret_cast<uintptr_t>(a.out[0]) & 15) == 0);
    const int nrows = min(UY, a.hi[1] - (y0 + cy));

    double Tprev[UY][2], Uprev[UY][2], Aprev[UY][2];
#pragma unroll
    for (int py = 0; py < UY; py++)
#pragma unroll
        for (int px = 0; px < 2; px++) Tprev[py][px] = Uprev[py][px] = Aprev[py][px] = 0.0;

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
        const double *pl = ring + ((p - p0) % NS) * PAL;
        // rows cy-1 .. cy+UY of the tile; columns [cx-1, cx+3) inside the aligned
        // smem span [cx, cx+6): w[r][1 + px + dx] is the tap (row r-1, px, dx)
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
        if constexpr (USE_TMA) {  // done with this slot
            __syncwarp();
            if ((t & 31) == 0)
                asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&empty[(p - p0) % NS]))
                             : "memory");
        }
        const int k = p - 1;  // output plane finished by this plane
        double *o = a.out[0] + ((zbase + k) * a.ny + (y0 + cy)) * a.nx + gi;
        const bool mp = MIR && mirror_plane(a, k);
#pragma unroll
        for (int py = 0; py < UY; py++) {
            double res[2];
#pragma unroll
            for (int px = 0; px < 2; px++) {
                const int c = ML + px;  // centre column in w
                const double s0 = w[py + 1][c];
                const double s1 = (w[py + 1][c - 1] + w[py + 1][c + 1]) + (w[py][c] + w[py + 2][c]);
                if constexpr (FORM == 0 || FORM == 2) {
                    const double s2 = (w[py][c - 1] + w[py][c + 1]) + (w[py + 2][c - 1] + w[py + 2][c + 1]);
                    const double cc = fma(w2, s2, fma(w1, s1, w0 * s0));
                    const double uu = fma(w3, s2, fma(w2, s1, w1 * s0));
                    if constexpr (FORM == 0)
                        res[px] = fma(nu, Tprev[py][px] + uu, Aprev[py][px]);  // B[k] = A[k] + nu(u_{k-1} + c_k + u_{k+1})
                    else
                        res[px] = Tprev[py][px] + uu;  // FORM 2: B[k] = u_{k-1} + c_k + u_{k+1}
                    Tprev[py][px] = Uprev[py][px] + cc;                   // u_{p-1} + c_p
                    Uprev[py][px] = uu;
                } else {
                    res[px] = ja * Aprev[py][px] - jc * (Tprev[py][px] + s0);      // B[k], k = p-1
                    Tprev[py][px] = fma(-6.0, s0, s1 + Aprev[py][px]);           // T_p
                }
                Aprev[py][px] = s0;
            }
            if (k >= kb && py < nrows) {
                if (vec) {
                    __stcs(reinterpret_cast<double2 *>(o), make_double2(res[0], res[1]));
                    if constexpr (MIR) if (mp) mirror2(a, k, o, res[0], res[1]);
                } else {
                    if (ok0) __stcs(o, res[0]);
                    if (ok1) __stcs(o + 1, res[1]);
                    if (MIR && mp && ok0) mirror1(a, k, o, res[0]);
                    if (MIR && mp && ok1) mirror1(a, k, o + 1, res[1]);
                }
            }
            o += a.nx;
        }
        if constexpr (!USE_TMA) __syncthreads();
    }
}

}  // namespace dev
}  // namespace sdag

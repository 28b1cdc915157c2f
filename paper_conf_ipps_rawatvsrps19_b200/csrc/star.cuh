// star.cuh -- sm_100a z-streaming kernel for axis-aligned star stencils
// (Listing 1's 7-point Jacobi, the 25-point radius-4 Laplacian).
//
// B200 design: the HBM roofline leaves ~0.7 SM
// clocks per output point, i.e. <= ~90 B of shared-memory traffic per point at
// 128 B/clk/SM, so the generic skeleton's all-taps-from-smem evaluation
// (~19 doubles/point for R=4) is shared-memory bound.  This kernel keeps
//  * the z-taps in a per-thread register queue of 2R+1 plane values
//    (serial streaming with register reuse along the streamed dimension,
//    P:611-638; the retiming idea of P:790-830 applied to the centre column),
//  * a 2-wide x patch read with 128-bit LDS (blocked unrolling):
//    each row window [x-R, x+2+R) is a few aligned double2 loads,
//  * a UY-tall y patch whose column [y-R, y+UY+R) is read once per plane,
// so each point costs ~9 doubles of smem reads for R=4 (4.5 for R=1).
// Planes arrive by TMA (cp.async.bulk.tensor.3d + mbarrier expect_tx) into a
// ring of R+1+PF slots: plane p is used first as the queue head (its centre
// values) and last, R iterations later, as the centre plane with its xy halo.
// Slots are recycled through per-slot "empty" mbarriers (one arrival per
// warp) instead of a CTA-wide barrier per plane, so warps do not wait for one
// another; only the TMA-issuing thread waits for a slot to drain.
//
// QMODE 0: the queue is shifted with register moves; with UNR > 1 the plane
//   loop is unrolled UNR times over a queue of NQ + UNR - 1 slots, so the
//   (NQ - 1)-slot shift happens once per UNR planes (UNR x the code, 1/UNR of
//   the moves);
// QMODE 1: the plane loop is dispatched to NQ phase copies so the queue
// rotates by compile-time indexing (no moves, NQ x the code);
// QMODE 4 ("late head", TMA): as QMODE 0, but plane p's barrier is only probed
//   (mbarrier.test_wait) at the start of its step; all taps of output k = p-R
//   except the z-tap at p are computed first, and the warp spins only if the
//   plane has still not landed -- the barrier latency leaves the critical path;
// QMODE 5: as QMODE 0 with the x taps in a separate accumulator chain;
// QMODE 6: the plane loop unrolled by the queue depth NQ (UNR == NQ): plane
//   p lives in slot (p - p0) mod NQ for its whole life, no moves, no dispatch.
//
// Arithmetic is re-associated relative to the spec (y/z taps first, then x,
// then the centre, each group as fma(c_r, sum, acc)); parity is by the scaled
// error gate (reading R13).
#pragma once

#ifdef __CUDACC_RTC__
// NVRTC (jit.cu): sweep.cuh's text precedes this one; the one std facility used
namespace std {
template <class T, T v>
struct integral_constant {
    static constexpr T value = v;
    using value_type = T;
    constexpr operator T() const { return v; }
};
}  // namespace std
#else
#include <type_traits>

#include "sweep.cuh"
#endif

namespace sdag {
namespace dev {

// 25-point radius-4 Laplacian: B = c0*A + sum_r c_r*(6 taps at distance r)
struct Lap25Star {
    static constexpr int R = 4, NIN = 1, NOUT = 1, NIO = 0, N1D = 0, RZ = 4, RY = 4, RX = 4, RZR = 4;
    static constexpr bool SPLIT_YZ = false;  // one coefficient for the y and z pair sums (yz)
    __host__ __device__ static constexpr int axis1d(int) { return 2; }
    __device__ __forceinline__ static void yz(double &acc, const SweepArgs &a, int r, double s) {
        acc = fma(a.s[r], s, acc);
    }
    __device__ __forceinline__ static void x(double &acc, const SweepArgs &a, int r, double s) {
        acc = fma(a.s[r], s, acc);
    }
    __device__ __forceinline__ static double finish(double acc, const SweepArgs &a, double ctr) {
        return fma(a.s[0], ctr, acc);
    }
};

// Listing 1: B = a*A - (b*h2inv)*(6 neighbours - 6*A); scalars (h2inv, a, b)
struct Jacobi7Star {
    static constexpr int R = 1, NIN = 1, NOUT = 1, NIO = 0, N1D = 0, RZ = 1, RY = 1, RX = 1, RZR = 1;
    static constexpr bool SPLIT_YZ = false;
    __host__ __device__ static constexpr int axis1d(int) { return 2; }
    __device__ __forceinline__ static void yz(double &acc, const SweepArgs &, int, double s) { acc += s; }
    __device__ __forceinline__ static void x(double &acc, const SweepArgs &, int, double s) { acc += s; }
    __device__ __forceinline__ static double finish(double acc, const SweepArgs &a, double ctr) {
        const double c = a.s[2] * a.s[0];
        return a.s[1] * ctr - c * fma(-6.0, ctr, acc);
    }
};

// compile-time loop: f(std::integral_constant<int, 0>) ... f(<N-1>)
template <int I, int N, class F>
__device__ __forceinline__ void static_for_impl(F &&f) {
    if constexpr (I < N) {
        f(std::integral_constant<int, I>{});
        static_for_impl<I + 1, N>(f);
    }
}
template <int N, class F>
__device__ __forceinline__ void static_for(F &&f) {
    static_for_impl<0, N>(f);
}

template <class B, int TX, int TY, int UY, int PF>
struct StarGeo {
    static constexpr int R = B::R;
    static constexpr int NTX = TX / 2, NTY = TY / UY, THREADS = NTX * NTY, NWARPS = (THREADS + 31) / 32;
    // left/right box margin ML = R rounded up to even, so the centre column
    // cx + ML and the aligned x-window start cx are both 16-B aligned in smem
    static constexpr int ML = R + (R % 2);
    static constexpr int PX = TX + 2 * ML, PY = TY + 2 * R, PLANE = PX * PY;
    static constexpr int WN = 2 * (R + 1 + (R % 2));  // x-window elements loaded per row (double2 aligned)
    static constexpr int PLANE_AL = ((PLANE * 8 + 127) / 128) * 128 / 8;
    static constexpr int NS = R + 1 + PF;  // ring slots
    static constexpr int NQ = 2 * R + 1;   // register queue depth
    static constexpr int SMEM = NS * PLANE_AL * 8 + 2 * NS * 8;  // ring + full/empty mbarriers
    static_assert(TX % 2 == 0 && TY % UY == 0, "tile");
    static_assert(PX <= 256 && PY <= 256, "TMA box");
};

template <class B, int TX, int TY, int UY, int PF, bool USE_TMA, int QMODE = 0, int MINB = 1, int UNR = 1,
          bool MIR = false>
__global__ void __launch_bounds__(StarGeo<B, TX, TY, UY, PF>::THREADS, MINB)
    sdag_star(const __grid_constant__ SweepArgs a) {
    using G = StarGeo<B, TX, TY, UY, PF>;
    constexpr int R = G::R, PX = G::PX, NS = G::NS, NQ = G::NQ, PAL = G::PLANE_AL, ML = G::ML, WN = G::WN;

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
    const int p0 = kb - R, plast = ke - 1 + R;
    const int64_t zbase = prob * a.nz;

    const int t = threadIdx.x;
    const int lx = t % G::NTX, ly = t / G::NTX;
    const int cx = 2 * lx;   // patch x offset inside the tile (even: 16-B aligned in smem)
    const int cy = UY * ly;  // patch y offset inside the tile

    auto issue = [&](int p) {
        const int slot = unsigned(p - p0) % NS;
        double *dst = ring + slot * PAL;
        if constexpr (USE_TMA) {
            if (t == 0) {
                // the previous occupant, plane p-NS, must have been released by every warp
                const int prev = p - NS;
                if (prev >= p0) mbar_wait(&empty[slot], (unsigned(prev - p0) / NS) & 1);
                mbar_expect_tx(&full[slot], uint32_t(G::PLANE * 8));
                tma_load_3d(dst, &a.tmap[0], &full[slot], x0 - ML, y0 - R, int(zbase + p));
            }
        } else {
            const int64_t pl = (zbase + p) * a.ny * a.nx;
            for (int e = t; e < G::PLANE; e += G::THREADS) {
                const int yy = e / PX, xx = e % PX;
                const int gx = x0 - ML + xx, gy = y0 - R + yy;
                const bool ok = gx >= 0 && gx < a.nx && gy >= 0 && gy < a.ny && p >= 0 && p < a.nz;
                cp_async8(dst + e, a.in[0] + (ok ? pl + int64_t(gy) * a.nx + gx : 0), ok);
            }
        }
    };
    auto release = [&](int p) {  // every warp is done with plane p's slot
        if constexpr (USE_TMA) {
            __syncwarp();
            if ((t & 31) == 0)
                asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&empty[unsigned(p - p0) % NS]))
                             : "memory");
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

    // per-thread store geometry (fixed for the whole z-stream)
    const int gi = x0 + cx;
    const bool ok0 = gi >= a.xmin && gi < a.hi[2];
    const bool ok1 = gi + 1 >= a.xmin && gi + 1 < a.hi[2];
    const bool vec = ok0 && ok1 && (a.nx % 2 == 0) && ((reinterpret_cast<uintptr_t>(a.out[0]) & 15) == 0);
    const int nrows = min(UY, a.hi[1] - (y0 + cy));

    constexpr bool ROT = QMODE == 1 || QMODE == 6;  // queue rotates by indexing, no moves
    static_assert(QMODE != 6 || UNR == NQ, "QMODE 6 unrolls the plane loop by the queue depth");
    constexpr int NQS = ROT ? NQ : NQ + UNR - 1;
    double q[NQS][UY][2];  // register z-queue (see QMODE)
    // queue slot of plane k + d (k = p - R) when plane p sits in slot PH
    auto qs = [](int ph, int d) { return ROT ? (ph + NQ - R + d) % NQ : ph - R + d; };

    auto step = [&](auto phase, int p, auto full_tag) {
        constexpr int PH = decltype(phase)::value;  // slot of plane p in q
        constexpr bool FULL = decltype(full_tag)::value;  // every output of this CTA is interior
        {
            const int pn = p + PF;
            if (pn <= plast) issue(pn);
            if constexpr (!USE_TMA) cp_async_commit();
        }
        if constexpr (QMODE == 4) {
            // late head (TMA only): the centre plane k = p - R has been resident
            // for R planes, so everything but the z-tap at k+R = p is computed
            // while plane p's barrier is probed; the warp spins (if at all)
            // only after that work, then folds in plane p's centre values.
            const int slot = unsigned(p - p0) % NS;
            const uint32_t par = (unsigned(p - p0) / NS) & 1;
            const bool ready = mbar_test(&full[slot], par);
            const int k = p - R;
            const double *hp = ring + slot * PAL + (cy + R) * PX + (cx + ML);
            if (k >= kb) {
                const double *cp = ring + (unsigned(k - p0) % NS) * PAL;
                double acc[UY][2], last[UY][2];
                double col[UY + 2 * R][2];
#pragma unroll
                for (int r = 0; r < UY + 2 * R; r++) {
                    const double2 v = *reinterpret_cast<const double2 *>(cp + (cy + r) * PX + (cx + ML));
                    col[r][0] = v.x;
                    col[r][1] = v.y;
                }
#pragma unroll
                for (int py = 0; py < UY; py++)
#pragma unroll
                    for (int px = 0; px < 2; px++) {
                        acc[py][px] = 0.0;
                        last[py][px] = (col[py + 2 * R][px] + col[py][px]) + q[qs(PH, -R)][py][px];
                    }
#pragma unroll
                for (int r = 1; r < R; r++)
#pragma unroll
                    for (int py = 0; py < UY; py++)
#pragma unroll
                        for (int px = 0; px < 2; px++) {
                            const double zp = q[qs(PH, r)][py][px];
                            const double zm = q[qs(PH, -r)][py][px];
                            B::yz(acc[py][px], a, r, (col[py + R + r][px] + col[py + R - r][px]) + (zp + zm));
                        }
#pragma unroll
                for (int py = 0; py < UY; py++) {
                    double w[WN];
                    const double *rp = cp + (cy + py + R) * PX + cx;
#pragma unroll
                    for (int c = 0; c < WN / 2; c++) {
                        const double2 v = *reinterpret_cast<const double2 *>(rp + 2 * c);
                        w[2 * c] = v.x;
                        w[2 * c + 1] = v.y;
                    }
#pragma unroll
                    for (int r = 1; r <= R; r++)
#pragma unroll
                        for (int px = 0; px < 2; px++) B::x(acc[py][px], a, r, w[ML + px + r] + w[ML + px - r]);
                }
                release(k);  // last use of plane k (as centre)
                if (!ready) mbar_wait(&full[slot], par);
#pragma unroll
                for (int py = 0; py < UY; py++) {
                    const double2 v = *reinterpret_cast<const double2 *>(hp + py * PX);
                    q[PH][py][0] = v.x;
                    q[PH][py][1] = v.y;
#pragma unroll
                    for (int px = 0; px < 2; px++) {
                        B::yz(acc[py][px], a, R, last[py][px] + q[PH][py][px]);
                        acc[py][px] = B::finish(acc[py][px], a, col[py + R][px]);
                    }
                }
                double *o = a.out[0] + ((zbase + k) * a.ny + (y0 + cy)) * a.nx + gi;
#pragma unroll
                for (int py = 0; py < UY; py++) {
                    if (py < nrows) {
                        if (vec) {
                            __stcs(reinterpret_cast<double2 *>(o), make_double2(acc[py][0], acc[py][1]));
                        } else {
                            if (ok0) __stcs(o, acc[py][0]);
                            if (ok1) __stcs(o + 1, acc[py][1]);
                        }
                    }
                    o += a.nx;
                }
            } else {
                if (!ready) mbar_wait(&full[slot], par);
#pragma unroll
                for (int py = 0; py < UY; py++) {
                    const double2 v = *reinterpret_cast<const double2 *>(hp + py * PX);
                    q[PH][py][0] = v.x;
                    q[PH][py][1] = v.y;
                }
                if (p < kb) release(p);  // a head-only plane (never a centre) is done
            }
            return;
        }
        if constexpr (USE_TMA) {
            mbar_wait(&full[unsigned(p - p0) % NS], (unsigned(p - p0) / NS) & 1);
        } else {
            cp_async_wait<PF>();
            __syncthreads();
        }
        {  // queue head: plane p's centre values
            const double *hp = ring + (unsigned(p - p0) % NS) * PAL + (cy + R) * PX + (cx + ML);
#pragma unroll
            for (int py = 0; py < UY; py++) {
                const double2 v = *reinterpret_cast<const double2 *>(hp + py * PX);
                q[PH][py][0] = v.x;
                q[PH][py][1] = v.y;
            }
        }
        const int k = p - R;
        if (k >= kb) {
            const double *cp = ring + (unsigned(k - p0) % NS) * PAL;  // centre plane k with its xy halo
            double acc[UY][2];
#pragma unroll
            for (int py = 0; py < UY; py++) acc[py][0] = acc[py][1] = 0.0;
            if constexpr (QMODE == 2) {
                // code differencing: memory pipeline only, no stencil arithmetic
#pragma unroll
                for (int py = 0; py < UY; py++) acc[py][0] = q[PH][py][0], acc[py][1] = q[PH][py][1];
            } else {
            // y and z taps: column rows [cy-R, cy+UY+R) of plane k; z from the queue
            {
                double col[UY + 2 * R][2];
#pragma unroll
                for (int r = 0; r < UY + 2 * R; r++) {
                    const double2 v = *reinterpret_cast<const double2 *>(cp + (cy + r) * PX + (cx + ML));
                    col[r][0] = v.x;
                    col[r][1] = v.y;
                }
                // r outermost: 2*UY independent accumulation chains per step
#pragma unroll
                for (int r = 1; r <= R; r++)
#pragma unroll
                    for (int py = 0; py < UY; py++)
#pragma unroll
                        for (int px = 0; px < 2; px++) {
                            // plane k+d (k = p-R) lives in slot (PH - R + d) mod NQ
                            const double zp = q[qs(PH, r)][py][px];
                            const double zm = q[qs(PH, -r)][py][px];
                            if constexpr (B::SPLIT_YZ) {  // distinct y and z coefficients (generated bodies)
                                B::y(acc[py][px], a, r, col[py + R + r][px] + col[py + R - r][px]);
                                B::z(acc[py][px], a, r, zp + zm);
                            } else {
                                B::yz(acc[py][px], a, r, (col[py + R + r][px] + col[py + R - r][px]) + (zp + zm));
                            }
                        }
            }
            // x taps: the row window [cx-R, cx+2+R) lies in the aligned span
            // [cx, cx+WN) of smem columns; w[ML + px + dx] is the tap (px, dx)
#pragma unroll
            for (int py = 0; py < UY; py++) {
                double w[WN];
                const double *rp = cp + (cy + py + R) * PX + cx;
#pragma unroll
                for (int c = 0; c < WN / 2; c++) {
                    const double2 v = *reinterpret_cast<const double2 *>(rp + 2 * c);
                    w[2 * c] = v.x;
                    w[2 * c + 1] = v.y;
                }
                if constexpr (QMODE == 5) {
                    // split accumulators: x taps in their own chain, joined
                    // before the centre term (dependency depth 2R+2, not 2R+1+...)
                    double ax[2] = {0.0, 0.0};
#pragma unroll
                    for (int r = 1; r <= R; r++)
#pragma unroll
                        for (int px = 0; px < 2; px++) B::x(ax[px], a, r, w[ML + px + r] + w[ML + px - r]);
#pragma unroll
                    for (int px = 0; px < 2; px++) acc[py][px] = B::finish(acc[py][px] + ax[px], a, w[ML + px]);
                } else {
#pragma unroll
                    for (int r = 1; r <= R; r++)
#pragma unroll
                        for (int px = 0; px < 2; px++) B::x(acc[py][px], a, r, w[ML + px + r] + w[ML + px - r]);
#pragma unroll
                    for (int px = 0; px < 2; px++) acc[py][px] = B::finish(acc[py][px], a, w[ML + px]);
                }
            }
            }
            release(k);  // last use of plane k (as centre)
            // interior-only streaming stores (16-B vector stores when both points are inside)
            double *o = a.out[0] + ((zbase + k) * a.ny + (y0 + cy)) * a.nx + gi;
            const bool mp = MIR && mirror_plane(a, k);  // dist p2p: also into a neighbour's ghosts
            if constexpr (FULL && QMODE != 3) {
                // a tile entirely inside the interior (the common case): 16-B
                // stores with no per-row / per-point conditions
#pragma unroll
                for (int py = 0; py < UY; py++) {
                    __stcs(reinterpret_cast<double2 *>(o), make_double2(acc[py][0], acc[py][1]));
                    if constexpr (MIR) if (mp) mirror2(a, k, o, acc[py][0], acc[py][1]);
                    o += a.nx;
                }
            } else {
#pragma unroll
            for (int py = 0; py < UY; py++) {
                // QMODE 3 (code differencing): arithmetic kept alive, stores (almost) never issued
                if (py < nrows && (QMODE != 3 || acc[py][0] == 12345.678)) {
                    if (vec) {
                        __stcs(reinterpret_cast<double2 *>(o), make_double2(acc[py][0], acc[py][1]));
                        if constexpr (MIR) if (mp) mirror2(a, k, o, acc[py][0], acc[py][1]);
                    } else {
                        if (ok0) __stcs(o, acc[py][0]);
                        if (ok1) __stcs(o + 1, acc[py][1]);
                        if (MIR && mp && ok0) mirror1(a, k, o, acc[py][0]);
                        if (MIR && mp && ok1) mirror1(a, k, o + 1, acc[py][1]);
                    }
                }
                o += a.nx;
            }
            }
        } else if (p < kb) {
            release(p);  // a head-only plane (never a centre) is done
        }
        if constexpr (!USE_TMA) __syncthreads();  // the LSU ring has no empty barriers
    };

    // the plane loop, compiled twice: tiles whose outputs are all interior (and
    // 16-B aligned) store without per-row / per-point conditions
    auto run = [&](auto full_tag) {
    if constexpr (QMODE == 6) {
        for (int p = p0; p <= plast; p += NQ)
            static_for<NQ>([&](auto I) {
                if (p + decltype(I)::value <= plast) step(I, p + decltype(I)::value, full_tag);
            });
    } else if constexpr (QMODE != 1) {
        for (int p = p0; p <= plast; p += UNR) {
            static_for<UNR>([&](auto I) {
                if (UNR == 1 || p + decltype(I)::value <= plast)
                    step(std::integral_constant<int, NQ - 1 + decltype(I)::value>{}, p + decltype(I)::value,
                         full_tag);
            });
#pragma unroll
            for (int d = 0; d < NQ - 1; d++)
#pragma unroll
                for (int py = 0; py < UY; py++) {
                    q[d][py][0] = q[d + UNR][py][0];
                    q[d][py][1] = q[d + UNR][py][1];
                }
        }
    } else {
        for (int p = p0; p <= plast; p++) {
            const int ph = unsigned(p - p0) % NQ;
            static_for<NQ>([&](auto I) {
                if (ph == decltype(I)::value) step(I, p, full_tag);
            });
        }
    }
    };
    const bool tile_full = x0 >= a.xmin && x0 + TX <= a.hi[2] && y0 + TY <= a.hi[1] && (a.nx % 2 == 0) &&
                      ((reinterpret_cast<uintptr_t>(a.out[0]) & 15) == 0);
    if (tile_full)
        run(std::integral_constant<bool, true>{});
    else
        run(std::integral_constant<bool, false>{});
}


// sdag_star2: same ring/patch design, but the z-taps k+1..k+R are read from the
// ring (those planes are resident anyway: plane p = k+R is the newest) and only
// k-1..k-R live in registers.  Halves the register queue (R instead of 2R+1
// values per point) and its per-plane shifting, for ~3 more doubles of smem
// reads per point (B200: the star kernel is issue-bound, not smem-bound).
template <class B, int TX, int TY, int UY, int PF, bool USE_TMA, int MINB = 1>
__global__ void __launch_bounds__(StarGeo<B, TX, TY, UY, PF>::THREADS, MINB)
    sdag_star2(const __grid_constant__ SweepArgs a) {
    using G = StarGeo<B, TX, TY, UY, PF>;
    constexpr int R = G::R, PX = G::PX, NS = G::NS, PAL = G::PLANE_AL, ML = G::ML, WN = G::WN;

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
    const int p0 = kb - R, plast = ke - 1 + R;
    const int64_t zbase = prob * a.nz;

    const int t = threadIdx.x;
    const int lx = t % G::NTX, ly = t / G::NTX;
    const int cx = 2 * lx, cy = UY * ly;

    auto issue = [&](int p) {
        const int slot = unsigned(p - p0) % NS;
        double *dst = ring + slot * PAL;
        if constexpr (USE_TMA) {
            if (t == 0) {
                const int prev = p - NS;
                if (prev >= p0) mbar_wait(&empty[slot], (unsigned(prev - p0) / NS) & 1);
                mbar_expect_tx(&full[slot], uint32_t(G::PLANE * 8));
                tma_load_3d(dst, &a.tmap[0], &full[slot], x0 - ML, y0 - R, int(zbase + p));
            }
        } else {
            const int64_t pl = (zbase + p) * a.ny * a.nx;
            for (int e = t; e < G::PLANE; e += G::THREADS) {
                const int yy = e / PX, xx = e % PX;
                const int gx = x0 - ML + xx, gy = y0 - R + yy;
                const bool ok = gx >= 0 && gx < a.nx && gy >= 0 && gy < a.ny && p >= 0 && p < a.nz;
                cp_async8(dst + e, a.in[0] + (ok ? pl + int64_t(gy) * a.nx + gx : 0), ok);
            }
        }
    };
    auto release = [&](int p) {
        if constexpr (USE_TMA) {
            __syncwarp();
            if ((t & 31) == 0)
                asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&empty[unsigned(p - p0) % NS]))
                             : "memory");
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

    const int gi = x0 + cx;
    const bool ok0 = gi >= a.xmin && gi < a.hi[2];
    const bool ok1 = gi + 1 >= a.xmin && gi + 1 < a.hi[2];
    const bool vec = ok0 && ok1 && (a.nx % 2 == 0) && ((reinterpret_cast<uintptr_t>(a.out[0]) & 15) == 0);
    const int nrows = min(UY, a.hi[1] - (y0 + cy));

    double qm[R][UY][2];  // qm[r-1] = centre values of plane k-r
#pragma unroll
    for (int r = 0; r < R; r++)
#pragma unroll
        for (int py = 0; py < UY; py++) qm[r][py][0] = qm[r][py][1] = 0.0;

    for (int p = p0; p <= plast; p++) {
        {
            const int pn = p + PF;
            if (pn <= plast) issue(pn);
            if constexpr (!USE_TMA) cp_async_commit();
        }
        if constexpr (USE_TMA) {
            mbar_wait(&full[unsigned(p - p0) % NS], (unsigned(p - p0) / NS) & 1);
        } else {
            cp_async_wait<PF>();
            __syncthreads();
        }
        const int k = p - R;  // plane k is the centre of this iteration
        if (k >= p0) {
            const double *cp = ring + (unsigned(k - p0) % NS) * PAL;
            double col[UY + 2 * R][2];  // rows [cy-R, cy+UY+R) of plane k, 2 centre columns
#pragma unroll
            for (int r = 0; r < UY + 2 * R; r++) {
                const double2 v = *reinterpret_cast<const double2 *>(cp + (cy + r) * PX + (cx + ML));
                col[r][0] = v.x;
                col[r][1] = v.y;
            }
            if (k >= kb) {
                double acc[UY][2];
#pragma unroll
                for (int py = 0; py < UY; py++) acc[py][0] = acc[py][1] = 0.0;
#pragma unroll
                for (int r = 1; r <= R; r++) {
                    const double *up = ring + ((k + r - p0) % NS) * PAL + (cy + R) * PX + (cx + ML);  // plane k+r
#pragma unroll
                    for (int py = 0; py < UY; py++) {
                        const double2 zp = *reinterpret_cast<const double2 *>(up + py * PX);
                        B::yz(acc[py][0], a, r, (col[py + R + r][0] + col[py + R - r][0]) + (zp.x + qm[r - 1][py][0]));
                        B::yz(acc[py][1], a, r, (col[py + R + r][1] + col[py + R - r][1]) + (zp.y + qm[r - 1][py][1]));
                    }
                }
#pragma unroll
                for (int py = 0; py < UY; py++) {
                    double w[WN];
                    const double *rp = cp + (cy + py + R) * PX + cx;
#pragma unroll
                    for (int c = 0; c < WN / 2; c++) {
                        const double2 v = *reinterpret_cast<const double2 *>(rp + 2 * c);
                        w[2 * c] = v.x;
                        w[2 * c + 1] = v.y;
                    }
#pragma unroll
                    for (int r = 1; r <= R; r++)
#pragma unroll
                        for (int px = 0; px < 2; px++) B::x(acc[py][px], a, r, w[ML + px + r] + w[ML + px - r]);
#pragma unroll
                    for (int px = 0; px < 2; px++) acc[py][px] = B::finish(acc[py][px], a, w[ML + px]);
                }
                release(k);
                double *o = a.out[0] + ((zbase + k) * a.ny + (y0 + cy)) * a.nx + gi;
#pragma unroll
                for (int py = 0; py < UY; py++) {
                    if (py < nrows) {
                        if (vec) {
                            __stcs(reinterpret_cast<double2 *>(o), make_double2(acc[py][0], acc[py][1]));
                        } else {
                            if (ok0) __stcs(o, acc[py][0]);
                            if (ok1) __stcs(o + 1, acc[py][1]);
                        }
                    }
                    o += a.nx;
                }
            } else {
                release(k);  // a plane below the chunk: only feeds the queue
            }
            // push plane k's centre values into the register queue
#pragma unroll
            for (int r = R - 1; r > 0; r--)
#pragma unroll
                for (int py = 0; py < UY; py++) {
                    qm[r][py][0] = qm[r - 1][py][0];
                    qm[r][py][1] = qm[r - 1][py][1];
                }
#pragma unroll
            for (int py = 0; py < UY; py++) {
                qm[0][py][0] = col[py + R][0];
                qm[0][py][1] = col[py + R][1];
            }
        }
        if constexpr (!USE_TMA) __syncthreads();
    }
}

}  // namespace dev
}  // namespace sdag

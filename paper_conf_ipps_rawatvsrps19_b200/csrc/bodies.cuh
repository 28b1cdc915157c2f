// bodies.cuh -- per-DAG point bodies for the sweep skeleton (a5).
//
// Each body evaluates the registered DAG of paper_conf_ipps_rawatvsrps19_b200/
// specs/<name>.sdag at one point.  The planner only dispatches a spec here
// after its canonical form (ir.hpp) equals the registered spec's, so the body
// and the spec denote the same DAG; parity against the independent oracle is
// tested in tests/test_gpu_parity.py.  nvcc contracts a*b+c into DFMA
// (--fmad=true, as the paper's --use_fast_math build), so
// results agree with the strict oracle to rounding (reading R12).
//
// Staged-array numbering = order of the 3D *inputs* among the formals;
// outputs / inouts = order of the written 3D formals.
#pragma once

namespace sdag {
namespace dev {

struct BodyBase {
    static constexpr int NIO = 0, N1D = 0;
    static constexpr int RZR = -1;  // shared-memory ring z-window; -1 = RZ (see ring_rz)
    __host__ __device__ static constexpr int axis1d(int) { return 2; }
};

// Listing 1: jacobi (B, A, h2inv, a, b)
struct Jacobi7 : BodyBase {
    static constexpr int NIN = 1, NOUT = 1, RZ = 1, RY = 1, RX = 1;
    template <class G>
    __device__ __forceinline__ static void eval(const G &g, double (&o)[NOUT]) {
        const double h2inv = g.s(0), a = g.s(1), b = g.s(2);
        const double c = b * h2inv;
        o[0] = a * g.at(0, 0, 0, 0) -
               c * (g.at(0, 0, 0, 1) + g.at(0, 0, 0, -1) + g.at(0, 0, 1, 0) + g.at(0, 0, -1, 0) + g.at(0, 1, 0, 0) +
                    g.at(0, -1, 0, 0) - g.at(0, 0, 0, 0) * 6.0);
    }
};

// 25-point radius-4 Laplacian (specs/lap25.sdag): lap25 (B, A, c0..c4)
struct Lap25 : BodyBase {
    static constexpr int NIN = 1, NOUT = 1, RZ = 4, RY = 4, RX = 4;
    template <class G>
    __device__ __forceinline__ static void eval(const G &g, double (&o)[NOUT]) {
        double acc = g.s(0) * g.at(0, 0, 0, 0);
#pragma unroll
        for (int r = 1; r <= 4; r++)
            acc += g.s(r) * (g.at(0, 0, 0, r) + g.at(0, 0, 0, -r) + g.at(0, 0, r, 0) + g.at(0, 0, -r, 0) +
                             g.at(0, r, 0, 0) + g.at(0, -r, 0, 0));
        o[0] = acc;
    }
};

// 27-point smoother (specs/smooth27.sdag): smooth27 (B, A, w0, w1, w2, w3, nu)
struct Smooth27 : BodyBase {
    static constexpr int NIN = 1, NOUT = 1, RZ = 1, RY = 1, RX = 1;
    template <class G>
    __device__ __forceinline__ static void eval(const G &g, double (&o)[NOUT]) {
        const double w0 = g.s(0), w1 = g.s(1), w2 = g.s(2), w3 = g.s(3), nu = g.s(4);
        // partial sums per plane: centre, in-plane faces, in-plane corners
        double s0[3], s1[3], s2[3];
#pragma unroll
        for (int d = -1; d <= 1; d++) {
            s0[d + 1] = g.at(0, d, 0, 0);
            s1[d + 1] = g.at(0, d, 0, -1) + g.at(0, d, 0, 1) + g.at(0, d, -1, 0) + g.at(0, d, 1, 0);
            s2[d + 1] = g.at(0, d, -1, -1) + g.at(0, d, -1, 1) + g.at(0, d, 1, -1) + g.at(0, d, 1, 1);
        }
        const double SF = s1[1] + (s0[0] + s0[2]);
        const double SE = s2[1] + (s1[0] + s1[2]);
        const double SC = s2[0] + s2[2];
        const double A = s0[1];
        o[0] = A + nu * (w0 * A + w1 * SF + w2 * SE + w3 * SC);
    }
};

// ExpCNS hypterm (specs/hypterm.sdag): inputs cons_1..4 (0..3), q_1..4 (4..7);
// outputs flux_0..4; scalars dxinv0..2, ALP, BET, GAM, DEL.
// v1 staging: the ring holds only the centre plane with its xy halo (8 arrays
// x 9 planes would not fit in 227 KB); z-taps come through L1/L2.
struct Hypterm : BodyBase {
    static constexpr int NIN = 8, NOUT = 5, RZ = 4, RY = 4, RX = 4, RZR = 0;
    template <class G>
    __device__ __forceinline__ static void eval(const G &g, double (&o)[NOUT]) {
        const double dxinv[3] = {g.s(0), g.s(1), g.s(2)};
        const double C[5] = {0.0, g.s(3), g.s(4), g.s(5), g.s(6)};
#pragma unroll
        for (int m = 0; m < 5; m++) o[m] = 0.0;
#pragma unroll
        for (int a = 0; a < 3; a++) {  // axis: 0 x (i), 1 y (j), 2 z (k)
            double t[5] = {0.0, 0.0, 0.0, 0.0, 0.0};
#pragma unroll
            for (int r = 1; r <= 4; r++) {
                const int dz = a == 2 ? r : 0, dy = a == 1 ? r : 0, dx = a == 0 ? r : 0;
                const int V = 4 + a;  // q_{1+a}: velocity along the axis
                const double vp = g.at(V, dz, dy, dx), vm = g.at(V, -dz, -dy, -dx);
                const double pp = g.at(7, dz, dy, dx), pm = g.at(7, -dz, -dy, -dx);
                double d[5];
                d[0] = g.at(a, dz, dy, dx) - g.at(a, -dz, -dy, -dx);  // mass: cons_{1+a}
#pragma unroll
                for (int m = 1; m <= 3; m++) {
                    d[m] = g.at(m - 1, dz, dy, dx) * vp - g.at(m - 1, -dz, -dy, -dx) * vm;
                    if (a == m - 1) d[m] += pp - pm;
                }
                d[4] = (g.at(3, dz, dy, dx) * vp - g.at(3, -dz, -dy, -dx) * vm) + (pp * vp - pm * vm);
#pragma unroll
                for (int m = 0; m < 5; m++) t[m] = (r == 1) ? C[1] * d[m] : t[m] + C[r] * d[m];
            }
#pragma unroll
            for (int m = 0; m < 5; m++) o[m] = (a == 0) ? -(t[m] * dxinv[0]) : o[m] - t[m] * dxinv[a];
        }
    }
};

// SW4 rhs4center (specs/rhs4center.sdag): staged u0,u1,u2,mu,la (0..4);
// inout uacc0..2; 1D strx (x), stry (y), strz (z); scalars tf, i6, i144, cof, a1.
struct Rhs4 : BodyBase {
    static constexpr int NIN = 5, NOUT = 3, NIO = 3, N1D = 3, RZ = 2, RY = 2, RX = 2;
    __host__ __device__ static constexpr int axis1d(int arr) { return arr == 0 ? 2 : (arr == 1 ? 1 : 0); }

    // offsets of `m` steps along axis b (0 x, 1 y, 2 z)
    __device__ __forceinline__ static int oz(int b, int m) { return b == 2 ? m : 0; }
    __device__ __forceinline__ static int oy(int b, int m) { return b == 1 ? m : 0; }
    __device__ __forceinline__ static int ox(int b, int m) { return b == 0 ? m : 0; }

    template <class G>
    __device__ __forceinline__ static double cs(const G &g, int coef, int b, int m) {
        // coef(p + m e_b) * str_b[idx_b + m]; str index: strx=0 (axis x), stry=1, strz=2
        return g.at(coef, oz(b, m), oy(b, m), ox(b, m)) * g.s1(b, m);
    }

    template <class G>
    __device__ __forceinline__ static double inner(const G &g, int coef, int u, int oa, int mo, int ob) {
        // coef(q)*(u(q-2e_b) - u(q+2e_b) + 8*(-u(q-e_b) + u(q+e_b))), q = p + mo e_a
        const int qz = oz(oa, mo), qy = oy(oa, mo), qx = ox(oa, mo);
        auto U = [&](int mb) { return g.at(u, qz + oz(ob, mb), qy + oy(ob, mb), qx + ox(ob, mb)); };
        return g.at(coef, qz, qy, qx) * (U(-2) - U(2) + 8.0 * (U(1) - U(-1)));
    }

    template <class G>
    __device__ __forceinline__ static void eval(const G &g, double (&o)[NOUT]) {
        const double tf = g.s(0), i6 = g.s(1), i144 = g.s(2), cof = g.s(3), a1 = g.s(4);
        constexpr int MU = 3, LA = 4;
        double mub[3][5];
#pragma unroll
        for (int b = 0; b < 3; b++) {
            const double m_2 = cs(g, MU, b, -2), m_1 = cs(g, MU, b, -1), m0 = cs(g, MU, b, 0), m1 = cs(g, MU, b, 1),
                         m2 = cs(g, MU, b, 2);
            mub[b][1] = m_1 - tf * (m0 + m_2);
            mub[b][2] = m_2 + m1 + 3.0 * (m0 + m_1);
            mub[b][3] = m_1 + m2 + 3.0 * (m1 + m0);
            mub[b][4] = m1 - tf * (m0 + m2);
        }
        const int sm[5] = {0, -2, -1, 1, 2};
        // mixed terms: (outer axis, inner axis, component, coef) in SW4 order
        const int T[3][4][4] = {
            {{0, 1, 1, LA}, {0, 2, 2, LA}, {1, 0, 1, MU}, {2, 0, 2, MU}},
            {{0, 1, 0, MU}, {1, 0, 0, LA}, {1, 2, 2, LA}, {2, 1, 2, MU}},
            {{0, 2, 0, MU}, {1, 2, 1, MU}, {2, 0, 0, LA}, {2, 1, 1, LA}},
        };
#pragma unroll
        for (int c = 0; c < 3; c++) {
            const double u0 = g.at(c, 0, 0, 0);
            double sumb = 0.0;
#pragma unroll
            for (int b = 0; b < 3; b++) {
                double sum = 0.0;
#pragma unroll
                for (int m = 1; m <= 4; m++) {
                    double K;
                    if (b == c) {
                        const double l_2 = cs(g, LA, b, -2), l_1 = cs(g, LA, b, -1), l0 = cs(g, LA, b, 0),
                                     l1 = cs(g, LA, b, 1), l2 = cs(g, LA, b, 2);
                        if (m == 1) K = 2.0 * mub[b][1] + l_1 - tf * (l0 + l_2);
                        else if (m == 2) K = 2.0 * mub[b][2] + l_2 + l1 + 3.0 * (l0 + l_1);
                        else if (m == 3) K = 2.0 * mub[b][3] + l_1 + l2 + 3.0 * (l1 + l0);
                        else K = 2.0 * mub[b][4] + l1 - tf * (l0 + l2);
                    } else {
                        K = mub[b][m];
                    }
                    const double du = g.at(c, oz(b, sm[m]), oy(b, sm[m]), ox(b, sm[m])) - u0;
                    sum = (m == 1) ? K * du : sum + K * du;
                }
                const double part = g.s1(b, 0) * sum;
                sumb = (b == 0) ? part : sumb + part;
            }
            double r = i6 * sumb;
#pragma unroll
            for (int q = 0; q < 4; q++) {
                const int oa = T[c][q][0], ob = T[c][q][1], comp = T[c][q][2], coef = T[c][q][3];
                const int lo = oa < ob ? oa : ob, hi = oa < ob ? ob : oa;
                const double D = inner(g, coef, comp, oa, -2, ob) - 8.0 * inner(g, coef, comp, oa, -1, ob) +
                                 8.0 * inner(g, coef, comp, oa, 1, ob) - inner(g, coef, comp, oa, 2, ob);
                r += g.s1(lo, 0) * g.s1(hi, 0) * i144 * D;
            }
            o[c] = a1 * g.io(c) + cof * r;
        }
    }
};

// toy: B = A(p + off), off = (s0, s1, s2) = (dz, dy, dx), |off| <= 4 (specs/shift.sdag)
struct Shift4 : BodyBase {
    static constexpr int NIN = 1, NOUT = 1, RZ = 4, RY = 4, RX = 4;
    template <class G>
    __device__ __forceinline__ static void eval(const G &g, double (&o)[NOUT]) {
        o[0] = g.at(0, int(g.s(0)), int(g.s(1)), int(g.s(2)));
    }
};

// Fig 1a j1d3pt: B[i] = c*(A[i+1] + A[i] + A[i-1]) / 3.0
struct J1d3pt : BodyBase {
    static constexpr int NIN = 1, NOUT = 1, RZ = 0, RY = 0, RX = 1;
    template <class G>
    __device__ __forceinline__ static void eval(const G &g, double (&o)[NOUT]) {
        o[0] = g.s(0) * (g.at(0, 0, 0, 1) + g.at(0, 0, 0, 0) + g.at(0, 0, 0, -1)) / 3.0;
    }
};

// Trivial-fission wrapper (Fig 3b): evaluate only output M of
// body B; the other outputs and every temporary they alone need are dead code.
template <class B, int M>
struct OnlyOut : B {
    static constexpr int NOUT = 1;
    template <class G>
    __device__ __forceinline__ static void eval(const G &g, double (&o)[1]) {
        double all[B::NOUT];
        B::eval(g, all);
        o[0] = all[M];
    }
};

}  // namespace dev
}  // namespace sdag

"""Pins for the CPU oracle (oracle/oracle.c) against what the mathematics fixes.

None of these re-type the oracle's formulas: they check it against
 - closed forms: a finite-difference operator applied to a polynomial of
   degree <= its exactness order equals the continuous derivative
   (computed symbolically by tests/polyexact.Poly), bit-for-bit;
 - invariants: constant fields, the abs-mode triangle bound, discrete
   self-adjointness of the SW4 operator, translation/iteration identities;
 - hand-expanded worked examples (tests/golden/, with citations).
The polynomial inputs use distinct random coefficients per axis and per
array, so a dropped term, a wrong sign, a wrong offset or a transposed
operand changes the result away from the closed form.
"""
from __future__ import annotations

import os
import random

import numpy as np
import pytest

import oracle
from polyexact import Poly, laplacian, random_poly

HERE = os.path.dirname(os.path.abspath(__file__))


def interior(shape, R):
    return tuple(slice(R[a], shape[a] - R[a]) for a in range(3))


def ring_mask(shape, R):
    m = np.ones(shape, dtype=bool)
    m[interior(shape, R)] = False
    return m


# --------------------------------------------------------------------------
# 7-point Jacobi, Listing 1
# --------------------------------------------------------------------------

@pytest.mark.parametrize("seed", range(4))
def test_jacobi7_polynomial_closed_form(seed):
    """a=1/2, b=1/4, h2inv=4 (c=b*h2inv=1): the 7-point sum minus 6*center is
    the exact Laplacian for per-axis degree <= 3, so B = p/2 - lap(p)."""
    rng = random.Random(seed)
    shape, origin = (14, 15, 16), (7, 7, 8)
    p = random_poly(rng, (3, 3, 3), coef=4, nterms=12)
    A = p.grid(shape, origin)
    expect = (p * Fraction2(1, 2) - laplacian(p)).grid(shape, origin)
    sentinel = np.full(shape, np.nan)
    B = oracle.jacobi7(A, 0.5, 0.25, 4.0, out=sentinel.copy())
    I = interior(shape, (1, 1, 1))
    assert np.array_equal(B[I], expect[I])
    assert np.all(np.isnan(B[ring_mask(shape, (1, 1, 1))]))  # ring never written


def Fraction2(a, b):
    from fractions import Fraction
    return Fraction(a, b)


def test_jacobi7_constant_field():
    A = np.full((6, 7, 8), 3.0)
    B = oracle.jacobi7(A, 0.5, 0.25, 4.0)
    assert np.all(B[1:-1, 1:-1, 1:-1] == 1.5)  # a*C - c*(6C - 6C)


def test_jacobi7_scalars_enter_as_listing1():
    """Vary a, b, h2inv separately on a quadratic: B = a p - (b h2inv) lap p."""
    shape, origin = (8, 8, 8), (4, 4, 4)
    p = Poly({(2, 0, 0): 1, (0, 2, 0): 2, (0, 0, 2): 5, (1, 1, 0): 3, (0, 0, 0): 7})  # lap = 16
    A = p.grid(shape, origin)
    for a, b, h in [(2.0, 0.5, 1.0), (0.25, 2.0, 0.5), (1.0, 0.125, 8.0)]:
        B = oracle.jacobi7(A, a, b, h)
        I = interior(shape, (1, 1, 1))
        assert np.array_equal(B[I], a * A[I] - (b * h) * 16.0)


# --------------------------------------------------------------------------
# 25-point radius-4 Laplacian
# --------------------------------------------------------------------------

@pytest.mark.parametrize("seed", range(3))
def test_lap25_x5040_polynomial_closed_form(seed):
    """Integer coefficients (-43050, 8064, -1008, 128, -9) = 5040 * the 8th-order
    central second difference, exact for per-axis degree <= 9: B = 5040 lap p.
    (c0 carries all three axes: 3 * -14350.)"""
    rng = random.Random(100 + seed)
    shape, origin = (17, 18, 19), (8, 9, 9)
    p = random_poly(rng, (6, 5, 4), coef=2, nterms=8)
    A = p.grid(shape, origin)
    expect = (laplacian(p) * 5040).grid(shape, origin)
    B = oracle.lap25(A, [-43050.0, 8064.0, -1008.0, 128.0, -9.0], out=np.full(shape, np.nan))
    I = interior(shape, (4, 4, 4))
    assert np.array_equal(B[I], expect[I])
    assert np.all(np.isnan(B[ring_mask(shape, (4, 4, 4))]))


def test_lap25_x5040_is_tight():
    """Degree 10 along one axis is NOT reproduced (the order-8 error term
    appears), so the pin above really constrains all nine taps."""
    shape, origin = (10, 10, 21), (5, 5, 10)
    p = Poly({(10, 0, 0): 1})
    A = p.grid(shape, origin)
    B = oracle.lap25(A, [-43050.0, 8064.0, -1008.0, 128.0, -9.0])
    I = interior(shape, (4, 4, 4))
    assert not np.array_equal(B[I], (laplacian(p) * 5040).grid(shape, origin)[I])


def test_lap25_real_coefficients_approximate_laplacian():
    from synth import LAP25_COEFS
    c = [LAP25_COEFS[k] for k in ("c0", "c1", "c2", "c3", "c4")]
    shape, origin = (12, 12, 12), (6, 6, 6)
    p = Poly({(2, 0, 0): 3, (0, 3, 1): 1, (1, 1, 1): 2, (0, 0, 4): 1})
    A = p.grid(shape, origin)
    B = oracle.lap25(A, c)
    E = laplacian(p).grid(shape, origin)
    I = interior(shape, (4, 4, 4))
    scale = oracle.lap25(np.abs(A), np.abs(c), absmode=True)
    assert np.max(np.abs(B[I] - E[I]) / scale[I]) < 1e-14


# --------------------------------------------------------------------------
# 27-point smoother (Table I)
# --------------------------------------------------------------------------

W_INT = [-128.0, 14.0, 3.0, 1.0]


@pytest.mark.parametrize("seed", range(3))
def test_smooth27_integer_weights_closed_form(seed):
    """w = (-128, 14, 3, 1): the weighted 27-point sum is 30 * lap p exactly
    for total degree <= 3; with nu = 1/32, B = p + (30/32) lap p."""
    rng = random.Random(200 + seed)
    shape, origin = (11, 12, 13), (5, 6, 6)
    p = random_poly(rng, (3, 3, 3), max_total=3, coef=5, nterms=14)
    A = p.grid(shape, origin)
    expect = (p + laplacian(p) * Fraction2(30, 32)).grid(shape, origin)
    B = oracle.smooth27(A, W_INT, 1.0 / 32.0, out=np.full(shape, np.nan))
    I = interior(shape, (1, 1, 1))
    assert np.array_equal(B[I], expect[I])
    assert np.all(np.isnan(B[ring_mask(shape, (1, 1, 1))]))


def test_smooth27_weights_each_class_matters():
    """Corner-only, edge-only and face-only weights on x*y*z, x^2 y, ...:
    each class has its own closed form (catches a neighbour put in the
    wrong class)."""
    shape, origin = (7, 7, 7), (3, 3, 3)
    A = Poly({(0, 0, 0): 1}).grid(shape, origin)
    I = interior(shape, (1, 1, 1))
    for w, expect in [([0, 1, 0, 0], 6.0), ([0, 0, 1, 0], 12.0), ([0, 0, 0, 1], 8.0), ([1, 0, 0, 0], 1.0)]:
        B = oracle.smooth27(A, w, 1.0)
        assert np.all(B[I] == 1.0 + expect)
    # x^2: faces see 2 (from +-x) + 4*0 ... second moments per class
    p = Poly({(2, 0, 0): 1})
    A = p.grid(shape, origin)
    x2 = A
    for w, sec in [([0, 1, 0, 0], 2.0), ([0, 0, 1, 0], 8.0), ([0, 0, 0, 1], 8.0)]:
        # sum over class of (x+dx)^2 = n_class*x^2 + sum dx^2
        ncls = {1: 6, 2: 12, 3: 8}[w.index(1)]
        B = oracle.smooth27(A, w, 1.0)
        assert np.array_equal(B[I], x2[I] + ncls * x2[I] + sec)


def test_smooth27_iterated_closed_form_region():
    """V8: with integer weights, nu=1/32 and a quadratic p, T sweeps with a
    fixed ring give A_T = p + T*(30/32)*lap p exactly where the distance to
    the ring is >= T, and deviate at distance T-1 (tight)."""
    shape, origin = (12, 12, 12), (6, 5, 6)
    p = Poly({(2, 0, 0): 3, (0, 2, 0): -2, (0, 0, 2): 5, (1, 1, 0): 1, (0, 1, 1): -3, (1, 0, 0): 2,
              (0, 0, 0): 11})
    A = p.grid(shape, origin)
    L = float(laplacian(p).c[(0, 0, 0)])
    kk, jj, ii = np.meshgrid(*[np.arange(n) for n in shape], indexing="ij")
    d = np.minimum.reduce([np.minimum(x, n - 1 - x) for x, n in zip((kk, jj, ii), shape)])
    for T in range(1, 5):
        AT = oracle.smooth27_iter(A, W_INT, 1.0 / 32.0, T)
        exact = A + T * (30.0 / 32.0) * L
        assert np.array_equal(AT[d >= T], exact[d >= T])
        assert not np.array_equal(AT[d == T - 1], exact[d == T - 1]) or T == 1
        assert np.array_equal(AT[d == 0], A[d == 0])  # ring untouched


def test_smooth27_iter_points_matches_full_iteration():
    from synth import uniform
    shape = (13, 14, 15)
    A = uniform(shape, -1, 1, "pin", "it27")
    w = [-128 / 30, 14 / 30, 3 / 30, 1 / 30]
    rng = np.random.default_rng(0)
    pts = np.stack([rng.integers(0, n, 300) for n in shape], axis=1)
    for T in (1, 2, 5):
        full = oracle.smooth27_iter(A, w, 0.125, T)
        got = oracle.smooth27_iter_points(A, w, 0.125, T, pts)
        assert np.array_equal(got, full[pts[:, 0], pts[:, 1], pts[:, 2]])


# --------------------------------------------------------------------------
# hypterm (Table I)
# --------------------------------------------------------------------------

def _hypterm_closed_form(cons, q, dxinv):
    """-840 * sum_a dxinv_a * d/dx_a of the flux components."""
    V = [q[0], q[1], q[2]]  # velocity along x, y, z
    F = []
    F.append([cons[0], cons[1], cons[2]])  # mass: M_a
    for m in range(3):
        F.append([cons[m] * V[a] + (q[3] if a == m else 0) for a in range(3)])
    F.append([(cons[3] + q[3]) * V[a] for a in range(3)])
    out = []
    for Fm in F:
        acc = Poly()
        for a in range(3):
            acc = acc + Fm[a].diff(a) * (Fraction2(1, 1) * dxinv[a])
        out.append(acc * (-840))
    return out


@pytest.mark.parametrize("seed", range(3))
@pytest.mark.parametrize("dxinv", [(1.0, 1.0, 1.0), (0.5, 0.25, 2.0)])
def test_hypterm_x840_polynomial_closed_form(seed, dxinv):
    """(ALP,BET,GAM,DEL)*840 = (672,-168,32,-3): the 8th-order central first
    difference is exact for degree <= 8, so with degree-2 fields (products of
    degree 4) flux_m = -840 sum_a dxinv_a d_a F_m,a exactly."""
    from fractions import Fraction
    rng = random.Random(300 + seed)
    shape, origin = (13, 14, 15), (6, 7, 7)
    cons = [random_poly(rng, (2, 2, 2), max_total=2, coef=3, nterms=6) for _ in range(4)]
    q = [random_poly(rng, (2, 2, 2), max_total=2, coef=3, nterms=6) for _ in range(4)]
    ins = [p.grid(shape, origin) for p in (*cons, *q)]
    expect = _hypterm_closed_form(cons, q, [Fraction(x) for x in dxinv])
    outs = oracle.hypterm(ins, dxinv, [672.0, -168.0, 32.0, -3.0],
                          outs=[np.full(shape, np.nan) for _ in range(5)])
    I = interior(shape, (4, 4, 4))
    for m in range(5):
        e = expect[m].grid(shape, origin)
        assert np.array_equal(outs[m][I], e[I]), f"flux_{m}"
        assert np.all(np.isnan(outs[m][ring_mask(shape, (4, 4, 4))]))


def test_hypterm_constant_fields_give_zero():
    shape = (10, 10, 10)
    ins = [np.full(shape, 1.0 + 0.25 * n) for n in range(8)]
    outs = oracle.hypterm(ins, (0.5, 0.25, 0.125), [0.8, -0.2, 4 / 105, -1 / 280])
    I = interior(shape, (4, 4, 4))
    for o in outs:
        assert np.all(o[I] == 0.0)


# --------------------------------------------------------------------------
# rhs4center (Table I)
# --------------------------------------------------------------------------

def _rhs4_closed_form(u, mu, la, st):
    """144 * L_c(u):
      L_c = sum_b str_b d_b(K_cb d_b u_c) + sum_{b!=c} str_c str_b [d_c(la d_b u_b) + d_b(mu d_c u_b)]
      K_cb = mu*str_b (b != c),  (2 mu + la)*str_c (b == c)."""
    out = []
    for c in range(3):
        acc = Poly()
        for b in range(3):
            K = (mu * 2 + la) * st[c] if b == c else mu * st[b]
            acc = acc + st[b] * (K * u[c].diff(b)).diff(b)
        for b in range(3):
            if b == c:
                continue
            acc = acc + st[c] * st[b] * ((la * u[b].diff(b)).diff(c) + (mu * u[b].diff(c)).diff(b))
        out.append(acc * 144)
    return out


@pytest.mark.parametrize("seed", range(3))
@pytest.mark.parametrize("a1", [0.0, 1.0])
def test_rhs4_polynomial_closed_form(seed, a1):
    """tf=3/4, i6=24, i144=1, cof=1: linear mu, la, str and u of total degree
    <= 3 make every SW4 difference exact, so uacc_new = a1*uacc + 144 L(u)."""
    rng = random.Random(400 + seed)
    shape, origin = (11, 12, 13), (5, 6, 6)
    u = [random_poly(rng, (3, 3, 3), max_total=3, coef=3, nterms=10) for _ in range(3)]
    mu = Poly({(0, 0, 0): rng.randint(5, 9), (1, 0, 0): rng.randint(-2, 2), (0, 1, 0): rng.randint(-2, 2),
               (0, 0, 1): rng.randint(-2, 2)})
    la = Poly({(0, 0, 0): rng.randint(5, 9), (1, 0, 0): rng.randint(-2, 2), (0, 1, 0): rng.randint(-2, 2),
               (0, 0, 1): rng.randint(-2, 2)})
    st = [Poly({(0, 0, 0): rng.randint(3, 5), tuple(1 if a == b else 0 for a in range(3)): rng.choice([-1, 1])})
          for b in range(3)]
    nz, ny, nx = shape
    oz, oy, ox = origin
    strx = np.array([float(st[0].c.get((0, 0, 0), 0) + st[0].c.get((1, 0, 0), 0) * (i - ox)) for i in range(nx)])
    stry = np.array([float(st[1].c.get((0, 0, 0), 0) + st[1].c.get((0, 1, 0), 0) * (j - oy)) for j in range(ny)])
    strz = np.array([float(st[2].c.get((0, 0, 0), 0) + st[2].c.get((0, 0, 1), 0) * (k - oz)) for k in range(nz)])
    U = [p.grid(shape, origin) for p in u]
    uacc_p = [random_poly(rng, (1, 1, 1), coef=3, nterms=3) for _ in range(3)]
    uacc = [p.grid(shape, origin) for p in uacc_p]
    outs = oracle.rhs4(U, mu.grid(shape, origin), la.grid(shape, origin), strx, stry, strz, uacc,
                       0.75, 24.0, 1.0, 1.0, a1)
    expect = _rhs4_closed_form(u, mu, la, st)
    I = interior(shape, (2, 2, 2))
    for c in range(3):
        e = (expect[c] + uacc_p[c] * Fraction2(int(a1), 1)).grid(shape, origin)
        assert np.array_equal(outs[c][I], e[I]), f"uacc{c}"
        ring = ring_mask(shape, (2, 2, 2))
        assert np.array_equal(outs[c][ring], uacc[c][ring])


def test_rhs4_constant_u_gives_zero():
    from synth import uniform
    shape = (9, 9, 9)
    U = [np.full(shape, 2.5)] * 3
    mu = uniform(shape, 1, 2, "pin", "mu")
    la = uniform(shape, 1, 2, "pin", "la")
    s = [uniform((n,), 0.5, 1.5, "pin", f"s{n}") for n in shape[::-1]]
    zero = [np.zeros(shape)] * 3
    outs = oracle.rhs4(U, mu, la, *s, zero, 0.75, 1 / 6, 1 / 144, 1.0, 0.0)
    I = interior(shape, (2, 2, 2))
    for o in outs:
        assert np.all(o[I] == 0.0)


def test_rhs4_self_adjoint_variable_coefficients():
    """V5: with variable mu, la, str and weight w = 1/(strx stry strz), the SW4
    operator is symmetric: <v, w A u> = <u, w A v> for u, v supported >= 2
    cells inside the interior.  (Catches index errors in mux1..muz4 and in
    the mixed-term inner/outer differences.)"""
    from synth import uniform
    shape = (14, 15, 16)
    nz, ny, nx = shape
    mu = uniform(shape, 1, 2, "pin", "sa-mu")
    la = uniform(shape, 1, 2, "pin", "sa-la")
    strx = uniform((nx,), 0.5, 1.5, "pin", "sa-sx")
    stry = uniform((ny,), 0.5, 1.5, "pin", "sa-sy")
    strz = uniform((nz,), 0.5, 1.5, "pin", "sa-sz")
    sup = np.zeros(shape)
    sup[4:-4, 4:-4, 4:-4] = 1.0
    u = [uniform(shape, -1, 1, "pin", "sa-u", c) * sup for c in range(3)]
    v = [uniform(shape, -1, 1, "pin", "sa-v", c) * sup for c in range(3)]
    zero = [np.zeros(shape)] * 3
    args = (0.75, 1 / 6, 1 / 144, 1.0, 0.0)
    Au = oracle.rhs4(u, mu, la, strx, stry, strz, zero, *args)
    Av = oracle.rhs4(v, mu, la, strx, stry, strz, zero, *args)
    w = 1.0 / (strz[:, None, None] * stry[None, :, None] * strx[None, None, :])
    lhs = sum(np.sum(v[c] * w * Au[c]) for c in range(3))
    rhs = sum(np.sum(u[c] * w * Av[c]) for c in range(3))
    mag = sum(np.sum(np.abs(v[c] * w * Au[c])) for c in range(3))
    assert abs(lhs - rhs) <= 1e-12 * mag
    # and the operator is not trivially symmetric in a broken way: swap mu/la
    Au2 = oracle.rhs4(u, la, mu, strx, stry, strz, zero, *args)
    assert not np.allclose(Au2[0], Au[0])


# --------------------------------------------------------------------------
# abs mode, toys
# --------------------------------------------------------------------------

def test_absmode_bounds_normal_mode():
    """|S(x)| <= S_abs(|x|) pointwise (triangle inequality) for every stencil."""
    from synth import hypterm_inputs, lap25_inputs, rhs4_inputs, uniform
    shape = (12, 13, 14)
    A = uniform(shape, -1, 1, "pin", "abs")
    B = oracle.jacobi7(A, 0.5, -0.25, 4.0)
    Ba = oracle.jacobi7(np.abs(A), 0.5, 0.25, 4.0, absmode=True)
    I = interior(shape, (1, 1, 1))
    assert np.all(np.abs(B[I]) <= Ba[I])
    ins, sc = lap25_inputs(shape, cfg="pin")
    c = list(sc.values())
    B = oracle.lap25(ins["A"], c)
    Ba = oracle.lap25(np.abs(ins["A"]), np.abs(c), absmode=True)
    I = interior(shape, (4, 4, 4))
    assert np.all(np.abs(B[I]) <= Ba[I])
    ins, sc = hypterm_inputs(shape, cfg="pin")
    arrs = list(ins.values())
    s = list(sc.values())
    F = oracle.hypterm(arrs, s[:3], s[3:])
    Fa = oracle.hypterm([np.abs(a) for a in arrs], np.abs(s[:3]), np.abs(s[3:]), absmode=True)
    for f, fa in zip(F, Fa):
        assert np.all(np.abs(f[I]) <= fa[I])
        assert np.all(fa[I] > 0)
    ins, sc = rhs4_inputs(shape, cfg="pin")
    R = oracle.rhs4([ins["u0"], ins["u1"], ins["u2"]], ins["mu"], ins["la"], ins["strx"], ins["stry"],
                    ins["strz"], [ins["uacc0"], ins["uacc1"], ins["uacc2"]], *sc.values())
    Ra = oracle.rhs4([np.abs(ins[k]) for k in ("u0", "u1", "u2")], np.abs(ins["mu"]), np.abs(ins["la"]),
                     ins["strx"], ins["stry"], ins["strz"], [np.abs(ins[f"uacc{c}"]) for c in range(3)],
                     *np.abs(list(sc.values())), absmode=True)
    I = interior(shape, (2, 2, 2))
    for r, ra in zip(R, Ra):
        assert np.all(np.abs(r[I]) <= ra[I])


@pytest.mark.parametrize("off", [(0, 0, 1), (0, 0, -2), (0, 3, 0), (-1, 0, 0), (2, -1, 3), (-4, 4, -4)])
def test_shift_is_a_plain_translation(off):
    shape = (10, 11, 12)
    A = np.arange(np.prod(shape), dtype=np.float64).reshape(shape)
    B = oracle.shift(A, off, out=np.full(shape, -1.0))
    R = [abs(o) for o in off]
    for k in range(shape[0]):
        for j in range(shape[1]):
            for i in range(shape[2]):
                inside = all(R[a] <= (k, j, i)[a] < shape[a] - R[a] for a in range(3))
                want = A[k + off[0], j + off[1], i + off[2]] if inside else -1.0
                assert B[k, j, i] == want


def test_j1d3pt_fig1a_golden():
    vals = {}
    with open(os.path.join(HERE, "golden", "j1d3pt_fig1a.txt")) as f:
        for line in f:
            if line.startswith("#") or not line.strip():
                continue
            k, *v = line.split()
            vals[k] = [float(x) for x in v]
    N, c, T = int(vals["N"][0]), vals["c"][0], int(vals["T"][0])
    A = np.array([vals["init"], vals["init"]])
    res = oracle.j1d3pt(A, c, T)
    assert list(res) == vals["expect"]
    assert N == len(res)

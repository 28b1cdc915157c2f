"""Integer-exact input cases of the five BASELINE DAGs (the closed forms of
tests/test_gpu_exact.py): integer/dyadic polynomial inputs whose stencil image
is known exactly (tests/polyexact.py), with the abs-mode bound that proves
every partial sum stays below 2^53.  No torch, no CUDA: the CPU suite checks
every case against the C oracle (tests/test_exact_cases.py), the GPU suite
runs the same cases through the hand-written kernels."""
from __future__ import annotations

from fractions import Fraction

import numpy as np

import oracle
from polyexact import Poly, laplacian, random_poly

TWO53 = 2.0 ** 53


def _centre(shape):
    return tuple(n // 2 for n in shape)


def _lap25_case(shape, rng, full):
    o = _centre(shape)
    if full:  # total degree <= 4, small coefficients: 5040*|c0|*max|p| << 2^53 at 512^3
        p = random_poly(rng, (4, 4, 4), max_total=4, coef=1, nterms=6)
    else:
        p = random_poly(rng, (5, 4, 4), max_total=5, coef=2, nterms=8)  # per-axis degree <= 5 on the 136-wide grid
    A = p.grid_fast(shape, o)
    exp = (laplacian(p) * 5040).grid_fast(shape, o)
    return dict(ins=[A], a1d=[], s=[-43050.0, 8064.0, -1008.0, 128.0, -9.0], exp=[exp], inout=None,
                absmode=lambda: [oracle.lap25(np.abs(A), [43050.0, 8064.0, 1008.0, 128.0, 9.0], absmode=True)],
                orc=lambda: [oracle.lap25(A, [-43050.0, 8064.0, -1008.0, 128.0, -9.0])])


def _smooth27_case(shape, rng, full):
    o = _centre(shape)
    p = random_poly(rng, (3, 3, 3), max_total=3, coef=3, nterms=14)
    A = p.grid_fast(shape, o)
    exp = (p + laplacian(p) * Fraction(30, 32)).grid_fast(shape, o)
    w = [-128.0, 14.0, 3.0, 1.0]
    return dict(ins=[A], a1d=[], s=[*w, 1.0 / 32.0], exp=[exp], inout=None,
                absmode=lambda: [oracle.smooth27(np.abs(A), np.abs(w), 1.0 / 32.0, absmode=True)],
                orc=lambda: [oracle.smooth27(A, w, 1.0 / 32.0)])


def _jacobi7_case(shape, rng, full):
    o = _centre(shape)
    p = random_poly(rng, (3, 3, 3), coef=4, nterms=12)
    A = p.grid_fast(shape, o)
    exp = (p * Fraction(1, 2) - laplacian(p)).grid_fast(shape, o)
    return dict(ins=[A], a1d=[], s=[4.0, 0.5, 0.25], exp=[exp], inout=None,
                absmode=lambda: [oracle.jacobi7(np.abs(A), 0.5, 0.25, 4.0, absmode=True)],
                orc=lambda: [oracle.jacobi7(A, 0.5, 0.25, 4.0)])


def _hypterm_closed_form(cons, q, dxinv):
    V = [q[0], q[1], q[2]]
    F = [[cons[0], cons[1], cons[2]]]
    for m in range(3):
        F.append([cons[m] * V[a] + (q[3] if a == m else 0) for a in range(3)])
    F.append([(cons[3] + q[3]) * V[a] for a in range(3)])
    out = []
    for Fm in F:
        acc = Poly()
        for a in range(3):
            acc = acc + Fm[a].diff(a) * Fraction(dxinv[a])
        out.append(acc * (-840))
    return out


def _hypterm_case(shape, rng, full, dxinv=(1.0, 1.0, 1.0)):
    o = _centre(shape)
    kw = dict(max_total=2, coef=1, nterms=4) if full else dict(max_total=2, coef=3, nterms=6)
    cons = [random_poly(rng, (2, 2, 2), **kw) for _ in range(4)]
    q = [random_poly(rng, (2, 2, 2), **kw) for _ in range(4)]
    ins = [p.grid_fast(shape, o) for p in (*cons, *q)]
    exp = [e.grid_fast(shape, o) for e in _hypterm_closed_form(cons, q, dxinv)]
    c = [672.0, -168.0, 32.0, -3.0]
    return dict(ins=ins, a1d=[], s=[*dxinv, *c], exp=exp, inout=None,
                absmode=lambda: oracle.hypterm([np.abs(x) for x in ins], np.abs(dxinv), np.abs(c), absmode=True),
                orc=lambda: oracle.hypterm(ins, dxinv, c))


def _rhs4_closed_form(u, mu, la, st):
    out = []
    for c in range(3):
        acc = Poly()
        for b in range(3):
            K = (mu * 2 + la) * st[c] if b == c else mu * st[b]
            acc = acc + st[b] * (K * u[c].diff(b)).diff(b)
        for b in range(3):
            if b != c:
                acc = acc + st[c] * st[b] * ((la * u[b].diff(b)).diff(c) + (mu * u[b].diff(c)).diff(b))
        out.append(acc * 144)
    return out


def _rhs4_case(shape, rng, full, a1=1.0):
    o = _centre(shape)
    oz, oy, ox = o
    if full:  # keep every SW4 partial sum < 2^53 at 320^3 (checked below by the abs-mode bound)
        u = [random_poly(rng, (2, 2, 2), max_total=2, coef=1, nterms=4) for _ in range(3)]
        mu = Poly({(0, 0, 0): rng.randint(2, 4), (1, 0, 0): rng.choice([-1, 1])})
        la = Poly({(0, 0, 0): rng.randint(2, 4), (0, 1, 0): rng.choice([-1, 1])})
        st = [Poly({(0, 0, 0): 1}), Poly({(0, 0, 0): 2}),
              Poly({(0, 0, 0): rng.randint(3, 5), (0, 0, 1): rng.choice([-1, 1])})]
    else:
        u = [random_poly(rng, (3, 3, 3), max_total=3, coef=3, nterms=10) for _ in range(3)]
        mu = Poly({(0, 0, 0): rng.randint(5, 9), (1, 0, 0): rng.randint(-2, 2), (0, 1, 0): rng.randint(-2, 2),
                   (0, 0, 1): rng.randint(-2, 2)})
        la = Poly({(0, 0, 0): rng.randint(5, 9), (1, 0, 0): rng.randint(-2, 2), (0, 1, 0): rng.randint(-2, 2),
                   (0, 0, 1): rng.randint(-2, 2)})
        st = [Poly({(0, 0, 0): rng.randint(3, 5), tuple(1 if a == b else 0 for a in range(3)): rng.choice([-1, 1])})
              for b in range(3)]
    nz, ny, nx = shape

    def line(p, axis, n, org):
        e = tuple(1 if a == axis else 0 for a in range(3))
        return np.array([float(p.c.get((0, 0, 0), 0) + p.c.get(e, 0) * (t - org)) for t in range(n)])

    strx, stry, strz = line(st[0], 0, nx, ox), line(st[1], 1, ny, oy), line(st[2], 2, nz, oz)
    U = [p.grid_fast(shape, o) for p in u]
    M, L = mu.grid_fast(shape, o), la.grid_fast(shape, o)
    ua_p = [random_poly(rng, (1, 1, 1), coef=3, nterms=3) for _ in range(3)]
    UA = [p.grid_fast(shape, o) for p in ua_p]
    exp = [(e + q * Fraction(int(a1), 1)).grid_fast(shape, o) for e, q in zip(_rhs4_closed_form(u, mu, la, st), ua_p)]
    s = [0.75, 24.0, 1.0, 1.0, a1]
    return dict(ins=[*U, M, L], a1d=[strx, stry, strz], s=s, exp=exp, inout=UA,
                absmode=lambda: oracle.rhs4([np.abs(x) for x in U], np.abs(M), np.abs(L), np.abs(strx), np.abs(stry),
                                            np.abs(strz), [np.abs(x) for x in UA], *np.abs(s), absmode=True),
                orc=lambda: oracle.rhs4(U, M, L, strx, stry, strz, UA, *s))


CASES = {"lap25": _lap25_case, "smooth27": _smooth27_case, "jacobi7": _jacobi7_case,
         "hypterm": _hypterm_case, "rhs4center": _rhs4_case}


def check_bound(case):
    for a in case["absmode"]():
        # margin 8: a kernel may form a scaled sub-sum (e.g. before a *3/4) above its share
        assert float(np.max(a)) < TWO53 / 8, "inputs too large for an exact test"


MULTI_TILE = {"lap25": (30, 70, 136), "smooth27": (21, 70, 136), "jacobi7": (21, 70, 136),
              "hypterm": (21, 38, 136), "rhs4center": (17, 38, 70)}

FULL = {"lap25": (512, 512, 512), "hypterm": (320, 320, 320), "rhs4center": (320, 320, 320),
        "smooth27": (512, 512, 512)}

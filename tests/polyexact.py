"""Exact multivariate polynomial arithmetic for the oracle pins.

Polynomials in (x, y, z) <-> grid axes (i, j, k) with integer (or Fraction)
coefficients.  Used to build inputs whose stencil image has a closed form
(continuous derivatives of a polynomial), evaluated exactly on the grid.
Independent of oracle/ and of the CUDA path.
"""
from __future__ import annotations

import random
from fractions import Fraction

import numpy as np


class Poly:
    __slots__ = ("c",)

    def __init__(self, c=None):
        self.c = {k: Fraction(v) for k, v in (c or {}).items() if v != 0}

    @staticmethod
    def const(v):
        return Poly({(0, 0, 0): v})

    @staticmethod
    def var(axis):  # axis 0=x(i) 1=y(j) 2=z(k)
        e = [0, 0, 0]
        e[axis] = 1
        return Poly({tuple(e): 1})

    def __add__(self, o):
        o = o if isinstance(o, Poly) else Poly.const(o)
        r = dict(self.c)
        for k, v in o.c.items():
            r[k] = r.get(k, 0) + v
        return Poly(r)

    __radd__ = __add__

    def __neg__(self):
        return Poly({k: -v for k, v in self.c.items()})

    def __sub__(self, o):
        return self + (-(o if isinstance(o, Poly) else Poly.const(o)))

    def __rsub__(self, o):
        return (-self) + o

    def __mul__(self, o):
        if not isinstance(o, Poly):
            return Poly({k: v * Fraction(o) for k, v in self.c.items()})
        r = {}
        for k1, v1 in self.c.items():
            for k2, v2 in o.c.items():
                k = (k1[0] + k2[0], k1[1] + k2[1], k1[2] + k2[2])
                r[k] = r.get(k, 0) + v1 * v2
        return Poly(r)

    __rmul__ = __mul__

    def diff(self, axis):
        r = {}
        for k, v in self.c.items():
            if k[axis] > 0:
                e = list(k)
                e[axis] -= 1
                r[tuple(e)] = r.get(tuple(e), 0) + v * k[axis]
        return Poly(r)

    def degree(self, axis=None):
        if not self.c:
            return 0
        if axis is None:
            return max(sum(k) for k in self.c)
        return max(k[axis] for k in self.c)

    def grid(self, shape, origin):
        """Exact values on the grid [nz][ny][nx] with x=i-ox, y=j-oy, z=k-oz.
        Returns float64; asserts every value (and partial sum) is an integer
        or dyadic of magnitude < 2^53 so the float is exact."""
        nz, ny, nx = shape
        oz, oy, ox = origin
        z = np.arange(nz, dtype=object)[:, None, None] - oz
        y = np.arange(ny, dtype=object)[None, :, None] - oy
        x = np.arange(nx, dtype=object)[None, None, :] - ox
        acc = np.zeros(shape, dtype=object)
        for (a, b, c), v in self.c.items():
            acc = acc + v * (x ** a) * (y ** b) * (z ** c)
        flat = acc.ravel()
        out = np.empty(flat.shape, dtype=np.float64)
        for n, q in enumerate(flat):
            q = Fraction(q)
            f = float(q)
            assert Fraction(f) == q, f"value {q} not exactly representable"
            assert abs(f) < 2.0 ** 53
            out[n] = f
        return out.reshape(shape)


    def grid_fast(self, shape, origin):
        """Same values as grid() for large grids: every coefficient must be a
        dyadic rational (denominator 2^e); D*p is evaluated in int64 numpy and
        divided by D = 2^e in float64 (exact).  The a-priori bound
        sum |D c| max|x|^a max|y|^b max|z|^c < 2^53 is asserted first, so no
        partial sum can overflow int64 or lose a bit in the final float."""
        D = 1
        for v in self.c.values():
            d = Fraction(v).denominator
            assert d & (d - 1) == 0, f"coefficient {v} is not dyadic"
            D = max(D, d)
        nz, ny, nx = shape
        oz, oy, ox = origin
        mx = max(abs(0 - ox), abs(nx - 1 - ox))
        my = max(abs(0 - oy), abs(ny - 1 - oy))
        mz = max(abs(0 - oz), abs(nz - 1 - oz))
        bound = sum(abs(int(Fraction(v) * D)) * mx ** a * my ** b * mz ** c for (a, b, c), v in self.c.items())
        assert bound < 2 ** 53, f"grid values may reach {bound} >= 2^53"
        x = np.arange(nx, dtype=np.int64) - ox
        y = np.arange(ny, dtype=np.int64) - oy
        z = np.arange(nz, dtype=np.int64) - oz
        acc = np.zeros(shape, dtype=np.int64)
        for (a, b, c), v in self.c.items():
            cv = int(Fraction(v) * D)
            yz = (cv * z[:, None] ** c) * (y[None, :] ** b)  # [nz][ny]
            acc += yz[:, :, None] * (x ** a)[None, None, :]
        out = acc.astype(np.float64)
        if D != 1:
            out /= float(D)
        return out

    def bound(self, shape, origin):
        """max over the grid of sum |c| |x|^a |y|^b |z|^c (exact, Fraction)."""
        nz, ny, nx = shape
        oz, oy, ox = origin
        mx = max(ox, nx - 1 - ox)
        my = max(oy, ny - 1 - oy)
        mz = max(oz, nz - 1 - oz)
        return sum(abs(Fraction(v)) * mx ** a * my ** b * mz ** c for (a, b, c), v in self.c.items())


def random_poly(rng: random.Random, max_deg_axis=(3, 3, 3), max_total=None, coef=3, nterms=8) -> Poly:
    terms = {}
    for _ in range(nterms):
        e = tuple(rng.randint(0, max_deg_axis[a]) for a in range(3))
        if max_total is not None and sum(e) > max_total:
            continue
        terms[e] = terms.get(e, 0) + rng.choice([v for v in range(-coef, coef + 1) if v != 0])
    terms[(0, 0, 0)] = terms.get((0, 0, 0), 0) + rng.randint(-coef, coef)
    return Poly(terms)


def laplacian(p: Poly) -> Poly:
    return p.diff(0).diff(0) + p.diff(1).diff(1) + p.diff(2).diff(2)

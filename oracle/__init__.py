"""CPU oracle for the sdag stencil DAGs -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline``
/ ``--impl reference`` legs may import this package.  The product package
``paper_conf_ipps_rawatvsrps19_b200`` never imports it; the two share no code.

The arithmetic lives in ``oracle.c`` (plain C loop nests, fp64, no FMA
contraction; each function cites the PAPER.md passage / SURVEY reading it
follows).  This module only builds the shared library with gcc and marshals
numpy arrays into it.

Parity status per function:
  jacobi7, lap25, smooth27 (+iter, +iter_points), hypterm, rhs4, shift, j1d3pt:
  pinned by tests/test_oracle_pins.py (closed forms on polynomials, invariants,
  symmetries, self-adjointness, hand-expanded toys).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# SDAG_ORACLE_SRC / SDAG_ORACLE_LIB: mutation testing of the pins only.
_SRC = os.environ.get("SDAG_ORACLE_SRC", os.path.join(_HERE, "oracle.c"))
_LIB = os.environ.get("SDAG_ORACLE_LIB", os.path.join(_HERE, "liboracle.so"))
_lock = threading.Lock()
_lib = None

CFLAGS = ["-O2", "-fopenmp", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared", "-std=c11"]


def build(force: bool = False) -> str:
    """Compile oracle.c -> liboracle.so (gcc, strict fp64)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


def lib():
    global _lib
    with _lock:
        if _lib is None:
            build()
            _lib = ctypes.CDLL(_LIB)
            _setup(_lib)
    return _lib


_dp = ctypes.POINTER(ctypes.c_double)
_i64p = ctypes.POINTER(ctypes.c_int64)
_i64 = ctypes.c_int64


def _setup(L):
    sig = {
        "orc_jacobi7": [_dp, _dp, _i64p, _dp, ctypes.c_int, _i64, _i64],
        "orc_lap25": [_dp, _dp, _i64p, _dp, ctypes.c_int, _i64, _i64],
        "orc_smooth27": [_dp, _dp, _i64p, _dp, ctypes.c_int, _i64, _i64],
        "orc_jacobi7_points": [_dp, _i64p, _dp, ctypes.c_int, _i64p, _i64, _dp],
        "orc_lap25_points": [_dp, _i64p, _dp, ctypes.c_int, _i64p, _i64, _dp],
        "orc_smooth27_points": [_dp, _i64p, _dp, ctypes.c_int, _i64p, _i64, _dp],
        "orc_smooth27_iter": [_dp, _dp, _i64p, _dp, ctypes.c_int, ctypes.c_int],
        "orc_smooth27_iter_points": [_dp, _i64p, _dp, ctypes.c_int, ctypes.c_int, _i64p, _i64, _dp],
        "orc_hypterm": [ctypes.c_void_p, ctypes.c_void_p, _i64p, _dp, ctypes.c_int, _i64, _i64],
        "orc_hypterm_points": [ctypes.c_void_p, _i64p, _dp, ctypes.c_int, _i64p, _i64, _dp],
        "orc_rhs4": [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, _i64p, _dp,
                     ctypes.c_int, _i64, _i64],
        "orc_rhs4_points": [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, _i64p, _dp, ctypes.c_int,
                            _i64p, _i64, _dp],
        "orc_shift": [_dp, _dp, _i64p, _i64p, _i64, _i64],
        "orc_j1d3pt": [_dp, _i64, ctypes.c_double, ctypes.c_int],
    }
    for name, args in sig.items():
        f = getattr(L, name)
        f.argtypes = args
        f.restype = None


def _d(a: np.ndarray):
    assert a.dtype == np.float64 and a.flags.c_contiguous
    return a.ctypes.data_as(_dp)


def _dims(shape):
    assert len(shape) == 3
    return (ctypes.c_int64 * 3)(*shape)


def _scal(s):
    s = np.ascontiguousarray(s, dtype=np.float64)
    return s, _d(s)


def _ptrs(arrs):
    for a in arrs:
        assert a.dtype == np.float64 and a.flags.c_contiguous
    return (ctypes.c_void_p * len(arrs))(*[a.ctypes.data for a in arrs])


def _pts(pts):
    pts = np.ascontiguousarray(pts, dtype=np.int64).reshape(-1, 3)
    return pts, pts.ctypes.data_as(_i64p), len(pts)


def _out_like(A, out):
    if out is None:
        out = np.zeros_like(A)
    return out


def _kr(krange):
    return (-1, -1) if krange is None else (int(krange[0]), int(krange[1]))


# ---- single-input stencils -------------------------------------------------

def _single(name, A, scal, absmode, out, krange):
    A = np.ascontiguousarray(A, dtype=np.float64)
    out = _out_like(A, out)
    s, sp = _scal(scal)
    getattr(lib(), name)(_d(A), _d(out), _dims(A.shape), sp, int(absmode), *_kr(krange))
    return out


def _single_points(name, A, scal, absmode, pts):
    A = np.ascontiguousarray(A, dtype=np.float64)
    s, sp = _scal(scal)
    pts, pp, n = _pts(pts)
    res = np.empty(n, dtype=np.float64)
    getattr(lib(), name)(_d(A), _dims(A.shape), sp, int(absmode), pp, n, _d(res))
    return res


def jacobi7(A, a, b, h2inv, absmode=False, out=None, krange=None):
    """Listing 1.  Returns B (ring of ``out`` untouched; zeros if new)."""
    return _single("orc_jacobi7", A, [a, b, h2inv], absmode, out, krange)


def jacobi7_points(A, a, b, h2inv, pts, absmode=False):
    return _single_points("orc_jacobi7_points", A, [a, b, h2inv], absmode, pts)


def lap25(A, c, absmode=False, out=None, krange=None):
    """25-point radius-4 Laplacian, c = (c0..c4)."""
    return _single("orc_lap25", A, c, absmode, out, krange)


def lap25_points(A, c, pts, absmode=False):
    return _single_points("orc_lap25_points", A, c, absmode, pts)


def smooth27(A, w, nu, absmode=False, out=None, krange=None):
    """27-point smoother, w = (w0..w3) (Table I)."""
    return _single("orc_smooth27", A, [*w, nu], absmode, out, krange)


def smooth27_points(A, w, nu, pts, absmode=False):
    return _single_points("orc_smooth27_points", A, [*w, nu], absmode, pts)


def smooth27_iter(A0, w, nu, T, absmode=False):
    """T ping-pong sweeps (Fig 1a); returns buf[T&1]."""
    b0 = np.array(A0, dtype=np.float64, order="C", copy=True)
    b1 = b0.copy()
    s, sp = _scal([*w, nu])
    lib().orc_smooth27_iter(_d(b0), _d(b1), _dims(b0.shape), sp, int(T), int(absmode))
    return b0 if (T & 1) == 0 else b1


def smooth27_iter_points(A0, w, nu, T, pts, absmode=False):
    A0 = np.ascontiguousarray(A0, dtype=np.float64)
    s, sp = _scal([*w, nu])
    pts, pp, n = _pts(pts)
    res = np.empty(n, dtype=np.float64)
    lib().orc_smooth27_iter_points(_d(A0), _dims(A0.shape), sp, int(T), int(absmode), pp, n, _d(res))
    return res


# ---- hypterm ----------------------------------------------------------------

HYPTERM_INPUTS = ("cons_1", "cons_2", "cons_3", "cons_4", "q_1", "q_2", "q_3", "q_4")


def hypterm(ins, dxinv, coefs, absmode=False, outs=None, krange=None):
    """ins: 8 arrays (cons_1..4, q_1..4); dxinv: 3; coefs: (ALP,BET,GAM,DEL).
    Returns the 5 flux arrays (Table I)."""
    ins = [np.ascontiguousarray(a, dtype=np.float64) for a in ins]
    assert len(ins) == 8
    if outs is None:
        outs = [np.zeros_like(ins[0]) for _ in range(5)]
    s, sp = _scal([*dxinv, *coefs])
    ip, op = _ptrs(ins), _ptrs(outs)
    lib().orc_hypterm(ip, op, _dims(ins[0].shape), sp, int(absmode), *_kr(krange))
    return outs


def hypterm_points(ins, dxinv, coefs, pts, absmode=False):
    ins = [np.ascontiguousarray(a, dtype=np.float64) for a in ins]
    s, sp = _scal([*dxinv, *coefs])
    pts, pp, n = _pts(pts)
    res = np.empty((n, 5), dtype=np.float64)
    lib().orc_hypterm_points(_ptrs(ins), _dims(ins[0].shape), sp, int(absmode), pp, n, _d(res))
    return res


# ---- rhs4center ---------------------------------------------------------------

def rhs4(u, mu, la, strx, stry, strz, uacc, tf, i6, i144, cof, a1, absmode=False, outs=None, krange=None):
    """SW4 rhs4center (Table I).  u, uacc: 3 arrays each.
    Returns the 3 new uacc arrays (ring copied from the old uacc)."""
    in3 = [np.ascontiguousarray(a, dtype=np.float64) for a in (*u, mu, la)]
    in1 = [np.ascontiguousarray(a, dtype=np.float64) for a in (strx, stry, strz)]
    ua = [np.ascontiguousarray(a, dtype=np.float64) for a in uacc]
    if outs is None:
        outs = [a.copy() for a in ua]
    s, sp = _scal([tf, i6, i144, cof, a1])
    lib().orc_rhs4(_ptrs(in3), _ptrs(in1), _ptrs(ua), _ptrs(outs), _dims(in3[0].shape), sp, int(absmode),
                   *_kr(krange))
    return outs


def rhs4_points(u, mu, la, strx, stry, strz, uacc, tf, i6, i144, cof, a1, pts, absmode=False):
    in3 = [np.ascontiguousarray(a, dtype=np.float64) for a in (*u, mu, la)]
    in1 = [np.ascontiguousarray(a, dtype=np.float64) for a in (strx, stry, strz)]
    ua = [np.ascontiguousarray(a, dtype=np.float64) for a in uacc]
    s, sp = _scal([tf, i6, i144, cof, a1])
    pts, pp, n = _pts(pts)
    res = np.empty((n, 3), dtype=np.float64)
    lib().orc_rhs4_points(_ptrs(in3), _ptrs(in1), _ptrs(ua), _dims(in3[0].shape), sp, int(absmode), pp, n,
                          _d(res))
    return res


# ---- toys -------------------------------------------------------------------

def shift(A, off, out=None, krange=None):
    A = np.ascontiguousarray(A, dtype=np.float64)
    out = _out_like(A, out)
    o = (ctypes.c_int64 * 3)(*[int(x) for x in off])
    lib().orc_shift(_d(A), _d(out), _dims(A.shape), o, *_kr(krange))
    return out


def j1d3pt(A2N, c, T):
    """Fig 1a.  A2N: [2][N] array, modified in place; returns A[T%2]."""
    A = np.ascontiguousarray(A2N, dtype=np.float64)
    assert A.ndim == 2 and A.shape[0] == 2
    lib().orc_j1d3pt(_d(A), A.shape[1], float(c), int(T))
    return A[T % 2]

"""Seeded synthetic inputs shared by the oracle tests, the GPU parity tests and
bench.py.  Holds NO stencil arithmetic -- only a counter-based generator
(splitmix64) and the per-config input recipes of SURVEY 8(d) / DESIGN.md
"Input recipe".

value(seed, key, n) = lo + (hi - lo) * (splitmix64(seed ^ key_hash + n) >> 11) * 2^-53

so any element can be regenerated independently (no sequential state), and
the same bytes go to the oracle and (copied) to the GPU.
"""
from __future__ import annotations

import hashlib

import numpy as np

MASTER_SEED = 20190520  # SURVEY 8(d) "Inputs"

_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)
_GOLD = np.uint64(0x9E3779B97F4A7C15)


def key_hash(*key) -> int:
    h = hashlib.sha256(repr(key).encode()).digest()
    return int.from_bytes(h[:8], "little")


def splitmix64(x: np.ndarray) -> np.ndarray:
    """Vectorised splitmix64 finaliser of (x + golden); x uint64."""
    with np.errstate(over="ignore"):
        z = x + _GOLD
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
        z = z ^ (z >> np.uint64(31))
    return z


def uniform(shape, lo: float, hi: float, *key, seed: int = MASTER_SEED, chunk: int = 1 << 24) -> np.ndarray:
    """Uniform doubles in [lo, hi) keyed by (seed, key); element n uses counter n."""
    n = int(np.prod(shape))
    base = np.uint64((seed ^ key_hash(*key)) & 0xFFFFFFFFFFFFFFFF)
    out = np.empty(n, dtype=np.float64)
    scale = (hi - lo) * 2.0 ** -53
    for s in range(0, n, chunk):
        e = min(n, s + chunk)
        with np.errstate(over="ignore"):
            ctr = np.arange(s, e, dtype=np.uint64) + base
        z = splitmix64(ctr) >> np.uint64(11)
        out[s:e] = z.astype(np.float64) * scale + lo
    return out.reshape(shape)


def uniform_at(lin_index, lo: float, hi: float, *key, seed: int = MASTER_SEED) -> np.ndarray:
    """The elements of uniform(shape, lo, hi, *key) at the given C-order linear
    indices (counter-based: no need to generate the whole array)."""
    idx = np.asarray(lin_index, dtype=np.uint64)
    base = np.uint64((seed ^ key_hash(*key)) & 0xFFFFFFFFFFFFFFFF)
    with np.errstate(over="ignore"):
        z = splitmix64(idx + base) >> np.uint64(11)
    return z.astype(np.float64) * ((hi - lo) * 2.0 ** -53) + lo


def uniform_torch(shape, lo: float, hi: float, *key, seed: int = MASTER_SEED, device="cuda", chunk: int = 1 << 26):
    """Same values as uniform(), generated on a torch device (for grids too large
    to build on the host).  int64 two's-complement arithmetic reproduces the
    uint64 splitmix64 bit for bit (logical shifts are masked)."""
    import torch

    n = int(np.prod(shape))
    base = (seed ^ key_hash(*key)) & 0xFFFFFFFFFFFFFFFF

    def s64(v):  # uint64 constant -> int64 bit pattern
        return v - (1 << 64) if v >= (1 << 63) else v

    m1, m2, gold = s64(0xBF58476D1CE4E5B9), s64(0x94D049BB133111EB), s64(0x9E3779B97F4A7C15)

    def lsr(x, s):
        return (x >> s) & ((1 << (64 - s)) - 1)

    out = torch.empty(n, dtype=torch.float64, device=device)
    scale = (hi - lo) * 2.0 ** -53
    for s0 in range(0, n, chunk):
        e = min(n, s0 + chunk)
        z = torch.arange(s0, e, dtype=torch.int64, device=device)
        z = z + s64(base)
        z = z + gold
        z = (z ^ lsr(z, 30)) * m1
        z = (z ^ lsr(z, 27)) * m2
        z = z ^ lsr(z, 31)
        z = lsr(z, 11)
        out[s0:e] = z.to(torch.float64) * scale + lo
    return out.view(*shape)


def integers(shape, lo: int, hi: int, *key, seed: int = MASTER_SEED) -> np.ndarray:
    """Uniform integers in [lo, hi) as float64 (exact), keyed like uniform()."""
    n = int(np.prod(shape))
    base = np.uint64((seed ^ key_hash(*key)) & 0xFFFFFFFFFFFFFFFF)
    with np.errstate(over="ignore"):
        ctr = np.arange(n, dtype=np.uint64) + base
    z = splitmix64(ctr) % np.uint64(hi - lo)
    return (z.astype(np.int64) + lo).astype(np.float64).reshape(shape)


# ---------------------------------------------------------------------------
# Input recipes.  Each returns a
# dict name -> numpy array plus the scalar list, in the stencil's formal order.
# ---------------------------------------------------------------------------

def jacobi7_inputs(dims, cfg="cfg1", batch=None):
    shape = tuple(dims) if batch is None else (batch, *dims)
    A = uniform(shape, -1.0, 1.0, cfg, "A")
    return {"A": A}, {"a": 0.5, "b": 0.25, "h2inv": 4.0}


LAP25_COEFS = {
    "c0": -205.0 / 24.0, "c1": 8.0 / 5.0, "c2": -1.0 / 5.0, "c3": 8.0 / 315.0, "c4": -1.0 / 560.0,
}
LAP25_COEFS_X5040 = {"c0": -43050.0, "c1": 8064.0, "c2": -1008.0, "c3": 128.0, "c4": -9.0}


def lap25_inputs(dims, cfg="cfg2"):
    return {"A": uniform(tuple(dims), -1.0, 1.0, cfg, "A")}, dict(LAP25_COEFS)


SMOOTH27_W = {"w0": -128.0 / 30.0, "w1": 14.0 / 30.0, "w2": 3.0 / 30.0, "w3": 1.0 / 30.0, "nu": 1.0 / 8.0}
SMOOTH27_W_INT = {"w0": -128.0, "w1": 14.0, "w2": 3.0, "w3": 1.0, "nu": 1.0 / 32.0}


def smooth27_inputs(dims, cfg="cfg5"):
    return {"A": uniform(tuple(dims), -1.0, 1.0, cfg, "A")}, dict(SMOOTH27_W)


HYPTERM_C = {"ALP": 0.8, "BET": -0.2, "GAM": 4.0 / 105.0, "DEL": -1.0 / 280.0}
HYPTERM_C_X840 = {"ALP": 672.0, "BET": -168.0, "GAM": 32.0, "DEL": -3.0}


def hypterm_inputs(dims, cfg="cfg3"):
    d = tuple(dims)
    ins = {}
    for m in (1, 2, 3, 4):
        ins[f"cons_{m}"] = uniform(d, 0.5, 1.5, cfg, f"cons_{m}")
    for m in (1, 2, 3):
        ins[f"q_{m}"] = uniform(d, -1.0, 1.0, cfg, f"q_{m}")
    ins["q_4"] = uniform(d, 0.5, 1.5, cfg, "q_4")
    scal = {"dxinv0": 0.5, "dxinv1": 0.25, "dxinv2": 0.125, **HYPTERM_C}
    return ins, scal


def rhs4_inputs(dims, cfg="cfg4"):
    d = tuple(dims)
    nz, ny, nx = d
    ins = {
        "u0": uniform(d, -1.0, 1.0, cfg, "u0"),
        "u1": uniform(d, -1.0, 1.0, cfg, "u1"),
        "u2": uniform(d, -1.0, 1.0, cfg, "u2"),
        "mu": uniform(d, 1.0, 2.0, cfg, "mu"),
        "la": uniform(d, 1.0, 2.0, cfg, "la"),
        "strx": uniform((nx,), 0.5, 1.5, cfg, "strx"),
        "stry": uniform((ny,), 0.5, 1.5, cfg, "stry"),
        "strz": uniform((nz,), 0.5, 1.5, cfg, "strz"),
        "uacc0": uniform(d, -1.0, 1.0, cfg, "uacc0"),
        "uacc1": uniform(d, -1.0, 1.0, cfg, "uacc1"),
        "uacc2": uniform(d, -1.0, 1.0, cfg, "uacc2"),
    }
    scal = {"tf": 0.75, "i6": 1.0 / 6.0, "i144": 1.0 / 144.0, "cof": 1.0, "a1": 1.0}
    return ins, scal


# ---------------------------------------------------------------------------
# The same recipes as data (bench.py builds the BASELINE-size inputs on the
# device from these with uniform_torch -- bit-identical to the *_inputs()
# arrays of the same cfg key, checked by tests/test_synth.py).
# recipe(name) -> (cfg key, {3D array: (lo, hi)}, {1D array: (lo, hi)}, scalars)
# ---------------------------------------------------------------------------

_RECIPES = {
    "jacobi7": ("cfg1", {"A": (-1.0, 1.0)}, {}, {"a": 0.5, "b": 0.25, "h2inv": 4.0}),
    "lap25": ("cfg2", {"A": (-1.0, 1.0)}, {}, LAP25_COEFS),
    "smooth27": ("cfg5", {"A": (-1.0, 1.0)}, {}, SMOOTH27_W),
    "hypterm": ("cfg3", {"cons_1": (0.5, 1.5), "cons_2": (0.5, 1.5), "cons_3": (0.5, 1.5), "cons_4": (0.5, 1.5),
                         "q_1": (-1.0, 1.0), "q_2": (-1.0, 1.0), "q_3": (-1.0, 1.0), "q_4": (0.5, 1.5)}, {},
                {"dxinv0": 0.5, "dxinv1": 0.25, "dxinv2": 0.125, **HYPTERM_C}),
    "rhs4center": ("cfg4", {"u0": (-1.0, 1.0), "u1": (-1.0, 1.0), "u2": (-1.0, 1.0), "mu": (1.0, 2.0),
                            "la": (1.0, 2.0), "uacc0": (-1.0, 1.0), "uacc1": (-1.0, 1.0), "uacc2": (-1.0, 1.0)},
                   {"strx": (0.5, 1.5), "stry": (0.5, 1.5), "strz": (0.5, 1.5)},
                   {"tf": 0.75, "i6": 1.0 / 6.0, "i144": 1.0 / 144.0, "cof": 1.0, "a1": 1.0}),
}


def recipe(name):
    cfg, a3, a1, sc = _RECIPES[name]
    return cfg, dict(a3), dict(a1), dict(sc)

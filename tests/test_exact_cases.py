"""The integer-exact cases the GPU bitwise tests use (tests/exactcases.py),
checked here on the CPU: every case stays below 2^53 (abs-mode bound) and the
C oracle reproduces its exact closed form bit for bit on the multi-tile shapes
the GPU tests run -- a further pin of the oracle and a guard
that the GPU tests' expected values are right before a kernel ever sees them."""
from __future__ import annotations

import random

import numpy as np
import pytest

from cases import RADIUS, interior
from exactcases import CASES, MULTI_TILE, _hypterm_case, _rhs4_case, check_bound


def _oracle_equals_closed_form(name, dims, case):
    check_bound(case)
    I = interior(dims, RADIUS[name])
    for m, (o, e) in enumerate(zip(case["orc"](), case["exp"])):
        assert np.array_equal(o[I], e[I]), f"{name} output {m}"


@pytest.mark.parametrize("name", list(CASES))
def test_exact_case_multitile(name):
    dims = MULTI_TILE[name]
    _oracle_equals_closed_form(name, dims, CASES[name](dims, random.Random(sum(map(ord, name))), False))


@pytest.mark.parametrize("dxinv", [(0.5, 0.25, 2.0), (2.0, 0.125, 4.0)])
def test_exact_case_hypterm_dxinv(dxinv):
    dims = MULTI_TILE["hypterm"]
    _oracle_equals_closed_form("hypterm", dims, _hypterm_case(dims, random.Random(17), False, dxinv=dxinv))


@pytest.mark.parametrize("a1", [0.0, 1.0])
def test_exact_case_rhs4_a1(a1):
    dims = MULTI_TILE["rhs4center"]
    _oracle_equals_closed_form("rhs4center", dims, _rhs4_case(dims, random.Random(int(a1) + 40), False, a1=a1))

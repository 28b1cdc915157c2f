"""NEXT-1 host logic on CPU: the temporal-fusion schedule of the C library
(sdag_fusion_schedule, deep tuning's DP opt(T) = min_x f(x) + opt(T - x),
P:1416-1440, plus the ping-pong parity constraint of apply_iterated) against
brute force over every composition of T into launch degrees."""
from __future__ import annotations

import itertools

import pytest

import paper_conf_ipps_rawatvsrps19_b200 as sdag


def brute(f, T):
    """Cheapest composition of T (ordered parts in f) with #parts == T (mod 2)."""
    best = None
    degs = sorted(f)

    def rec(rem, parts):
        nonlocal best
        if rem == 0:
            if len(parts) % 2 == T % 2:
                c = sum(f[d] for d in parts)
                if best is None or c < best - 1e-12:
                    best = c
            return
        for d in degs:
            if d <= rem:
                rec(rem - d, parts + [d])

    rec(T, [])
    return best


COSTS = [
    {1: 1.0},
    {1: 1.0, 2: 1.15},
    {1: 1.0, 2: 1.73},
    {1: 1.0, 2: 2.5},  # fusion slower than two sweeps: never used
    {1: 1.0, 2: 1.2, 3: 1.5},
    {1: 1.0, 3: 1.4},
    {1: 1.0, 2: 1.9, 4: 2.2},
]


@pytest.mark.parametrize("f", COSTS, ids=lambda f: "_".join(f"{k}:{v}" for k, v in f.items()))
@pytest.mark.parametrize("T", list(range(0, 13)))
def test_schedule_is_optimal_and_valid(f, T):
    seq, cost = sdag.fusion_schedule(f, T)
    assert sum(seq) == T
    assert len(seq) % 2 == T % 2  # the result lands in buf[T & 1]
    assert all(d in f for d in seq)
    assert cost == pytest.approx(sum(f[d] for d in seq))
    assert cost == pytest.approx(brute(f, T))


def test_schedule_examples():
    f = {1: 1.0, 2: 1.15}
    assert sdag.fusion_schedule(f, 12)[0] == [2] * 6
    s5 = sdag.fusion_schedule(f, 5)[0]
    assert sorted(s5) == [1, 2, 2]
    # a single 2-sweep launch cannot land in buf[0]: T = 2 -> two sweeps
    assert sdag.fusion_schedule(f, 2)[0] == [1, 1]
    assert sdag.fusion_schedule(f, 3)[0] == [1, 1, 1]
    assert sdag.fusion_schedule({1: 1.0, 2: 2.5}, 8)[0] == [1] * 8


@pytest.mark.parametrize("bad", [
    dict(f={1: 0.0, 2: 1.0}, T=4),   # no single-sweep kernel
    dict(f={1: 1.0}, T=-1),
    dict(f={1: 1.0, 9: 1.0}, T=4),   # maxdeg out of range
])
def test_schedule_errors(bad):
    with pytest.raises(sdag.SdagError):
        sdag.fusion_schedule(bad["f"], bad["T"])


def test_compositions_enumerated_match_count():
    # sanity of the brute force itself: compositions of 6 into {1,2} = Fib(7) = 13
    n = sum(1 for k in range(1, 7) for c in itertools.product((1, 2), repeat=k) if sum(c) == 6)
    assert n == 13

"""Integer-exact BITWISE pins of the hand-written, timed sm_100a kernels
(Table I P:1664-1701 for the five DAGs).

Each DAG gets scalars that make every coefficient an integer or a dyadic
rational and inputs that are integer polynomials of degree <= the stencil's
exactness order (tests/polyexact.Poly).  Then every value the kernel forms --
in any association, with or without FMA contraction -- is an exactly
representable integer/dyadic below 2^53 (asserted through the abs-mode bound:
every partial sum of any evaluation order is bounded by the abs-mode value),
so the GPU result must equal the continuous closed form BIT FOR BIT:

  lap25    c = (-43050, 8064, -1008, 128, -9) = 5040 x the 8th-order 2nd difference
           -> 5040 lap p  (per-axis degree <= 9; we use <= 4 at full size)
  smooth27 w = (-128, 14, 3, 1), nu = 1/32 -> p + (30/32) lap p   (total degree <= 3)
           iterated (V8): p + T (30/32) lap p where the ring distance >= T (quadratic p)
  hypterm  (ALP..DEL) x 840 = (672, -168, 32, -3) -> -840 sum_a dxinv_a d_a F_a
           (degree-2 fields, degree-4 flux products)
  rhs4     tf = 3/4, i6 = 24, i144 = 1, cof = 1, a1 in {0, 1} -> a1 uacc + 144 L(u)
           (linear mu, la, str; u of total degree <= 3)
  jacobi7  a = 1/2, b = 1/4, h2inv = 4 -> p/2 - lap p (per-axis degree <= 3)

Each runs (i) on a multi-tile shape with ragged tails through EVERY registered
variant of the DAG, also against the C oracle bitwise, and (ii) at the BASELINE
size in the launch configuration bench.py times (the default plan and the
tune=1 plan).  The expected values come from the closed form (exact rational
calculus in tests/polyexact.py), never from the CUDA path.
"""
from __future__ import annotations

import random
from fractions import Fraction

import numpy as np
import pytest

from cases import RADIUS, interior, ring_mask
from exactcases import (CASES, FULL, MULTI_TILE, _centre, _hypterm_case, _rhs4_case, check_bound, laplacian,
                        random_poly)

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("no CUDA device", allow_module_level=True)

import paper_conf_ipps_rawatvsrps19_b200 as sdag  # noqa: E402

def _run(plan, case, dims):
    dev = [torch.from_numpy(np.ascontiguousarray(x)).cuda() for x in case["ins"]]
    if case["inout"] is not None:
        outs = [torch.from_numpy(x.copy()).cuda() for x in case["inout"]]
    else:
        outs = [torch.full(tuple(dims), float("nan"), dtype=torch.float64, device="cuda") for _ in case["exp"]]
    a1d = [torch.from_numpy(x).cuda() for x in case["a1d"]]
    plan.apply(outs + dev, a1d, case["s"])
    torch.cuda.synchronize()
    res = [t.cpu().numpy() for t in outs]
    del dev, outs
    return res


def _assert_exact(name, dims, got, case, tag):
    R = RADIUS[name]
    I = interior(dims, R)
    ring = ring_mask(dims, R)
    for m, (g, e) in enumerate(zip(got, case["exp"])):
        bad = np.count_nonzero(g[I] != e[I])
        assert bad == 0, f"{name} {tag} output {m}: {bad} interior points differ from the exact closed form"
        if case["inout"] is not None:
            assert np.array_equal(g[ring], case["inout"][m][ring]), f"{name} {tag} output {m}: ring modified"
        else:
            assert np.all(np.isnan(g[ring])), f"{name} {tag} output {m}: wrote outside the interior"


@pytest.mark.parametrize("name", list(CASES))
def test_every_variant_bitwise_exact_multitile(name):
    """(i) multi-tile, ragged: every registered variant of the hand-written
    kernels == the exact closed form == the C oracle, bit for bit."""
    dims = MULTI_TILE[name]
    case = CASES[name](dims, random.Random(sum(map(ord, name))), False)
    check_bound(case)
    orc = case["orc"]()
    R = RADIUS[name]
    I = interior(dims, R)
    for m, e in enumerate(case["exp"]):
        assert np.array_equal(orc[m][I], e[I]), f"oracle vs closed form, output {m}"
    spec = sdag.spec_text(name)
    variants = sdag.Plan(spec, dims).variants()
    assert variants
    for v in variants:
        got = _run(sdag.Plan(spec, dims, variant=v), case, dims)
        _assert_exact(name, dims, got, case, v)


@pytest.mark.parametrize("dxinv", [(0.5, 0.25, 2.0), (2.0, 0.125, 4.0)])
def test_hypterm_dyadic_dxinv_bitwise(dxinv):
    """dxinv enters per axis (a wrong axis would still pass with dxinv = 1)."""
    dims = MULTI_TILE["hypterm"]
    case = _hypterm_case(dims, random.Random(17), False, dxinv=dxinv)
    check_bound(case)
    got = _run(sdag.Plan(sdag.spec_text("hypterm"), dims), case, dims)
    _assert_exact("hypterm", dims, got, case, f"dxinv={dxinv}")


@pytest.mark.parametrize("a1", [0.0, 1.0])
def test_rhs4_a1_bitwise(a1):
    dims = MULTI_TILE["rhs4center"]
    case = _rhs4_case(dims, random.Random(int(a1) + 40), False, a1=a1)
    check_bound(case)
    for v in sdag.Plan(sdag.spec_text("rhs4center"), dims).variants():
        got = _run(sdag.Plan(sdag.spec_text("rhs4center"), dims, variant=v), case, dims)
        _assert_exact("rhs4center", dims, got, case, f"{v} a1={a1}")


@pytest.mark.parametrize("tune", [False, True])
@pytest.mark.parametrize("name", list(FULL))
def test_bench_geometry_bitwise_exact(name, tune):
    """(ii) BASELINE size, bench.py's launch configuration (default and tune=1
    plan): every interior point equals the exact closed form."""
    dims = FULL[name]
    case = CASES[name](dims, random.Random(7), True)
    check_bound(case)
    plan = sdag.Plan(sdag.spec_text(name), dims, tune=tune)
    got = _run(plan, case, dims)
    _assert_exact(name, dims, got, case, plan.info["variant"])


@pytest.mark.parametrize("a1", [0.0, 1.0])
def test_rhs4_bench_geometry_a1_bitwise(a1):
    dims = FULL["rhs4center"]
    case = _rhs4_case(dims, random.Random(3), True, a1=a1)
    check_bound(case)
    got = _run(sdag.Plan(sdag.spec_text("rhs4center"), dims), case, dims)
    _assert_exact("rhs4center", dims, got, case, f"a1={a1}")


@pytest.mark.parametrize("tune", [False, True])
def test_jacobi7_batched_bench_geometry_bitwise(tune):
    """config 1b: 128 x 64^3 in one launch, a different polynomial per problem."""
    dims, batch = (64, 64, 64), 128
    rng = random.Random(11)
    polys = [random_poly(rng, (3, 3, 3), coef=4, nterms=12) for _ in range(8)]
    o = _centre(dims)
    grids = [p.grid_fast(dims, o) for p in polys]
    exps = [(p * Fraction(1, 2) - laplacian(p)).grid_fast(dims, o) for p in polys]
    A = np.stack([grids[b % 8] for b in range(batch)])
    plan = sdag.Plan(sdag.spec_text("jacobi7"), dims, batch=batch, tune=tune)
    dA = torch.from_numpy(A).cuda()
    dB = torch.full(A.shape, float("nan"), dtype=torch.float64, device="cuda")
    plan.apply_batched(batch, [dB, dA], scalars=[4.0, 0.5, 0.25])
    torch.cuda.synchronize()
    G = dB.cpu().numpy()
    I = interior(dims, 1)
    for b in range(batch):
        assert np.array_equal(G[b][I], exps[b % 8][I]), f"problem {b}"
        assert np.all(np.isnan(G[b][ring_mask(dims, 1)]))


@pytest.mark.parametrize("tune", [False, True])
def test_smooth27_iterated_1024_closed_form_bitwise(tune):
    """config 5 on one GPU (1024^3, T = 12, the fused kernels bench.py times):
    integer weights, nu = 1/32, quadratic p -> every value exact, so
    A_T = p + T (30/32) lap p bit for bit wherever the ring distance d >= T
    (V8; the ring itself stays p).  Built and checked on the device, plane
    block by plane block, from the closed form."""
    dims, T = (1024, 1024, 1024), 12
    nz, ny, nx = dims
    c = {"ii": 3, "jj": -2, "kk": 5, "ij": 1, "jk": -3, "i": 2, "1": 11}
    L = 2 * (c["ii"] + c["jj"] + c["kk"])
    dev = "cuda"
    i = torch.arange(nx, device=dev, dtype=torch.int64) - nx // 2
    j = torch.arange(ny, device=dev, dtype=torch.int64) - ny // 2

    def p_block(z0, z1):
        k = torch.arange(z0, z1, device=dev, dtype=torch.int64)[:, None, None] - nz // 2
        jj, ii = j[None, :, None], i[None, None, :]
        v = (c["ii"] * ii * ii + c["jj"] * jj * jj + c["kk"] * k * k + c["ij"] * ii * jj + c["jk"] * jj * k
             + c["i"] * ii + c["1"])
        return v.to(torch.float64)

    b0 = torch.empty(dims, dtype=torch.float64, device=dev)
    for z0 in range(0, nz, 64):
        b0[z0:z0 + 64] = p_block(z0, z0 + 64)
    b1 = b0.clone()
    plan = sdag.Plan(sdag.spec_text("smooth27"), dims, tune=tune)
    plan.apply_iterated(b0, b1, T, scalars=[-128.0, 14.0, 3.0, 1.0, 1.0 / 32.0])
    torch.cuda.synchronize()
    res = b0 if T % 2 == 0 else b1
    add = T * (30.0 / 32.0) * L
    dj = torch.minimum(torch.arange(ny, device=dev), ny - 1 - torch.arange(ny, device=dev))
    di = torch.minimum(torch.arange(nx, device=dev), nx - 1 - torch.arange(nx, device=dev))
    dxy = torch.minimum(dj[:, None], di[None, :])
    bad = 0
    for z0 in range(0, nz, 64):
        kz = torch.arange(z0, z0 + 64, device=dev)
        dz = torch.minimum(kz, nz - 1 - kz)
        d = torch.minimum(dz[:, None, None], dxy[None])
        p = p_block(z0, z0 + 64)
        exact = torch.where(d >= T, p + add, res[z0:z0 + 64])
        ring = d == 0
        bad += int((res[z0:z0 + 64] != exact).sum())
        bad += int((res[z0:z0 + 64][ring] != p[ring]).sum())
    assert bad == 0, f"{bad} points differ from the V8 closed form ({plan.info['variant']})"

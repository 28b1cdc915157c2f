"""GPU parity: the sm_100a path through the C ABI vs the CPU oracle on the same
seeded inputs, element by element (scaled-error gate, R13), plus
bit-exact bookkeeping: interior-only writes, untouched rings, integer-coded
shift stencils, P-slab loopback == 1-GPU."""
from __future__ import annotations

import numpy as np
import pytest

import oracle
import synth
from cases import RADIUS, TOL, check, interior, make_case, ring_mask, run_gpu, scaled_err

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("no CUDA device", allow_module_level=True)

import paper_conf_ipps_rawatvsrps19_b200 as sdag  # noqa: E402

NAMES = ["jacobi7", "lap25", "smooth27", "hypterm", "rhs4center"]


def _min_dims(name):
    R = RADIUS[name]
    return (2 * R + 1, 2 * R + 1, 2 * R + 2)  # one interior point in z,y; x even for the TMA path


# odd nx -> LSU loader; even nx -> TMA; several tiles and ragged tails in x/y/z
SHAPES = [(37, 41, 43), (20, 34, 70), (13, 70, 136)]


@pytest.mark.parametrize("name", NAMES)
@pytest.mark.parametrize("dims", SHAPES, ids=lambda d: "x".join(map(str, d)))
def test_parity_small(name, dims):
    case = make_case(name, dims)
    g, plan = run_gpu(name, dims, case)
    check(name, dims, g, case)


@pytest.mark.parametrize("name", NAMES)
def test_parity_minimal_grid(name):
    dims = _min_dims(name)
    case = make_case(name, dims)
    g, _ = run_gpu(name, dims, case)
    check(name, dims, g, case)


@pytest.mark.parametrize("name", NAMES)
def test_every_variant(name):
    dims = (18, 37, 66)
    case = make_case(name, dims)
    plan = sdag.Plan(sdag.spec_text(name), dims, device=0)
    for v in plan.variants():
        g, p = run_gpu(name, dims, case, variant=v)
        assert p.info["variant"] == v
        check(name, dims, g, case)


def test_lsu_variants_on_odd_nx():
    dims = (11, 13, 35)
    for name in NAMES:
        plan = sdag.Plan(sdag.spec_text(name), dims)
        assert all("tma" not in v for v in plan.variants())
        case = make_case(name, dims)
        g, _ = run_gpu(name, dims, case)
        check(name, dims, g, case)


def test_tuned_plan_is_correct():
    dims = (24, 40, 72)
    case = make_case("lap25", dims)
    g, plan = run_gpu("lap25", dims, case, tune=True)
    assert "[tuned]" in plan.describe()
    check("lap25", dims, g, case)


def test_unaligned_pointer_uses_lsu_twin():
    dims = (12, 14, 16)
    case = make_case("jacobi7", dims)
    plan = sdag.Plan(sdag.spec_text("jacobi7"), dims)
    n = int(np.prod(dims))
    big = torch.zeros(n + 1, dtype=torch.float64, device="cuda")
    A = big[1:].view(dims)  # 8-byte but not 16-byte aligned
    A.copy_(torch.from_numpy(case["inputs"][0]))
    B = torch.full(dims, float("nan"), dtype=torch.float64, device="cuda")
    plan.apply([B, A], scalars=case["s"])
    torch.cuda.synchronize()
    check("jacobi7", dims, [B.cpu().numpy()], case)


def test_batched_jacobi7():
    dims, batch = (16, 18, 20), 6
    ins, sc = synth.jacobi7_inputs(dims, cfg="batched", batch=batch)
    A = ins["A"]
    plan = sdag.Plan(sdag.spec_text("jacobi7"), dims, batch=batch)
    dA = torch.from_numpy(A).cuda()
    dB = torch.full(A.shape, float("nan"), dtype=torch.float64, device="cuda")
    plan.apply_batched(batch, [dB, dA], scalars=[sc["h2inv"], sc["a"], sc["b"]])
    torch.cuda.synchronize()
    G = dB.cpu().numpy()
    I = interior(dims, 1)
    for b in range(batch):
        o = oracle.jacobi7(A[b], sc["a"], sc["b"], sc["h2inv"])
        a = oracle.jacobi7(np.abs(A[b]), sc["a"], sc["b"], sc["h2inv"], absmode=True)
        assert scaled_err(G[b][I], o[I], a[I]) <= TOL
        assert np.all(np.isnan(G[b][ring_mask(dims, 1)]))


def test_iterated_smooth27_matches_oracle():
    dims, T = (20, 22, 24), 5
    ins, sc = synth.smooth27_inputs(dims, cfg="iter")
    A = ins["A"]
    w = [sc[k] for k in ("w0", "w1", "w2", "w3")]
    plan = sdag.Plan(sdag.spec_text("smooth27"), dims)
    b0 = torch.from_numpy(A).cuda()
    b1 = b0.clone()
    plan.apply_iterated(b0, b1, T, scalars=[*w, sc["nu"]])
    torch.cuda.synchronize()
    G = (b0 if T % 2 == 0 else b1).cpu().numpy()
    O = oracle.smooth27_iter(A, w, sc["nu"], T)
    Aabs = oracle.smooth27_iter(np.abs(A), np.abs(w), sc["nu"], T, absmode=True)
    # rounding accumulates over T sweeps: bound T * TOL (reading R13)
    assert scaled_err(G, O, Aabs) <= T * TOL
    assert np.array_equal(G[ring_mask(dims, 1)], A[ring_mask(dims, 1)])


def test_iterated_smooth27_exact_closed_form():
    """V8 on the GPU: integer weights, nu = 1/32, quadratic input -> every value
    exact, so the GPU result equals p + T*(30/32)*lap(p) bit for bit where the
    distance to the ring is >= T."""
    dims, T = (16, 18, 20), 4
    k, j, i = np.meshgrid(*[np.arange(n, dtype=np.float64) - n // 2 for n in dims], indexing="ij")
    p = 3 * i * i - 2 * j * j + 5 * k * k + i * j - 3 * j * k + 2 * i + 11
    L = 2 * (3 - 2 + 5)
    plan = sdag.Plan(sdag.spec_text("smooth27"), dims)
    b0 = torch.from_numpy(p.copy()).cuda()
    b1 = b0.clone()
    plan.apply_iterated(b0, b1, T, scalars=[-128.0, 14.0, 3.0, 1.0, 1.0 / 32.0])
    torch.cuda.synchronize()
    G = (b0 if T % 2 == 0 else b1).cpu().numpy()
    kk, jj, ii = np.meshgrid(*[np.arange(n) for n in dims], indexing="ij")
    d = np.minimum.reduce([np.minimum(x, n - 1 - x) for x, n in zip((kk, jj, ii), dims)])
    exact = p + T * (30.0 / 32.0) * L
    assert np.array_equal(G[d >= T], exact[d >= T])
    assert np.array_equal(G, oracle.smooth27_iter(p, [-128.0, 14.0, 3.0, 1.0], 1 / 32, T))


@pytest.mark.parametrize("off", [(1, 0, 0), (0, -2, 3), (-4, 4, -1), (2, 1, -4), (0, 0, 0)])
def test_shift_bitwise(off):
    dims = (14, 15, 18)
    R = [abs(o) for o in off]
    spec = ("iterator k, j, i;\ndouble in[L,M,N], out[L,M,N];\nstencil s (B, A) {\n"
            f"B[k][j][i] = A[k{off[0]:+d}][j{off[1]:+d}][i{off[2]:+d}];\n}}\ns (out, in);\n")
    A = np.arange(np.prod(dims), dtype=np.float64).reshape(dims)
    plan = sdag.Plan(spec, dims)
    assert plan.info["dag"] == "shift"
    dA = torch.from_numpy(A).cuda()
    dB = torch.full(dims, -1.0, dtype=torch.float64, device="cuda")
    plan.apply([dB, dA])
    torch.cuda.synchronize()
    G = dB.cpu().numpy()
    O = oracle.shift(A, off, out=np.full(dims, -1.0))
    assert np.array_equal(G, O)
    assert plan.info["radius"] == tuple(R)


def test_j1d3pt_fig1a_on_gpu():
    """Fig 1a, hand-expanded in tests/golden/j1d3pt_fig1a.txt."""
    plan = sdag.Plan(sdag.spec_text("j1d3pt"), (1, 1, 5))
    b0 = torch.tensor([1.0, 2, 3, 4, 5], dtype=torch.float64, device="cuda").view(1, 1, 5)
    b1 = b0.clone()
    plan.apply_iterated(b0, b1, 2, scalars=[3.0])
    torch.cuda.synchronize()
    assert b0.flatten().tolist() == [1.0, 16.0, 27.0, 26.0, 5.0]


def test_apply_host_end_to_end():
    dims = (20, 24, 30)
    case = make_case("lap25", dims)
    plan = sdag.Plan(sdag.spec_text("lap25"), dims)
    out = np.full(dims, np.nan)
    up, down = plan.apply_host([out, case["inputs"][0]], scalars=case["s"])
    assert up == case["inputs"][0].nbytes
    assert down == 8 * (dims[0] - 8) * (dims[1] - 8) * (dims[2] - 8)
    check("lap25", dims, [out], case)


@pytest.mark.parametrize("name,gdims,T", [("smooth27", (30, 20, 22), 6), ("lap25", (44, 18, 20), 3)])
@pytest.mark.parametrize("P", [1, 2, 3, 4])
def test_loopback_slabs_bitwise_equal_single_gpu(name, gdims, T, P):
    """a7 bookkeeping: P z-slabs with the halo schedule of the NCCL path
    (moved by cudaMemcpy) reproduce the single-GPU iteration bit for bit."""
    case = make_case(name, gdims, cfg="slab")
    A = case["inputs"][0]
    s = case["s"]
    spec = sdag.spec_text(name)
    full = sdag.Plan(spec, gdims)
    b0 = torch.from_numpy(A).cuda()
    b1 = b0.clone()
    full.apply_iterated(b0, b1, T, scalars=s)
    ref = (b0 if T % 2 == 0 else b1).cpu().numpy()

    dists = [sdag.Dist(spec, gdims, r, P) for r in range(P)]
    bufs0, bufs1 = [], []
    for d in dists:
        (nza, ny, nx), g0 = d.layout()
        loc = np.zeros((nza, ny, nx))
        lo, hi = max(g0, 0), min(g0 + nza, gdims[0])
        loc[lo - g0:hi - g0] = A[lo:hi]
        bufs0.append(torch.from_numpy(loc).cuda())
        bufs1.append(torch.from_numpy(loc.copy()).cuda())
    sdag.Dist.apply_iterated_loopback(dists, bufs0, bufs1, T, scalars=s)
    torch.cuda.synchronize()
    res = bufs0 if T % 2 == 0 else bufs1
    for r, d in enumerate(dists):
        part = sdag.slab_partition(gdims[0], RADIUS[name], P, r)
        (nza, ny, nx), g0 = d.layout()
        z0, n = part["z0"], part["nz_own"]
        got = res[r].cpu().numpy()[z0 - g0:z0 - g0 + n]
        assert np.array_equal(got, ref[z0:z0 + n]), f"rank {r} of {P}"


def test_full_size_lap25_sampled():
    """BASELINE config 2 (512^3) in the launch configuration bench.py times,
    checked on sampled points the oracle computes one by one."""
    dims = (512, 512, 512)
    ins, sc = synth.lap25_inputs(dims)
    A = ins["A"]
    c = [sc[k] for k in ("c0", "c1", "c2", "c3", "c4")]
    plan = sdag.Plan(sdag.spec_text("lap25"), dims)
    dA = torch.from_numpy(A).cuda()
    dB = torch.full(dims, float("nan"), dtype=torch.float64, device="cuda")
    plan.apply([dB, dA], scalars=c)
    torch.cuda.synchronize()
    rng = np.random.default_rng(7)
    pts = np.stack([rng.integers(4, n - 4, 4000) for n in dims], axis=1)
    # include tile/chunk seams and the interior corners
    pts = np.concatenate([pts, np.array([[4, 4, 4], [507, 507, 507], [4, 507, 4], [255, 256, 67], [300, 63, 64]])])
    o = oracle.lap25_points(A, c, pts)
    a = oracle.lap25_points(np.abs(A), np.abs(c), pts, absmode=True)
    g = dB[pts[:, 0], pts[:, 1], pts[:, 2]].cpu().numpy()
    assert scaled_err(g, o, a) <= TOL
    ring = np.array([[0, 0, 0], [3, 100, 100], [508, 10, 10], [100, 3, 100], [100, 100, 511]])
    assert torch.isnan(dB[ring[:, 0], ring[:, 1], ring[:, 2]]).all()

"""GPU parity: the sm_100a path through the C ABI vs the CPU oracle on the same
seeded inputs, element by element (scaled-error gate, R13), plus
bit-exact bookkeeping: interior-only writes, untouched rings, integer-coded
shift stencils, P-slab loopback == 1-GPU."""
from __future__ import annotations

import numpy as np
import pytest

import oracle
import synth
from cases import RADIUS, check, gate, interior, make_case, ring_mask, run_gpu

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


@pytest.mark.parametrize("name", NAMES)
@pytest.mark.parametrize("dims", [(13, 22, 40), (11, 13, 35)], ids=["tma", "lsu"])
def test_batched_every_dag(name, dims):
    """sdag_apply_batched: B independent problems laid out [batch][nz][ny][nx]
    (1D arrays [batch][len], include/sdag.h) in one launch; every problem
    matches its own oracle and keeps its own ring (rhs4center's strx/stry/strz
    are per problem, so a wrong 1D batch stride fails here)."""
    B = 3
    cases = [make_case(name, dims, cfg=f"batch{b}") for b in range(B)]
    plan = sdag.Plan(sdag.spec_text(name), dims, batch=B)
    dev = [torch.from_numpy(np.ascontiguousarray(np.stack([c["inputs"][q] for c in cases]))).cuda()
           for q in range(len(cases[0]["inputs"]))]
    if cases[0]["inout"]:
        outs = [torch.from_numpy(np.stack([c["inout"][m] for c in cases])).cuda() for m in range(len(cases[0]["inout"]))]
    else:
        outs = [torch.full((B, *dims), np.nan, dtype=torch.float64, device="cuda") for _ in range(cases[0]["outs"])]
    a1d = [torch.from_numpy(np.concatenate([c["a1d"][q] for c in cases])).cuda() for q in range(len(cases[0]["a1d"]))]
    for c in cases[1:]:
        assert c["s"] == cases[0]["s"], "scalars are shared by the batch"
    plan.apply_batched(B, outs + dev, a1d, cases[0]["s"])
    torch.cuda.synchronize()
    for b, c in enumerate(cases):
        check(name, dims, [t[b].cpu().numpy() for t in outs], c)


@pytest.mark.parametrize("name", ["jacobi7", "smooth27", "lap25"])
def test_iterated_zero_sweeps_leaves_both_buffers(name):
    """T = 0 (the degenerate iteration): nothing is launched, the result is buf0
    as given and buf1 is untouched (bitwise)."""
    dims = (14, 20, 36)
    case = make_case(name, dims)
    plan = sdag.Plan(sdag.spec_text(name), dims)
    b0 = torch.from_numpy(case["inputs"][0].copy()).cuda()
    b1 = torch.full(dims, np.nan, dtype=torch.float64, device="cuda")
    l0 = sdag.launch_count()
    plan.apply_iterated(b0, b1, 0, case["s"])
    torch.cuda.synchronize()
    assert sdag.launch_count() == l0
    assert np.array_equal(b0.cpu().numpy(), case["inputs"][0])
    assert np.all(np.isnan(b1.cpu().numpy()))


def test_batch_beyond_the_launch_grid_is_refused():
    """The largest batch one launch can carry: grid.z = z-chunks x batch <= 65535.
    65535 one-plane problems run; 65536 are refused with DOMAIN before anything
    is enqueued (the outputs keep their sentinel)."""
    dims = (3, 3, 4)  # one interior point per problem
    for B, ok in ((65535, True), (65536, False)):
        plan = sdag.Plan(sdag.spec_text("jacobi7"), dims, batch=B)
        A = torch.rand((B, *dims), dtype=torch.float64, device="cuda")
        out = torch.full((B, *dims), np.nan, dtype=torch.float64, device="cuda")
        if ok:
            plan.apply_batched(B, [out, A], scalars=[4.0, 0.5, 0.25])
            torch.cuda.synchronize()
            a = A[:, 1, 1, 1:3].cpu().numpy()
            nb = (A[:, 0, 1, 1:3] + A[:, 2, 1, 1:3] + A[:, 1, 0, 1:3] + A[:, 1, 2, 1:3]).cpu().numpy()
            nb = nb + np.stack([A[:, 1, 1, 0].cpu().numpy(), A[:, 1, 1, 1].cpu().numpy()], 1) \
                + np.stack([A[:, 1, 1, 2].cpu().numpy(), A[:, 1, 1, 3].cpu().numpy()], 1)
            ref = 0.5 * a - (0.25 * 4.0) * (nb - 6.0 * a)
            got = out[:, 1, 1, 1:3].cpu().numpy()
            assert np.max(np.abs(got - ref) / np.maximum(np.abs(ref), 1.0)) < 1e-12
        else:
            with pytest.raises(sdag.SdagError) as e:
                plan.apply_batched(B, [out, A], scalars=[4.0, 0.5, 0.25])
            assert e.value.code == "DOMAIN"
            torch.cuda.synchronize()
            assert torch.all(torch.isnan(out))


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
    assert "[tuned: " in plan.describe()  # hierarchical: geometries, then their variants, then z-chunks
    check("lap25", dims, g, case)


def test_persistent_tune_cache(tmp_path, monkeypatch):
    """NEXT-3 persistent plan cache: a tune=1 plan appends its choice to
    $SDAG_TUNE_CACHE; the next plan of the same shape restores it without timing."""
    path = tmp_path / "tune.txt"
    monkeypatch.setenv("SDAG_TUNE_CACHE", str(path))
    dims = (40, 48, 64)
    p1 = sdag.Plan(sdag.spec_text("smooth27"), dims, tune=True)
    assert "[tuned: " in p1.describe()
    lines = path.read_text().splitlines()
    assert len(lines) == 1 and p1.info["variant"] in lines[0]
    p2 = sdag.Plan(sdag.spec_text("smooth27"), dims, tune=True)
    assert "from $SDAG_TUNE_CACHE" in p2.describe()
    assert p2.info["variant"] == p1.info["variant"]
    assert len(path.read_text().splitlines()) == 1
    f1 = [ln for ln in p1.describe().splitlines() if "f(1)=" in ln]
    f2 = [ln for ln in p2.describe().splitlines() if "f(1)=" in ln]
    assert [x.split(":", 1)[1] for x in f1] == [x.split(":", 1)[1] for x in f2]
    z1 = [w for w in p1.describe().split("  ") if w.startswith("z-chunk")]
    z2 = [w for w in p2.describe().split("  ") if w.startswith("z-chunk")]
    assert z1 == z2  # the tuned z-chunk length is restored too
    case = make_case("smooth27", dims)
    g1, _ = run_gpu("smooth27", dims, case, variant=p1.info["variant"])
    check("smooth27", dims, g1, case)
    # another shape misses and appends
    sdag.Plan(sdag.spec_text("smooth27"), (40, 48, 66), tune=True)
    assert len(path.read_text().splitlines()) == 2


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
        gate(G[b][I], o[I], a[I])
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
    # the north-star gate holds for the iterate too: A_p is the abs-mode T-sweep iterate (R13)
    gate(G, O, Aabs)
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


@pytest.mark.parametrize("name", NAMES)
def test_apply_host_pipelined_chunks(name):
    """sdag_apply_host over several z-chunks (H2D / sweep / D2H overlapped on
    three streams): same values as the oracle, ring untouched, each input byte
    uploaded once, only the interior box downloaded."""
    dims = (70, 22, 34)  # >= 6 chunks for every radius
    case = make_case(name, dims)
    plan = sdag.Plan(sdag.spec_text(name), dims)
    R = RADIUS[name]
    if case["inout"]:
        outs = [x.copy() for x in case["inout"]]
    else:
        outs = [np.full(dims, np.nan) for _ in range(case["outs"])]
    ins = [np.ascontiguousarray(x) for x in case["inputs"]]
    up, down = plan.apply_host(outs + ins, case["a1d"], scalars=case["s"])
    n_up = len(ins) + len(case["inout"])
    assert up == n_up * ins[0].nbytes + sum(x.nbytes for x in case["a1d"])
    assert down == len(outs) * 8 * (dims[0] - 2 * R) * (dims[1] - 2 * R) * (dims[2] - 2 * R)
    check(name, dims, outs, case)
    # a second call on the same plan (workspace and copy streams reused) is identical
    outs2 = [x.copy() for x in case["inout"]] if case["inout"] else [np.full(dims, np.nan) for _ in outs]
    plan.apply_host(outs2 + ins, case["a1d"], scalars=case["s"])
    for a, b in zip(outs, outs2):
        assert np.array_equal(a, b, equal_nan=True)


@pytest.mark.parametrize("name,gdims,T,tt", [("smooth27", (30, 20, 22), 6, 1), ("lap25", (44, 18, 20), 3, 1),
                                             ("smooth27", (30, 20, 22), 6, 2), ("smooth27", (31, 22, 24), 5, 2),
                                             ("smooth27", (40, 26, 30), 12, 2)])
@pytest.mark.parametrize("P", [1, 2, 3, 4])
def test_loopback_slabs_bitwise_equal_single_gpu(name, gdims, T, tt, P):
    """a7 bookkeeping: P z-slabs with the halo schedule of the NCCL path
    (moved by cudaMemcpy) reproduce the single-GPU iteration bit for bit.
    tt = 2 (NEXT-1, communication-avoiding): ghost depth 2 R_z, fused 2-sweep
    launches, one exchange of 2 R_z planes per launch."""
    case = make_case(name, gdims, cfg="slab")
    A = case["inputs"][0]
    s = case["s"]
    spec = sdag.spec_text(name)
    full = sdag.Plan(spec, gdims)
    b0 = torch.from_numpy(A).cuda()
    b1 = b0.clone()
    full.apply_iterated(b0, b1, T, scalars=s)
    ref = (b0 if T % 2 == 0 else b1).cpu().numpy()

    dists = [sdag.Dist(spec, gdims, r, P, time_tile=tt) for r in range(P)]
    bufs0, bufs1 = [], []
    for d in dists:
        (nza, ny, nx), g0 = d.layout()
        loc = np.zeros((nza, ny, nx))
        lo, hi = max(g0, 0), min(g0 + nza, gdims[0])
        loc[lo - g0:hi - g0] = A[lo:hi]
        bufs0.append(torch.from_numpy(loc).cuda())
        bufs1.append(torch.from_numpy(loc.copy()).cuda())
    n0 = sdag.launch_count()
    sdag.Dist.apply_iterated_loopback(dists, bufs0, bufs1, T, scalars=s)
    torch.cuda.synchronize()
    nl = sdag.launch_count() - n0
    if tt == 2 and T >= 4:  # fused launches: at most 3 per rank per pair of sweeps
        assert nl <= P * 3 * ((T + 1) // 2 + 1) and nl < P * 3 * T
    res = bufs0 if T % 2 == 0 else bufs1
    for r, d in enumerate(dists):
        part = sdag.slab_partition2(gdims[0], RADIUS[name], tt, P, r)
        (nza, ny, nx), g0 = d.layout()
        z0, n = part["z0"], part["nz_own"]
        got = res[r].cpu().numpy()[z0 - g0:z0 - g0 + n]
        assert np.array_equal(got, ref[z0:z0 + n]), f"rank {r} of {P}"


@pytest.mark.parametrize("variant,tt", [("fuse3_tma_60x28_u2x2_pf2_mb1", 3), ("fuse4_tma_58x26_u2x2_pf2_mb1", 4)])
@pytest.mark.parametrize("P", [1, 2, 3])
def test_loopback_slabs_fusion_degree(variant, tt, P):
    """NEXT-1 x a7: slabs with ghost depth tt R_z run the forced tt-sweep kernel
    (one exchange of tt R_z planes per launch) bit-identical to one GPU."""
    name, gdims, T = "smooth27", (46, 34, 66), 12
    case = make_case(name, gdims, cfg="slab")
    A = case["inputs"][0]
    s = case["s"]
    spec = sdag.spec_text(name)
    full = sdag.Plan(spec, gdims, variant=variant)
    b0 = torch.from_numpy(A).cuda()
    b1 = b0.clone()
    full.apply_iterated(b0, b1, T, scalars=s)
    ref = (b0 if T % 2 == 0 else b1).cpu().numpy()
    dists = [sdag.Dist(spec, gdims, r, P, time_tile=tt, variant=variant) for r in range(P)]
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
        part = sdag.slab_partition2(gdims[0], RADIUS[name], tt, P, r)
        (nza, ny, nx), g0 = d.layout()
        z0, n = part["z0"], part["nz_own"]
        got = res[r].cpu().numpy()[z0 - g0:z0 - g0 + n]
        assert np.array_equal(got, ref[z0:z0 + n]), f"rank {r} of {P}"
    O = oracle.smooth27_iter(A, s[:4], s[4], T)
    Aabs = oracle.smooth27_iter(np.abs(A), np.abs(s[:4]), s[4], T, absmode=True)
    gate(ref, O, Aabs)


FUSED = ["fuse2_tma_62x14_u2x2_pf2_mb2", "fuse2_tma_30x14_u2x2_pf2_mb3", "fuse2_tma_126x14_u2x4_pf2", "fuse2_tma_62x30_u2x2_pf2",
         "fuse2_tma_126x14_u2x2_pf2", "fuse2_tma_62x14_u4x2_pf2",
         "fuse2o_tma_62x14_u2x2_pf2_mb2", "fuse2o_tma_30x14_u2x2_pf2_mb3", "fuse2o_tma_126x14_u2x4_pf2",
         "fuse2o_tma_62x14_u4x2_pf2_mb2",
         "fuse3_tma_60x28_u2x2_pf2_mb1", "fuse3o_tma_60x28_u2x2_pf2_mb1", "fuse3_tma_124x12_u2x2_pf2_mb1",
         "fuse4_tma_58x26_u2x2_pf2_mb1", "fuse4_tma_58x10_u2x2_pf2_mb2"]


@pytest.mark.parametrize("variant", FUSED)
@pytest.mark.parametrize("dims", [(26, 30, 40), (33, 20, 132), (9, 70, 260)], ids=lambda d: "x".join(map(str, d)))
def test_temporal_fusion_matches_oracle_and_unfused(variant, dims):
    """NEXT-1: two sweeps per launch (overlapped tiling in x/y, retimed z);
    the DP schedule mixes 2-sweep and 1-sweep launches to keep the ping-pong
    parity.  Same result as T single sweeps (and the oracle) for odd and even T."""
    ins, sc = synth.smooth27_inputs(dims, cfg="fuse")
    A = ins["A"]
    w = [sc[k] for k in ("w0", "w1", "w2", "w3")]
    s = [*w, sc["nu"]]
    fused = sdag.Plan(sdag.spec_text("smooth27"), dims, variant=variant)
    plain = sdag.Plan(sdag.spec_text("smooth27"), dims, fusion=False)
    for T in (1, 2, 3, 5, 12):
        outs = []
        for plan in (fused, plain):
            b0 = torch.from_numpy(A).cuda()
            b1 = b0.clone()
            n0 = sdag.launch_count()
            plan.apply_iterated(b0, b1, T, scalars=s)
            torch.cuda.synchronize()
            outs.append(((b0 if T % 2 == 0 else b1).cpu().numpy(), sdag.launch_count() - n0))
        (gf, nf), (gp, np_) = outs
        # launches flip the ping-pong pair once each, so #launches == T (mod 2)
        assert np_ == T and nf == _expected_launches(fused, T, variant)
        O = oracle.smooth27_iter(A, w, sc["nu"], T)
        Aabs = oracle.smooth27_iter(np.abs(A), np.abs(w), sc["nu"], T, absmode=True)
        gate(gf, O, Aabs)
        gate(gp, O, Aabs)
        assert np.array_equal(gf[ring_mask(dims, 1)], A[ring_mask(dims, 1)])


def _expected_launches(plan, T, variant):
    """Launches of apply_iterated with one forced x-sweep kernel: the DP schedule
    over the plan's own f(x) (sdag_plan_describe) with the parity rule."""
    import re
    line = [ln for ln in plan.describe().splitlines() if "f(1)=" in ln][0]
    deg = int(variant[4])  # "fuseN..."
    f = {int(x): float(v) for x, v in re.findall(r"f\((\d)\)=([0-9.eE+-]+)", line) if int(x) in (1, deg)}
    seq, _ = sdag.fusion_schedule(f, T)
    assert len(seq) % 2 == T % 2 and sum(seq) == T
    return len(seq)


FUSED_J7 = ["fuse2o_tma_62x14_u2x2_pf2_mb2", "fuse2o_tma_30x14_u2x2_pf2_mb3", "fuse2o_tma_126x14_u2x4_pf2",
            "fuse2_tma_62x14_u2x2_pf2_mb2", "fuse3_tma_60x28_u2x2_pf2_mb1", "fuse3o_tma_60x28_u2x2_pf2_mb1",
            "fuse4_tma_58x26_u2x2_pf2_mb1", "fuse4_tma_58x10_u2x2_pf2_mb2"]


def _jacobi7_iter(A, a, b, h2inv, T, absmode=False):
    """T oracle sweeps, ping-pong with a fixed ring (Fig 1a semantics, reading R1)."""
    cur = np.array(A, copy=True)
    for _ in range(T):
        cur = oracle.jacobi7(cur, a, b, h2inv, absmode=absmode, out=cur.copy())
    return cur


@pytest.mark.parametrize("variant", FUSED_J7)
@pytest.mark.parametrize("dims", [(26, 30, 40), (9, 70, 260)], ids=lambda d: "x".join(map(str, d)))
def test_temporal_fusion_jacobi7(variant, dims):
    """NEXT-1 on Listing 1's 7-point Jacobi (the paper's 7pt-smoother, Table II):
    two sweeps per launch vs T oracle sweeps, odd and even T, ring untouched."""
    ins, sc = synth.jacobi7_inputs(dims, cfg="fuse")
    A = ins["A"]
    s = [sc["h2inv"], sc["a"], sc["b"]]
    fused = sdag.Plan(sdag.spec_text("jacobi7"), dims, variant=variant)
    for T in (1, 2, 5, 6):
        b0 = torch.from_numpy(A).cuda()
        b1 = b0.clone()
        n0 = sdag.launch_count()
        fused.apply_iterated(b0, b1, T, scalars=s)
        torch.cuda.synchronize()
        g = (b0 if T % 2 == 0 else b1).cpu().numpy()
        # launches flip the ping-pong pair once each, so #launches == T (mod 2)
        assert sdag.launch_count() - n0 == _expected_launches(fused, T, variant)
        O = _jacobi7_iter(A, sc["a"], sc["b"], sc["h2inv"], T)
        Aabs = _jacobi7_iter(np.abs(A), sc["a"], sc["b"], sc["h2inv"], T, absmode=True)
        gate(g, O, Aabs)
        assert np.array_equal(g[ring_mask(dims, 1)], A[ring_mask(dims, 1)])


def test_temporal_fusion_exact_closed_form():
    """V8 through the fused kernels: integer weights, quadratic input, bit-exact."""
    dims, T = (16, 18, 20), 4
    k, j, i = np.meshgrid(*[np.arange(n, dtype=np.float64) - n // 2 for n in dims], indexing="ij")
    p = 3 * i * i - 2 * j * j + 5 * k * k + i * j - 3 * j * k + 2 * i + 11
    plan = sdag.Plan(sdag.spec_text("smooth27"), dims)
    assert "temporal fusion" in plan.describe()
    b0 = torch.from_numpy(p.copy()).cuda()
    b1 = b0.clone()
    n0 = sdag.launch_count()
    plan.apply_iterated(b0, b1, T, scalars=[-128.0, 14.0, 3.0, 1.0, 1.0 / 32.0])
    torch.cuda.synchronize()
    assert sdag.launch_count() - n0 == 2  # two fused launches
    G = b0.cpu().numpy()
    assert np.array_equal(G, oracle.smooth27_iter(p, [-128.0, 14.0, 3.0, 1.0], 1 / 32, T))


@pytest.mark.parametrize("name", ["jacobi7", "smooth27"])
def test_iterated_cuda_graph_replay_is_bitwise(name, monkeypatch):
    """launch-bound iterations are replayed as a CUDA graph (2nd call captures,
    later calls replay): every call bitwise equal to plain launches, and the
    launch counter still counts the sweeps' kernels"""
    dims, T = (64, 64, 64), 12
    case = make_case(name, (20, 21, 22))  # scalars only
    s = case["s"]
    A = synth.uniform(dims, -1.0, 1.0, "graph", name)
    plan = sdag.Plan(sdag.spec_text(name), dims)
    monkeypatch.setenv("SDAG_GRAPHS", "0")
    r0 = torch.from_numpy(A).cuda()
    r1 = r0.clone()
    plan.apply_iterated(r0, r1, T, scalars=s)
    torch.cuda.synchronize()
    ref = r0.cpu().numpy()
    n_plain = None
    monkeypatch.setenv("SDAG_GRAPHS", "1")
    b0 = torch.from_numpy(A).cuda()
    b1 = b0.clone()
    for call in range(4):  # plain, capture + replay, replay, replay
        b0.copy_(torch.from_numpy(A))
        b1.copy_(b0)
        n0 = sdag.launch_count()
        plan.apply_iterated(b0, b1, T, scalars=s)
        torch.cuda.synchronize()
        n = sdag.launch_count() - n0
        n_plain = n if n_plain is None else n_plain
        assert n == n_plain > 0, (call, n, n_plain)
        assert np.array_equal(b0.cpu().numpy(), ref), call


@pytest.mark.parametrize("name,gdims", [("lap25", (44, 18, 20)), ("smooth27", (30, 20, 22))])
@pytest.mark.parametrize("P", [1, 3])
def test_dist_apply_host_bitwise_equal_single_gpu(name, gdims, P):
    """end to end per slab (host buffers with ghost planes, pipelined H2D /
    sweep / D2H): each rank's planes of the global interior equal the
    single-GPU sweep bitwise; every other output plane is left untouched"""
    case = make_case(name, gdims, cfg="slab")
    A = case["inputs"][0]
    s = case["s"]
    spec = sdag.spec_text(name)
    full = sdag.Plan(spec, gdims)
    dA = torch.from_numpy(A).cuda()
    dB = torch.full(gdims, float("nan"), dtype=torch.float64, device="cuda")
    full.apply([dB, dA], scalars=s)
    ref = dB.cpu().numpy()
    R = RADIUS[name]
    for r in range(P):
        d = sdag.Dist(spec, gdims, r, P)
        (nza, ny, nx), g0 = d.layout()
        hA = np.zeros((nza, ny, nx))
        lo, hi = max(g0, 0), min(g0 + nza, gdims[0])
        hA[lo - g0:hi - g0] = A[lo:hi]
        hB = np.full((nza, ny, nx), np.nan)
        up, down = d.apply_host([hB, hA], scalars=s)
        part = sdag.slab_partition(gdims[0], R, P, r)
        k0, k1 = part["k_lo"], part["k_hi"]  # local planes computed (global interior only)
        got = hB[k0:k1]
        assert np.array_equal(got, ref[g0 + k0:g0 + k1], equal_nan=True), f"rank {r} of {P}"
        untouched = np.ones(nza, bool)
        untouched[k0:k1] = False
        assert np.all(np.isnan(hB[untouched]))
        assert up == hA.nbytes and down == (k1 - k0) * (ny - 2 * R) * (nx - 2 * R) * 8


@pytest.mark.parametrize("T", [5, 12])
def test_generated_box_form_iterated_with_temporal_fusion(T):
    """the 27-point smoother forced through the generator is in box form: its
    single sweeps run the box kernel (FORM 2) and apply_iterated fuses pairs of
    sweeps with the FORM-2 fused kernel -- against the C oracle's T-sweep
    iteration under the 1e-12 gate (A_p = abs-mode iterate), ring fixed"""
    dims = (20, 22, 24)
    ins, sc = synth.smooth27_inputs(dims, cfg="iter")
    A = ins["A"]
    w = [sc[k] for k in ("w0", "w1", "w2", "w3")]
    plan = sdag.Plan(sdag.spec_text("smooth27"), dims, variant="jit")
    assert plan.info["variant"].startswith("jitbox_")
    b0 = torch.from_numpy(A).cuda()
    b1 = b0.clone()
    n0 = sdag.launch_count()
    plan.apply_iterated(b0, b1, T, scalars=[*w, sc["nu"]])
    torch.cuda.synchronize()
    assert sdag.launch_count() - n0 < T  # fused 2-sweep launches
    G = (b0 if T % 2 == 0 else b1).cpu().numpy()
    O = oracle.smooth27_iter(A, w, sc["nu"], T)
    Aabs = oracle.smooth27_iter(np.abs(A), np.abs(w), sc["nu"], T, absmode=True)
    gate(G, O, Aabs)
    assert np.array_equal(G[ring_mask(dims, 1)], A[ring_mask(dims, 1)])


def _shift_spec(off):
    return ("iterator k, j, i;\ndouble in[L,M,N], out[L,M,N];\nstencil s (B, A) {\n"
            f"B[k][j][i] = A[k{off[0]:+d}][j{off[1]:+d}][i{off[2]:+d}];\n}}\ns (out, in);\n")


def _shift_iter_oracle(A, off, T):
    cur = np.array(A, copy=True)
    for _ in range(T):
        cur = oracle.shift(cur, off, out=cur.copy())  # ring fixed (Fig 1a ping-pong semantics)
    return cur


@pytest.mark.parametrize("off", [(1, 0, 0), (-2, 1, 0), (4, -1, 2), (-3, 0, -1)])
@pytest.mark.parametrize("P", [2, 3, 4])
def test_shift_integer_coded_loopback_slabs_bitwise(off, P):
    """SURVEY 8(c) c4 "Halo bookkeeping": integer-coded input v = i + nx (j + ny k)
    (exact < 2^53) through a z-shift stencil iterated T times on P z-slabs with
    the NCCL path's halo schedule (moved by cudaMemcpy): every owned plane equals
    the global oracle bit for bit -- a ghost plane from the wrong rank, a wrong
    plane offset or a stale exchange shows up as a wrong integer."""
    gdims, T = (40, 14, 18), 5
    nz, ny, nx = gdims
    A = np.arange(nz * ny * nx, dtype=np.float64).reshape(gdims)
    ref = _shift_iter_oracle(A, off, T)
    spec = _shift_spec(off)
    dists = [sdag.Dist(spec, gdims, r, P) for r in range(P)]
    bufs0, bufs1 = [], []
    for d in dists:
        (nza, _, _), g0 = d.layout()
        loc = np.full((nza, ny, nx), -1.0)
        lo, hi = max(g0, 0), min(g0 + nza, nz)
        loc[lo - g0:hi - g0] = A[lo:hi]
        bufs0.append(torch.from_numpy(loc).cuda())
        bufs1.append(torch.from_numpy(loc.copy()).cuda())
    sdag.Dist.apply_iterated_loopback(dists, bufs0, bufs1, T)
    torch.cuda.synchronize()
    res = bufs0 if T % 2 == 0 else bufs1
    for r, d in enumerate(dists):
        part = sdag.slab_partition(nz, abs(off[0]), P, r)
        (_, _, _), g0 = d.layout()
        z0, n = part["z0"], part["nz_own"]
        got = res[r].cpu().numpy()[z0 - g0:z0 - g0 + n]
        assert np.array_equal(got, ref[z0:z0 + n]), f"rank {r} of {P}"

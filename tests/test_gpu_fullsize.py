"""Full-size parity, EVERY point: the BASELINE workloads (SURVEY 8(d) table,
configs 1b-5) in the launch configuration bench.py times (default plan and
tune=1 plan), compared element by element with a full oracle sweep of the
same seeded input under the north-star gate e_p <= 1e-12 (tests/cases.gate,
DESIGN R13).  Config 5 (1024^3, T = 12) is compared on whole z-slab regions
(all 1024 x 1024 points of each plane) -- bottom ring, a z-chunk seam, top
ring -- which the oracle iterates on a plane window wide enough (T + 1 planes
beyond each side) that its own window faces cannot reach the compared planes.
"""
from __future__ import annotations

import numpy as np
import pytest

import oracle
import synth
from cases import gate, interior, ring_mask

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("no CUDA device", allow_module_level=True)

import paper_conf_ipps_rawatvsrps19_b200 as sdag  # noqa: E402


def _nan(dims, n):
    return [torch.full(tuple(dims), float("nan"), dtype=torch.float64, device="cuda") for _ in range(n)]


@pytest.mark.parametrize("tune", [False, True])
def test_full_lap25_every_point(tune):
    """config 2: 512^3, 128 M interior points, all compared."""
    dims = (512, 512, 512)
    ins, sc = synth.lap25_inputs(dims)
    A = ins["A"]
    c = [sc[k] for k in ("c0", "c1", "c2", "c3", "c4")]
    plan = sdag.Plan(sdag.spec_text("lap25"), dims, tune=tune)
    dA = torch.from_numpy(A).cuda()
    (dB,) = _nan(dims, 1)
    plan.apply([dB, dA], scalars=c)
    torch.cuda.synchronize()
    del dA
    G = dB.cpu().numpy()
    del dB
    I = interior(dims, 4)
    o = oracle.lap25(A, c)
    a = oracle.lap25(np.abs(A), np.abs(c), absmode=True)
    gate(G[I], o[I], a[I], what=plan.info["variant"])
    assert np.all(np.isnan(G[ring_mask(dims, 4)]))


@pytest.mark.parametrize("tune", [False, True])
def test_full_hypterm_every_point(tune):
    """config 3: 320^3, 8 inputs, 5 outputs, every interior point of every flux."""
    dims = (320, 320, 320)
    ins, sc = synth.hypterm_inputs(dims)
    arrs = [ins[k] for k in oracle.HYPTERM_INPUTS]
    s = [sc[k] for k in ("dxinv0", "dxinv1", "dxinv2", "ALP", "BET", "GAM", "DEL")]
    plan = sdag.Plan(sdag.spec_text("hypterm"), dims, tune=tune)
    dev = [torch.from_numpy(x).cuda() for x in arrs]
    outs = _nan(dims, 5)
    plan.apply(outs + dev, scalars=s)
    torch.cuda.synchronize()
    del dev
    G = [t.cpu().numpy() for t in outs]
    del outs
    o = oracle.hypterm(arrs, s[:3], s[3:])
    a = oracle.hypterm([np.abs(x) for x in arrs], np.abs(s[:3]), np.abs(s[3:]), absmode=True)
    I = interior(dims, 4)
    ring = ring_mask(dims, 4)
    for m in range(5):
        gate(G[m][I], o[m][I], a[m][I], what=f"flux_{m} {plan.info['variant']}")
        assert np.all(np.isnan(G[m][ring]))


@pytest.mark.parametrize("tune", [False, True])
def test_full_rhs4_every_point(tune):
    """config 4: 320^3, uacc inout with a1 = 1, every interior point."""
    dims = (320, 320, 320)
    ins, sc = synth.rhs4_inputs(dims)
    u = [ins["u0"], ins["u1"], ins["u2"]]
    ua = [ins["uacc0"], ins["uacc1"], ins["uacc2"]]
    a1d = [ins["strx"], ins["stry"], ins["strz"]]
    s = [sc[k] for k in ("tf", "i6", "i144", "cof", "a1")]
    plan = sdag.Plan(sdag.spec_text("rhs4center"), dims, tune=tune)
    d_ua = [torch.from_numpy(x.copy()).cuda() for x in ua]
    d_in = [torch.from_numpy(x).cuda() for x in (*u, ins["mu"], ins["la"])]
    plan.apply(d_ua + d_in, [torch.from_numpy(x).cuda() for x in a1d], s)
    torch.cuda.synchronize()
    del d_in
    G = [t.cpu().numpy() for t in d_ua]
    del d_ua
    o = oracle.rhs4(u, ins["mu"], ins["la"], *a1d, ua, *s)
    a = oracle.rhs4([np.abs(x) for x in u], np.abs(ins["mu"]), np.abs(ins["la"]), *[np.abs(x) for x in a1d],
                    [np.abs(x) for x in ua], *np.abs(s), absmode=True)
    I = interior(dims, 2)
    ring = ring_mask(dims, 2)
    for c in range(3):
        gate(G[c][I], o[c][I], a[c][I], what=f"uacc{c} {plan.info['variant']}")
        assert np.array_equal(G[c][ring], ua[c][ring])


@pytest.mark.parametrize("tune", [False, True])
def test_full_jacobi7_batched_every_point(tune):
    """config 1b: 128 independent 64^3 problems in one launch, every problem."""
    dims, batch = (64, 64, 64), 128
    ins, sc = synth.jacobi7_inputs(dims, cfg="cfg1", batch=batch)
    A = ins["A"]
    plan = sdag.Plan(sdag.spec_text("jacobi7"), dims, batch=batch, tune=tune)
    dA = torch.from_numpy(A).cuda()
    dB = torch.full(A.shape, float("nan"), dtype=torch.float64, device="cuda")
    plan.apply_batched(batch, [dB, dA], scalars=[sc["h2inv"], sc["a"], sc["b"]])
    torch.cuda.synchronize()
    G = dB.cpu().numpy()
    I = interior(dims, 1)
    ring = ring_mask(dims, 1)
    for b in range(batch):
        o = oracle.jacobi7(A[b], sc["a"], sc["b"], sc["h2inv"])
        a = oracle.jacobi7(np.abs(A[b]), sc["a"], sc["b"], sc["h2inv"], absmode=True)
        gate(G[b][I], o[I], a[I], what=plan.info["variant"])
        assert np.all(np.isnan(G[b][ring]))


def _plane_window(z0, z1, dims, T):
    """planes [z0, z1) to compare; the oracle iterates planes [w0, w1) with
    w0 = max(0, z0 - T - 1), w1 = min(nz, z1 + T + 1): a window face that is not
    a global face is >= T + 1 planes from every compared plane, and after T
    sweeps a value depends only on inputs within distance T."""
    return max(0, z0 - T - 1), min(dims[0], z1 + T + 1)


@pytest.mark.parametrize("tune", [False, True])
def test_full_smooth27_iterated_slabs_every_point(tune):
    """config 5 on one GPU (the per-GPU slab of the weak-scaled run): 1024^3,
    T = 12, the fused kernels and DP schedule bench.py times.  Three 24-plane
    slabs compared at all 1024 x 1024 points: the bottom (global ring plane 0
    and the planes the DP's first launches touch), one across the middle
    (z-chunk seams), and the top."""
    dims, T = (1024, 1024, 1024), 12
    nz, ny, nx = dims
    w = [synth.SMOOTH27_W[k] for k in ("w0", "w1", "w2", "w3")]
    nu = synth.SMOOTH27_W["nu"]
    b0 = synth.uniform_torch(dims, -1.0, 1.0, "cfg5", "A")
    b1 = b0.clone()
    plan = sdag.Plan(sdag.spec_text("smooth27"), dims, tune=tune)
    plan.apply_iterated(b0, b1, T, scalars=[*w, nu])
    torch.cuda.synchronize()
    res = b0 if T % 2 == 0 else b1
    for z0, z1 in [(0, 24), (500, 524), (nz - 24, nz)]:
        w0, w1 = _plane_window(z0, z1, dims, T)
        lin0, lin1 = w0 * ny * nx, w1 * ny * nx
        win = synth.uniform_at(np.arange(lin0, lin1, dtype=np.int64), -1.0, 1.0, "cfg5", "A").reshape(w1 - w0, ny, nx)
        o = oracle.smooth27_iter(win, w, nu, T)[z0 - w0:z1 - w0]
        a = oracle.smooth27_iter(np.abs(win), np.abs(w), nu, T, absmode=True)[z0 - w0:z1 - w0]
        g = res[z0:z1].cpu().numpy()
        gate(g, o, a, what=f"planes [{z0},{z1}) {plan.info['variant']}")
        del win, o, a, g


@pytest.mark.parametrize("name", ["lap25", "hypterm", "rhs4center", "smooth27"])
def test_large_ragged_every_point(name):
    """A large grid ragged in every axis (no extent a multiple of any tile or
    z-chunk; nx even so the TMA path runs): every interior point vs the oracle,
    every ring point untouched -- the tile and chunk tails at scale."""
    from cases import make_case, run_gpu, check
    dims = {"lap25": (389, 262, 514), "hypterm": (211, 197, 302), "rhs4center": (203, 181, 266),
            "smooth27": (401, 277, 390)}[name]
    case = make_case(name, dims, cfg="ragged")
    g, plan = run_gpu(name, dims, case)
    assert "tma" in plan.info["variant"]
    check(name, dims, g, case)

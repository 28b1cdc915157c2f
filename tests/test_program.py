"""Multi-stencil programs (Fig 3c).

CPU part (-m "not gpu"):
* the oracle's program evaluator (oracle/interp.py evaluate_program) pinned to
  things other than itself: the paper's own Fig 3c trivial fission of
  rhs4center must reproduce the hand-written C oracle bitwise (each stage
  keeps the original statements, in order); the two-stage Laplacian of a
  Laplacian is the exact biharmonic of a per-axis-cubic integer polynomial;
  abs-mode bounds;
* the C++ front-end's program analysis on host-only plans: argument order
  (declaration order), program-level roles, per-stage canonical counts (Fig 3:
  the fission replicates the 84-flop mu/la temporaries, 3 x 278 flops),
  error statuses.
GPU part (-m gpu): the same programs through sdag_program_apply vs the oracle."""
from __future__ import annotations

import numpy as np
import pytest

import oracle
import paper_conf_ipps_rawatvsrps19_b200 as sdag
import synth
from cases import gate
from oracle import interp
from specgen import BIHARM, rhs4_fission_program

HOST = -2  # SDAG_DEVICE_NONE: analysis-only plans, no GPU


def _cubic_poly(seed):
    """Integer polynomial sum_t f_t(z) g_t(y) h_t(x), every factor cubic; returns
    (p, biharmonic of p) as functions of centred integer coordinates."""
    rng = np.random.default_rng(seed)
    P = np.polynomial.Polynomial
    terms = [[P(rng.integers(-3, 4, 4).astype(float)) for _ in range(3)] for _ in range(3)]

    def p(z, y, x):
        return sum(f(z) * g(y) * h(x) for f, g, h in terms)

    def lap(z, y, x):  # Delta p (the 7-point Laplacian is exact for per-axis cubics)
        return sum(f.deriv(2)(z) * g(y) * h(x) + f(z) * g.deriv(2)(y) * h(x) + f(z) * g(y) * h.deriv(2)(x)
                   for f, g, h in terms)

    def bih(z, y, x):  # Delta^2 p: fourth derivatives of cubics vanish
        out = 0.0
        for f, g, h in terms:
            f2, g2, h2 = f.deriv(2), g.deriv(2), h.deriv(2)
            out = out + 2.0 * (f2(z) * g2(y) * h(x) + f2(z) * g(y) * h2(x) + f(z) * g2(y) * h2(x))
        return out

    return p, lap, bih


def _grid(dims):
    z, y, x = np.meshgrid(*[np.arange(n, dtype=float) - n // 2 for n in dims], indexing="ij")
    return z, y, x


# ---------------------------------------------------------------- oracle pins

def test_program_biharmonic_closed_form():
    dims = (13, 14, 16)
    p, lap, bih = _cubic_poly(7)
    z, y, x = _grid(dims)
    A = p(z, y, x)
    T0 = np.zeros(dims)
    B0 = np.full(dims, np.nan)
    out = interp.evaluate_program(BIHARM, dims, {"A": A, "T": T0, "B": B0}, {"c": 1.0})
    assert set(out) == {"T", "B"}
    I2 = (slice(2, -2),) * 3
    assert np.array_equal(out["B"][I2], bih(z, y, x)[I2])  # exact: integers < 2^53
    # stage 1 alone is the 7-point Laplacian (exact for cubics): Delta p
    I1 = (slice(1, -1),) * 3
    assert np.array_equal(out["T"][I1], lap(z, y, x)[I1])
    # B outside its own interior [1, n-1) is untouched
    ring = np.ones(dims, bool)
    ring[I1] = False
    assert np.all(np.isnan(out["B"][ring]))


def test_fig3c_fission_program_equals_c_oracle_bitwise():
    dims = (12, 13, 15)
    ins, sc = synth.rhs4_inputs(dims, cfg="prog")
    prog = rhs4_fission_program(sdag.spec_text("rhs4center"))
    arrays = {k: ins[k] for k in ("uacc0", "uacc1", "uacc2", "u0", "u1", "u2", "mu", "la", "strx", "stry", "strz")}
    out = interp.evaluate_program(prog, dims, arrays, sc)
    ref = oracle.rhs4([ins["u0"], ins["u1"], ins["u2"]], ins["mu"], ins["la"], ins["strx"], ins["stry"], ins["strz"],
                      [ins["uacc0"], ins["uacc1"], ins["uacc2"]], sc["tf"], sc["i6"], sc["i144"], sc["cof"], sc["a1"])
    for m in range(3):
        assert np.array_equal(out[f"uacc{m}"], ref[m]), f"uacc{m}"


def test_program_absmode_bound():
    dims = (12, 12, 12)
    rng = np.random.default_rng(3)
    A = rng.uniform(-1, 1, dims)
    T0 = np.zeros(dims)
    o = interp.evaluate_program(BIHARM, dims, {"A": A, "T": T0, "B": np.zeros(dims)}, {"c": -0.7})
    a = interp.evaluate_program(BIHARM, dims, {"A": np.abs(A), "T": T0, "B": np.zeros(dims)}, {"c": -0.7},
                                absmode=True)
    for k in ("T", "B"):
        assert np.all(np.abs(o[k]) <= a[k])


def test_program_stages_split():
    st = interp.program_stages(BIHARM)
    assert [b for _, b in st] == [{"out": "T", "in": "A", "c": "c"}, {"out": "B", "in": "T", "c": "c"}]


# ------------------------------------------------------ C++ front-end (host)

def test_program_host_analysis_biharmonic():
    g = sdag.Program(BIHARM, (20, 21, 22), device=HOST)
    assert g.counts == {"n_stages": 2, "n_arrays3d": 3, "n_arrays1d": 0, "n_scalars": 1}
    assert g.args() == [(0, 0, "A", 0), (0, 1, "T", 1), (0, 2, "B", 1), (2, 0, "c", -1)]
    for s in range(2):
        i = g.stage(s).info
        assert i["radius"] == (1, 1, 1) and i["flops_per_point"] == 8.0


def test_program_host_analysis_fig3c_fission():
    g = sdag.Program(rhs4_fission_program(sdag.spec_text("rhs4center")), (20, 20, 20), device=HOST)
    c = g.counts
    assert c == {"n_stages": 3, "n_arrays3d": 8, "n_arrays1d": 3, "n_scalars": 5}
    names = [a[2] for a in g.args()]
    assert names == ["uacc0", "uacc1", "uacc2", "u0", "u1", "u2", "mu", "la", "strx", "stry", "strz",
                     "tf", "i6", "i144", "cof", "a1"]
    roles = {a[2]: a[3] for a in g.args() if a[0] == 0}
    assert roles == {"uacc0": 2, "uacc1": 2, "uacc2": 2, "u0": 0, "u1": 0, "u2": 0, "mu": 0, "la": 0}
    # Fig 3: every fission stage replicates the 84-flop mu/la temporaries: 84 + 75 + 116 + 3 = 278 per output
    flops = [g.stage(s).info["flops_per_point"] for s in range(3)]
    assert flops == [278.0, 278.0, 278.0]
    assert sum(flops) - 2 * 84 == 666.0  # = Table I's rhs4center when the temporaries are shared


def _status(fn):
    with pytest.raises(sdag.SdagError) as e:
        fn()
    return e.value.status


def test_program_errors():
    assert _status(lambda: sdag.Plan(BIHARM, (20, 20, 20), device=HOST)) == 4  # UNSUPPORTED: use a program
    undefined = BIHARM.replace("lap(B, T, c);", "lop(B, T, c);")
    assert _status(lambda: sdag.Program(undefined, (20, 20, 20), device=HOST)) == 3  # SEMANTIC
    twice = BIHARM.replace("lap(T, A, c);", "stencil lap (o, a) { o[k][j][i] = a[k][j][i]; }\nlap(T, A, c);")
    assert _status(lambda: sdag.Program(twice, (20, 20, 20), device=HOST)) == 3
    nocall = BIHARM.replace("lap(T, A, c);\nlap(B, T, c);", "stencil cp (o, a) { o[k][j][i] = a[k][j][i]; }")
    assert _status(lambda: sdag.Program(nocall, (20, 20, 20), device=HOST)) == 3
    arity = BIHARM.replace("lap(B, T, c);", "lap(B, T);")
    assert _status(lambda: sdag.Program(arity, (20, 20, 20), device=HOST)) == 3
    # a single-call spec is a one-stage program with formal == declared order
    g = sdag.Program(sdag.spec_text("lap25"), (20, 20, 20), device=HOST)
    assert g.counts["n_stages"] == 1


# ------------------------------------------------------------------- GPU

@pytest.mark.gpu
def test_gpu_program_biharmonic():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    dims = (40, 36, 50)
    A = synth.uniform(dims, -1.0, 1.0, "prog", "A")
    T0 = np.zeros(dims)
    B0 = np.full(dims, np.nan)
    c = 0.25
    g = sdag.Program(BIHARM, dims)
    d = [torch.from_numpy(x.copy()).cuda() for x in (A, T0, B0)]
    n0 = sdag.launch_count()
    g.apply(d, [], [c])
    torch.cuda.synchronize()
    assert sdag.launch_count() - n0 == 2
    o = interp.evaluate_program(BIHARM, dims, {"A": A, "T": T0, "B": B0}, {"c": c})
    a = interp.evaluate_program(BIHARM, dims, {"A": np.abs(A), "T": T0, "B": np.zeros(dims)}, {"c": c}, absmode=True)
    I = (slice(1, -1),) * 3
    gT, gB = d[1].cpu().numpy(), d[2].cpu().numpy()
    gate(gT[I], o["T"][I], a["T"][I])
    gate(gB[I], o["B"][I], a["B"][I])  # two stages, same 1e-12 gate vs the abs-mode composition (R13, R21)
    ring = np.ones(dims, bool)
    ring[I] = False
    assert np.all(np.isnan(gB[ring])) and np.all(gT[ring] == 0.0)


@pytest.mark.gpu
def test_gpu_program_fig3c_fission_matches_oracle():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    dims = (22, 37, 40)
    ins, sc = synth.rhs4_inputs(dims, cfg="prog")
    prog = rhs4_fission_program(sdag.spec_text("rhs4center"))
    g = sdag.Program(prog, dims)
    names3 = ["uacc0", "uacc1", "uacc2", "u0", "u1", "u2", "mu", "la"]
    d3 = [torch.from_numpy(ins[k].copy()).cuda() for k in names3]
    d1 = [torch.from_numpy(ins[k]).cuda() for k in ("strx", "stry", "strz")]
    g.apply(d3, d1, [sc[k] for k in ("tf", "i6", "i144", "cof", "a1")])
    torch.cuda.synchronize()
    u = [ins["u0"], ins["u1"], ins["u2"]]
    ua = [ins["uacc0"], ins["uacc1"], ins["uacc2"]]
    s = [sc[k] for k in ("tf", "i6", "i144", "cof", "a1")]
    o = oracle.rhs4(u, ins["mu"], ins["la"], ins["strx"], ins["stry"], ins["strz"], ua, *s)
    a = oracle.rhs4([np.abs(x) for x in u], np.abs(ins["mu"]), np.abs(ins["la"]),
                    *[np.abs(ins[k]) for k in ("strx", "stry", "strz")], [np.abs(x) for x in ua], *np.abs(s),
                    absmode=True)
    I = (slice(2, -2),) * 3
    for m in range(3):
        gm = d3[m].cpu().numpy()
        gate(gm[I], o[m][I], a[m][I], what=f"uacc{m}")
        ring = np.ones(dims, bool)
        ring[I] = False
        assert np.array_equal(gm[ring], ua[m][ring])


@pytest.mark.gpu
def test_gpu_program_validates_before_enqueue():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    dims = (20, 20, 20)
    g = sdag.Program(BIHARM, dims)
    A = torch.rand(dims, dtype=torch.float64, device="cuda")
    T = torch.zeros(dims, dtype=torch.float64, device="cuda")
    n0 = sdag.launch_count()
    with pytest.raises(sdag.SdagError):
        g.apply([A, T], [], [1.0])  # missing B
    with pytest.raises(sdag.SdagError):
        g.apply([A, T, T], [], [1.0])  # stage 2 writes B == T, which it reads: aliasing
    assert sdag.launch_count() == n0  # nothing enqueued, not even stage 1

#!/usr/bin/env python3
"""One small launch of every sm_100a kernel family, for compute-sanitizer
(memcheck / synccheck / racecheck of the TMA + mbarrier rings and
the P2P flag protocol).  Small grids keep the instrumented run short.

usage: compute-sanitizer --tool TOOL python tools/sanitize_run.py [FAMILY ...]
families: star box27 fuse2 fuseN hyp hypc rhs4 rhs4f sweep lsu jit p2p
"""
import sys
from pathlib import Path

import numpy as np
import torch

sys.path.insert(0, str(Path(__file__).resolve().parents[1]))
import paper_conf_ipps_rawatvsrps19_b200 as sdag  # noqa: E402
import synth  # noqa: E402

SCAL = {"lap25": list(synth.LAP25_COEFS.values()), "jacobi7": [4.0, 0.5, 0.25],
        "smooth27": [synth.SMOOTH27_W[k] for k in ("w0", "w1", "w2", "w3", "nu")],
        "hypterm": [0.5, 0.25, 0.125, 0.8, -0.2, 4 / 105, -1 / 280],
        "rhs4center": [0.75, 1 / 6, 1 / 144, 1.0, 1.0]}


def one(name, dims, variant=None, iterated=0, deg=2):
    plan = sdag.Plan(sdag.spec_text(name), dims, variant=variant)
    info = plan.info
    g = torch.Generator(device="cuda").manual_seed(3)
    arrs = [torch.rand(dims, dtype=torch.float64, device="cuda", generator=g) + 0.5 for _ in range(info["n_arrays3d"])]
    a1 = [torch.rand(dims[2 - q], dtype=torch.float64, device="cuda") + 0.5 for q in range(info["n_arrays1d"])]
    if iterated:
        plan.apply_iterated(arrs[0], arrs[1], iterated, SCAL[name])
    else:
        plan.apply(arrs, a1, SCAL[name])
    torch.cuda.synchronize()
    if iterated:  # the fused kernel apply_iterated launched (temporal fusion of `iterated` sweeps)
        fl = [ln.strip() for ln in plan.describe().splitlines() if "temporal fusion" in ln]
        print(f"{name} {fl[0] if fl else info['variant']} | {plan.kernel_name(deg)} ok", flush=True)
    else:
        print(f"{name} {info['variant']} {plan.kernel_name(1)} ok", flush=True)


def p2p():
    spec = sdag.spec_text("smooth27")
    gdims = (24, 20, 22)
    P = 2
    dists = [sdag.Dist(spec, gdims, r, P, time_tile=2) for r in range(P)]
    A = synth.uniform(gdims, -1.0, 1.0, "san", "A")
    for r, d in enumerate(dists):
        b0, _ = d.p2p_alloc()
        (nza, ny, nx), g0 = d.layout()
        part = sdag.slab_partition2(gdims[0], 1, 2, P, r)
        z0, n = part["z0"], part["nz_own"]
        b0[z0 - g0:z0 - g0 + n] = torch.from_numpy(np.ascontiguousarray(A[z0:z0 + n])).cuda()
    dists[0].p2p_attach(1, dists[1])
    dists[1].p2p_attach(0, dists[0])
    streams = [torch.cuda.Stream() for _ in range(P)]
    torch.cuda.synchronize()
    for d, st in zip(dists, streams):
        d.p2p_apply_iterated(4, scalars=SCAL["smooth27"], stream=st)
    torch.cuda.synchronize()
    print("p2p 2 slabs ok", flush=True)


FAM = {
    "star": lambda: one("lap25", (20, 40, 72)),
    "box27": lambda: one("smooth27", (12, 34, 140)),
    "fuse2": lambda: one("smooth27", (12, 34, 140), "fuse2o_tma_62x14_u2x2_pf2_mb2", iterated=4),
    "fuseN": lambda: one("smooth27", (12, 34, 140), "fuse3_tma_60x28_u2x2_pf2_mb1", iterated=3, deg=3),
    "hyp": lambda: one("hypterm", (12, 20, 72)),
    "hypc": lambda: one("hypterm", (12, 20, 72), "hypc_tma_64x8_u2x1_pf2"),
    "rhs4": lambda: one("rhs4center", (9, 20, 36)),
    "rhs4f": lambda: [one("rhs4center", (9, 20, 36), v) for v in ("r4f_tma_32x16_u2x1_pf1", "r4g_tma_32x16_u2x1_pf0")],
    "sweep": lambda: one("lap25", (12, 20, 72), "tma_64x16_u1x4_pf1"),
    "lsu": lambda: [one(n, (11, 13, 35)) for n in ("lap25", "smooth27", "hypterm", "rhs4center", "jacobi7")],
    "jit": lambda: one("lap25", (12, 20, 40), "jit"),
    "p2p": p2p,
}

if __name__ == "__main__":
    for f in sys.argv[1:] or list(FAM):
        FAM[f]()

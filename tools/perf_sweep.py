#!/usr/bin/env python3
"""Time every candidate variant of every BASELINE stencil on the GPU (CUDA
events, inputs > L2, warm-up first) and print one JSON line per (dag, variant)
with GFLOP/s, algorithmic GB/s and the HBM roofline fraction.  Development
tool (the headline number is bench.py's)."""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_rawatvsrps19_b200 as sdag  # noqa: E402

PEAK = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"] if os.path.exists(
    os.path.join(ROOT, "MEASURED_PEAKS.json")) else 6650.0

CFG = {
    "lap25": ((512, 512, 512), 1, [-205 / 24, 8 / 5, -0.2, 8 / 315, -1 / 560]),
    "jacobi7": ((64, 64, 64), 128, [4.0, 0.5, 0.25]),
    "smooth27": ((512, 512, 512), 1, [-128 / 30, 14 / 30, 3 / 30, 1 / 30, 0.125]),
    "hypterm": ((320, 320, 320), 1, [0.5, 0.25, 0.125, 0.8, -0.2, 4 / 105, -1 / 280]),
    "rhs4center": ((320, 320, 320), 1, [0.75, 1 / 6, 1 / 144, 1.0, 1.0]),
}


def run(name, reps, only=None):
    dims, batch, scal = CFG[name]
    spec = sdag.spec_text(name)
    base = sdag.Plan(spec, dims, batch=batch)
    info = base.info
    n3, n1 = info["n_arrays3d"], info["n_arrays1d"]
    shape = (batch, *dims) if batch > 1 else dims
    g = torch.Generator(device="cuda").manual_seed(1)
    arrs = [torch.rand(shape, dtype=torch.float64, device="cuda", generator=g) + 0.5 for _ in range(n3)]
    # 1D arrays in formal order strx (nx), stry (ny), strz (nz)
    a1 = [torch.rand(dims[2 - q], dtype=torch.float64, device="cuda") + 0.5 for q in range(n1)]
    flops = info["flops_per_point"] * info["points"] * batch
    byts = info["bytes_per_point"] * info["points"] * batch
    out = []
    for v in base.variants():
        if only and only not in v:
            continue
        p = sdag.Plan(spec, dims, batch=batch, variant=v)
        f = (lambda: p.apply_batched(batch, arrs, a1, scal)) if batch > 1 else (lambda: p.apply(arrs, a1, scal))
        for _ in range(3):
            f()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(reps):
            f()
        e1.record()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / reps
        r = {"dag": name, "variant": v, "ms": round(ms, 4), "gflops": round(flops / ms / 1e6, 1),
             "gbs": round(byts / ms / 1e6, 1), "hbm_frac": round(byts / ms / 1e6 / PEAK, 4)}
        print(json.dumps(r), flush=True)
        out.append(r)
    return out


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("dags", nargs="*", default=list(CFG))
    ap.add_argument("--reps", type=int, default=10)
    ap.add_argument("--only", default=None)
    a = ap.parse_args()
    for n in a.dags:
        run(n, a.reps, a.only)

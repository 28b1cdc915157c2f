#!/usr/bin/env python3
"""apply_iterated on a small grid (config 1's 64^3 Jacobi, T sweeps): plain
launches vs CUDA-graph replay (ms per sweep)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import paper_conf_ipps_rawatvsrps19_b200 as sdag  # noqa: E402

for n, T in ((64, 100), (128, 100), (256, 24)):
    dims = (n, n, n)
    b0 = torch.rand(dims, dtype=torch.float64, device="cuda")
    b1 = b0.clone()
    out = {"dims": list(dims), "T": T}
    for g in ("0", "1"):
        os.environ["SDAG_GRAPHS"] = g
        plan = sdag.Plan(sdag.spec_text("jacobi7"), dims)
        for _ in range(3):
            plan.apply_iterated(b0, b1, T, [4.0, 0.5, 0.25])
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record()
        for _ in range(10):
            plan.apply_iterated(b0, b1, T, [4.0, 0.5, 0.25])
        e1.record()
        torch.cuda.synchronize()
        out["graph_us_per_sweep" if g == "1" else "plain_us_per_sweep"] = round(e0.elapsed_time(e1) / 10 / T * 1e3, 2)
    print(json.dumps(out), flush=True)

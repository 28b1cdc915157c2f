#!/usr/bin/env python3
"""Profile-guided classification (paper Section IV) of every BASELINE stencil's
default kernel at its BASELINE size: one JSON line per stencil (Plan.profile)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_ipps_rawatvsrps19_b200 as sdag  # noqa: E402
from tools.perf_sweep import CFG  # noqa: E402

peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))).get("hbm_gbs", 0.0) \
    if os.path.exists(os.path.join(ROOT, "MEASURED_PEAKS.json")) else 0.0
fp64 = sdag.fp64_peak() / 1e12
for name, (dims, batch, scal) in CFG.items():
    if batch > 1:
        dims = (64, 256, 256)  # profile() takes one problem: config 1b's bytes as one grid
    plan = sdag.Plan(sdag.spec_text(name), dims)
    g = torch.Generator(device="cuda").manual_seed(1)
    a3 = [torch.rand(dims, dtype=torch.float64, device="cuda", generator=g) + 0.5 for _ in range(plan.info["n_arrays3d"])]
    a1 = [torch.rand(dims[2 - q], dtype=torch.float64, device="cuda", generator=g) + 0.5
          for q in range(plan.info["n_arrays1d"])]
    pr = plan.profile(a3, a1, scal, peak_hbm_gbs=peak, peak_fp64_tflops=fp64)
    pr.update({"dag": name, "dims": list(dims)})
    print(json.dumps(pr), flush=True)
    del a3, a1
    torch.cuda.empty_cache()

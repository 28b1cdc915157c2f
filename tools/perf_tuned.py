#!/usr/bin/env python3
"""Heuristic vs hierarchical tune=1 plan of a BASELINE stencil at its BASELINE
size: chosen variant, z-chunk and time (CUDA events).  One JSON line."""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_ipps_rawatvsrps19_b200 as sdag  # noqa: E402
from tools.perf_sweep import CFG  # noqa: E402

name = sys.argv[1]
dims, batch, scal = CFG[name]
spec = sdag.spec_text(name)
out = {"dag": name}
for tune in (False, True):
    t0 = time.perf_counter()
    p = sdag.Plan(spec, dims, batch=batch, tune=tune)
    tplan = time.perf_counter() - t0
    info = p.info
    shape = (batch, *dims) if batch > 1 else dims
    g = torch.Generator(device="cuda").manual_seed(1)
    a3 = [torch.rand(shape, dtype=torch.float64, device="cuda", generator=g) + 0.5 for _ in range(info["n_arrays3d"])]
    a1 = [torch.rand(dims[2 - q], dtype=torch.float64, device="cuda") + 0.5 for q in range(info["n_arrays1d"])]
    f = (lambda: p.apply_batched(batch, a3, a1, scal)) if batch > 1 else (lambda: p.apply(a3, a1, scal))
    for _ in range(3):
        f()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record()
    for _ in range(20):
        f()
    e1.record()
    torch.cuda.synchronize()
    zl = [w for w in p.describe().split("  ") if w.startswith("z-chunk")]
    out["tuned" if tune else "heuristic"] = {"variant": info["variant"], "ms": e0.elapsed_time(e1) / 20,
                                             "plan_s": round(tplan, 2), "zchunk": zl[0] if zl else None}
    del a3, a1
    torch.cuda.empty_cache()
print(json.dumps(out), flush=True)

#!/usr/bin/env python3
"""Run one DAG at its BASELINE size a few times (for ncu captures)."""
import sys, os
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT); sys.path.insert(0, os.path.join(ROOT, "tools"))
import torch
from perf_sweep import CFG
import paper_conf_ipps_rawatvsrps19_b200 as sdag
name = sys.argv[1]; variant = sys.argv[2] if len(sys.argv) > 2 and sys.argv[2] != "-" else None
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 4
dims, batch, scal = CFG[name]
p = sdag.Plan(sdag.spec_text(name), dims, batch=batch, variant=variant)
i = p.info
shape = (batch, *dims) if batch > 1 else dims
arrs = [torch.rand(shape, dtype=torch.float64, device="cuda") + 0.5 for _ in range(i["n_arrays3d"])]
a1 = [torch.rand(dims[2 - q], dtype=torch.float64, device="cuda") + 0.5 for q in range(i["n_arrays1d"])]
for _ in range(reps):
    if batch > 1: p.apply_batched(batch, arrs, a1, scal)
    else: p.apply(arrs, a1, scal)
torch.cuda.synchronize()
print(name, i["variant"], "ok")

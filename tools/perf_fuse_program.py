#!/usr/bin/env python3
"""Staged program vs its maxfuse (recomputation) on the GPU: the Laplacian of a
Laplacian at 512^3 -- two sweeps through HBM (A -> T -> B) vs one fused
generated stencil (A -> B, T recomputed at its 7 read offsets)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import torch  # noqa: E402

import paper_conf_ipps_rawatvsrps19_b200 as sdag  # noqa: E402
from specgen import BIHARM  # noqa: E402

n = 512
dims = (n, n, n)
A = torch.rand(dims, dtype=torch.float64, device="cuda")
T = torch.zeros_like(A)
B = torch.zeros_like(A)


def timed(f, reps=10):
    for _ in range(3):
        f()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record()
    for _ in range(reps):
        f()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


prog = sdag.Program(BIHARM, dims)
ms_staged = timed(lambda: prog.apply([A, T, B], [], [0.25]))
fused = sdag.Plan(sdag.fuse_program(BIHARM, keep_intermediates=False), dims, tune=True)
names = [nm for kind, _, nm, _ in fused.args() if kind == 0]
arr = {"A": A, "T": T, "B": B}
ms_fused = timed(lambda: fused.apply([arr[x] for x in names], [], [0.25]))
print(json.dumps({"staged_ms": round(ms_staged, 4), "fused_ms": round(ms_fused, 4),
                  "fused_variant": fused.info["variant"], "fused_flops_per_point": fused.info["flops_per_point"],
                  "speedup": round(ms_staged / ms_fused, 3)}))

#!/usr/bin/env python3
"""Ablation of the z-chunking heuristic (concurrent streaming):
time one DAG's default variant with SDAG_NCHUNK forced to each value.
Usage: python tools/chunk_sweep.py DAG N1 N2 ... (each value runs in a fresh process)"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CHILD = r'''
import sys, os, json
sys.path.insert(0, os.path.join(sys.argv[1], "tools")); sys.path.insert(0, sys.argv[1])
from perf_sweep import CFG
import torch
import paper_conf_ipps_rawatvsrps19_b200 as sdag
name = sys.argv[2]
dims, batch, scal = CFG[name]
p = sdag.Plan(sdag.spec_text(name), dims, batch=batch)
i = p.info
shape = (batch, *dims) if batch > 1 else dims
arrs = [torch.rand(shape, dtype=torch.float64, device="cuda") + 0.5 for _ in range(i["n_arrays3d"])]
a1 = [torch.rand(dims[2 - q], dtype=torch.float64, device="cuda") + 0.5 for q in range(i["n_arrays1d"])]
f = (lambda: p.apply_batched(batch, arrs, a1, scal)) if batch > 1 else (lambda: p.apply(arrs, a1, scal))
for _ in range(3): f()
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(20): f()
e1.record(); torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / 20
print(json.dumps({"dag": name, "variant": i["variant"], "nchunk": os.environ.get("SDAG_NCHUNK", "auto"), "ms": round(ms, 4),
                  "GBps": round(i["bytes_per_point"] * i["points"] * batch / ms / 1e6, 1)}))
'''


def main():
    name, vals = sys.argv[1], sys.argv[2:] or ["auto"]
    for v in vals:
        env = dict(os.environ)
        if v != "auto":
            env["SDAG_NCHUNK"] = v
        r = subprocess.run([sys.executable, "-c", CHILD, ROOT, name], env=env, capture_output=True, text=True)
        print(r.stdout.strip() or json.dumps({"nchunk": v, "error": r.stderr[-300:]}), flush=True)


if __name__ == "__main__":
    main()

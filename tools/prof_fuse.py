"""Fused 2-sweep launches (T=4 -> 2 launches) of the 27-point smoother (for ncu captures).
usage: prof_fuse.py VARIANT [N]"""
import sys
from pathlib import Path

import torch

sys.path.insert(0, str(Path(__file__).resolve().parents[1]))
import paper_conf_ipps_rawatvsrps19_b200 as sdag  # noqa: E402

v = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 512
dims = (n, n, n)
p = sdag.Plan(sdag.spec_text("smooth27"), dims, variant=v)
b0 = torch.rand(dims, dtype=torch.float64, device="cuda")
b1 = b0.clone()
for _ in range(2):
    p.apply_iterated(b0, b1, 4, [-128 / 30, 14 / 30, 3 / 30, 1 / 30, 0.125])
torch.cuda.synchronize()
print(v, "ok")

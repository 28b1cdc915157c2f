#!/usr/bin/env python3
"""e2e (apply_host) time of the headline 512^3 Laplacian vs the host chunk count."""
import json
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import paper_conf_ipps_rawatvsrps19_b200 as sdag  # noqa: E402

dims = (512, 512, 512)
c = [-205 / 24, 1.6, -0.2, 8 / 315, -1 / 560]
hA = torch.rand(dims, dtype=torch.float64).pin_memory().numpy()
hB = torch.zeros(dims, dtype=torch.float64).pin_memory().numpy()
for ch in sys.argv[1:]:
    os.environ["SDAG_HOST_CHUNKS"] = ch
    plan = sdag.Plan(sdag.spec_text("lap25"), dims)
    plan.apply_host([hB, hA], scalars=c)
    ts = []
    for _ in range(5):
        t0 = time.perf_counter()
        plan.apply_host([hB, hA], scalars=c)
        ts.append(time.perf_counter() - t0)
    print(json.dumps({"chunks": int(ch), "ms": round(statistics.median(ts) * 1e3, 2)}), flush=True)

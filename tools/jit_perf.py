#!/usr/bin/env python3
"""Time the NVRTC-generated generic kernels (NEXT-4) against the hand-written
ones on every BASELINE stencil: plan with variant="jit" (code generation into
the sweep.cuh skeleton) vs the default plan.  One JSON line per DAG."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))
import torch  # noqa: E402

import paper_conf_ipps_rawatvsrps19_b200 as sdag  # noqa: E402
from perf_sweep import CFG  # noqa: E402


def timed(p, arrs, a1, scal, batch, reps=10):
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
    return e0.elapsed_time(e1) / reps


def main():
    names = sys.argv[1:] or list(CFG)
    for name in names:
        dims, batch, scal = CFG[name]
        spec = sdag.spec_text(name)
        hand = sdag.Plan(spec, dims, batch=batch)
        i = hand.info
        shape = (batch, *dims) if batch > 1 else dims
        arrs = [torch.rand(shape, dtype=torch.float64, device="cuda") + 0.5 for _ in range(i["n_arrays3d"])]
        a1 = [torch.rand(dims[2 - q], dtype=torch.float64, device="cuda") + 0.5 for q in range(i["n_arrays1d"])]
        rec = {"dag": name, "hand_variant": i["variant"], "hand_ms": round(timed(hand, arrs, a1, scal, batch), 4)}
        jit = sdag.Plan(spec, dims, batch=batch, variant="jit")
        rec["jit_variant"] = jit.info["variant"]
        rec["jit_variants"] = jit.variants()
        rec["jit_ms"] = round(timed(jit, arrs, a1, scal, batch), 4)
        best = None
        for v in jit.variants():
            if "lsu" in v:
                continue
            pv = sdag.Plan(spec, dims, batch=batch, variant=v)
            ms = timed(pv, arrs, a1, scal, batch, reps=5)
            if best is None or ms < best[1]:
                best = (v, ms)
        rec["jit_best"] = [best[0], round(best[1], 4)] if best else None
        bpp = i["bytes_per_point"] * i["points"] * batch
        rec["hand_GBps"] = round(bpp / rec["hand_ms"] / 1e6, 1)
        rec["jit_GBps"] = round(bpp / rec["jit_ms"] / 1e6, 1)
        print(json.dumps(rec), flush=True)


if __name__ == "__main__":
    main()

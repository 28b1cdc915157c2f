#!/usr/bin/env python3
"""Fig 6-style ablation on B200 (paper P:2265-2349): for every BASELINE stencil
at its BASELINE size, the same DAG through

  gen_base   the generated (NVRTC) skeleton, fixed thread block -- (32,16) for
             the iterative stencils, (16,16) for the spatial ones (the paper's
             baselines), unroll 1, TMA-staged ring;
  gen_tb     the generated skeleton, thread block / unroll / queue form tuned
             (tune=1: hierarchical, register caps);
  hand       the hand-written sm_100a kernel (register z-queues, retiming,
             computation folding, 128-bit patches, TMA rings), heuristic pick;
  hand_tuned the same with tune=1;
  fused      iterated stencils only: per-sweep time of apply_iterated(T=12)
             with temporal fusion (deep-tuning DP), at the 1024^3 of config 5.

One JSON line per stencil: ms per sweep and the HBM roofline fraction."""
import json
import os
import re
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_ipps_rawatvsrps19_b200 as sdag  # noqa: E402
from tools.perf_sweep import CFG, PEAK  # noqa: E402

ITERATIVE = {"jacobi7", "smooth27"}


def with_block(spec, bx, by):
    """the spec with '#pragma stream k block (bx,by)' (unroll removed)"""
    lines = [ln for ln in spec.splitlines() if not ln.strip().startswith("#pragma")]
    out = []
    for ln in lines:
        if ln.startswith("stencil "):
            out.append(f"#pragma stream k block ({bx},{by})")
        out.append(ln)
    return "\n".join(out) + "\n"


def timed(f, reps=20):
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


def main():
    names = sys.argv[1:] or list(CFG)
    for name in names:
        dims, batch, scal = CFG[name]
        spec = sdag.spec_text(name)
        ref = sdag.Plan(spec, dims, batch=batch)
        info = ref.info
        byts = info["bytes_per_point"] * info["points"] * batch
        shape = (batch, *dims) if batch > 1 else dims
        g = torch.Generator(device="cuda").manual_seed(1)
        a3 = [torch.rand(shape, dtype=torch.float64, device="cuda", generator=g) + 0.5
              for _ in range(info["n_arrays3d"])]
        a1 = [torch.rand(dims[2 - q], dtype=torch.float64, device="cuda") + 0.5 for q in range(info["n_arrays1d"])]
        row = {"dag": name, "dims": list(dims), "batch": batch}

        def run(plan):
            f = (lambda: plan.apply_batched(batch, a3, a1, scal)) if batch > 1 else (lambda: plan.apply(a3, a1, scal))
            ms = timed(f)
            return {"variant": plan.info["variant"], "ms": round(ms, 4),
                    "hbm_frac": round(byts / (ms * 1e-3) / 1e9 / PEAK, 3)}

        bx, by = (32, 16) if name in ITERATIVE else (16, 16)
        try:
            row["gen_base"] = run(sdag.Plan(with_block(spec, bx, by), dims, batch=batch, variant="jit"))
        except sdag.SdagError as e:
            row["gen_base"] = {"error": str(e)[:120]}
        try:
            row["gen_tb"] = run(sdag.Plan(re.sub(r"#pragma[^\n]*\n", "", spec), dims, batch=batch, variant="jit",
                                          tune=True))
        except sdag.SdagError as e:
            row["gen_tb"] = {"error": str(e)[:120]}
        row["hand"] = run(ref)
        row["hand_tuned"] = run(sdag.Plan(spec, dims, batch=batch, tune=True))
        del a3, a1
        torch.cuda.empty_cache()
        if name in ITERATIVE:
            n = 1024
            T = 12
            b0 = torch.rand((n, n, n), dtype=torch.float64, device="cuda", generator=g)
            b1 = b0.clone()
            sc = scal if name == "smooth27" else [4.0, 0.5, 0.25]
            for fusion in (False, True):
                p = sdag.Plan(spec, (n, n, n), fusion=fusion)
                ms = timed(lambda: p.apply_iterated(b0, b1, T, sc), reps=3) / T
                sweep_b = p.info["bytes_per_point"] * p.info["points"]
                row["unfused_1024" if not fusion else "fused_1024"] = {
                    "ms_per_sweep": round(ms, 4), "sweep_equiv_frac": round(sweep_b / (ms * 1e-3) / 1e9 / PEAK, 3)}
            del b0, b1
            torch.cuda.empty_cache()
        print(json.dumps(row), flush=True)


if __name__ == "__main__":
    main()

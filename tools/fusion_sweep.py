"""Time every temporal-fusion kernel of the 27-point smoother on B200
(apply_iterated, T sweeps), against the unfused plan and the tuned plan.
Usage: python tools/fusion_sweep.py [--dims 1024 1024 1024] [--T 12]"""
import argparse
import json
import sys
from pathlib import Path

import torch

sys.path.insert(0, str(Path(__file__).resolve().parents[1]))
import paper_conf_ipps_rawatvsrps19_b200 as sdag  # noqa: E402


def fused_variants(plan):
    for line in plan.describe().splitlines():
        if "temporal fusion" in line:
            return [w for w in line.split(":", 1)[1].split() if w.startswith("fuse")]
    return []


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--dims", type=int, nargs=3, default=[1024, 1024, 1024])
    ap.add_argument("--T", type=int, default=12)
    ap.add_argument("--reps", type=int, default=3)
    a = ap.parse_args()
    dims, T = tuple(a.dims), a.T
    s = [-128 / 30, 14 / 30, 3 / 30, 1 / 30, 0.125]
    b0 = torch.rand(dims, dtype=torch.float64, device="cuda")
    b1 = b0.clone()
    base = sdag.Plan(sdag.spec_text("smooth27"), dims)
    cfgs = [("plain", {"fusion": False}), ("default", {}), ("tuned", {"tune": True})]
    cfgs += [(v, {"variant": v}) for v in fused_variants(base)]
    bpp = base.info["bytes_per_point"] * base.info["points"]
    for name, kw in cfgs:
        p = sdag.Plan(sdag.spec_text("smooth27"), dims, **kw)
        p.apply_iterated(b0, b1, T, s)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        n0 = sdag.launch_count()
        e0.record()
        for _ in range(a.reps):
            p.apply_iterated(b0, b1, T, s)
        e1.record()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / a.reps / T
        rec = {"cfg": name, "ms_per_sweep": round(ms, 4), "launches": (sdag.launch_count() - n0) // a.reps,
               "GBps_single_sweep_equiv": round(bpp / ms / 1e6, 1)}
        if name == "tuned":
            rec["describe"] = [ln.strip() for ln in p.describe().splitlines() if "f(" in ln or "fusion" in ln]
        print(json.dumps(rec), flush=True)


if __name__ == "__main__":
    main()

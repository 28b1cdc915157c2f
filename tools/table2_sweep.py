#!/usr/bin/env python3
"""The paper's Table II / Fig 4 experiment on B200: the 7pt-smoother (Listing 1
Jacobi, Table I: 512^3, T = 12) with temporal fusion degree 1 (plain sweeps) and
2 (fused launches, DP schedule), plus the 27pt-smoother for comparison.
Prints one JSON line per (stencil, configuration): ms per sweep and the
single-sweep-equivalent algorithmic HBM bandwidth.
Usage: python tools/table2_sweep.py [--n 512] [--T 12]"""
import argparse
import json
import sys
from pathlib import Path

import torch

sys.path.insert(0, str(Path(__file__).resolve().parents[1]))
import paper_conf_ipps_rawatvsrps19_b200 as sdag  # noqa: E402

SC = {"jacobi7": [4.0, 0.5, 0.25], "smooth27": [-128 / 30, 14 / 30, 3 / 30, 1 / 30, 0.125]}


def run(name, dims, T, reps, **kw):
    p = sdag.Plan(sdag.spec_text(name), dims, **kw)
    b0 = torch.rand(dims, dtype=torch.float64, device="cuda")
    b1 = b0.clone()
    p.apply_iterated(b0, b1, T, SC[name])
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    n0 = sdag.launch_count()
    e0.record()
    for _ in range(reps):
        p.apply_iterated(b0, b1, T, SC[name])
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / reps / T
    bpp = p.info["bytes_per_point"] * p.info["points"]
    fl = [ln.strip() for ln in p.describe().splitlines() if "temporal fusion" in ln]
    return {"dag": name, "dims": list(dims), "T": T, "cfg": kw, "ms_per_sweep": round(ms, 4),
            "launches_per_T": (sdag.launch_count() - n0) // reps,
            "GBps_single_sweep_equiv": round(bpp / ms / 1e6, 1),
            "fused_kernel": fl[0].split(":", 1)[1].split()[0] if fl and kw.get("fusion", True) else None}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=512)
    ap.add_argument("--T", type=int, default=12)
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--all", action="store_true", help="also time every fused kernel forced")
    a = ap.parse_args()
    dims = (a.n, a.n, a.n)
    for name in ("jacobi7", "smooth27"):
        cfgs = [{"fusion": False}, {}, {"tune": True}]
        if a.all:
            base = sdag.Plan(sdag.spec_text(name), dims)
            for ln in base.describe().splitlines():
                if "temporal fusion" in ln:
                    cfgs += [{"variant": w} for w in ln.split(":", 1)[1].split() if w.startswith("fuse")]
        for kw in cfgs:
            rec = run(name, dims, a.T, a.reps, **kw)
            if "variant" in kw:
                rec["fused_kernel"] = kw["variant"]
            print(json.dumps(rec), flush=True)


if __name__ == "__main__":
    main()

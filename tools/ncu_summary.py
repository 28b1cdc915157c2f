#!/usr/bin/env python3
"""Summarise an ncu report (--set full) into markdown + JSON for profiles/.

usage: ncu_summary.py REPORT.ncu-rep OUT_PREFIX [--variant NAME] [--alg-bytes B] [--flops F]
Writes OUT_PREFIX.md and OUT_PREFIX.json and merges DRAM bytes/launch into
profiles/ncu_traffic.json under NAME (read by bench.py's roofline.traffic)."""
import argparse
import csv
import io
import json
import os
import subprocess

KEYS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_bytes.sum",
    "sm__cycles_elapsed.avg.per_second", "sm__inst_executed.sum", "smsp__inst_executed_pipe_fp64.sum",
    "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active", "sm__warps_active.avg.pct_of_peak_sustained_active",
    "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
    "smsp__sass_thread_inst_executed_op_dfma_pred_on.sum", "smsp__sass_thread_inst_executed_op_dadd_pred_on.sum",
    "smsp__sass_thread_inst_executed_op_dmul_pred_on.sum", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "smsp__issue_active.avg.pct_of_peak_sustained_active",
]


def raw(report):
    out = subprocess.run(["ncu", "-i", report, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, u = rows[0], rows[1]
    kernels = []
    for v in rows[2:]:
        d = {}
        for n, un, val in zip(h, u, v):
            d[n] = (val, un)
        kernels.append(d)
    return kernels


def stalls(k):
    s = {}
    for n, (v, _) in k.items():
        if n.startswith("smsp__pcsamp_warps_issue_stalled_") and not n.endswith("_not_issued"):
            try:
                s[n.replace("smsp__pcsamp_warps_issue_stalled_", "")] = int(float(v.replace(",", "")))
            except ValueError:
                pass
    return dict(sorted(s.items(), key=lambda x: -x[1])[:8])


def num(k, n):
    v, u = k.get(n, ("", ""))
    try:
        x = float(v.replace(",", ""))
    except ValueError:
        return None, u
    return x, u


def to_bytes(x, u):
    return x * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}.get(u, 1)


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("report")
    ap.add_argument("out")
    ap.add_argument("--variant", help="traffic key: VARIANT@[batchx]NZxNYxNX")
    ap.add_argument("--alg-bytes", type=float)
    ap.add_argument("--flops", type=float)
    a = ap.parse_args()
    ks = raw(a.report)
    k = ks[0]
    res = {"kernel": k.get("Kernel Name", ("", ""))[0], "metrics": {}, "stalls": stalls(k)}
    for n in KEYS:
        x, u = num(k, n)
        if x is not None:
            res["metrics"][n] = {"value": x, "unit": u}
    fp = [num(k, f"smsp__sass_thread_inst_executed_op_{o}_pred_on.sum")[0] for o in ("dfma", "dadd", "dmul")]
    if all(x is not None for x in fp):
        res["fp64_thread_inst_per_launch"] = {"dfma": fp[0], "dadd": fp[1], "dmul": fp[2]}
        res["fp64_flops_executed_per_launch"] = 2 * fp[0] + fp[1] + fp[2]
    rb = num(k, "dram__bytes_read.sum")
    wb = num(k, "dram__bytes_write.sum")
    if rb[0] is not None and wb[0] is not None:
        res["dram_bytes_per_launch"] = to_bytes(*rb) + to_bytes(*wb)
    t = num(k, "gpu__time_duration.sum")
    tsec = t[0] * {"nsecond": 1e-9, "ns": 1e-9, "usecond": 1e-6, "us": 1e-6, "msecond": 1e-3, "ms": 1e-3}.get(t[1], 1e-9) if t[0] else None
    if a.alg_bytes and tsec:
        res["alg_bytes_per_launch"] = a.alg_bytes
        res["alg_GBps_under_ncu"] = a.alg_bytes / tsec / 1e9
        if "dram_bytes_per_launch" in res:
            res["traffic_over_alg"] = res["dram_bytes_per_launch"] / a.alg_bytes
    if a.flops and tsec:
        res["GFLOPs_under_ncu"] = a.flops / tsec / 1e9
    with open(a.out + ".json", "w") as f:
        json.dump(res, f, indent=1)
    with open(a.out + ".md", "w") as f:
        f.write(f"# ncu --set full: {res['kernel']}\n\n")
        f.write(f"report: `{os.path.basename(a.report)}` (clock-control none; numbers under the profiler are "
                f"cold-cache/serialised -- use shares, not absolutes)\n\n| metric | value | unit |\n|---|---|---|\n")
        for n, v in res["metrics"].items():
            f.write(f"| {n} | {v['value']:.6g} | {v['unit']} |\n")
        for n in ("dram_bytes_per_launch", "alg_bytes_per_launch", "traffic_over_alg", "alg_GBps_under_ncu",
                  "GFLOPs_under_ncu", "fp64_flops_executed_per_launch"):
            if n in res:
                f.write(f"| {n} | {res[n]:.6g} | |\n")
        f.write("\nTop warp stall reasons (pc samples):\n\n")
        for n, v in res["stalls"].items():
            f.write(f"- {n}: {v}\n")
    if a.variant and "dram_bytes_per_launch" in res:
        # per-launch counters read by bench.py (roofline.traffic, the F = min(canonical, executed) rule)
        p = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles", "ncu_counters.json")
        d = json.load(open(p)) if os.path.exists(p) else {}
        e = {"dram_bytes": res["dram_bytes_per_launch"], "source": os.path.basename(a.report)}
        if "fp64_flops_executed_per_launch" in res:
            e["fp64_flops"] = res["fp64_flops_executed_per_launch"]
        d[a.variant] = e
        json.dump(d, open(p, "w"), indent=1, sort_keys=True)
    print(json.dumps({k2: res[k2] for k2 in res if k2 != "metrics"}, indent=1))

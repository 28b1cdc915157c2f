#!/usr/bin/env python3
"""Rewrite the per-config table and the number bullets of profiles/<round>/INDEX.md
from that directory's bench.json, bench_reference.json and ncu/*_ncu.json (so the
index always quotes the committed files).  usage: tools/refresh_index.py r02"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PTS = {"lap25": 504 ** 3, "jacobi7": 128 * 62 ** 3, "hypterm": 312 ** 3, "rhs4center": 316 ** 3, "fuse2": 1022 ** 3}


def main(rnd):
    P = os.path.join(ROOT, "profiles", rnd)
    d = json.load(open(os.path.join(P, "bench.json")))
    ref = json.load(open(os.path.join(P, "bench_reference.json")))
    pc = d["per_config"]

    def ncu(n):
        return json.load(open(os.path.join(P, "ncu", f"{n}_ncu.json")))

    def row(cfg, var, ms, r, n):
        j = ncu(n)
        m = j["metrics"]
        ex = j["fp64_flops_executed_per_launch"] / r["canonical_flops_per_launch"]
        tr = j["dram_bytes_per_launch"] / r["alg_bytes_per_launch"]
        wf = m["l1tex__data_pipe_lsu_wavefronts_mem_shared.sum"]["value"] / PTS[n]
        fp = m["sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active"]["value"]
        iss = m["smsp__issue_active.avg.pct_of_peak_sustained_active"]["value"]
        return (f"| {cfg} | {var} | {ms:.4f} | {r['bound']} {r['achieved']:.1f} of {r['peak']:.1f} {r['unit']} | "
                f"**{r['frac']:.3f}** | {tr:.3f} | {ex:.3f} | {wf:.2f} | {fp:.1f} % | {iss:.1f} % |")

    rows = [row("2 (headline)", d["plan"]["variant"], d["ms_per_step"], d["roofline"], "lap25")]
    for cid, n in (("1b", "jacobi7"), ("3", "hypterm"), ("4", "rhs4center")):
        v = pc[cid]
        rows.append(row(cid, v["variant"], v["ms_per_step"], v["roofline"], n))
    v = pc["5"]
    rows.append(row("5 (per fused launch = 2 sweeps)", v["variant"], v["roofline"]["kernel_ms"], v["roofline"], "fuse2"))
    p = os.path.join(P, "INDEX.md")
    s = open(p).read()
    i, j = s.index("| 2 (headline)"), s.index("* config 1 (one")
    s = s[:i] + "\n".join(rows) + "\n\n" + s[j:]
    out = []
    for ln in s.split("\n"):
        if ln.startswith("* config 1 (one 64^3"):
            ln = (f"* config 1 (one 64^3 problem, L2 flushed before every launch): {pc['1']['ms_per_step'] * 1e3:.1f} us "
                  f"median, {pc['1']['us_min']:.1f} us min -- latency, not throughput.")
        elif ln.startswith("* config 4 by canonical"):
            ln = (f"* config 4 by canonical flops (666/pt): {pc['4']['roofline']['frac_canonical_flops']:.3f} of the "
                  f"measured DFMA rate {pc['fp64_peak_tflops_measured']:.2f} TFLOP/s; the table uses F = min(canonical, "
                  f"executed).")
        elif ln.startswith("* config 5: "):
            ln = (f"* config 5: {v['ms_per_step']:.2f} ms per 12-sweep step = {v['ms_per_step'] / 12:.3f} ms per sweep; "
                  f"sweep-equivalent {v['roofline']['sweep_equivalent']['frac_of_unfused_roofline']:.3f} of the unfused "
                  f"HBM roofline; clocks {v['clocks']}.")
        elif ln.startswith("* headline: "):
            cb = d["cpu_baseline"]
            ln = (f"* headline: {d['value']:.0f} GFLOP/s, {d['hbm_gbs']:.0f} GB/s; e2e (sdag_apply_host) "
                  f"{d['e2e']['value']:.1f} GFLOP/s ({d['e2e']['ms_per_step']:.1f} ms per step); cpu_baseline "
                  f"{cb['value']:.1f} GFLOP/s on {cb['cores']} cores ({cb.get('cpu_model', '')}); reference arm "
                  f"(`--impl reference`, same box) {ref['value']:.1f} GFLOP/s; clocks {d['clocks']}.")
        out.append(ln)
    open(p, "w").write("\n".join(out))
    print("\n".join(rows))


if __name__ == "__main__":
    main(sys.argv[1])

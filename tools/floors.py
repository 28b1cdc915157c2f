#!/usr/bin/env python3
"""Per-kernel resource floors from one `ncu --set full` capture each (the
reports tools/measure_round.sh writes): for every hot kernel the time the
launch would take if ONE resource ran at its peak and nothing else mattered,

  HBM    DRAM bytes (read + write)            / measured copy bandwidth (MEASURED_PEAKS.json)
  FP64   DFMA + DADD + DMUL thread instr.     / (148 SMs x 64 lanes x clock)
  smem   LSU shared wavefronts + TMA fill/128 / (148 SMs x 1 wavefront (128 B) x clock)
  issue  warp instructions                    / (148 SMs x 4 schedulers x clock)

and the launch's measured time under ncu (cold, serialised; clock = the
capture's own sm__cycles_elapsed rate).  The largest floor is the kernel's
binding roofline; time / floor says how close the kernel runs to it.

usage: tools/floors.py MEAS_DIR OUT_PREFIX   (reads MEAS_DIR/prof_*.ncu-rep)"""
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SMS = 148
UNIT = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12,
        "nsecond": 1e-9, "usecond": 1e-6, "msecond": 1e-3, "second": 1.0, "ns": 1e-9, "us": 1e-6, "ms": 1e-3, "s": 1.0,
        "hz": 1.0, "Khz": 1e3, "Mhz": 1e6, "Ghz": 1e9, "": 1.0, "inst": 1.0, "warp": 1.0}
WANT = {
    "t": "gpu__time_duration.sum",
    "clk": "sm__cycles_elapsed.avg.per_second",
    "dram_r": "dram__bytes_read.sum",
    "dram_w": "dram__bytes_write.sum",
    "lsu_wf": "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
    "tma_bytes": "l1tex__m_xbar2l1tex_read_bytes_mem_global_op_tma_ld.sum",
    "inst": "smsp__inst_executed.sum",
    "dfma": "smsp__sass_thread_inst_executed_op_dfma_pred_on.sum",
    "dadd": "smsp__sass_thread_inst_executed_op_dadd_pred_on.sum",
    "dmul": "smsp__sass_thread_inst_executed_op_dmul_pred_on.sum",
}
KERNELS = [("lap25", "25-pt Laplacian 512^3 (headline)"), ("jacobi7", "7-pt Jacobi 128 x 64^3"),
           ("hypterm", "hypterm 320^3"), ("rhs4center", "rhs4center 320^3"), ("smooth27", "27-pt smoother 512^3"),
           ("fuse2", "27-pt smoother 1024^3, 2 sweeps fused")]


def raw(report):
    out = subprocess.run(["ncu", "-i", report, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, u, v = rows[0], rows[1], rows[2]
    got = {}
    for key, name in WANT.items():
        if name in h:
            i = h.index(name)
            try:
                got[key] = float(v[i].replace(",", "")) * UNIT.get(u[i], 1.0)
            except ValueError:
                pass
    got["kernel"] = v[h.index("Kernel Name")] if "Kernel Name" in h else ""
    return got


def main(meas, out):
    peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"] * 1e9
    res = {}
    for name, label in KERNELS:
        rep = os.path.join(meas, f"prof_{name}.ncu-rep")
        if not os.path.exists(rep):
            continue
        m = raw(rep)
        clk = m["clk"]
        fl = {
            "hbm": (m["dram_r"] + m["dram_w"]) / peak,
            "fp64": (m["dfma"] + m["dadd"] + m["dmul"]) / (SMS * 64 * clk),
            "smem": (m["lsu_wf"] + m.get("tma_bytes", 0.0) / 128.0) / (SMS * clk),
            "issue": m["inst"] / (SMS * 4 * clk),
        }
        bind = max(fl, key=fl.get)
        res[name] = {"label": label, "kernel": m["kernel"], "t_ms": m["t"] * 1e3, "clock_ghz": clk / 1e9,
                     "floors_ms": {k: v * 1e3 for k, v in fl.items()}, "binding": bind,
                     "frac_of_binding": fl[bind] / m["t"], "raw": m}
    json.dump(res, open(out + ".json", "w"), indent=1)
    lines = ["# Resource floors per hot kernel (tools/floors.py)", "",
             "From one `ncu --set full` capture per kernel (cold, serialised; each floor uses the capture's own SM "
             "clock). HBM = DRAM bytes / measured copy bandwidth; FP64 = FP64 thread instructions / (148 x 64 lanes "
             "x clock); smem = (LSU shared wavefronts + TMA fill bytes / 128) / (148 x clock); issue = warp "
             "instructions / (148 x 4 x clock). The largest floor is the binding roofline.", "",
             "| kernel | ncu time (ms) | HBM | FP64 | smem | issue | binding | time at binding floor |",
             "|---|---|---|---|---|---|---|---|"]
    for name, r in res.items():
        f = r["floors_ms"]
        lines.append(f"| {r['label']} | {r['t_ms']:.3f} | {f['hbm']:.3f} | {f['fp64']:.3f} | {f['smem']:.3f} | "
                     f"{f['issue']:.3f} | {r['binding']} | **{r['frac_of_binding']:.2f}** |")
    open(out + ".md", "w").write("\n".join(lines) + "\n")
    print("\n".join(lines))


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2])

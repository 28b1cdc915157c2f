#!/usr/bin/env python3
"""Run every (dag, variant) on one shape in a fresh subprocess; report ok / error
and the scaled error vs the oracle (debug aid for the GPU box)."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

CHILD = r'''
import sys, json
sys.path.insert(0, ROOT); sys.path.insert(0, ROOT + "/tests")
from cases import make_case, run_gpu, check
name, dims, v = NAME, DIMS, VAR
case = make_case(name, dims)
g, p = run_gpu(name, dims, case, variant=v)
print(json.dumps({"worst": check(name, dims, g, case)}))
'''

if __name__ == "__main__":
    import paper_conf_ipps_rawatvsrps19_b200 as sdag
    dims = tuple(int(x) for x in (sys.argv[1] if len(sys.argv) > 1 else "20,34,70").split(","))
    names = sys.argv[2].split(",") if len(sys.argv) > 2 else ["jacobi7", "lap25", "smooth27", "hypterm", "rhs4center"]
    for name in names:
        for v in sdag.Plan(sdag.spec_text(name), dims, device="none").variants():
            code = CHILD.replace("ROOT", repr(ROOT)).replace("NAME", repr(name)).replace("DIMS", repr(dims)).replace(
                "VAR", repr(v))
            r = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, timeout=300)
            last = (r.stdout.strip().splitlines() or [""])[-1]
            err = [l for l in r.stderr.splitlines() if "Error" in l or "error" in l][-1:] if r.returncode else []
            print(json.dumps({"dag": name, "variant": v, "rc": r.returncode, "out": last, "err": err}), flush=True)

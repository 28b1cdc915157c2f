#!/usr/bin/env python3
"""Randomised GPU parity sweep of the generated (NVRTC) path: N random DAGs
(tests/specgen.user_spec), each with random user guidance (#pragma block /
unroll / occupancy, #assign gmem), every generated variant vs the oracle's
spec interpreter under the R13 gate.  Prints one line per failure and a
summary; exit 1 on any failure."""
import os
import random
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

from specgen import user_spec  # noqa: E402
from test_gpu_jit import compare, run_user  # noqa: E402

import paper_conf_ipps_rawatvsrps19_b200 as sdag  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 40
fails = runs = 0
for seed in range(100, 100 + n):
    text, desc = user_spec(seed)
    rnd = random.Random(seed)
    g = text
    ins = [f"in{q}" for q in range(8) if f"in{q}[" in text]
    if len(ins) >= 2 and rnd.random() < 0.4:
        g = g.replace("{\n", "{\n#assign gmem (" + rnd.choice(ins) + ")\n", 1)
    prag = []
    if rnd.random() < 0.4:
        prag.append(f"block ({rnd.choice([16, 32, 64])},{rnd.choice([4, 8, 16])})")
        if rnd.random() < 0.5:
            prag.append(f"unroll j={rnd.choice([1, 2])}")
    if rnd.random() < 0.3:
        prag.append(f"occupancy {rnd.choice([0.25, 0.5, 0.75])}")
    if prag:
        g = g.replace("\nstencil ", "\n#pragma stream k " + " ".join(prag) + "\nstencil ", 1)
    dims = (9 + 2 * desc["R"][0] + rnd.randrange(8), 11 + 2 * desc["R"][1] + rnd.randrange(20),
            30 + 2 * desc["R"][2] + rnd.randrange(40))
    try:
        variants = sdag.Plan(g, dims).variants()
    except sdag.SdagError as e:
        print("plan error", seed, e)
        fails += 1
        continue
    for v in variants:
        runs += 1
        try:
            plan, arrs, sc, got = run_user(g, desc, dims, seed, variant=v)
            compare(text, dims, arrs, sc, got)
        except Exception as e:  # noqa: BLE001
            fails += 1
            print("FAIL", seed, v, dims, prag, type(e).__name__, str(e)[:200], flush=True)
print(f"jit fuzz: {n} DAGs, {runs} variant runs, {fails} failures")
sys.exit(1 if fails else 0)

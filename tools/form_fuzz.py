#!/usr/bin/env python3
"""Randomised GPU parity sweep of the generated star- and box-form kernels:
random linear, mirror-symmetric star DAGs (radius 1-4, per-axis coefficients
from scalars and literals, optional affine term) and random class-weighted
3x3x3 box DAGs, every generated form variant vs the oracle's spec interpreter
under the R13 gate.  Exit 1 on any failure."""
import os
import random
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_rawatvsrps19_b200 as sdag  # noqa: E402
from test_gpu_jit import compare  # noqa: E402


def tap(d, off):
    idx = ["k", "j", "i"]
    o = [0, 0, 0]
    o[d] = off
    return "A" + "".join(f"[{idx[a]}{'+' if o[a] > 0 else '-'}{abs(o[a])}]" if o[a] else f"[{idx[a]}]" for a in range(3))


def star_spec(rnd):
    R = rnd.randint(1, 4)
    coef = lambda: rnd.choice(["s0", "s1", "s2", f"{rnd.uniform(-1, 1):.6f}", "(s0*s1)", f"(s2/{rnd.randint(2, 9)}.0)"])
    terms = [f"{coef()}*A[k][j][i]"]
    same_yz = rnd.random() < 0.5
    for r in range(1, R + 1):
        cx, cy = coef(), coef()
        cz = cy if same_yz else coef()
        terms.append(f"{cx}*({tap(2, r)} + {tap(2, -r)})")
        terms.append(f"{cy}*({tap(1, r)} + {tap(1, -r)})")
        terms.append(f"{cz}*({tap(0, r)} + {tap(0, -r)})")
    if rnd.random() < 0.3:
        terms.append("s2")
    body = " + ".join(terms)
    return f"""iterator k, j, i;
double out[64,64,64], A[64,64,64], s0, s1, s2;
stencil st (out, A, s0, s1, s2) {{
  out[k][j][i] = {body};
}}
""", "jitstar_"


def box_spec(rnd):
    w = [rnd.choice(["s0", "s1", f"{rnd.uniform(-1, 1):.5f}", "(s0-s2)"]) for _ in range(4)]
    cls = {0: [], 1: [], 2: [], 3: []}
    for dz in (-1, 0, 1):
        for dy in (-1, 0, 1):
            for dx in (-1, 0, 1):
                idx = "".join(f"[{v}{'+' if o > 0 else '-'}{abs(o)}]" if o else f"[{v}]"
                              for v, o in zip(("k", "j", "i"), (dz, dy, dx)))
                cls[(dz != 0) + (dy != 0) + (dx != 0)].append("A" + idx)
    body = " + ".join(f"{w[c]}*(" + " + ".join(cls[c]) + ")" for c in range(4) if rnd.random() < 0.9 or c == 0)
    return f"""iterator k, j, i;
double out[64,64,64], A[64,64,64], s0, s1, s2;
stencil bx (out, A, s0, s1, s2) {{
  out[k][j][i] = {body};
}}
""", "jitbox_"


def main():
    n = int(sys.argv[1]) if len(sys.argv) > 1 else 30
    fails = runs = 0
    for seed in range(n):
        rnd = random.Random(1000 + seed)
        text, prefix = (star_spec if seed % 2 == 0 else box_spec)(rnd)
        R = 4
        dims = (2 * R + 3 + rnd.randrange(10), 2 * R + 5 + rnd.randrange(20), 2 * R + 20 + 2 * rnd.randrange(20))
        try:
            p0 = sdag.Plan(text, dims)
        except sdag.SdagError as e:
            print("plan error", seed, e)
            fails += 1
            continue
        forms = [v for v in p0.variants() if v.startswith(prefix)]
        if not forms:
            print("FORM NOT DETECTED", seed, prefix, p0.variants()[:3])
            fails += 1
            continue
        g = np.random.default_rng(seed)
        A = g.uniform(-1, 1, dims)
        sc = {"s0": 0.7, "s1": -0.4, "s2": 1.3}
        for v in forms:
            runs += 1
            try:
                plan = sdag.Plan(text, dims, variant=v)
                dev = [torch.full(dims, float("nan"), dtype=torch.float64, device="cuda"), torch.from_numpy(A).cuda()]
                plan.apply(dev, [], [sc["s0"], sc["s1"], sc["s2"]])
                torch.cuda.synchronize()
                compare(text, dims, {"A": A}, sc, {"out": dev[0].cpu().numpy(), "A": A})
            except Exception as e:  # noqa: BLE001
                fails += 1
                print("FAIL", seed, v, dims, type(e).__name__, str(e)[:300], flush=True)
    print(f"form fuzz: {n} DAGs, {runs} variant runs, {fails} failures")
    return 1 if fails else 0


if __name__ == "__main__":
    sys.exit(main())

#!/usr/bin/env python3
"""Embed specs/*.sdag into a C++ initializer list (build step)."""
import os
import sys

out, d = sys.argv[1], sys.argv[2]
order = ["jacobi7", "lap25", "smooth27", "hypterm", "rhs4center", "shift", "j1d3pt"]
names = sorted((f[:-5] for f in os.listdir(d) if f.endswith(".sdag")),
               key=lambda n: (order.index(n) if n in order else 99, n))
lines = []
for n in names:
    t = open(os.path.join(d, n + ".sdag")).read()
    assert ')SDAG"' not in t
    lines.append(f'{{"{n}", R"SDAG({t})SDAG"}},')
tmp = out + ".tmp"
with open(tmp, "w") as f:
    f.write("\n".join(lines) + "\n")
os.replace(tmp, out)

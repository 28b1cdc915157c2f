#!/usr/bin/env python3
"""Embed a text file as a C++ raw string constant (build step).
usage: embed_text.py OUT.inc VARNAME FILE"""
import os
import sys

out, var, src = sys.argv[1], sys.argv[2], sys.argv[3]
t = open(src).read()
assert ')SDAGTXT"' not in t
tmp = out + ".tmp"
with open(tmp, "w") as f:
    f.write(f'static const char *{var} = R"SDAGTXT({t})SDAGTXT";\n')
os.replace(tmp, out)

"""Mutation check of the oracle pins: each plausible slip (wrong tap, swapped
coefficient array, wrong velocity component, dropped corner, ...) injected
into a copy of oracle/oracle.c must make tests/test_oracle_pins.py fail.
Runs the pins in a subprocess against the mutant library."""
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

MUTATIONS = [
    ("rhs4-mux2-tap", "mub[b][2] = MUS(-2) + MUS(1)", "mub[b][2] = MUS(-2) + MUS(2)", "rhs4"),
    ("rhs4-mixed-la-mu", "{0, 1, 1, 1}, {0, 2, 2, 1}, {1, 0, 1, 0}", "{0, 1, 1, 0}, {0, 2, 2, 1}, {1, 0, 1, 1}", "rhs4"),
    ("rhs4-inner-tap", "8 * (NEG(u[q - sb]) + u[q + sb])", "8 * (NEG(u[q - sb]) + u[q + 2 * sb])", "rhs4"),
    ("rhs4-tf-sign", "mub[b][4] = SUB(MUS(1), tf", "mub[b][4] = (MUS(1) + tf", "rhs4"),
    ("hypterm-pressure", "d = d + SUB(q[4][pp], q[4][pm]);", "d = d + SUB(q[4][pp], q[4][pp - sa]);", "hypterm"),
    ("hypterm-velocity", "const double *V = q[1 + a];", "const double *V = q[1 + (a + 1) % 3];", "hypterm"),
    ("hypterm-dxinv", "SUB(acc, term * dxinv[a])", "SUB(acc, term * dxinv[0])", "hypterm"),
    ("smooth27-corner", "A_(1, -1, -1) + A_(1, -1, 1)", "A_(1, -1, -1) + A_(1, -1, 0)", "smooth27"),
    ("smooth27-nu", "return A_(0, 0, 0) + nu *", "return A_(0, 0, 0) + 0.5 * nu *", "smooth27"),
    ("lap25-ztap", "A_(r, 0, 0) + A_(-r, 0, 0)", "A_(r, 0, 0) + A_(-r, 0, 1)", "lap25"),
    ("jacobi7-center", "A_(0, 0, 0) * 6.0", "A_(0, 0, 0) * 5.0", "jacobi7"),
    ("jacobi7-ynbr", "A_(0, 1, 0) + A_(0, -1, 0)", "A_(0, 1, 0) + A_(0, 1, 0)", "jacobi7"),
]


@pytest.mark.parametrize("name,old,new,k", MUTATIONS, ids=[m[0] for m in MUTATIONS])
def test_mutant_is_killed(tmp_path, name, old, new, k):
    src = open(os.path.join(ROOT, "oracle", "oracle.c")).read()
    assert src.count(old) >= 1, f"mutation anchor not found: {old}"
    mut = tmp_path / f"{name}.c"
    mut.write_text(src.replace(old, new))
    env = dict(os.environ, SDAG_ORACLE_SRC=str(mut), SDAG_ORACLE_LIB=str(tmp_path / f"{name}.so"))
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-p", "no:cacheprovider",
                        os.path.join(ROOT, "tests", "test_oracle_pins.py"), "-k", k],
                       env=env, cwd=ROOT, capture_output=True, text=True, timeout=600)
    assert r.returncode != 0, f"mutant {name} survived:\n{r.stdout[-2000:]}"

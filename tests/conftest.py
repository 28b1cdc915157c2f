import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)
HERE = os.path.dirname(os.path.abspath(__file__))
if HERE not in sys.path:
    sys.path.insert(0, HERE)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a)")
    config.addinivalue_line("markers", "slow: long-running CPU test")


def pytest_terminal_summary(terminalreporter):
    """Print the worst scaled error e_p per parity test (tests/cases.gate) and
    write them to $SDAG_PARITY_LOG as JSON when that is set."""
    cases = sys.modules.get("cases")
    worst = getattr(cases, "WORST", None) if cases else None
    if not worst:
        return
    tr = terminalreporter
    tr.section("worst scaled error e_p per parity check (gate 1e-12)")
    for k in sorted(worst, key=lambda k: -worst[k]["e_p"]):
        w = worst[k]
        tr.write_line(f"{w['e_p']:.3e}  normwise {w['normwise']:.3e}  {w['points']:>11d} pts  {k}")
    path = os.environ.get("SDAG_PARITY_LOG")
    if path:
        import json
        with open(path, "w") as f:
            json.dump({"gate": 1e-12, "checks": worst}, f, indent=1, sort_keys=True)

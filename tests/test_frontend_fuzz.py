"""Front-end robustness (a1-a2, host only): the C++ parser/analyser must answer
every input with a plan or an sdag_status -- never a crash, hang or exception
other than SdagError -- on random text and on single-character mutations of
the registered specs and generated DAGs (hypothesis)."""
from __future__ import annotations

import pytest

hypothesis = pytest.importorskip("hypothesis")
from hypothesis import HealthCheck, given, settings  # noqa: E402
from hypothesis import strategies as st  # noqa: E402

import paper_conf_ipps_rawatvsrps19_b200 as sdag  # noqa: E402
from specgen import user_spec  # noqa: E402

SPECS = [sdag.spec_text(n) for n in ("jacobi7", "lap25", "smooth27", "hypterm", "rhs4center")] + \
        [user_spec(s)[0] for s in range(4)]
ALPHABET = "abcijkABXYZ0123456789.+-*/=;,()[]{}#\n \t_eE" + "stencil double iterator parameter"
CODES = {"PARSE", "SEMANTIC", "UNSUPPORTED", "DOMAIN", "INVALID_ARG"}


def _plan(text):
    try:
        p = sdag.Plan(text, (12, 13, 14), device="none")
    except sdag.SdagError as e:
        assert e.code in CODES, e
        return None
    assert p.info["radius"] is not None
    return p


@settings(max_examples=300, deadline=None, derandomize=True, suppress_health_check=[HealthCheck.too_slow])
@given(st.text(alphabet=ALPHABET, max_size=300))
def test_random_text_is_rejected_cleanly(text):
    _plan(text)


@settings(max_examples=300, deadline=None, derandomize=True, suppress_health_check=[HealthCheck.too_slow])
@given(st.sampled_from(SPECS), st.integers(min_value=0, max_value=10 ** 6), st.sampled_from(["del", "dup", "sub"]),
       st.sampled_from(list("()[]{};,=+-*/0123456789kji.")))
def test_mutated_specs_plan_or_fail_cleanly(spec, pos, op, ch):
    i = pos % len(spec)
    if op == "del":
        text = spec[:i] + spec[i + 1:]
    elif op == "dup":
        text = spec[:i] + spec[i] + spec[i:]
    else:
        text = spec[:i] + ch + spec[i + 1:]
    _plan(text)


@settings(max_examples=100, deadline=None, derandomize=True)
@given(st.sampled_from(SPECS), st.sampled_from(["maxfuse", "trivial"]))
def test_fission_of_valid_specs_reparses(spec, kind):
    try:
        text = sdag.fission(spec, kind)
    except sdag.SdagError as e:
        assert e.code == "UNSUPPORTED"
        return
    g = sdag.Program(text, (20, 20, 20), device=-2)
    assert g.counts["n_stages"] >= 1

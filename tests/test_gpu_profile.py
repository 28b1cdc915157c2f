"""Profile-guided classification (paper Section IV; SURVEY 8(f)
NEXT-3) on the B200 kernels: roofline placement against the measured DRAM and
FP64 peaks, code-differenced twins, the bound and the IV-A hints."""
from __future__ import annotations

import json
import os

import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("no CUDA device", allow_module_level=True)

import paper_conf_ipps_rawatvsrps19_b200 as sdag  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _hbm_peak():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    return json.load(open(p)).get("hbm_gbs", 0.0) if os.path.exists(p) else 0.0


def _arrays(name, dims):
    plan = sdag.Plan(sdag.spec_text(name), dims)
    g = torch.Generator(device="cuda").manual_seed(7)
    a3 = [torch.rand(dims, dtype=torch.float64, device="cuda", generator=g) + 0.5
          for _ in range(plan.info["n_arrays3d"])]
    a1 = [torch.rand(dims[2 - q], dtype=torch.float64, device="cuda", generator=g) + 0.5
          for q in range(plan.info["n_arrays1d"])]
    return plan, a3, a1


def test_profile_lap25_is_dram_bound_with_code_differencing():
    plan, a3, a1 = _arrays("lap25", (512, 512, 512))
    pr = plan.profile(a3, a1, scalars=[-205 / 24, 1.6, -0.2, 8 / 315, -1 / 560], peak_hbm_gbs=_hbm_peak())
    assert pr["variant"] == plan.info["variant"]
    assert pr["ms"] > 0 and pr["flops"] == pytest.approx(29 * 504 ** 3)
    assert pr["frac_dram"] == pytest.approx(pr["bytes"] / (pr["peak_hbm_gbs"] * 1e9) * 1e3 / pr["ms"])
    assert pr["oi_dram"] < pr["ridge"]
    assert pr["bound"] == "dram", pr
    # the registered twins of the star kernel (DESIGN 6.4): memory-only and arithmetic-only
    assert 0 < pr["ms_diff_mem"] and 0 < pr["ms_diff_arith"]
    assert pr["hints"], pr


def test_profile_rhs4_is_not_dram_bound_and_reports_register_pressure():
    plan, a3, a1 = _arrays("rhs4center", (320, 320, 320))
    pr = plan.profile(a3, a1, scalars=[0.75, 1 / 6, 1 / 144, 1.0, 1.0], peak_hbm_gbs=_hbm_peak())
    assert pr["oi_dram"] > pr["ridge"]  # above the ridge: FP64 is the attainable bound
    assert pr["bound"] in ("compute", "latency")
    assert pr["regs"] >= 224 and pr["warps_per_sm"] >= 4
    assert any("register pressure" in h for h in pr["hints"]), pr["hints"]
    assert pr["ms_diff_mem"] == 0.0  # no twins registered for this kernel


def test_profile_iterative_dram_bound_hints_fusion():
    plan, a3, a1 = _arrays("smooth27", (512, 512, 512))
    pr = plan.profile(a3, a1, scalars=[-128 / 30, 14 / 30, 3 / 30, 1 / 30, 0.125], peak_hbm_gbs=_hbm_peak())
    assert pr["bound"] == "dram", pr
    assert any("fusion degree" in h for h in pr["hints"]), pr["hints"]

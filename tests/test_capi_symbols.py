"""The C-ABI library loads without a GPU and exports every entry point that
include/sdag.h declares (no compute calls)."""
import os
import re

import pytest
import subprocess

import paper_conf_ipps_rawatvsrps19_b200 as sdag
from paper_conf_ipps_rawatvsrps19_b200 import _capi

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def header_functions():
    text = open(os.path.join(ROOT, "include", "sdag.h")).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return sorted(set(re.findall(r"\b(sdag_[a-z0-9_]+)\s*\(", text)))


def test_header_and_binding_agree():
    assert header_functions() == sorted(_capi.EXPORTED)


def test_every_declared_symbol_is_exported():
    out = subprocess.run(["nm", "-D", "--defined-only", _capi.LIB_PATH], capture_output=True, text=True).stdout
    exported = set(re.findall(r"\bT (sdag_[a-z0-9_]+)", out))
    missing = [f for f in header_functions() if f not in exported]
    assert not missing, missing
    L = _capi.lib()
    for f in header_functions():
        assert getattr(L, f) is not None


def test_library_is_sm100a_only():
    """libsdag.so carries sm_100a SASS (and no other arch)."""
    out = subprocess.run(["cuobjdump", "--list-elf", _capi.LIB_PATH], capture_output=True, text=True).stdout
    archs = set(re.findall(r"sm_(\d+a?)", out))
    assert archs == {"100a"}, archs


def test_version_and_launch_counter():
    assert "sm_100a" in sdag.version()
    assert sdag.launch_count() >= 0


def test_profile_struct_layout():
    """ctypes mirror of sdag_profile: 96-byte name, 11 doubles, 5 int32, 1024-byte hints"""
    import ctypes

    from paper_conf_ipps_rawatvsrps19_b200 import _capi
    assert _capi.Profile.hints.offset == 96 + 11 * 8 + 5 * 4
    assert ctypes.sizeof(_capi.Profile) == 96 + 11 * 8 + 5 * 4 + 1024 + 4  # padded to 8


def test_plain_c_client(tmp_path):
    """the boundary is a C ABI: examples/c_api_host.c (no Python, no torch) builds
    against include/sdag.h + libsdag.so, plans Listing 1 host-only, reads the
    analysis and writes the trivial fission of rhs4center"""
    import os
    import shutil
    import subprocess

    if not shutil.which("gcc"):
        pytest.skip("no C compiler")
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    lib = os.path.join(root, "paper_conf_ipps_rawatvsrps19_b200", "lib")
    exe = str(tmp_path / "c_api_host")
    subprocess.check_call(["gcc", "-std=c99", "-Wall", "-Werror", "-I" + os.path.join(root, "include"),
                           os.path.join(root, "examples", "c_api_host.c"), "-L" + lib, "-lsdag",
                           "-Wl,-rpath," + lib, "-o", exe])
    out = subprocess.run([exe, os.path.join(root, "paper_conf_ipps_rawatvsrps19_b200", "specs", "rhs4center.sdag")],
                         capture_output=True, text=True, timeout=120)
    assert out.returncode == 0, out.stderr
    assert "dag jacobi7" in out.stdout and "radius 1 1 1 flops/pt 10" in out.stdout
    assert "array B role 1" in out.stdout and "array A role 0" in out.stdout
    assert "bad spec -> status 2 (PARSE)" in out.stdout
    assert "trivial fission: 3 stencils" in out.stdout


def test_binding_rejects_undersized_host_buffers():
    """the binding checks element counts before handing raw pointers
    to the C ABI (an undersized buffer would be read/written out of bounds)."""
    import numpy as np
    import pytest as _pt

    import paper_conf_ipps_rawatvsrps19_b200 as sdag
    plan = sdag.Plan(sdag.spec_text("jacobi7"), (8, 9, 10), device="none")
    ok = np.zeros((8, 9, 10))
    with _pt.raises(ValueError, match="elements"):
        plan.apply_host([np.zeros((8, 9, 9)), ok], scalars=[4.0, 0.5, 0.25])
    r4 = sdag.Plan(sdag.spec_text("rhs4center"), (8, 9, 10), device="none")
    g = [np.zeros((8, 9, 10)) for _ in range(8)]
    with _pt.raises(ValueError, match="axis"):  # strz has the y extent
        r4.apply_host(g, [np.zeros(10), np.zeros(9), np.zeros(9)], scalars=[0.75, 1 / 6, 1 / 144, 1.0, 1.0])


def _build_device_client(tmp_path):
    import os
    import shutil
    import subprocess

    if not shutil.which("gcc"):
        pytest.skip("no C compiler")
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    lib = os.path.join(root, "paper_conf_ipps_rawatvsrps19_b200", "lib")
    cuda = "/usr/local/cuda"
    exe = str(tmp_path / "c_api_device")
    subprocess.check_call(["gcc", "-std=c99", "-Wall", "-Werror", "-I" + os.path.join(root, "include"),
                           "-I" + cuda + "/include", os.path.join(root, "examples", "c_api_device.c"), "-L" + lib,
                           "-lsdag", "-Wl,-rpath," + lib, "-L" + cuda + "/lib64", "-lcudart",
                           "-Wl,-rpath," + cuda + "/lib64", "-o", exe])
    return exe, os.path.join(root, "paper_conf_ipps_rawatvsrps19_b200", "specs", "lap25.sdag")


def test_plain_c_device_client_builds(tmp_path):
    """examples/c_api_device.c (device pointers, cudaMalloc, sdag_apply on a
    stream) compiles with -Werror against include/sdag.h and links libsdag.so"""
    _build_device_client(tmp_path)


@pytest.mark.gpu
def test_plain_c_device_client_runs(tmp_path):
    """the plain-C client on device pointers: every interior point of the
    5040-scaled Laplacian of x^2 + 2y^2 - z^2 is exactly 20160, the ring keeps
    its sentinel, an aliased output is refused"""
    import subprocess
    exe, spec = _build_device_client(tmp_path)
    out = subprocess.run([exe, spec], capture_output=True, text=True, timeout=300)
    assert out.returncode == 0, out.stdout + out.stderr
    assert "mismatches 0" in out.stdout and "aliased output -> status 1" in out.stdout
    assert "device C ABI ok" in out.stdout and "sdag_star" in out.stdout

"""The C-ABI library loads without a GPU and exports every entry point that
include/sdag.h declares (no compute calls)."""
import os
import re
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

"""The C-ABI library builds for sm_100a, loads, and exports every symbol include/hirace.h
declares; without a GPU it fails loudly instead of falling back to the CPU."""
import os
import re
import subprocess

import pytest

from paper_conf_sc_jacobsonbg24_b200 import build, hirace

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    src = open(os.path.join(ROOT, "include", "hirace.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(hirace_[a-z_]+)\s*\(", src)))


def test_header_declares_the_boundary():
    names = _declared()
    for must in ("hirace_shadow_alloc", "hirace_barrier", "hirace_replay_trace", "hirace_collect_races",
                 "hirace_bucket_events"):
        assert must in names
    assert sorted(hirace.EXPORTS) == names


def test_library_exports_every_declared_symbol():
    so = build.build()
    out = subprocess.check_output(["nm", "-D", "--defined-only", so], text=True)
    exported = set(re.findall(r"\bT (hirace_\w+)", out))
    missing = set(_declared()) - exported
    assert not missing, missing
    lib = hirace.load()
    for name in _declared():
        assert hasattr(lib, name)


def test_library_targets_sm100a_only():
    so = build.build()
    out = subprocess.check_output(["/usr/local/cuda/bin/cuobjdump", "--list-elf", so], text=True)
    assert "sm_100a" in out
    assert not re.search(r"sm_(?!100a)\d+", out)


def test_no_cpu_fallback_without_gpu():
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    with pytest.raises(hirace.HiraceError) as e:
        hirace.Checker(1, 32, 32, 16, 0)
    assert e.value.status == -3  # HIRACE_E_CUDA


def test_status_strings_and_version():
    lib = hirace.load()
    assert lib.hirace_status_string(-6) == b"bad trace"
    assert b"sm_100a" in lib.hirace_version()

"""The replay kernel's raw-flag label (include/hirace_device.cuh label_raw + expand_raw_table)
selects the canonical FSM entry for every state / kind / relation / epoch difference: a host
C++ check compiled with g++ against the library's canonical table (no GPU)."""
import os
import subprocess

import numpy as np
import pytest

import paper_conf_sc_jacobsonbg24_b200 as hr

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.parametrize("policy", [hr.POLICY_STRICT, hr.POLICY_RELAXED_READ_ATOMIC])
def test_label_raw_matches_canonical_table(tmp_path, policy):
    exe = tmp_path / "label_raw_check"
    subprocess.check_call(["g++", "-O2", "-std=c++17", "-I", os.path.join(ROOT, "include"),
                           os.path.join(ROOT, "tests", "native", "label_raw_check.cpp"), "-o", str(exe)])
    tab = tmp_path / "table.bin"
    hr.fsm_table(policy).astype(np.uint8).tofile(tab)
    out = subprocess.run([str(exe), str(tab)], capture_output=True, text=True)
    assert out.returncode == 0, out.stdout + out.stderr
    assert out.stdout.startswith("ok")

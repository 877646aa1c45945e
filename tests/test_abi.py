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


def test_ctypes_structs_match_the_c_header(tmp_path):
    """The binding's ctypes mirrors of hirace_config / hirace_dev_ctx / hirace_epoch_limits have
    the C layout (the library writes whole structs into them)."""
    import ctypes
    import subprocess

    from paper_conf_sc_jacobsonbg24_b200 import hirace as hb
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    src = tmp_path / "sz.c"
    fields = [f for f, _ in hb.DevCtx._fields_]
    src.write_text("#include <stdio.h>\n#include <stddef.h>\n#include \"hirace.h\"\nint main(){\n"
                   "printf(\"%zu %zu %zu\\n\", sizeof(hirace_config), sizeof(hirace_dev_ctx), sizeof(hirace_epoch_limits));\n"
                   + "".join(f"printf(\"%zu\\n\", offsetof(hirace_dev_ctx, {f}));\n" for f in fields) + "return 0;}\n")
    exe = tmp_path / "sz"
    subprocess.check_call(["gcc", "-I", os.path.join(root, "include"), str(src), "-o", str(exe)])
    out = subprocess.check_output([str(exe)], text=True).split()
    assert [int(x) for x in out[:3]] == [ctypes.sizeof(hb.Config), ctypes.sizeof(hb.DevCtx),
                                        ctypes.sizeof(hb.EpochLimits)]
    assert [int(x) for x in out[3:]] == [getattr(hb.DevCtx, f).offset for f in fields]


def test_cluster_dev_ctx_mirror_matches_the_c_header(tmp_path):
    import ctypes
    import subprocess

    from paper_conf_sc_jacobsonbg24_b200 import hirace as hb
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    fields = [f for f, _ in hb.ClusterDevCtx._fields_]
    src = tmp_path / "csz.c"
    src.write_text("#include <stdio.h>\n#include <stddef.h>\n#include \"hirace.h\"\nint main(){\n"
                   "printf(\"%zu %zu\\n\", sizeof(hirace_cluster_dev_ctx), sizeof(hirace_warp_sync));\n"
                   + "".join(f"printf(\"%zu\\n\", offsetof(hirace_cluster_dev_ctx, {f}));\n" for f in fields)
                   + "return 0;}\n")
    exe = tmp_path / "csz"
    subprocess.check_call(["gcc", "-I", os.path.join(root, "include"), str(src), "-o", str(exe)])
    out = [int(x) for x in subprocess.check_output([str(exe)], text=True).split()]
    assert out[:2] == [ctypes.sizeof(hb.ClusterDevCtx), hb.WARP_SYNC_DTYPE.itemsize]
    assert out[2:] == [getattr(hb.ClusterDevCtx, f).offset for f in fields]


def test_ws_ctx_mirror_matches_the_c_header(tmp_path):
    import ctypes
    import subprocess

    from paper_conf_sc_jacobsonbg24_b200 import hirace as hb
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    fields = [f for f, _ in hb.WsCtx._fields_]
    src = tmp_path / "wsz.c"
    src.write_text("#include <stdio.h>\n#include <stddef.h>\n#include \"hirace.h\"\nint main(){\n"
                   "printf(\"%zu\\n\", sizeof(hirace_ws_ctx));\n"
                   + "".join(f"printf(\"%zu\\n\", offsetof(hirace_ws_ctx, {f}));\n" for f in fields)
                   + "return 0;}\n")
    exe = tmp_path / "wsz"
    subprocess.check_call(["gcc", "-I", os.path.join(root, "include"), str(src), "-o", str(exe)])
    out = [int(x) for x in subprocess.check_output([str(exe)], text=True).split()]
    assert out[0] == ctypes.sizeof(hb.WsCtx)
    assert out[1:] == [getattr(hb.WsCtx, f).offset for f in fields]

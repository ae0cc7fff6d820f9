"""CPU-side checks of the C-ABI library: it loads and exports every symbol that
include/rw.h declares (no compute calls without a GPU)."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_symbols():
    src = open(os.path.join(ROOT, "include", "rw.h")).read()
    return sorted(set(re.findall(r"^\s*(?:rw_status|void|int64_t|const char \*)\s*\*?\s*(rw_\w+)\s*\(", src, re.M)))


def test_header_declares_the_boundary():
    names = declared_symbols()
    for n in ["rw_plan_create", "rw_plan_add_select", "rw_plan_add_project", "rw_plan_add_join",
              "rw_plan_add_agg", "rw_plan_execute", "rw_plan_explain", "rw_plan_destroy"]:
        assert n in names


def test_library_loads_and_exports_every_declared_symbol():
    from paper_conf_micro_wudcy12_b200 import _build
    lib_path = _build.build()
    lib = ctypes.CDLL(lib_path)
    missing = [n for n in declared_symbols() if not hasattr(lib, n)]
    assert not missing, missing
    from paper_conf_micro_wudcy12_b200 import rw
    assert set(rw.EXPORTS) <= set(declared_symbols())
    rw.lib()


def test_status_strings_without_gpu():
    from paper_conf_micro_wudcy12_b200 import rw
    L = rw.lib()
    for code, name in rw.STATUS.items():
        assert L.rw_status_str(code).decode() == name


def test_create_fails_loudly_without_device():
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    from paper_conf_micro_wudcy12_b200 import rw
    o = rw.rw_plan_opts()
    o.fuse = 1
    h = ctypes.c_void_p()
    st = rw.lib().rw_plan_create(ctypes.byref(h), ctypes.byref(o))
    assert st == -8 or st == -1   # RW_E_CUDA / RW_E_ARG: no silent CPU path


def test_kernels_are_sm100a_sass():
    import subprocess
    from paper_conf_micro_wudcy12_b200 import _build
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "-lelf", _build.build()], capture_output=True, text=True).stdout
    assert "sm_100a" in out
    sass = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "-sass", _build.build()], capture_output=True, text=True).stdout
    assert "UBLKCP" in sass          # TMA bulk copies (cp.async.bulk) in the scan chain
    assert "VOTE" in sass            # warp ballot compaction

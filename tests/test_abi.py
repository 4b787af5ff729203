"""Host-side checks of the C-ABI library (CPU only, no compute calls): it builds for
sm_100a, loads, exports every symbol include/topk.h declares, and the product package
neither imports the oracle nor has a CPU path."""
import ctypes
import os
import re

import pytest
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_sigmod_shanbhagpm18_b200")


def header_functions():
    src = open(os.path.join(ROOT, "include", "topk.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(topk_[a-z0-9_]+)\s*\(", src)))


@pytest.fixture(scope="module")
def lib():
    from paper_conf_sigmod_shanbhagpm18_b200 import _build, _lib
    _build.build()
    return _lib.load(build_if_missing=False)


def test_exports_every_header_symbol(lib):
    from paper_conf_sigmod_shanbhagpm18_b200 import _lib
    names = header_functions()
    assert len(names) >= 13
    assert sorted(_lib.SYMBOLS) == names
    for name in names:
        assert getattr(lib, name) is not None


def test_sass_is_sm100a():
    from paper_conf_sigmod_shanbhagpm18_b200 import _build
    import subprocess
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", _build.LIB],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_host_only_calls(lib):
    assert lib.topk_abi_version() == 1
    assert b"INVALID" in lib.topk_status_string(1)
    assert lib.topk_launch_count() == 0
    # argument errors are synchronous and need no device
    assert lib.topk_select(0, None, None, 10, 0, 3, 0, 0, None, None, None, None, 0, None) == 1
    assert lib.topk_select(0, ctypes.c_void_p(16), None, 10, 0, 0, 0, 0, None, None, None,
                           None, 0, None) == 1
    assert lib.topk_select(0, ctypes.c_void_p(16), None, 10, 0, 11, 0, 0, None, None, None,
                           None, 0, None) == 1
    assert lib.topk_select(0, ctypes.c_void_p(16), None, 5000, 0, 2049, 0, 0, None, None, None,
                           None, 0, None) == 1
    assert lib.topk_select(0, ctypes.c_void_p(18), None, 10, 0, 1, 0, 0, None, None, None,
                           None, 0, None) == 1  # misaligned f32 pointer
    assert lib.topk_merge(0, None, None, None, 1, 4, 2, 0, None, None, None, None, 0, None) == 1


def test_product_never_imports_oracle():
    for dirpath, _, files in os.walk(PKG):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                src = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in src and "from oracle" not in src, f
                assert "topk_oracle" not in src, f


def test_no_cpu_path():
    import paper_conf_sigmod_shanbhagpm18_b200 as tk
    with pytest.raises(ValueError):
        tk.topk(torch.zeros(100), 5)

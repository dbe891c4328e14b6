"""The C ABI library: builds, loads without a GPU, exports every symbol
include/spline_builder.h declares, and reports errors through status codes
(no compute calls -- this file runs on CPU)."""
import ctypes
import os
import re
import subprocess

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "spline_builder.h")


@pytest.fixture(scope="module")
def lib():
    from paper_conf_sc_asahilbpbgo24_b200 import _lib, build
    build.build()
    return _lib.load()


def declared_functions():
    text = open(HEADER).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    names = set(re.findall(r"\b(spline_builder_\w+)\s*\(", text))
    return sorted(names)


def test_header_declares_expected_entry_points():
    names = declared_functions()
    for must in ("spline_builder_create", "spline_builder_solve", "spline_builder_destroy"):
        assert must in names


def test_every_declared_symbol_is_exported(lib):
    from paper_conf_sc_asahilbpbgo24_b200 import _lib
    names = declared_functions()
    assert set(names) == set(_lib.EXPORTS), "binding EXPORTS out of sync with the header"
    for name in names:
        assert hasattr(lib, name), name
    out = subprocess.run(["nm", "-D", "--defined-only", _lib.LIB_PATH], capture_output=True, text=True).stdout
    exported = set(re.findall(r"\bT (spline_builder_\w+)", out))
    assert set(names) <= exported


def test_library_has_no_torch_dependency(lib):
    from paper_conf_sc_asahilbpbgo24_b200 import _lib
    out = subprocess.run(["ldd", _lib.LIB_PATH], capture_output=True, text=True).stdout
    assert "torch" not in out and "libc10" not in out


def test_sm100a_code_present(lib):
    from paper_conf_sc_asahilbpbgo24_b200 import _lib
    out = subprocess.run(["cuobjdump", "--list-elf", _lib.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_tma_in_sass(lib):
    """the tile kernel issues TMA (UTMALDG) and the mbarrier pipeline (SYNCS)."""
    from paper_conf_sc_asahilbpbgo24_b200 import _lib
    out = subprocess.run(["cuobjdump", "-sass", _lib.LIB_PATH], capture_output=True, text=True).stdout
    assert "UTMALDG" in out
    assert "SYNCS" in out


def test_invalid_arguments_return_null_with_status(lib):
    from paper_conf_sc_asahilbpbgo24_b200 import _lib
    assert not lib.spline_builder_create_ex(0, 100, 0, None, -1, -1, 1)
    assert lib.spline_builder_last_status() == _lib.SB_INVALID_ARG
    assert b"degree" in lib.spline_builder_last_error()
    bad = np.array([0.0, 0.5, 0.4, 1.0])
    assert not lib.spline_builder_create_ex(3, 3, 0, ctypes.c_void_p(bad.ctypes.data), -1, -1, 1)
    assert lib.spline_builder_last_status() == _lib.SB_INVALID_ARG
    assert not lib.spline_builder_create_ex(3, 100, 7, None, -1, -1, 1)
    assert not lib.spline_builder_create_ex(3, 100, 0, None, 1, 1, 1)  # periodic needs split_lo == 0


def test_host_only_handle(lib):
    from paper_conf_sc_asahilbpbgo24_b200 import SplineBuilder, _lib
    sb = SplineBuilder(3, 1000, 0, host_only=True)
    assert sb.n == 1000
    info = sb.info()
    assert info["nbasis"] == 1000 and info["k"] == 1
    # a host-only handle never launches: solve reports UNSUPPORTED (batch 0 is a no-op)
    assert sb._lib.spline_builder_solve(sb._h, ctypes.c_void_p(16), 10, 1, None) == _lib.SB_UNSUPPORTED
    assert sb._lib.spline_builder_solve_host(sb._h, ctypes.c_void_p(16), 0, 10, 10) == _lib.SB_UNSUPPORTED
    sb.close()


def test_null_handle_is_safe(lib):
    from paper_conf_sc_asahilbpbgo24_b200 import _lib
    lib.spline_builder_destroy(None)
    assert lib.spline_builder_solve(None, None, 1, 1, None) == _lib.SB_INVALID_ARG
    assert lib.spline_builder_nbasis(None) == -1
    assert lib.spline_builder_version().startswith(b"b200-spline-build")


def test_device_create_without_gpu_fails_cleanly(lib):
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    from paper_conf_sc_asahilbpbgo24_b200 import _lib
    h = lib.spline_builder_create(3, 100, 0, None)
    assert not h
    assert lib.spline_builder_last_status() == _lib.SB_CUDA


def test_product_path_does_not_import_oracle():
    """the package never imports oracle/ (test infrastructure only)."""
    pkg = os.path.join(ROOT, "paper_conf_sc_asahilbpbgo24_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cpp", ".cu", ".cuh", ".hpp", ".h")):
                text = open(os.path.join(dirpath, f), errors="ignore").read()
                assert "import oracle" not in text and "from oracle" not in text, f
                assert "spline_oracle" not in text, f

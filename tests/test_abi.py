"""Host-side checks of the C-ABI library: it loads, exports every symbol the
header declares, and fails loudly (no CPU fallback) without a GPU.  CPU only:
no compute calls are made here."""
import ctypes
import os
import re

import pytest

from paper_conf_ipps_ribizela19_b200 import _abi, build

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "sampleselect.h")


@pytest.fixture(scope="module")
def lib():
    build.build()
    return _abi.lib()


def _declared():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(ss_[a-z_0-9]+)\s*\(", src)))


def test_header_declares_expected_api():
    decl = _declared()
    assert decl == sorted(_abi.EXPORTS)
    for name in ["ss_select", "ss_approx_select", "ss_create", "ss_destroy"]:
        assert name in decl


def test_library_exports_every_declared_symbol(lib):
    for name in _declared():
        assert hasattr(lib, name), name
    assert lib.ss_abi_version() == 7


def test_exported_symbols_are_c_linkage(lib):
    out = os.popen(f"nm -D --defined-only {_abi.LIB_PATH}").read()
    syms = set(re.findall(r"\bT (ss_[a-z_0-9]+)\b", out))
    assert set(_declared()) <= syms


def test_status_strings(lib):
    for code, name in _abi.STATUS.items():
        assert lib.ss_status_string(code).decode() == name


def test_create_rejects_bad_arguments(lib):
    assert lib.ss_create(0, None) == 1
    h = ctypes.c_void_p()
    assert lib.ss_create(-1, ctypes.byref(h)) == 1


def test_no_gpu_fails_loudly(lib):
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is visible")
    h = ctypes.c_void_p()
    assert lib.ss_create(0, ctypes.byref(h)) == 2  # SS_ERR_CUDA, no fallback
    from paper_conf_ipps_ribizela19_b200 import Context, SSError
    with pytest.raises(SSError):
        Context(0)


def test_null_context_argument_checks(lib):
    """Argument validation happens before any device work."""
    out = ctypes.c_float()
    assert lib.ss_select(None, 0, ctypes.c_void_p(16), 10, 0, ctypes.byref(out), None) == 1
    assert lib.ss_last_error(None) == b"NULL context"


def test_product_never_imports_oracle():
    """The product package must not reference the test oracle."""
    pkg = os.path.join(ROOT, "paper_conf_ipps_ribizela19_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                src = open(os.path.join(dirpath, f)).read()
                assert not re.search(r"^\s*(import|from)\s+oracle\b", src, re.M), f
                assert "oracle.c" not in src and "liboracle" not in src, f

"""CPU-side checks of the C ABI: libbar.so builds for sm_100a, loads, and exports every symbol
include/bar.h declares (no compute calls: there is no GPU here)."""
import ctypes
import os
import re
import subprocess

import pytest

from conftest import ROOT

HEADER = os.path.join(ROOT, "include", "bar.h")
LIB = os.path.join(ROOT, "paper_conf_ipps_anzttdh12_b200", "libbar.so")


def _declared():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(bar_[a-z_0-9]+)\s*\(", src)))


@pytest.fixture(scope="module")
def lib():
    from tools.build import build_bar

    try:
        build_bar()
    except RuntimeError as e:  # pragma: no cover
        pytest.fail(f"libbar.so does not build: {e}")
    return ctypes.CDLL(LIB)


def test_header_declares_the_contract():
    d = _declared()
    for name in ("bar_create_csr", "bar_solve", "bar_residual", "bar_destroy", "bar_last_error"):
        assert name in d


def test_every_declared_symbol_is_exported(lib):
    for name in _declared():
        assert hasattr(lib, name), name
    out = subprocess.run(["nm", "-D", "--defined-only", LIB], capture_output=True, text=True).stdout
    exported = set(re.findall(r" T (bar_[a-z_0-9]+)$", out, flags=re.M))
    assert set(_declared()) <= exported
    # the binding names the same symbols
    import importlib

    bar = importlib.import_module("paper_conf_ipps_anzttdh12_b200.bar")
    assert set(bar.EXPORTS) == set(_declared())


def test_sass_is_sm100a(lib):
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", LIB], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_null_safe_without_gpu(lib):
    """Argument validation happens before any device work."""
    lib.bar_last_error.restype = ctypes.c_char_p
    lib.bar_destroy(None)
    st = lib.bar_create_csr(ctypes.c_int64(0), ctypes.c_int64(0), None, None, None, 128, 0, None)
    assert st == 1  # BAR_ERR_INVALID_ARG
    assert lib.bar_last_error()

"""Host-side checks of the C ABI boundary (no GPU needed): the library builds,
loads, and exports every symbol include/spbla_b200.h declares; the Python
binding declares the same set; calls fail cleanly without a device."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "spbla_b200.h")


def header_symbols():
    txt = open(HEADER).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(spbla_[A-Za-z_]+)\s*\(", txt)))


@pytest.fixture(scope="module")
def lib():
    from paper_conf_ipps_orachevkkg21_b200 import _build, _capi
    _build.build_library()
    return _capi.load()


def test_header_declares_the_paper_operations():
    syms = header_symbols()
    for s in ["spbla_Matrix_New", "spbla_Matrix_Build", "spbla_Matrix_ExtractPairs", "spbla_MxM",
              "spbla_Matrix_EWiseAdd", "spbla_Kronecker", "spbla_Matrix_Transpose", "spbla_Matrix_Reduce",
              "spbla_Matrix_ExtractSubMatrix", "spbla_TransitiveClosure", "spbla_Matrix_Free"]:
        assert s in syms


def test_library_exports_every_header_symbol(lib):
    missing = [s for s in header_symbols() if not hasattr(lib, s)]
    assert not missing, missing


def test_binding_covers_header():
    from paper_conf_ipps_orachevkkg21_b200 import _capi
    assert sorted(_capi.SIGNATURES) == header_symbols()


def test_sm100a_code_in_library():
    from paper_conf_ipps_orachevkkg21_b200 import _build
    import subprocess
    out = subprocess.run(["cuobjdump", "--list-elf", _build.LIB], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_calls_fail_cleanly_without_device(lib):
    import torch
    if torch.cuda.is_available():
        pytest.skip("device present")
    st = lib.spbla_Initialize(0)
    assert st != 0
    h = ctypes.c_void_p()
    assert lib.spbla_Matrix_New(ctypes.byref(h), 4, 4) == 4  # INVALID_STATE
    assert b"Initialize" in lib.spbla_GetLastErrorMessage()

"""C-ABI boundary checks that need no GPU: the library loads, exports every
symbol include/ks.h declares, and refuses to run without an sm_100 device
(no CPU fallback).  Also: the product package never touches oracle/."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "ks.h")
PKG = os.path.join(ROOT, "paper_conf_icppw_wangkbgj16_b200")


def declared_symbols():
    txt = open(HEADER).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(ks_[a-z_0-9]+)\s*\(", txt)))


@pytest.fixture(scope="module")
def lib():
    from paper_conf_icppw_wangkbgj16_b200 import build
    build.build()
    return ctypes.CDLL(build.LIB)


def test_header_declares_expected_api():
    syms = declared_symbols()
    for s in ("ks_create", "ks_set_sources", "ks_eval", "ks_destroy", "ks_get_info", "ks_last_error"):
        assert s in syms


def test_library_exports_every_declared_symbol(lib):
    for s in declared_symbols():
        assert hasattr(lib, s), f"libks.so does not export {s}"


def test_binding_lists_every_symbol():
    import paper_conf_icppw_wangkbgj16_b200 as ks
    assert sorted(ks.EXPORTED) == declared_symbols()


def test_only_abi_symbols_exported(lib):
    """-fvisibility=hidden: the .so exports the ABI, not internals."""
    import subprocess
    from paper_conf_icppw_wangkbgj16_b200 import build
    out = subprocess.run(["nm", "-D", "--defined-only", build.LIB], capture_output=True, text=True).stdout
    ours = [l.split()[-1] for l in out.splitlines() if l.split()[-1].startswith("ks")]
    assert sorted(set(ours)) == declared_symbols()


def test_status_strings(lib):
    lib.ks_status_str.restype = ctypes.c_char_p
    names = [lib.ks_status_str(i).decode() for i in range(6)]
    assert names == ["KS_OK", "KS_EINVAL", "KS_ESTATE", "KS_ENOMEM", "KS_ECUDA", "KS_EUNSUPPORTED"]
    lib.ks_version.restype = ctypes.c_char_p
    assert b"sm_100a" in lib.ks_version()


def test_argument_errors_without_gpu(lib):
    """Validation happens before any device call; NULL-safe entry points."""
    lib.ks_create.argtypes = [ctypes.c_int, ctypes.c_float, ctypes.POINTER(ctypes.c_void_p)]
    lib.ks_last_error.restype = ctypes.c_char_p
    out = ctypes.c_void_p()
    assert lib.ks_create(0, 1.0, ctypes.byref(out)) == 1          # K < 1
    assert lib.ks_create(4097, 1.0, ctypes.byref(out)) == 1       # K > 4096
    assert lib.ks_create(4, 0.0, ctypes.byref(out)) == 1          # h <= 0
    assert lib.ks_create(4, float("nan"), ctypes.byref(out)) == 1
    assert lib.ks_create(4, float("inf"), ctypes.byref(out)) == 1
    assert lib.ks_create(4, 1e-30, ctypes.byref(out)) == 1        # c overflows FP32
    assert b"h=" in lib.ks_last_error()
    assert lib.ks_create(4, 1.0, None) == 1
    lib.ks_destroy.argtypes = [ctypes.c_void_p]
    assert lib.ks_destroy(None) == 0                               # NULL is a no-op
    lib.ks_eval.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p]
    assert lib.ks_eval(None, None, 0, None) == 1


def test_no_gpu_means_error_not_fallback(lib):
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    lib.ks_create.argtypes = [ctypes.c_int, ctypes.c_float, ctypes.POINTER(ctypes.c_void_p)]
    out = ctypes.c_void_p()
    rc = lib.ks_create(4, 1.0, ctypes.byref(out))
    assert rc in (4, 5) and not out.value


def test_product_never_imports_oracle():
    for dirpath, _, files in os.walk(PKG):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                txt = open(os.path.join(dirpath, f)).read()
                assert not re.search(r"\boracle\b", txt.replace("# oracle-free", "")), \
                    f"{f} references the oracle"

"""The C-ABI library loads and exports every symbol include/mp.h declares (no GPU needed)."""
import ctypes
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HDR = os.path.join(ROOT, "include", "mp.h")


def declared_symbols():
    txt = open(HDR).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(mp_[a-z_]+)\s*\(", txt)))


@pytest.fixture(scope="module")
def libmp():
    from paper_conf_ipps_tayebbfg24_b200 import build as b
    path = b.build()
    return ctypes.CDLL(path), path


def test_header_declares_north_star_calls():
    syms = declared_symbols()
    for s in ("mp_build_dag", "mp_bottom_level", "mp_affinity", "mp_score", "mp_build_queues", "mp_free",
              "mp_replicas_run"):
        assert s in syms


def test_library_exports_every_declared_symbol(libmp):
    lib, path = libmp
    out = subprocess.run(["nm", "-D", "--defined-only", path], capture_output=True, text=True).stdout
    exported = set(re.findall(r"\s[TW]\s+(mp_\w+)", out))
    for s in declared_symbols():
        assert s in exported, s
        assert hasattr(lib, s)


def test_status_strings_and_build_info(libmp):
    lib, _ = libmp
    lib.mp_status_str.restype = ctypes.c_char_p
    lib.mp_build_info.restype = ctypes.c_char_p
    assert lib.mp_status_str(0) == b"MP_OK"
    assert lib.mp_status_str(2) == b"MP_ERR_CYCLE"
    assert b"sm_100a" in lib.mp_build_info()
    lib.mp_free(None)  # NULL-safe, no GPU touched


def test_library_is_sm100a_cubin(libmp):
    _, path = libmp
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", path], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_arg_errors_without_gpu(libmp):
    """Host-side argument checks return before any launch."""
    lib, _ = libmp
    h = ctypes.c_void_p()
    lib.mp_build_dag.argtypes = [ctypes.c_int32, ctypes.c_int64, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
                                 ctypes.POINTER(ctypes.c_void_p)]
    assert lib.mp_build_dag(-1, 0, None, None, None, ctypes.byref(h)) == 1
    assert lib.mp_build_dag(4, 3, None, None, None, ctypes.byref(h)) == 1

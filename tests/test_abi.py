"""The C-ABI library loads and exports every symbol include/proclus.h
declares; argument validation that needs no GPU; the oracle / library
separation (CPU only, no compute calls)."""
import ctypes as C
import os
import re
import subprocess

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "proclus.h")
PKG = os.path.join(ROOT, "paper_conf_edbt_jorgensensape22_b200")


def declared_symbols():
    src = open(HEADER).read()
    return sorted(set(re.findall(r"PROCLUS_API\s+[\w\s\*]+?\b(proclus_\w+)\s*\(", src)))


@pytest.fixture(scope="module")
def pk():
    import paper_conf_edbt_jorgensensape22_b200 as pk

    pk.lib()
    return pk


def test_header_declares_the_boundary():
    syms = declared_symbols()
    for want in ("proclus_create", "proclus_create_ex", "proclus_run", "proclus_run_multi",
                 "proclus_destroy", "proclus_last_error", "proclus_load"):
        assert want in syms


def test_library_exports_every_declared_symbol(pk):
    out = subprocess.check_output(["nm", "-D", "--defined-only", pk.LIB_PATH]).decode()
    exported = set(re.findall(r"\bT (proclus_\w+)", out))
    assert set(declared_symbols()) <= exported
    # and the binding binds exactly the declared set, by the same names
    assert sorted(n for n, _, _ in pk.SIGNATURES) == declared_symbols()


def test_library_is_sm100a(pk):
    out = subprocess.check_output(["cuobjdump", "--list-elf", pk.LIB_PATH]).decode()
    assert "sm_100a" in out
    assert pk.proclus_target_sm() == 100
    assert pk.proclus_abi_version() == 1


def test_validation_without_gpu(pk):
    L = pk.lib()
    h = C.c_void_p()
    data = np.zeros((10, 3), np.float32)
    assert L.proclus_create(None, 10, 3, C.byref(h)) == pk.EINVAL
    assert L.proclus_create(data.ctypes.data, 0, 3, C.byref(h)) == pk.EINVAL
    assert L.proclus_create(data.ctypes.data, 10, 1, C.byref(h)) == pk.EINVAL
    assert "d must be" in pk.proclus_last_error()
    assert L.proclus_create(data.ctypes.data, 10, 2000, C.byref(h)) == pk.EINVAL
    o = pk.proclus_options_init()
    o.metric = 7
    assert L.proclus_create_ex(data.ctypes.data, 10, 3, C.byref(o), C.byref(h)) == pk.EINVAL
    o = pk.proclus_options_init()
    o.world_size, o.rank = 2, 2
    assert L.proclus_create_ex(data.ctypes.data, 10, 3, C.byref(o), C.byref(h)) == pk.EINVAL
    res = pk.proclus_result()
    assert L.proclus_run(None, 5, 3, 100, 10, 0.7, 5, 1, C.byref(res)) == pk.EINVAL
    L.proclus_destroy(None)  # NULL-safe
    assert pk.proclus_last_launches(None) == -1


def test_options_defaults(pk):
    o = pk.proclus_options_init()
    assert (o.device, o.metric, o.max_iter, o.world_size, o.trace) == (-1, 0, 10000, 1, 0)


def test_oracle_and_library_share_nothing():
    """The oracle (test infrastructure) and the CUDA path share no code."""
    for dirpath, _, files in os.walk(PKG):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                src = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in src and "from oracle" not in src, f
                assert "proclus_oracle" not in src and "liboracle" not in src, f
    for f in os.listdir(os.path.join(ROOT, "oracle")):
        if f.endswith((".c", ".h", ".py")):
            src = open(os.path.join(ROOT, "oracle", f)).read()
            assert not re.search(r'#include\s*[<"][^>"]*proclus\.h', src), f
            assert not re.search(r"^\s*(import|from)\s+paper_conf_edbt", src, re.M), f
            assert "libproclus" not in src, f

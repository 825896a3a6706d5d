"""The C-ABI library loads and exports every symbol include/cg.h declares (no GPU needed),
argument errors are reported before any device work, and the product package carries no
route to the oracle."""
import ctypes
import os
import re

import pytest

from paper_conf_eurosys_0002a0a024_b200 import _build, _lib

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def L():
    return _lib.lib(build=True)


def test_exports_every_header_symbol(L):
    names = _lib.header_functions()
    assert len(names) >= 15
    for name in names:
        assert hasattr(L, name), name
    assert set(names) == set(_lib._SIGS), "binding and header disagree"


def test_sm100a_cubin_embedded():
    out = os.popen(f"/usr/local/cuda/bin/cuobjdump --list-elf {_build.LIB} 2>&1").read()
    assert "sm_100a" in out


def test_status_strings(L):
    for code, name in _lib.STATUS.items():
        assert L.cg_status_string(code).decode() == name


def test_argument_errors_without_device(L):
    h = ctypes.c_void_p()
    assert L.cg_graph_create(0, 0, 0, None, None, None, None, ctypes.byref(h)) == -1
    assert b"n must be" in L.cg_last_error()
    assert L.cg_graph_create(0, 5, 3, None, None, None, None, ctypes.byref(h)) == -1
    assert L.cg_graph_create(0, 5, 0, None, None, None, None, None) == -1
    assert L.cg_graph_info(None, None, None, None) == -1
    assert L.cg_query(None, 0, None, 0, 0, None, None, None) == -1
    assert L.cg_build(None, 0, 20, 0, None, 0, None) == -1
    assert L.cg_graph_destroy(None) == 0
    with pytest.raises(_lib.CGInvalid):
        _lib.call("cg_graph_info", None, None, None, None)


def test_allocator_pairing(L):
    assert L.cg_set_allocator(_lib.ALLOC_FN(), _lib.FREE_FN(), None) == 0  # NULL, NULL restores cudaMalloc
    a = _lib.ALLOC_FN(lambda n, s, c: None)
    assert L.cg_set_allocator(a, _lib.FREE_FN(), None) == -1


def test_product_never_imports_oracle():
    pkg = os.path.join(ROOT, "paper_conf_eurosys_0002a0a024_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".hpp", ".h", ".cpp")):
                text = open(os.path.join(dirpath, f)).read()
                assert not re.search(r"^\s*(import|from)\s+oracle\b", text, re.M), f
                assert "oracle.c" not in text and "liboracle" not in text, f

"""C-ABI library checks that need no GPU: it loads, exports every symbol that
include/sssp.h declares, and rejects bad arguments before touching a device."""
import ctypes
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HDR = os.path.join(ROOT, "include", "sssp.h")


@pytest.fixture(scope="module")
def lib():
    import __graft_entry__

    __graft_entry__.build_cuda()
    import paper_conf_icppw_zhangczsdhay23_b200 as pkg

    return pkg


def declared_functions():
    txt = open(HDR).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(sssp_[a-z_0-9]+)\s*\(", txt)))


def test_header_declares_the_boundary():
    names = declared_functions()
    for n in ("sssp_graph_create", "sssp_reorder", "sssp_run", "sssp_distances", "sssp_destroy"):
        assert n in names


def test_exports_every_declared_symbol(lib):
    out = subprocess.check_output(["nm", "-D", "--defined-only", lib.LIB_PATH]).decode()
    exported = set(re.findall(r"\bT (sssp_\w+)", out))
    missing = set(declared_functions()) - exported
    assert not missing, missing
    assert set(lib.EXPORTS) == set(declared_functions())


def test_library_is_sm100a(lib):
    out = subprocess.check_output(["cuobjdump", "--list-elf", lib.LIB_PATH]).decode()
    assert "sm_100a" in out


def test_status_strings(lib):
    f = lib._lib.sssp_status_string
    assert f(0) == b"SSSP_OK"
    assert f(1) == b"SSSP_ERR_INVALID_ARGUMENT"
    assert f(5) == b"SSSP_ERR_OVERFLOW"
    assert f(99) == b"SSSP_UNKNOWN_STATUS"


def test_null_handle_paths(lib):
    L = lib._lib
    L.sssp_destroy(None)  # NULL-safe
    assert L.sssp_run(None, 0, 1.0) == lib.SSSP_ERR_INVALID_ARGUMENT
    assert L.sssp_reorder(None) == lib.SSSP_ERR_INVALID_ARGUMENT
    assert L.sssp_distances(None, None, 0) == lib.SSSP_ERR_INVALID_ARGUMENT
    assert L.sssp_get_stats(None, None) == lib.SSSP_ERR_INVALID_ARGUMENT
    assert L.sssp_set_param(None, 0, 8) == lib.SSSP_ERR_INVALID_ARGUMENT
    assert b"null" in L.sssp_last_error()


def test_create_rejects_bad_sizes_without_device(lib):
    L = lib._lib
    h = ctypes.c_void_p()
    import numpy as np

    row = np.zeros(2, np.int64)
    assert L.sssp_graph_create(ctypes.byref(h), 0, 0, 0, row.ctypes.data, None, None, 0, 0, None) == 1
    assert L.sssp_graph_create(ctypes.byref(h), 0, 1, -1, row.ctypes.data, None, None, 0, 0, None) == 1
    assert L.sssp_graph_create(None, 0, 1, 0, row.ctypes.data, None, None, 0, 0, None) == 1
    assert L.sssp_graph_create(ctypes.byref(h), 0, 1, 0, row.ctypes.data, None, None, 7, 0, None) == 1


def test_no_oracle_in_product_path():
    """The product package never imports or links the oracle (test infrastructure)."""
    pkg = os.path.join(ROOT, "paper_conf_icppw_zhangczsdhay23_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                txt = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in txt and "from oracle" not in txt and "oracle.h" not in txt, f
    out = subprocess.check_output(["nm", "-D", os.path.join(pkg, "libsssp.so")]).decode()
    assert "oracle_" not in out


def test_binding_constants_match_header(lib):
    """Every SSSP_* enumerator of include/sssp.h has the same value in the binding."""
    txt = re.sub(r"/\*.*?\*/", "", open(HDR).read(), flags=re.S)
    consts = {k: int(v) for k, v in re.findall(r"\b(SSSP_[A-Z0-9_]+)\s*=\s*(\d+)", txt)}
    assert "SSSP_PARAM_LOCAL_CHASE" in consts
    for k, v in consts.items():
        if k.startswith("SSSP_PARAM_"):
            assert getattr(lib, k) == v, k
    for k, v in consts.items():
        if hasattr(lib, k):
            assert getattr(lib, k) == v, k

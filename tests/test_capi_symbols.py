"""CPU-side checks of the C ABI: the library loads without a GPU and exports
every entry point include/gs.h declares; host-side argument validation."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_symbols():
    src = open(os.path.join(ROOT, "include", "gs.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    names = set(re.findall(r"\b(gs_[a-z_]+)\s*\(", src))
    return sorted(n for n in names if not n.endswith("_fn"))


@pytest.fixture(scope="module")
def lib():
    import __graft_entry__
    __graft_entry__.build()
    from paper_conf_sosp_gonglmc0lwl23_b200 import gs
    return gs.load_library()


def test_all_declared_symbols_exported(lib):
    from paper_conf_sosp_gonglmc0lwl23_b200 import gs
    decl = declared_symbols()
    assert len(decl) >= 15
    for name in decl:
        assert hasattr(lib, name), f"{name} declared in gs.h but not exported"
    assert sorted(gs.EXPORTS) == decl


def test_status_strings_and_version(lib):
    assert lib.gs_status_string(0) == b"GS_OK"
    assert lib.gs_status_string(7) == b"GS_ERR_CAPACITY"
    assert lib.gs_version() >= 100


def test_host_validation_without_gpu(lib):
    # invalid arguments are rejected on the host before any CUDA call
    out = ctypes.c_void_p()
    st = lib.gs_graph_create(None, None, None, 10, 5, 0, None, ctypes.byref(out))
    assert st == 1
    assert b"null" in lib.gs_last_error()
    fan = (ctypes.c_int * 2)(5, 0)
    st = lib.gs_sample_neighbors(None, None, 0, 1, 0, fan, 2, 0, 0, ctypes.c_uint64(0), None,
                                 ctypes.byref(out))
    assert st == 1
    st = lib.gs_random_walk(None, None, 0, 0, 3, ctypes.c_float(1), ctypes.c_float(1),
                            ctypes.c_uint64(0), 0, None, None)
    assert st == 1


def test_sources_have_no_oracle_dependency():
    """The product path shares no code with oracle/ (no include, import or link)."""
    pkg = os.path.join(ROOT, "paper_conf_sosp_gonglmc0lwl23_b200")
    banned = ["import oracle", "from oracle", "gso.h", "liboracle", "gso_"]
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                txt = open(os.path.join(dirpath, f)).read()
                for b in banned:
                    assert b not in txt, f"{f} references the oracle ({b})"


def test_host_validation_new_entry_points(lib):
    """GraphSAINT-RW, PinSAGE-style and the Table-4 operators reject bad
    arguments on the host (no CUDA call)."""
    out = ctypes.c_void_p()
    assert lib.gs_sample_saint_rw(None, None, 0, 1, 0, 2, ctypes.c_uint64(0), None,
                                  ctypes.byref(out)) == 1
    k = (ctypes.c_int * 2)(5, 5)
    assert lib.gs_sample_pinsage(None, None, 0, 1, 0, k, 2, 10, 3, ctypes.c_float(0.5),
                                 ctypes.c_uint64(0), None, ctypes.byref(out)) == 1
    assert lib.gs_matrix_slice_columns(None, None, 0, None, ctypes.byref(out)) == 1
    assert lib.gs_matrix_slice_rows(None, None, 0, None, ctypes.byref(out)) == 1
    assert lib.gs_matrix_sum(None, 0, None, None) == 1
    assert lib.gs_matrix_broadcast(None, 0, None, 0, None) == 1
    assert lib.gs_matrix_elementwise(None, 9, ctypes.c_float(1.0), None) == 1
    n = ctypes.c_int64()
    assert lib.gs_matrix_row_ids(None, None, ctypes.byref(n), None) == 1
    assert b"null" in lib.gs_last_error()

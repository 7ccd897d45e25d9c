"""The C ABI as a plain C99 consumer sees it (gs.h must compile
without any CUDA header).  CPU: gcc -std=c99 -pedantic -Wall -Werror compiles
and links tests/c/gs_c_client.c against libgsb200.so.  GPU: the client runs
gs_graph_create(HOST_PTRS) + gs_sample_neighbors and its block matches the
oracle."""
import os
import subprocess

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_sosp_gonglmc0lwl23_b200")


def _compile(tmp_path):
    import __graft_entry__
    __graft_entry__.build()
    exe = str(tmp_path / "gs_c_client")
    cmd = ["gcc", "-std=c99", "-pedantic", "-Wall", "-Wextra", "-Werror",
           "-I", os.path.join(ROOT, "include"), os.path.join(ROOT, "tests", "c", "gs_c_client.c"),
           "-L", PKG, "-lgsb200", f"-Wl,-rpath,{PKG}", "-L/usr/local/cuda/lib64", "-lcudart",
           "-Wl,-rpath,/usr/local/cuda/lib64", "-o", exe]
    subprocess.check_call(cmd)
    return exe


def test_header_compiles_as_c99(tmp_path):
    exe = _compile(tmp_path)
    assert os.path.exists(exe)
    # the header alone, as C89-compatible C99 with every warning an error
    src = tmp_path / "only_header.c"
    src.write_text('#include "gs.h"\nint main(void) { return gs_version() > 0 ? 0 : 1; }\n')
    subprocess.check_call(["gcc", "-std=c99", "-pedantic", "-Wall", "-Werror", "-fsyntax-only",
                           "-I", os.path.join(ROOT, "include"), str(src)])


@pytest.mark.gpu
def test_c_client_matches_oracle(tmp_path, oracle_lib):
    exe = _compile(tmp_path)
    out = subprocess.run([exe], capture_output=True, text=True, timeout=120)
    assert out.returncode == 0, out.stderr
    lines = out.stdout.strip().split("\n")
    T, R, E = (int(x) for x in lines[0].split())
    eid = np.array([int(x) for x in lines[1].split()], dtype=np.int64)
    rows = np.array([int(x) for x in lines[2].split()], dtype=np.int32) if R else np.zeros(0, np.int32)
    indptr = np.array([0, 3, 6, 8, 9, 12, 14], dtype=np.int64)
    indices = np.array([1, 2, 4, 0, 3, 5, 0, 1, 2, 0, 1, 3, 2, 4], dtype=np.int32)
    O = oracle_lib.Graph(indptr, indices, None)
    ref = oracle_lib.sample_neighbors(O, np.array([0, 1, 4], np.int32), [2, 2], batch_size=3,
                                      rng_key=42)
    blk = ref[0][0]
    assert (T, R, E) == (3, len(blk["row_map"]), len(blk["eid"]))
    assert np.array_equal(eid, blk["eid"])
    assert np.array_equal(rows, blk["row_map"])

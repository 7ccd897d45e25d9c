"""Builds libgsb200.so (sm_100a) in-tree with nvcc.

Flags: -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -fmad=false
(no FMA contraction on the parity-relevant fp32/fp64 paths, R19).
"""
from __future__ import annotations

import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
ROOT = os.path.dirname(HERE)
LIB = os.path.join(HERE, "libgsb200.so")
SOURCES = ["capi.cu", "nodewise_wave.cu", "nodewise_hop.cu", "shadow.cu", "layerwise.cu", "layerwise_sm.cu", "layerwise_bm.cu", "walk.cu", "pack.cu", "pinsage.cu", "ops.cu", "pass_att.cu"]
HEADERS = ["common.cuh", "gs_internal.h", "nodewise_common.cuh"]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
# -cudart shared: the static runtime would embed the name table of every
# runtime entry point (including batched-copy APIs this pool forbids) in the .so
FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-fmad=false",
         "-cudart", "shared",
         "-std=c++17", "-Xcompiler", "-fPIC", "-I", os.path.join(ROOT, "include")]


def _stale(target, deps):
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False) -> str:
    deps_common = [os.path.join(CSRC, h) for h in HEADERS] + [os.path.join(ROOT, "include", "gs.h")]
    objs = []
    objdir = os.path.join(CSRC, "build")
    os.makedirs(objdir, exist_ok=True)
    for src in SOURCES:
        s = os.path.join(CSRC, src)
        o = os.path.join(objdir, src.replace(".cu", ".o"))
        if force or _stale(o, [s] + deps_common):
            cmd = [NVCC] + FLAGS + (["-Xptxas", "-v"] if verbose else []) + ["-c", s, "-o", o]
            if verbose:
                print(" ".join(cmd), file=sys.stderr)
            subprocess.check_call(cmd)
        objs.append(o)
    if force or _stale(LIB, objs):
        tmp = LIB + ".tmp"
        subprocess.check_call([NVCC, "-shared", "-gencode", "arch=compute_100a,code=sm_100a",
                               "-cudart", "shared", "-o", tmp] + objs +
                              ["-lcublas", "-Xlinker", "-rpath=/usr/local/cuda/lib64"])
        os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))

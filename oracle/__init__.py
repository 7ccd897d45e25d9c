"""CPU oracle for the gSampler ECSF hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package.  The
product package (``paper_conf_sosp_gonglmc0lwl23_b200``) never imports it and
shares no code with it (see gso.h / gso.cpp for the algorithm and citations).

This module only marshals arguments to/from ``liboracle_gso.so`` (ctypes).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle_gso.so")
_SRC = [os.path.join(_HERE, "gso.cpp")]
_HDR = os.path.join(_HERE, "gso.h")

UNIFORM, EDGE, PASS_COLNORM = 0, 1, 2
LADIES, DEGREE, COUNT = 0, 1, 2


def build(force: bool = False) -> str:
    """Compile the oracle with -ffp-contract=off (no FMA contraction, R19)."""
    newest = max(os.path.getmtime(p) for p in _SRC + [_HDR])
    if not force and os.path.exists(_SO) and os.path.getmtime(_SO) >= newest:
        return _SO
    cmd = ["g++", "-O2", "-std=c++17", "-ffp-contract=off", "-fno-fast-math", "-fopenmp",
           "-shared", "-fPIC", "-o", _SO + ".tmp"] + _SRC
    subprocess.check_call(cmd)
    os.replace(_SO + ".tmp", _SO)
    return _SO


class _Graph(ctypes.Structure):
    _fields_ = [("num_nodes", ctypes.c_int64), ("num_edges", ctypes.c_int64),
                ("indptr", ctypes.c_void_p), ("indices", ctypes.c_void_p),
                ("weights", ctypes.c_void_p)]


class _View(ctypes.Structure):
    _fields_ = [("n_cols", ctypes.c_int64), ("n_rows", ctypes.c_int64),
                ("n_edges", ctypes.c_int64),
                ("col_map", ctypes.c_void_p), ("row_map", ctypes.c_void_p),
                ("indptr", ctypes.c_void_p), ("row_local", ctypes.c_void_p),
                ("eid", ctypes.c_void_p), ("val", ctypes.c_void_p),
                ("row_prob", ctypes.c_void_p)]


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_SO)
        vp, i64, i32, u64 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int, ctypes.c_uint64
        L.gso_philox4x32_10.argtypes = [vp, vp, vp]
        L.gso_uniform_below.argtypes = [u64, ctypes.c_uint32, ctypes.c_uint32]
        L.gso_uniform_below.restype = u64
        L.gso_ares_key.argtypes = [ctypes.c_uint32, ctypes.c_double]
        L.gso_ares_key.restype = ctypes.c_double
        L.gso_sample_neighbors.argtypes = [vp, vp, i64, i64, i64, vp, i32, i32, i32, u64, i32,
                                           ctypes.POINTER(vp)]
        L.gso_sample_layerwise.argtypes = [vp, vp, i64, i64, i64, vp, i32, i32, u64, i32,
                                           ctypes.POINTER(vp)]
        L.gso_shadow.argtypes = [vp, vp, i64, i64, i64, vp, i32, i32, u64, i32,
                                 ctypes.POINTER(vp)]
        L.gso_saint_rw.argtypes = [vp, vp, i64, i64, i64, i32, u64, i32, ctypes.POINTER(vp)]
        L.gso_pinsage.argtypes = [vp, vp, i64, i64, i64, vp, i32, i32, i32, ctypes.c_float, u64,
                                  i32, ctypes.POINTER(vp)]
        L.gso_random_walk.argtypes = [vp, vp, i64, i64, i32, ctypes.c_float, ctypes.c_float,
                                      u64, i32, i32, vp]
        L.gso_result_num_batches.argtypes = [vp]
        L.gso_result_num_batches.restype = i64
        L.gso_result_num_layers.argtypes = [vp]
        L.gso_result_view.argtypes = [vp, i64, i32, ctypes.POINTER(_View)]
        L.gso_result_free.argtypes = [vp]
        _lib = L
    return _lib


class OracleError(RuntimeError):
    def __init__(self, code, where):
        super().__init__(f"{where} failed with status {code}")
        self.code = code


class Graph:
    """Host CSC graph handed to the oracle (keeps the numpy arrays alive)."""

    def __init__(self, indptr, indices, weights=None):
        self.indptr = np.ascontiguousarray(indptr, dtype=np.int64)
        self.indices = np.ascontiguousarray(indices, dtype=np.int32)
        self.weights = None if weights is None else np.ascontiguousarray(weights, dtype=np.float32)
        self.num_nodes = len(self.indptr) - 1
        self.num_edges = len(self.indices)
        self._c = _Graph(self.num_nodes, self.num_edges, self.indptr.ctypes.data,
                         self.indices.ctypes.data,
                         None if self.weights is None else self.weights.ctypes.data)

    @property
    def ptr(self):
        return ctypes.addressof(self._c)


def philox4x32_10(ctr, key):
    c = np.asarray(ctr, dtype=np.uint32)
    k = np.asarray(key, dtype=np.uint32)
    out = np.zeros(4, dtype=np.uint32)
    lib().gso_philox4x32_10(c.ctypes.data, k.ctypes.data, out.ctypes.data)
    return [int(x) for x in out]


def uniform_below(n, r0, r1):
    return int(lib().gso_uniform_below(n, r0, r1))


def ares_key(r, bias):
    return float(lib().gso_ares_key(r, bias))


def _arr(ptr, n, dtype):
    if n == 0 or not ptr:
        return np.zeros(0, dtype=dtype)
    ct = {np.int32: ctypes.c_int32, np.int64: ctypes.c_int64, np.float32: ctypes.c_float}[dtype]
    buf = (ct * n).from_address(ptr)
    return np.ctypeslib.as_array(buf).copy()


def _collect(res):
    L = lib()
    nb = L.gso_result_num_batches(res)
    nl = L.gso_result_num_layers(res)
    out = []
    v = _View()
    for b in range(nb):
        layers = []
        for l in range(nl):
            st = L.gso_result_view(res, b, l, ctypes.byref(v))
            if st:
                raise OracleError(st, "gso_result_view")
            layers.append({
                "col_map": _arr(v.col_map, v.n_cols, np.int32),
                "row_map": _arr(v.row_map, v.n_rows, np.int32),
                "indptr": _arr(v.indptr, v.n_cols + 1, np.int64),
                "row_local": _arr(v.row_local, v.n_edges, np.int32),
                "eid": _arr(v.eid, v.n_edges, np.int64),
                "val": None if not v.val else _arr(v.val, v.n_edges, np.float32),
                "row_prob": None if not v.row_prob else _arr(v.row_prob, v.n_rows, np.float32),
            })
        out.append(layers)
    L.gso_result_free(res)
    return out


def _seeds(seeds):
    return np.ascontiguousarray(seeds, dtype=np.int32)


def sample_neighbors(g: Graph, seeds, fanouts, batch_size=None, batch_index_base=0,
                     replace=False, bias_mode=UNIFORM, rng_key=0, num_threads=0):
    """Returns blocks[batch][layer] -> dict of numpy arrays."""
    s = _seeds(seeds)
    f = np.ascontiguousarray(fanouts, dtype=np.int32)
    bs = batch_size or max(1, len(s))
    res = ctypes.c_void_p()
    st = lib().gso_sample_neighbors(g.ptr, s.ctypes.data, len(s), bs, batch_index_base,
                                    f.ctypes.data, len(f), int(replace), bias_mode, rng_key,
                                    num_threads, ctypes.byref(res))
    if st:
        raise OracleError(st, "gso_sample_neighbors")
    return _collect(res)


def sample_layerwise(g: Graph, seeds, n_per_layer, batch_size=None, batch_index_base=0,
                     prob_mode=LADIES, rng_key=0, num_threads=0):
    s = _seeds(seeds)
    f = np.ascontiguousarray(n_per_layer, dtype=np.int32)
    bs = batch_size or max(1, len(s))
    res = ctypes.c_void_p()
    st = lib().gso_sample_layerwise(g.ptr, s.ctypes.data, len(s), bs, batch_index_base,
                                    f.ctypes.data, len(f), prob_mode, rng_key, num_threads,
                                    ctypes.byref(res))
    if st:
        raise OracleError(st, "gso_sample_layerwise")
    return _collect(res)


def shadow(g: Graph, seeds, fanouts, batch_size=None, batch_index_base=0, bias_mode=UNIFORM,
           rng_key=0, num_threads=0):
    s = _seeds(seeds)
    f = np.ascontiguousarray(fanouts, dtype=np.int32)
    bs = batch_size or max(1, len(s))
    res = ctypes.c_void_p()
    st = lib().gso_shadow(g.ptr, s.ctypes.data, len(s), bs, batch_index_base, f.ctypes.data,
                          len(f), bias_mode, rng_key, num_threads, ctypes.byref(res))
    if st:
        raise OracleError(st, "gso_shadow")
    return [blocks[0] for blocks in _collect(res)]


def saint_rw(g: Graph, roots, walk_length, batch_size=None, batch_index_base=0, rng_key=0,
             num_threads=0):
    """GraphSAINT-RW (Table 2; DESIGN R26): DeepWalk walks from the roots,
    then per batch the subgraph induced on the visited nodes (one block per batch)."""
    s = _seeds(roots)
    bs = batch_size or max(1, len(s))
    res = ctypes.c_void_p()
    st = lib().gso_saint_rw(g.ptr, s.ctypes.data, len(s), bs, batch_index_base, walk_length,
                            rng_key, num_threads, ctypes.byref(res))
    if st:
        raise OracleError(st, "gso_saint_rw")
    return [blocks[0] for blocks in _collect(res)]


def pinsage(g: Graph, seeds, topk, num_walks, walk_length, restart_prob, batch_size=None,
            batch_index_base=0, rng_key=0, num_threads=0):
    """PinSAGE-style sampling (Table 2; DESIGN R27): restart walks from every
    frontier, its topk[l] most visited nodes as neighbours (val = visit count)."""
    s = _seeds(seeds)
    f = np.ascontiguousarray(topk, dtype=np.int32)
    bs = batch_size or max(1, len(s))
    res = ctypes.c_void_p()
    st = lib().gso_pinsage(g.ptr, s.ctypes.data, len(s), bs, batch_index_base, f.ctypes.data,
                           len(f), num_walks, walk_length, restart_prob, rng_key, num_threads,
                           ctypes.byref(res))
    if st:
        raise OracleError(st, "gso_pinsage")
    return _collect(res)


def random_walk(g: Graph, starts, length, p=1.0, q=1.0, walker_index_base=0, rng_key=0,
                force_node2vec=False, num_threads=0):
    s = _seeds(starts)
    traces = np.empty((len(s), length + 1), dtype=np.int32)
    st = lib().gso_random_walk(g.ptr, s.ctypes.data, len(s), walker_index_base, length, p, q,
                               rng_key, int(force_node2vec), num_threads, traces.ctypes.data)
    if st:
        raise OracleError(st, "gso_random_walk")
    return traces

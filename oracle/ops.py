"""CPU ORACLE for the matrix-centric operators of Table 4.

TEST INFRASTRUCTURE ONLY: only tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / --impl reference legs may import this module; the product path
(paper_conf_sosp_gonglmc0lwl23_b200/, include/gs.h) never does, and the two
share no code.

Every operator here is a plain definition, written with numpy
in the order the paper states it; sums accumulate in fp64 and round once to
fp32 (R19).  A sub-matrix is a dict over GLOBAL ids:
  cols   int32[n_cols]   the column (frontier) node of each local column
  indptr int64[n_cols+1] CSC over the local columns
  row    int32[nnz]      global row id of each entry
  eid    int64[nnz]      position of the entry in the graph's indices
  val    float32[nnz]    the entry's value (the edge weight; 1 if unweighted)
Entries of a column keep the graph's CSC order (ascending position).
"""
from __future__ import annotations

import numpy as np

# element-wise / broadcast operators (Table 4: add, sub, mul, div, **)
ADD, SUB, MUL, DIV, POW = 0, 1, 2, 3, 4


def slice_columns(indptr, indices, weights, cols):
    """A[:, columns] (Table 4 Extract): the columns' entries, in order."""
    cols = np.asarray(cols, dtype=np.int32)
    ip = [0]
    row, eid, val = [], [], []
    for v in cols.tolist():
        for e in range(int(indptr[v]), int(indptr[v + 1])):
            row.append(int(indices[e]))
            eid.append(e)
            val.append(1.0 if weights is None else float(weights[e]))
        ip.append(len(eid))
    return {"cols": cols, "indptr": np.array(ip, np.int64), "row": np.array(row, np.int32),
            "eid": np.array(eid, np.int64), "val": np.array(val, np.float32)}


def slice_rows(m, rows):
    """A[rows, :] (Table 4 Extract): the entries whose row is in `rows`."""
    keep_set = set(np.asarray(rows, dtype=np.int64).tolist())
    ip = [0]
    keep = []
    for c in range(len(m["cols"])):
        for i in range(int(m["indptr"][c]), int(m["indptr"][c + 1])):
            if int(m["row"][i]) in keep_set:
                keep.append(i)
        ip.append(len(keep))
    keep = np.array(keep, np.int64)
    return {"cols": m["cols"].copy(), "indptr": np.array(ip, np.int64),
            "row": m["row"][keep] if len(keep) else np.zeros(0, np.int32),
            "eid": m["eid"][keep] if len(keep) else np.zeros(0, np.int64),
            "val": m["val"][keep] if len(keep) else np.zeros(0, np.float32)}


def col_sum(m):
    """A.sum(axis=0) (Table 4 Compute; R1: per column): fp32(sum_fp64)."""
    out = np.zeros(len(m["cols"]), np.float32)
    for c in range(len(m["cols"])):
        s = 0.0
        for i in range(int(m["indptr"][c]), int(m["indptr"][c + 1])):
            s += float(m["val"][i])
        out[c] = np.float32(s)
    return out


def row_sum(m, num_nodes):
    """A.sum(axis=1) (Table 4 Compute; R1: per row, keyed by global row id,
    the LADIES bias of Fig. 2): dense float32[num_nodes]."""
    acc = np.zeros(num_nodes, np.float64)
    for i in range(len(m["row"])):
        acc[int(m["row"][i])] += float(m["val"][i])
    return acc.astype(np.float32)


def _apply(op, a, b):
    a = np.float32(a)
    b = np.float32(b)
    if op == ADD:
        return np.float32(a + b)
    if op == SUB:
        return np.float32(a - b)
    if op == MUL:
        return np.float32(a * b)
    if op == DIV:
        return np.float32(a / b)
    if op == POW:
        return np.float32(np.power(np.float64(a), np.float64(b)))  # fp64 pow, rounded once
    raise ValueError(op)


def broadcast(m, op, V, axis):
    """A.<op>(V, axis) (Table 4 Compute): axis 0 -> V is indexed by the
    local column (one value per frontier), axis 1 -> by the global row id."""
    out = dict(m)
    val = m["val"].copy()
    with np.errstate(divide="ignore", invalid="ignore", over="ignore"):
        for c in range(len(m["cols"])):
            for i in range(int(m["indptr"][c]), int(m["indptr"][c + 1])):
                x = V[c] if axis == 0 else V[int(m["row"][i])]
                val[i] = _apply(op, val[i], x)
    out["val"] = val
    return out


def elementwise(m, op, scalar):
    """A <op> v (Table 4 Compute): every entry with a number."""
    out = dict(m)
    with np.errstate(divide="ignore", invalid="ignore", over="ignore"):
        out["val"] = np.array([_apply(op, x, scalar) for x in m["val"].tolist()], np.float32)
    return out


def row_ids(m):
    """A.row() (Table 4 Finalize; R3): the distinct row ids, ascending."""
    return np.array(sorted(set(m["row"].tolist())), np.int32)

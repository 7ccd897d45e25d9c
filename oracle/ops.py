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


# ---------------------------------------------------------------------------
# Select operators (Table 4 Select) and the fused chains /
# learned bias of SURVEY 8(f) f3.  Randomness: the samplers' Philox keying
# (R4): column node v and the entry's position p inside the sub-matrix column
# for individual_sample, the row node u for collective_sample, with the
# caller's layer and global batch index.
# ---------------------------------------------------------------------------
def _philox(c0, c1, c2, c3, key):
    from oracle import philox4x32_10
    return philox4x32_10([c0 & 0xFFFFFFFF, c1 & 0xFFFFFFFF, c2 & 0xFFFFFFFF, c3 & 0xFFFFFFFF],
                         [key & 0xFFFFFFFF, (key >> 32) & 0xFFFFFFFF])


def _draw_below(n, r0, r1):
    return ((r1 << 32 | r0) * n) >> 64      # floor(r n / 2^64), R23


def _ares_key(r, bias):
    import math
    return -math.log((r + 0.5) * 2.0 ** -32) / float(bias)    # R6, fp64


def _submatrix(m, keep):
    keep = np.asarray(keep, np.int64)
    ip = [0]
    ks = set(keep.tolist())
    out_idx = []
    for c in range(len(m["cols"])):
        for i in range(int(m["indptr"][c]), int(m["indptr"][c + 1])):
            if i in ks:
                out_idx.append(i)
        ip.append(len(out_idx))
    idx = np.array(out_idx, np.int64)
    return {"cols": m["cols"].copy(), "indptr": np.array(ip, np.int64),
            "row": m["row"][idx] if len(idx) else np.zeros(0, np.int32),
            "eid": m["eid"][idx] if len(idx) else np.zeros(0, np.int64),
            "val": m["val"][idx] if len(idx) else np.zeros(0, np.float32)}


def individual_sample(m, K, rng_key, layer=0, batch=0, use_values=False, replace=False):
    """A.individual_sample(K, probs) (Table 4 Select): every
    column (frontier) samples K of its entries independently.  probs omitted
    (use_values False): uniform -- without replacement Robert Floyd's
    algorithm (R5), the column's d <= K entries all kept; with replacement K
    i.i.d. draws in slot order (R10).  probs = the matrix's values (use_values):
    A-Res without replacement on them (R6: value <= 0 ineligible, every
    eligible one when at most K, else the K smallest keys, ties -> smaller
    position).  Kept entries in ascending position (slot order with
    replacement); returns the sub-matrix (duplicated entries with replacement)."""
    out = {"cols": m["cols"].copy(), "indptr": [0], "row": [], "eid": [], "val": []}
    for c in range(len(m["cols"])):
        v = int(m["cols"][c])
        lo, hi = int(m["indptr"][c]), int(m["indptr"][c + 1])
        d = hi - lo
        if replace:
            pos = []
            if d > 0:
                for s in range(K):
                    r = _philox(v, s, layer | (2 << 24), batch, rng_key)
                    pos.append(_draw_below(d, r[0], r[1]))
        elif not use_values:
            if d <= K:
                pos = list(range(d))
            else:
                S = set()
                for s in range(K):
                    r = _philox(v, s, layer | (1 << 24), batch, rng_key)
                    mm = d - K + s
                    t = _draw_below(mm + 1, r[0], r[1])
                    S.add(mm if t in S else t)
                pos = sorted(S)
        else:
            elig = [p for p in range(d) if m["val"][lo + p] > 0]
            if len(elig) <= K:
                pos = elig
            else:
                keys = []
                for p in elig:
                    r = _philox(v, p >> 2, layer | (3 << 24), batch, rng_key)[p & 3]
                    keys.append((_ares_key(r, np.float64(m["val"][lo + p])), p))
                pos = sorted(p for _, p in sorted(keys)[:K])
        for p in pos:
            out["row"].append(int(m["row"][lo + p]))
            out["eid"].append(int(m["eid"][lo + p]))
            out["val"].append(float(m["val"][lo + p]))
        out["indptr"].append(len(out["eid"]))
    return {"cols": out["cols"], "indptr": np.array(out["indptr"], np.int64),
            "row": np.array(out["row"], np.int32), "eid": np.array(out["eid"], np.int64),
            "val": np.array(out["val"], np.float32)}


def collective_sample(m, K, rng_key, layer=0, batch=0, node_probs=None):
    """A.collective_sample(K, node_probs) (Table 4 Select):
    sample K of the matrix's row nodes C (the distinct rows) by the bias
    b(u) = node_probs[u] (a dense per-node vector, used unnormalised), or,
    node_probs omitted, b(u) = fp32(number of entries of u) ("the sampling bias
    on each edge is 1 and automatically aggregates"): b <= 0
    ineligible; every eligible row when at most K (R24), else the K smallest
    A-Res keys E/b(u) (R6, word 0 of philox(u, 0, layer | 4<<24, batch); ties ->
    smaller u).  Returns (the sub-matrix of the entries whose row was selected,
    in CSC order; S ascending)."""
    C = row_ids(m)
    if node_probs is None:
        cnt = {}
        for u in m["row"].tolist():
            cnt[u] = cnt.get(u, 0) + 1
        b = {int(u): np.float32(cnt[int(u)]) for u in C}
    else:
        b = {int(u): np.float32(node_probs[int(u)]) for u in C}
    elig = [u for u in C.tolist() if b[u] > 0]
    if len(elig) <= K:
        S = sorted(elig)
    else:
        keys = []
        for u in elig:
            r = _philox(u, 0, layer | (4 << 24), batch, rng_key)[0]
            keys.append((_ares_key(r, np.float64(b[u])), u))
        S = sorted(u for _, u in sorted(keys)[:K])
    Sset = set(S)
    keep = [i for i in range(len(m["row"])) if int(m["row"][i]) in Sset]
    return _submatrix(m, keep), np.array(S, np.int32)


def map_reduce(m, ops, scalars, axis, num_nodes=None):
    """An Edge-Map chain fused with an Edge-Reduce: the entry
    values after the element-wise operators (ops[i], scalars[i]) applied in
    order -- exactly elementwise(...elementwise(m, ops[0], scalars[0])...) --
    then summed over `axis` (0: per column, 1: per global row; fp64, one fp32
    rounding, R19).  axis None: the mapped matrix itself (Edge-Map fusion)."""
    x = m
    for op, s in zip(ops, scalars):
        x = elementwise(x, op, s)
    if axis is None:
        return x
    return col_sum(x) if axis == 0 else row_sum(x, num_nodes)


def asgcn_bias(m, X, wg, num_nodes):
    """AS-GCN-style learned layer-wise bias (Table 2: "sampling bias ...
    computed using trainable model"; R30): per row node u of the
    extracted matrix, b(u) = fp32(s(u) * g(u)) with s = A.sum(axis=1) (fp64,
    rounded once: the frontiers' aggregated edge values) and the learned
    self-dependent score g(u) = relu(fp32(sum_fp64_f X[u, f] wg[f])) (X: node
    features, wg: the trainable projection, seeded synthetic).  Dense
    float32[num_nodes] (0 off the rows of m): the node_probs of
    collective_sample."""
    s = row_sum(m, num_nodes)
    X = np.asarray(X, np.float64)
    wg = np.asarray(wg, np.float32).astype(np.float64)
    out = np.zeros(num_nodes, np.float32)
    for u in row_ids(m).tolist():
        g = np.float32(float(np.sum(X[u] * wg)))
        g = g if g > 0 else np.float32(0.0)
        out[u] = np.float32(np.float32(s[u]) * g)
    return out


# ---------------------------------------------------------------------------
# Heterogeneous graphs ("each type of edges is modeled as a sparse
# matrix to conduct the same sampling workflow as homogeneous graphs"; SURVEY
# 8(f) f4).  Relation r is its own CSC matrix whose columns are nodes of type
# dst[r] and whose rows are nodes of type src[r] (ids local to each type).
# Layer l: every relation r samples fanouts[l][r] entries of each frontier
# column of type dst[r] (A_r[:, F_dst].individual_sample, uniform without
# replacement, R5) with the relation's key (R33); the next frontier of type t
# is the union of the rows of the relations whose src is t, ascending (A.row()
# of each, merged).
# ---------------------------------------------------------------------------
def relation_key(rng_key, r):
    """R33: the RNG key of relation r -- rng_key XOR (r + 1) times the 64-bit
    golden ratio, so relations never share a Philox stream."""
    return (int(rng_key) ^ ((0x9E3779B97F4A7C15 * (r + 1)) & 0xFFFFFFFFFFFFFFFF)) & 0xFFFFFFFFFFFFFFFF


def hetero_sample_neighbors(rels, num_nodes, seeds, fanouts, rng_key):
    """rels[r] = (src_type, dst_type, indptr, indices); num_nodes[t]; seeds[t]
    (int32 array, possibly empty); fanouts[l][r] (0: relation skipped at l).
    Returns (blocks, frontiers): blocks[l][r] the sampled sub-matrix (or None),
    frontiers[l][t] for l = 0 .. L (frontiers[0] = the seeds)."""
    T = len(num_nodes)
    frontiers = [[np.asarray(seeds[t], np.int32) for t in range(T)]]
    blocks = []
    for l, fl in enumerate(fanouts):
        bl = []
        for r, (st, dt, ip, ix) in enumerate(rels):
            F = frontiers[l][dt]
            if fl[r] == 0 or len(F) == 0:
                bl.append(None)
                continue
            m = slice_columns(ip, ix, None, F)
            bl.append(individual_sample(m, fl[r], relation_key(rng_key, r), layer=l, batch=0))
        blocks.append(bl)
        nxt = []
        for t in range(T):
            rows = set()
            for r, (st, dt, ip, ix) in enumerate(rels):
                if st == t and bl[r] is not None:
                    rows |= set(row_ids(bl[r]).tolist())
            nxt.append(np.array(sorted(rows), np.int32))
        frontiers.append(nxt)
    return blocks, frontiers

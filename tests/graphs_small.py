"""Hand-built tiny graphs used by the oracle pins and the GPU parity tests."""
import numpy as np


def csc_from_columns(n, columns, weighted=True):
    """columns: {v: [(u, w), ...]} -> (indptr, indices, weights) with sorted rows."""
    indptr = [0]
    indices, weights = [], []
    for v in range(n):
        col = sorted(columns.get(v, []))
        indices += [u for u, _ in col]
        weights += [w for _, w in col]
        indptr.append(len(indices))
    return (np.array(indptr, np.int64), np.array(indices, np.int32),
            np.array(weights, np.float32) if weighted else None)


# Figure 1 toy graph as narrated at P:105-117: frontier a; in-neighbours of a
# are {b, c, e}; in-neighbours of b and e together are {c, d, f, g, h}; the
# only weights the paper prints are w_fb = 0.7 and w_fe = 0.3 (B_f = 0.58,
# P:117); every other weight is chosen here.
A, B, C, D, E, F, G, H = range(8)
FIG1 = {
    A: [(B, 0.5), (C, 0.4), (E, 0.6)],
    B: [(C, 0.2), (D, 0.9), (F, 0.7)],
    E: [(F, 0.3), (G, 0.8), (H, 0.1)],
}


def fig1_graph():
    return csc_from_columns(8, FIG1)


def star_graph(d, weights=None):
    """Node 0 has in-neighbours 1..d (weights optional)."""
    w = weights if weights is not None else [1.0] * d
    return csc_from_columns(d + 1, {0: [(i + 1, float(w[i])) for i in range(d)]})

"""Pins for the oracle's random walks (DeepWalk P:75, Node2Vec P:82) and the
ShaDow induced subgraph.

Walk pins: the exact path law prod 1/deg(v) enumerated on a 5-node graph
(chi-square), dead-end padding, the Node2Vec second-order transition law
bias(prev, x) / sum bias = 1/9, 2/9, 2/9, 4/9 at p = 2, q = 0.5, and Node2Vec
at p = q = 1 realising the DeepWalk law.  ShaDow pin: brute-force induced edge
set {u -> v in E : u, v in U}.
"""
from collections import Counter

import numpy as np
import pytest

import synth
from tests._stats import chi_square_p
from tests.graphs_small import csc_from_columns

# in-neighbour lists; node 4 has no in-neighbours (dead end)
WALK5 = {0: [(1, 1.0), (2, 1.0)], 1: [(0, 1.0), (2, 1.0), (3, 1.0)], 2: [(0, 1.0), (4, 1.0)],
         3: [(1, 1.0)]}


def path_law(cols, start, length):
    law = {}

    def rec(path, p):
        if len(path) == length + 1:
            law[tuple(path)] = law.get(tuple(path), 0.0) + p
            return
        v = path[-1]
        nb = [u for u, _ in cols.get(v, [])] if v >= 0 else []
        if not nb:
            rec(path + [-1], p)
            return
        for u in nb:
            rec(path + [u], p / len(nb))

    rec([start], 1.0)
    return law


@pytest.mark.parametrize("force_n2v", [False, True])
def test_deepwalk_path_law(oracle_lib, force_n2v):
    ip, ix, _ = csc_from_columns(5, WALK5)
    og = oracle_lib.Graph(ip, ix)
    n = 60_000
    tr = oracle_lib.random_walk(og, np.zeros(n, np.int32), 3, rng_key=31,
                                force_node2vec=force_n2v)
    cnt = Counter(tuple(r) for r in tr.tolist())
    law = path_law(WALK5, 0, 3)
    assert chi_square_p(cnt, law, n) > 1e-3


def test_dead_end_padding(oracle_lib):
    ip, ix, _ = csc_from_columns(5, WALK5)
    og = oracle_lib.Graph(ip, ix)
    tr = oracle_lib.random_walk(og, np.array([4, 2, 3], np.int32), 5, p=2.0, q=0.5)
    assert tr[0].tolist() == [4, -1, -1, -1, -1, -1]
    for row in tr:
        seen_dead = False
        for x in row:
            seen_dead |= x == -1
            assert (x == -1) == seen_dead or not seen_dead
    tr0 = oracle_lib.random_walk(og, np.array([1], np.int32), 0)
    assert tr0.tolist() == [[1]]


def test_node2vec_second_order_law(oracle_lib):
    """prev = t, N(v) = {t, x1, x2, y}, x1, x2 in N(t): 1/9, 2/9, 2/9, 4/9 (p=2, q=0.5)."""
    t, v, x1, x2, y = range(5)
    cols = {t: [(v, 1.0), (x1, 1.0), (x2, 1.0)], v: [(t, 1.0), (x1, 1.0), (x2, 1.0), (y, 1.0)],
            x1: [(t, 1.0)], x2: [(t, 1.0)], y: [(v, 1.0)]}
    ip, ix, _ = csc_from_columns(5, cols)
    og = oracle_lib.Graph(ip, ix)
    n = 150_000
    tr = oracle_lib.random_walk(og, np.full(n, t, np.int32), 2, p=2.0, q=0.5, rng_key=41)
    sel = tr[tr[:, 1] == v][:, 2]
    cnt = Counter(sel.tolist())
    law = {t: 1 / 9, x1: 2 / 9, x2: 2 / 9, y: 4 / 9}
    assert chi_square_p(cnt, law, len(sel)) > 1e-3
    # step 1 has no previous node: uniform over N(t)
    cnt1 = Counter(tr[:, 1].tolist())
    assert chi_square_p(cnt1, {v: 1 / 3, x1: 1 / 3, x2: 1 / 3}, n) > 1e-3


@pytest.fixture(scope="module")
def tiny(oracle_lib):
    g = synth.make_graph("tiny")
    return oracle_lib.Graph(g["indptr"].numpy(), g["indices"].numpy(), g["weights"].numpy())


@pytest.mark.parametrize("pq", [(1.0, 1.0), (2.0, 0.5)])
def test_walk_edges_exist(oracle_lib, tiny, pq):
    starts = synth.make_seeds("tiny", 2000).numpy()
    tr = oracle_lib.random_walk(tiny, starts, 20, p=pq[0], q=pq[1], rng_key=5)
    ip, ix = tiny.indptr, tiny.indices
    assert np.array_equal(tr[:, 0], starts)
    for row in tr[:300]:
        for a, b in zip(row[:-1], row[1:]):
            if b < 0:
                assert a < 0 or ip[a + 1] == ip[a]
            else:
                assert b in ix[ip[a]:ip[a + 1]]
    # walker_index_base keys the stream by global walker index
    part = oracle_lib.random_walk(tiny, starts[1000:], 20, p=pq[0], q=pq[1], rng_key=5,
                                  walker_index_base=1000)
    assert np.array_equal(part, tr[1000:])


@pytest.mark.parametrize("bias_mode", [0, 1])
def test_shadow_brute_force(oracle_lib, tiny, bias_mode):
    seeds = synth.make_seeds("tiny", 300).numpy()
    fan = [10, 5]
    ind = oracle_lib.shadow(tiny, seeds, fan, batch_size=100, bias_mode=bias_mode, rng_key=8)
    nw = oracle_lib.sample_neighbors(tiny, seeds, fan, batch_size=100, bias_mode=bias_mode,
                                     rng_key=8)
    ip, ix = tiny.indptr, tiny.indices
    for b, blk in enumerate(ind):
        # R12: U = unique of the seeds and every hop's rows, ascending
        U = sorted(set(np.concatenate([seeds[b * 100:(b + 1) * 100]] +
                                      [L["row_map"] for L in nw[b]]).tolist()))
        assert blk["row_map"].tolist() == U and blk["col_map"].tolist() == U
        Uset = set(U)
        want = sorted(e for v in U for e in range(ip[v], ip[v + 1]) if ix[e] in Uset)
        got = blk["eid"].tolist()
        assert sorted(got) == want and len(got) == len(want)
        # CSC over local ids: column c holds edges into U[c]
        for c, v in enumerate(U):
            lo, hi = blk["indptr"][c], blk["indptr"][c + 1]
            assert np.all((blk["eid"][lo:hi] >= ip[v]) & (blk["eid"][lo:hi] < ip[v + 1]))
        assert np.all(np.array(U)[blk["row_local"]] == ix[blk["eid"]])

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


# ---- GraphSAINT-RW (Table 2; DESIGN R26): walk, then induce on the visited nodes ----

def test_saint_rw_visited_set_law(oracle_lib):
    """One root per batch on the 5-node graph: U's law is the DeepWalk path law
    (prod 1/deg) pushed through path -> set of visited nodes; every block's edges
    are exactly {u -> v in E : u, v in U} read off the column lists."""
    ip, ix, _ = csc_from_columns(5, WALK5)
    og = oracle_lib.Graph(ip, ix)
    n = 20_000
    blocks = oracle_lib.saint_rw(og, np.zeros(n, np.int32), 3, batch_size=1, rng_key=77)
    assert len(blocks) == n
    law = Counter()
    for path, p in path_law(WALK5, 0, 3).items():
        law[tuple(sorted(set(x for x in path if x >= 0)))] += p
    cnt = Counter(tuple(b["row_map"].tolist()) for b in blocks)
    assert chi_square_p(cnt, dict(law), n) > 1e-3
    edges = {(u, v) for v, col in WALK5.items() for u, _ in col}
    for b in blocks[:500]:
        U = b["row_map"].tolist()
        assert b["col_map"].tolist() == U
        got = {(U[r], U[c]) for c in range(len(U))
               for r in b["row_local"][b["indptr"][c]:b["indptr"][c + 1]].tolist()}
        assert got == {(u, v) for (u, v) in edges if u in U and v in U}


def test_saint_rw_special_cases(oracle_lib):
    # walk_length 0: U = the batch's distinct roots; complete digraph K_6:
    # the induced block has |U| (|U| - 1) edges
    n = 6
    ip, ix, _ = csc_from_columns(n, {v: [(u, 1.0) for u in range(n) if u != v] for v in range(n)})
    og = oracle_lib.Graph(ip, ix)
    roots = np.array([4, 1, 4, 0, 5, 5], np.int32)
    blocks = oracle_lib.saint_rw(og, roots, 0, batch_size=3)
    assert [b["row_map"].tolist() for b in blocks] == [[1, 4], [0, 5]]
    assert [len(b["eid"]) for b in blocks] == [2, 2]
    # walks on K_6 never stop: U covers every visited node, edges |U|(|U|-1)
    blocks = oracle_lib.saint_rw(og, roots, 4, batch_size=2, rng_key=9)
    for b in blocks:
        k = len(b["row_map"])
        assert 1 <= k <= 2 * 5 and len(b["eid"]) == k * (k - 1)
    # a root with no in-neighbours: its walk stops at once (R13)
    ip, ix, _ = csc_from_columns(5, WALK5)
    blocks = oracle_lib.saint_rw(oracle_lib.Graph(ip, ix), np.array([4], np.int32), 5)
    assert blocks[0]["row_map"].tolist() == [4] and len(blocks[0]["eid"]) == 0


def test_saint_rw_brute_force_tiny(oracle_lib, tiny):
    roots = synth.make_seeds("tiny", 600).numpy()
    bs, L = 200, 4
    blocks = oracle_lib.saint_rw(tiny, roots, L, batch_size=bs, rng_key=12)
    tr = oracle_lib.random_walk(tiny, roots, L, rng_key=12)   # DeepWalk, global walker ids
    ip, ix = tiny.indptr, tiny.indices
    for b, blk in enumerate(blocks):
        t = tr[b * bs:(b + 1) * bs].ravel()
        U = sorted(set(t[t >= 0].tolist()))
        assert blk["row_map"].tolist() == U
        Uset = set(U)
        want = [e for v in U for e in range(ip[v], ip[v + 1]) if ix[e] in Uset]
        assert blk["eid"].tolist() == want   # CSC order: columns in U order, positions ascending
        assert np.all(np.array(U)[blk["row_local"]] == ix[blk["eid"]])
        assert np.all(np.diff(blk["indptr"]) >= 0) and blk["indptr"][-1] == len(want)
    # global batch index keying: batch 2 alone, based at 2, is the same block
    part = oracle_lib.saint_rw(tiny, roots[2 * bs:], L, batch_size=bs, batch_index_base=2,
                               rng_key=12)
    for k in ["row_map", "indptr", "row_local", "eid"]:
        assert np.array_equal(part[0][k], blocks[2][k])

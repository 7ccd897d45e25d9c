"""Pins for the oracle's PinSAGE-style sampler (Table 2; DESIGN R27):
restart walks from every frontier, the k most visited nodes as its neighbours.

  * directed cycle (one in-neighbour per node), restart 0: every walk visits
    v-1, v-2, ..., v-T, so the counts are closed form (num_walks each), the
    tie rule (id ascending) decides the top-k, and v itself is never counted;
  * restart_prob = 1: no step is ever taken (empty blocks, empty next layers);
  * first-step law: one walk of one step from the centre of a star picks each
    in-neighbour with probability 1/d (chi-square over many batches);
  * restart law: on a long cycle the number of steps of one walk is the
    truncated geometric law P(s) = (1-r)^s r (s < T), (1-r)^T (s = T);
  * on the tiny R-MAT graph: each selected node lies within T in-edge hops of
    v, counts <= num_walks * T, rank order, k bound, layer chaining, batch keying.
"""
from collections import Counter, deque

import numpy as np
import pytest

import synth
from tests._stats import chi_square_p
from tests.graphs_small import csc_from_columns, star_graph


def cycle(n):
    return csc_from_columns(n, {v: [((v - 1) % n, 1.0)] for v in range(n)})


def test_cycle_closed_form(oracle_lib):
    ip, ix, _ = cycle(10)
    og = oracle_lib.Graph(ip, ix)
    seeds = np.array([1, 5], np.int32)
    blk = oracle_lib.pinsage(og, seeds, [2], 5, 3, 0.0)[0][0]
    # v = 1 visits 0, 9, 8 five times each -> top-2 by id: 0, 8; v = 5 -> 2, 3
    assert blk["row_map"].tolist() == [0, 2, 3, 8]
    assert blk["indptr"].tolist() == [0, 2, 4]
    assert blk["row_map"][blk["row_local"]].tolist() == [0, 8, 2, 3]
    assert blk["val"].tolist() == [5.0] * 4 and blk["eid"].tolist() == [-1] * 4
    # a 3-cycle returns to v at step 3: v is never its own neighbour
    ip, ix, _ = cycle(3)
    blk = oracle_lib.pinsage(oracle_lib.Graph(ip, ix), np.array([0], np.int32), [3], 4, 3,
                             0.0)[0][0]
    assert blk["row_map"].tolist() == [1, 2] and blk["val"].tolist() == [4.0, 4.0]


def test_restart_one_takes_no_step(oracle_lib):
    ip, ix, _ = cycle(10)
    r = oracle_lib.pinsage(oracle_lib.Graph(ip, ix), np.arange(10, dtype=np.int32), [3, 3], 8, 4,
                           1.0, batch_size=4)
    for layers in r:
        assert all(len(b["eid"]) == 0 for b in layers)
        assert len(layers[1]["col_map"]) == 0


def test_first_step_law(oracle_lib):
    ip, ix, _ = star_graph(4)
    og = oracle_lib.Graph(ip, ix)
    n = 40_000
    r = oracle_lib.pinsage(og, np.zeros(n, np.int32), [1], 1, 1, 0.0, batch_size=1, rng_key=5)
    cnt = Counter(int(layers[0]["row_map"][0]) for layers in r)
    assert chi_square_p(cnt, {1: .25, 2: .25, 3: .25, 4: .25}, n) > 1e-3


def test_restart_law(oracle_lib):
    ip, ix, _ = cycle(50)
    og = oracle_lib.Graph(ip, ix)
    n, T, rp = 40_000, 4, 0.3
    r = oracle_lib.pinsage(og, np.full(n, 25, np.int32), [T], 1, T, rp, batch_size=1, rng_key=6)
    cnt = Counter(len(layers[0]["eid"]) for layers in r)   # distinct visits = steps taken
    law = {s: (1 - rp) ** s * rp for s in range(T)}
    law[T] = (1 - rp) ** T
    assert chi_square_p(cnt, law, n) > 1e-3


@pytest.fixture(scope="module")
def tiny(oracle_lib):
    g = synth.make_graph("tiny")
    return oracle_lib.Graph(g["indptr"].numpy(), g["indices"].numpy(), g["weights"].numpy())


def within_hops(ip, ix, v, T):
    dist = {v: 0}
    q = deque([v])
    while q:
        x = q.popleft()
        if dist[x] == T:
            continue
        for u in ix[ip[x]:ip[x + 1]].tolist():
            if u not in dist:
                dist[u] = dist[x] + 1
                q.append(u)
    return dist


def test_invariants_tiny(oracle_lib, tiny):
    seeds = synth.make_seeds("tiny", 400).numpy()
    W, T, k = 8, 3, [6, 4]
    r = oracle_lib.pinsage(tiny, seeds, k, W, T, 0.4, batch_size=100, rng_key=11)
    ip, ix = tiny.indptr, tiny.indices
    for b, layers in enumerate(r):
        assert layers[0]["col_map"].tolist() == seeds[b * 100:(b + 1) * 100].tolist()
        for l, blk in enumerate(layers):
            if l:
                assert blk["col_map"].tolist() == layers[l - 1]["row_map"].tolist()
            rows = blk["row_map"]
            assert np.all(np.diff(rows) > 0)
            for c, v in enumerate(blk["col_map"].tolist()[:40]):
                lo, hi = blk["indptr"][c], blk["indptr"][c + 1]
                assert hi - lo <= k[l]
                sel = rows[blk["row_local"][lo:hi]].tolist()
                cnt = blk["val"][lo:hi].tolist()
                assert v not in sel and len(set(sel)) == len(sel)
                assert all(1 <= x <= W * T for x in cnt)
                assert all((a > b2) or (a == b2 and s1 < s2)
                           for a, b2, s1, s2 in zip(cnt, cnt[1:], sel, sel[1:]))
                reach = within_hops(ip, ix, v, T)
                assert all(x in reach for x in sel)
    part = oracle_lib.pinsage(tiny, seeds[200:], k, W, T, 0.4, batch_size=100,
                              batch_index_base=2, rng_key=11)
    for l in range(2):
        for key in ["row_map", "indptr", "row_local", "val"]:
            assert np.array_equal(part[0][l][key], r[2][l][key])

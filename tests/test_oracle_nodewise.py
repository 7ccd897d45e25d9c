"""Pins for the oracle's node-wise path: GraphSAGE (Floyd), KGCN (replacement),
weighted A-Res, PASS-style A3 probabilities, and the Finalize relabel.

Pins: structural invariants (every sampled edge exists, count = min(k, d), no
duplicates without replacement, row() = the block's unique rows ascending and
row_local their ranks, R3), exact sampling laws
by enumeration + chi-square (p > 0.001), and the paper's Fig. 1(b) narration
(two frontiers that both sample f give 3 layer-2 nodes).
"""
import itertools
import math
from collections import Counter

import numpy as np
import pytest

import synth
from tests._stats import chi_square_p, successive_sampling_law
from tests.graphs_small import B, C, D, E, F, G, H, fig1_graph, star_graph


def _og(oracle, indptr, indices, weights=None):
    return oracle.Graph(indptr, indices, weights)


@pytest.fixture(scope="module")
def tiny(oracle_lib):
    g = synth.make_graph("tiny")
    return oracle_lib.Graph(g["indptr"].numpy(), g["indices"].numpy(), g["weights"].numpy())


def check_block_invariants(og, blk, k=None, replace=False, exact_count=True):
    ip, ix = og.indptr, og.indices
    n_cols = len(blk["col_map"])
    assert blk["indptr"][0] == 0 and len(blk["indptr"]) == n_cols + 1
    assert np.all(np.diff(blk["indptr"]) >= 0)
    assert blk["indptr"][-1] == len(blk["eid"]) == len(blk["row_local"])
    # row_map: no duplicates; row_map[row_local[e]] is the edge's source node
    assert len(set(blk["row_map"].tolist())) == len(blk["row_map"])
    assert np.all(blk["row_map"][blk["row_local"]] == ix[blk["eid"]])
    # R3: row_map is exactly the set of the block's rows, ascending
    assert blk["row_map"].tolist() == sorted(set(ix[blk["eid"]].tolist()))
    for j in range(n_cols):
        v = blk["col_map"][j]
        lo, hi = blk["indptr"][j], blk["indptr"][j + 1]
        eids = blk["eid"][lo:hi]
        d = ip[v + 1] - ip[v]
        assert np.all((eids >= ip[v]) & (eids < ip[v + 1])), "edge not in column v"
        if k is not None and exact_count:
            want = (k if d > 0 else 0) if replace else min(k, d)
            assert hi - lo == want
        if not replace:
            assert np.all(np.diff(eids) > 0), "positions must be distinct and ascending"


@pytest.mark.parametrize("replace", [False, True])
def test_invariants_tiny(oracle_lib, tiny, replace):
    seeds = synth.make_seeds("tiny", 512).numpy()
    res = oracle_lib.sample_neighbors(tiny, seeds, [5, 5], batch_size=128, replace=replace,
                                      rng_key=0x5EED)
    assert len(res) == 4
    for b, layers in enumerate(res):
        assert np.array_equal(layers[0]["col_map"], seeds[b * 128:(b + 1) * 128])
        for l, blk in enumerate(layers):
            check_block_invariants(tiny, blk, k=5, replace=replace)
            if l > 0:  # next frontiers = previous A.row()
                assert np.array_equal(blk["col_map"], layers[l - 1]["row_map"])


def test_deterministic_and_batch_keyed(oracle_lib, tiny):
    seeds = synth.make_seeds("tiny", 256).numpy()
    a = oracle_lib.sample_neighbors(tiny, seeds, [5, 5], batch_size=64, rng_key=1)
    b = oracle_lib.sample_neighbors(tiny, seeds, [5, 5], batch_size=64, rng_key=1)
    for x, y in zip(a, b):
        for bx, by in zip(x, y):
            assert np.array_equal(bx["eid"], by["eid"])
    # batch 2 of the full call == a call on its seeds alone with batch_index_base = 2
    c = oracle_lib.sample_neighbors(tiny, seeds[128:192], [5, 5], batch_size=64,
                                    batch_index_base=2, rng_key=1)
    for l in range(2):
        assert np.array_equal(a[2][l]["eid"], c[0][l]["eid"])
        assert np.array_equal(a[2][l]["row_map"], c[0][l]["row_map"])


def test_floyd_exact_law(oracle_lib):
    """Uniform k-subset law 1/C(d,k) (GraphSAGE), d=6, k=3: 20 cells."""
    og = _og(oracle_lib, *star_graph(6))
    n = 100_000
    res = oracle_lib.sample_neighbors(og, np.zeros(n, np.int32), [3], batch_size=1, rng_key=11)
    cnt = Counter(tuple(r[0]["eid"].tolist()) for r in res)
    law = {s: 1.0 / math.comb(6, 3) for s in itertools.combinations(range(6), 3)}
    assert chi_square_p(cnt, law, n) > 1e-3


def test_floyd_small_degree_identity(oracle_lib):
    og = _og(oracle_lib, *star_graph(4))
    for k in [4, 5, 25]:
        res = oracle_lib.sample_neighbors(og, np.zeros(50, np.int32), [k], batch_size=1)
        for r in res:
            assert r[0]["eid"].tolist() == [0, 1, 2, 3]


def test_replace_exact_law(oracle_lib):
    """KGCN reading (R10): ordered k-tuples uniform over d^k; d=4, k=3: 64 cells."""
    og = _og(oracle_lib, *star_graph(4))
    n = 128_000
    res = oracle_lib.sample_neighbors(og, np.zeros(n, np.int32), [3], batch_size=1,
                                      replace=True, rng_key=12)
    cnt = Counter(tuple(r[0]["eid"].tolist()) for r in res)
    law = {t: 1.0 / 64 for t in itertools.product(range(4), repeat=3)}
    assert chi_square_p(cnt, law, n) > 1e-3
    # dedup of rows still applies (Finalize); count = k * [d > 0]
    for r in res[:200]:
        blk = r[0]
        assert len(blk["eid"]) == 3
        assert len(blk["row_map"]) == len(set(blk["eid"].tolist()))


def test_ares_exact_law(oracle_lib):
    """Weighted without replacement (R6): successive-sampling law, w=[1,2,3,4,10], k=2."""
    w = [1.0, 2.0, 3.0, 4.0, 10.0]
    og = _og(oracle_lib, *star_graph(5, w))
    n = 100_000
    res = oracle_lib.sample_neighbors(og, np.zeros(n, np.int32), [2], batch_size=1,
                                      bias_mode=oracle_lib.EDGE, rng_key=13)
    cnt = Counter(tuple(r[0]["eid"].tolist()) for r in res)
    law = successive_sampling_law(w, 2)
    assert law[(3, 4)] == pytest.approx(0.325, abs=1e-6)  # SURVEY 8(c) c.5 value
    assert chi_square_p(cnt, law, n) > 1e-3


def test_ares_equal_weights_uniform(oracle_lib):
    og = _og(oracle_lib, *star_graph(6, [0.25] * 6))
    n = 60_000
    res = oracle_lib.sample_neighbors(og, np.zeros(n, np.int32), [3], batch_size=1,
                                      bias_mode=oracle_lib.EDGE, rng_key=14)
    cnt = Counter(tuple(r[0]["eid"].tolist()) for r in res)
    law = {s: 1.0 / 20 for s in itertools.combinations(range(6), 3)}
    assert chi_square_p(cnt, law, n) > 1e-3


def test_ares_zero_weight_ineligible(oracle_lib):
    og = _og(oracle_lib, *star_graph(6, [1.0, 0.0, 2.0, 0.0, 3.0, 1.0]))
    res = oracle_lib.sample_neighbors(og, np.zeros(2000, np.int32), [3], batch_size=1,
                                      bias_mode=oracle_lib.EDGE)
    for r in res:
        e = r[0]["eid"].tolist()
        assert len(e) == 3 and 1 not in e and 3 not in e
    # |eligible| <= k: take all eligible, no randomness
    res = oracle_lib.sample_neighbors(og, np.zeros(5, np.int32), [4], batch_size=1,
                                      bias_mode=oracle_lib.EDGE)
    for r in res:
        assert r[0]["eid"].tolist() == [0, 2, 4, 5]


def test_pass_colnorm_closed_form(oracle_lib, tiny):
    """PASS A3 = sub_A.div(sub_A.sum(axis=0)) (R1, R11): prob_e is the
    edge weight over its full column sum, so summing it over ALL of a column's
    edges gives 1."""
    seeds = synth.make_seeds("tiny", 256).numpy()
    res = oracle_lib.sample_neighbors(tiny, seeds, [4, 4], batch_size=256,
                                      bias_mode=oracle_lib.PASS_COLNORM, rng_key=3)
    ip, w = tiny.indptr, tiny.weights
    for blk in res[0]:
        check_block_invariants(tiny, blk, k=None)
        assert blk["val"] is not None
        for j, v in enumerate(blk["col_map"]):
            lo, hi = blk["indptr"][j], blk["indptr"][j + 1]
            full = w[ip[v]:ip[v + 1]].astype(np.float64)
            if hi > lo:
                np.testing.assert_allclose(blk["val"][lo:hi] * full.sum(),
                                           w[blk["eid"][lo:hi]], rtol=1e-6)
    # the selection is the EDGE (A-Res) selection
    ref = oracle_lib.sample_neighbors(tiny, seeds, [4, 4], batch_size=256,
                                      bias_mode=oracle_lib.EDGE, rng_key=3)
    for a, b in zip(res[0], ref[0]):
        assert np.array_equal(a["eid"], b["eid"])


def test_fig1b_two_frontiers_share_f(oracle_lib):
    """b and e each sample 2 in-neighbours and both pick f -> 3 layer-2 nodes."""
    ip, ix, w = fig1_graph()
    og = _og(oracle_lib, ip, ix, w)
    found = 0
    for key in range(400):
        res = oracle_lib.sample_neighbors(og, np.array([B, E], np.int32), [2], rng_key=key)
        blk = res[0][0]
        rows_b = set(ix[blk["eid"][0:2]].tolist())
        rows_e = set(ix[blk["eid"][2:4]].tolist())
        assert rows_b <= {C, D, F} and rows_e <= {F, G, H}
        if F in rows_b and F in rows_e:
            found += 1
            assert len(blk["row_map"]) == 3
            # R3: the union of both picks, ascending
            assert blk["row_map"].tolist() == sorted(rows_b | rows_e)
        else:
            assert len(blk["row_map"]) == 4
    assert found > 0

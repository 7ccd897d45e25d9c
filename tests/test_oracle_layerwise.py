"""Pins for the oracle's layer-wise path (collective_sample) with
LADIES / FastGCN / COUNT biases (Table 2, Fig. 3(b)).

Pins: the paper's worked value B_f = w_fb^2 + w_fe^2 = 0.58, Fig. 1(c)
"sample 4 of {c,d,f,g,h} -> 4 nodes", the closed form of the LADIES
edge weights after the B-cancelling rewrite val_e = (w_e / b_u) / sum_col(w / b),
column normalisation (columns sum to 1), the successive-sampling law of the
K-of-|C| selection (chi-square), the identity LADIES(w == 1) == COUNT and the
FastGCN degree bias, plus brute-force block membership on the tiny graph.
"""
import json
import os
from collections import Counter

import numpy as np
import pytest

import synth
from tests._stats import chi_square_p, successive_sampling_law
from tests.graphs_small import B, C, D, E, F, G, H, FIG1, fig1_graph

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "ladies_fig1.json")


@pytest.fixture(scope="module")
def fig1(oracle_lib):
    return oracle_lib.Graph(*fig1_graph())


def test_paper_bias_of_f(oracle_lib, fig1):
    gold = json.load(open(GOLDEN))
    res = oracle_lib.sample_layerwise(fig1, np.array([B, E], np.int32), [5],
                                      prob_mode=oracle_lib.LADIES)
    blk = res[0][0]
    assert blk["row_map"].tolist() == [C, D, F, G, H]          # S = C, ascending
    # B_f = 0.49 + 0.09 = 0.58; p(f) = B_f / B with B = sum over C
    bias = {C: 0.04, D: 0.81, F: 0.58, G: 0.64, H: 0.01}
    Btot = sum(bias.values())
    p = dict(zip(blk["row_map"].tolist(), blk["row_prob"].tolist()))
    assert p[F] * Btot == pytest.approx(gold["B_f"], rel=2e-7)
    assert gold["B_f"] == 0.58
    assert sum(p.values()) == pytest.approx(1.0, rel=1e-6)
    for u in bias:
        assert p[u] == pytest.approx(bias[u] / Btot, rel=1e-6)


def test_ladies_val_closed_form(oracle_lib, fig1):
    res = oracle_lib.sample_layerwise(fig1, np.array([B, E], np.int32), [5])
    blk = res[0][0]
    bias = {C: 0.04, D: 0.81, F: 0.58, G: 0.64, H: 0.01}
    for j, v in enumerate([B, E]):
        lo, hi = blk["indptr"][j], blk["indptr"][j + 1]
        col = FIG1[v]
        assert hi - lo == len(col)
        denom = sum(w / bias[u] for u, w in col)
        want = [(w / bias[u]) / denom for u, w in col]
        np.testing.assert_allclose(blk["val"][lo:hi], want, rtol=2e-6)
        assert blk["val"][lo:hi].astype(np.float64).sum() == pytest.approx(1.0, rel=1e-6)


def test_fig1c_four_of_five(oracle_lib, fig1):
    """layer-wise sampling of 4 nodes among {c,d,f,g,h} gives 4 nodes."""
    for key in range(50):
        blk = oracle_lib.sample_layerwise(fig1, np.array([B, E], np.int32), [4],
                                          rng_key=key)[0][0]
        assert len(blk["row_map"]) == 4
        assert set(blk["row_map"].tolist()) <= {C, D, F, G, H}
        assert np.all(np.diff(blk["row_map"]) > 0)
        # column-normalised val (Fig. 3(b) line 7)
        for j in range(2):
            lo, hi = blk["indptr"][j], blk["indptr"][j + 1]
            if hi > lo:
                assert blk["val"][lo:hi].astype(np.float64).sum() == pytest.approx(1, rel=1e-6)


@pytest.mark.parametrize("K", [4, 2])
def test_selection_law(oracle_lib, fig1, K):
    """collective_sample without replacement by node bias (R6/R7): successive sampling."""
    n = 60_000
    seeds = np.tile(np.array([B, E], np.int32), n)
    res = oracle_lib.sample_layerwise(fig1, seeds, [K], batch_size=2, rng_key=21)
    cnt = Counter(tuple(r[0]["row_map"].tolist()) for r in res)
    nodes = [C, D, F, G, H]
    bias = [0.04, 0.81, 0.58, 0.64, 0.01]
    law = {tuple(nodes[i] for i in s): p for s, p in successive_sampling_law(bias, K).items()}
    assert chi_square_p(cnt, law, n) > 1e-3


@pytest.fixture(scope="module")
def tiny(oracle_lib):
    g = synth.make_graph("tiny")
    return oracle_lib.Graph(g["indptr"].numpy(), g["indices"].numpy(), g["weights"].numpy())


@pytest.mark.parametrize("mode", [0, 1, 2])
def test_block_is_extract_restricted_to_S(oracle_lib, tiny, mode):
    seeds = synth.make_seeds("tiny", 512).numpy()
    res = oracle_lib.sample_layerwise(tiny, seeds, [64, 64, 64], batch_size=256,
                                      prob_mode=mode, rng_key=5)
    ip, ix = tiny.indptr, tiny.indices
    for layers in res:
        for l, blk in enumerate(layers):
            S = blk["row_map"]
            assert np.all(np.diff(S) > 0) and len(S) <= 64
            cand = set()
            for v in blk["col_map"]:
                cand |= set(ix[ip[v]:ip[v + 1]].tolist())
            assert len(S) == min(64, len(cand))   # every candidate has b(u) > 0 here
            Sset = set(S.tolist())
            for j, v in enumerate(blk["col_map"]):
                lo, hi = blk["indptr"][j], blk["indptr"][j + 1]
                want = [e for e in range(ip[v], ip[v + 1]) if ix[e] in Sset]
                assert blk["eid"][lo:hi].tolist() == want
                assert np.all(S[blk["row_local"][lo:hi]] == ix[blk["eid"][lo:hi]])
                if hi > lo:
                    assert blk["val"][lo:hi].astype(np.float64).sum() == pytest.approx(1, rel=1e-5)
            if l > 0:
                assert np.array_equal(blk["col_map"], layers[l - 1]["row_map"])


def test_ladies_unit_weights_equals_count(oracle_lib, tiny):
    ones = oracle_lib.Graph(tiny.indptr, tiny.indices, np.ones_like(tiny.weights))
    seeds = synth.make_seeds("tiny", 300).numpy()
    a = oracle_lib.sample_layerwise(ones, seeds, [50, 50], batch_size=100, prob_mode=0, rng_key=9)
    b = oracle_lib.sample_layerwise(ones, seeds, [50, 50], batch_size=100, prob_mode=2, rng_key=9)
    for x, y in zip(a, b):
        for bx, by in zip(x, y):
            for k in ["row_map", "eid", "row_local"]:
                assert np.array_equal(bx[k], by[k])
            assert np.array_equal(bx["val"], by["val"])
            assert np.array_equal(bx["row_prob"], by["row_prob"])


def test_fastgcn_degree_bias(oracle_lib, tiny):
    """FastGCN: the sampling bias of a node is its degree (Table 2; R9)."""
    seeds = synth.make_seeds("tiny", 100).numpy()
    ip, ix = tiny.indptr, tiny.indices
    blk = oracle_lib.sample_layerwise(tiny, seeds, [100000], prob_mode=1)[0][0]
    cand = sorted(set(np.concatenate([ix[ip[v]:ip[v + 1]] for v in seeds]).tolist()))
    # candidates with in-degree 0 have bias 0 and are not eligible (R6)
    cand = [u for u in cand if ip[u + 1] > ip[u]]
    assert blk["row_map"].tolist() == cand
    deg = np.array([ip[u + 1] - ip[u] for u in cand], dtype=np.float64)
    np.testing.assert_allclose(blk["row_prob"], deg / deg.sum(), rtol=1e-6)


def test_empty_candidates_propagate(oracle_lib):
    ip = np.zeros(5, np.int64)
    og = oracle_lib.Graph(ip, np.zeros(0, np.int32), None)
    res = oracle_lib.sample_layerwise(og, np.array([0, 1], np.int32), [3, 3])
    for blk in res[0]:
        assert len(blk["row_map"]) == 0 and len(blk["eid"]) == 0
    assert len(res[0][1]["col_map"]) == 0

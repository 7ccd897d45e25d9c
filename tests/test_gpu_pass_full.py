"""GPU parity: PASS learned bias in full (Fig. 3(c) lines 3-10; DESIGN
R29) -- gs_pass_attention (tensor-core projection GEMM + SDDMM/mix kernel) vs
oracle/pass_att.py bit for bit, then line 10's weighted node-wise sampling over
att (gs_graph_set_weights + gs_sample_neighbors(EDGE)) vs the oracle's A-Res
sampler over the oracle's att, element by element."""
import numpy as np
import pytest
import torch

import synth
from oracle import pass_att
from tests.parity import compare_all, host_graph

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def gs():
    from paper_conf_sosp_gonglmc0lwl23_b200 import gs as _gs
    _gs.load_library()
    _gs.use_torch_allocator()
    return _gs


def inputs(N, F, H, seed):
    X = synth.make_grid_matrix(seed, N, F, device="cuda")
    W1 = synth.make_grid_matrix(seed + 1, F, H, device="cuda")
    W2 = synth.make_grid_matrix(seed + 2, F, H, device="cuda")
    return X, W1, W2


@pytest.mark.parametrize("H,F,W3", [(32, 128, [0.2, -0.4, 0.9]), (8, 64, [1.0, 1.0, 1.0]),
                                    (64, 32, [-3.0, 2.0, 0.0]), (16, 128, [0.0, 0.0, 5.0])])
def test_attention_tiny(gs, H, F, W3):
    g = synth.make_graph("tiny", device="cuda")
    G = gs.Graph(g["indptr"], g["indices"], g["weights"])
    X, W1, W2 = inputs(10_000, F, H, 31)
    att = gs.pass_attention(G, X, W1, W2, W3).cpu().numpy()
    ip, ix, w = host_graph(g)
    ref = pass_att.pass_attention(ip, ix, w, X.float().cpu().numpy(), W1.float().cpu().numpy(),
                                  W2.float().cpu().numpy(), W3)
    assert np.array_equal(att, ref), f"{np.sum(att != ref)} of {len(ref)} differ"
    assert (ref > 0).any() and (ref == 0).any()   # both relu branches exercised


def test_attention_unweighted(gs):
    g = synth.small_graph(20_000, 200_000, undirected=True, weights=None, seed=5, device="cuda")
    G = gs.Graph(g["indptr"], g["indices"], None)
    X, W1, W2 = inputs(20_000, 128, 32, 41)
    att = gs.pass_attention(G, X, W1, W2, [0.1, 0.2, 0.3]).cpu().numpy()
    ip, ix, _ = host_graph(g)
    ref = pass_att.pass_attention(ip, ix, None, X.float().cpu().numpy(), W1.float().cpu().numpy(),
                                  W2.float().cpu().numpy(), [0.1, 0.2, 0.3])
    assert np.array_equal(att, ref)


def test_pass_full_sampling_medium(gs, oracle_lib):
    g = synth.small_graph(200_000, 3_000_000, undirected=True, weights="uniform", seed=77,
                          device="cuda")
    G = gs.Graph(g["indptr"], g["indices"], g["weights"])
    X, W1, W2 = inputs(200_000, 128, 32, 51)
    W3 = [0.2, -0.4, 0.9]
    att = gs.pass_attention(G, X, W1, W2, W3)
    ip, ix, w = host_graph(g)
    ref_att = pass_att.pass_attention(ip, ix, w, X.float().cpu().numpy(), W1.float().cpu().numpy(),
                                      W2.float().cpu().numpy(), W3)
    assert np.array_equal(att.cpu().numpy(), ref_att)
    Ga = gs.Graph(g["indptr"], g["indices"], g["weights"])
    Ga.set_weights(att)
    seeds = synth.make_seeds(synth.GraphSpec("m", 200_000, 1, True, None, 6), 3000)
    out = gs.sample_neighbors(Ga, seeds.cuda(), [10, 10], batch_size=1024, bias_mode=1,
                              rng_key=61).to_host()
    O = oracle_lib.Graph(ip, ix, ref_att)
    ref = oracle_lib.sample_neighbors(O, seeds.numpy(), [10, 10], batch_size=1024, bias_mode=1,
                                      rng_key=61)
    compare_all(out, ref, "PASS full [10,10]")


def test_pass_attention_pdw_full_size(gs):
    """The bench configuration (PDw, 128-d features, H = 32): att of 300 random
    columns and the 20 highest-degree columns recomputed by the oracle."""
    g = synth.make_graph("PDw", device="cuda")
    G = gs.Graph(g["indptr"], g["indices"], g["weights"])
    N = g["indptr"].numel() - 1
    X = synth.make_grid_matrix(21, N, 128, device="cuda")
    W1 = synth.make_grid_matrix(22, 128, 32, device="cuda")
    W2 = synth.make_grid_matrix(23, 128, 32, device="cuda")
    W3 = [0.2, -0.4, 0.9]
    att = gs.pass_attention(G, X, W1, W2, W3)
    ip = g["indptr"].cpu().numpy()
    deg = np.diff(ip)
    cols = sorted(set(np.random.default_rng(3).integers(0, N, 300).tolist()) |
                  set(np.argsort(deg)[-20:].tolist()))
    ix = g["indices"].cpu().numpy()
    w = g["weights"].cpu().numpy()
    ref = pass_att.pass_attention_columns(ip, ix, w, X.float().cpu().numpy(),
                                          W1.float().cpu().numpy(), W2.float().cpu().numpy(), W3, cols)
    a = att.cpu().numpy()
    for v in cols:
        assert np.array_equal(a[ip[v]:ip[v + 1]], ref[v]), f"column {v}"

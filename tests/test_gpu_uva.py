"""GPU parity: graphs whose index / weight arrays stay in pinned host memory
(GS_GRAPH_HOST_MAPPED: every kernel reads them over the host link, P:415's UVA
mode).  Every sampler must return exactly what it returns on
the HBM-resident graph (and hence what the oracle returns)."""
import numpy as np
import pytest
import torch

import synth
from tests.parity import compare_all, host_graph

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def gs():
    from paper_conf_sosp_gonglmc0lwl23_b200 import gs as _gs
    _gs.load_library()
    _gs.use_torch_allocator()
    return _gs


@pytest.fixture(scope="module")
def graphs(gs):
    g = synth.small_graph(200_000, 3_000_000, undirected=True, weights="uniform", seed=77,
                          device="cuda")
    Gd = gs.Graph(g["indptr"], g["indices"], g["weights"])
    Gh = gs.Graph(g["indptr"], g["indices"], g["weights"], host_mapped=True)
    assert Gh.host_mapped and not Gd.host_mapped
    return g, Gd, Gh


def seeds(n, s=6):
    return synth.make_seeds(synth.GraphSpec("m", 200_000, 1, True, None, s), n).cuda()


def test_uva_nodewise_and_weighted(gs, graphs, oracle_lib):
    g, Gd, Gh = graphs
    for bias in (0, 1, 2):
        a = gs.sample_neighbors(Gh, seeds(3000), [10, 5], batch_size=1024, bias_mode=bias, rng_key=5).to_host()
        b = gs.sample_neighbors(Gd, seeds(3000), [10, 5], batch_size=1024, bias_mode=bias, rng_key=5).to_host()
        compare_all(a, b, f"uva nodewise bias={bias}")
    O = oracle_lib.Graph(*host_graph(g))
    ref = oracle_lib.sample_neighbors(O, seeds(3000).cpu().numpy(), [10, 5], batch_size=1024, rng_key=5)
    a = gs.sample_neighbors(Gh, seeds(3000), [10, 5], batch_size=1024, rng_key=5).to_host()
    compare_all(a, ref, "uva nodewise vs oracle")


def test_uva_layerwise_shadow_saint_pinsage(gs, graphs):
    g, Gd, Gh = graphs
    pairs = [
        lambda G: gs.sample_layerwise(G, seeds(2000), [256, 256], batch_size=512, prob_mode=0, rng_key=3),
        lambda G: gs.sample_layerwise(G, seeds(2000), [256, 256], batch_size=512, prob_mode=1, rng_key=3),
        lambda G: gs.sample_shadow(G, seeds(1000), [5, 3], batch_size=256, rng_key=4),
        lambda G: gs.sample_saint_rw(G, seeds(4000), 2, batch_size=1000, rng_key=6),
        lambda G: gs.sample_pinsage(G, seeds(2000), [6, 4], 8, 3, 0.5, batch_size=512, rng_key=7),
    ]
    for k, f in enumerate(pairs):
        compare_all(f(Gh).to_host(), f(Gd).to_host(), f"uva sampler {k}")


def test_uva_walks(gs, graphs):
    g, Gd, Gh = graphs
    st = seeds(20_000)
    for pq in [(1.0, 1.0), (2.0, 0.5)]:
        a = gs.random_walk(Gh, st, 20, p=pq[0], q=pq[1], rng_key=9)
        b = gs.random_walk(Gd, st, 20, p=pq[0], q=pq[1], rng_key=9)
        assert torch.equal(a, b)


@pytest.mark.parametrize("budget_frac", [0.0, 0.3, 1.0])
def test_uva_hot_page_cache(gs, budget_frac, oracle_lib):
    """gs_graph_cache_hot: the node-wise sampler reads cached pages from HBM and
    the rest over the host link -- the same blocks as without a cache (and as
    the oracle), uniform, weighted and PASS-style, whatever the budget."""
    g = synth.small_graph(200_000, 3_000_000, undirected=True, weights="uniform", seed=78, device="cuda")
    Gd = gs.Graph(g["indptr"], g["indices"], g["weights"])
    Gh = gs.Graph(g["indptr"], g["indices"], g["weights"], host_mapped=True)
    budget = int(budget_frac * (g["indices"].numel() + 16384) * 8)  # whole pages
    cached = Gh.cache_hot(budget)
    if budget_frac == 1.0:
        assert cached >= g["indices"].numel()
    elif budget_frac == 0.0:
        assert cached == 0
    else:
        assert 0 < cached < g["indices"].numel()
    for bias in (0, 1, 2):
        a = gs.sample_neighbors(Gh, seeds(3000, 8), [10, 5], batch_size=1024, bias_mode=bias, rng_key=9).to_host()
        b = gs.sample_neighbors(Gd, seeds(3000, 8), [10, 5], batch_size=1024, bias_mode=bias, rng_key=9).to_host()
        compare_all(a, b, f"uva cache {budget_frac} bias={bias}")
    O = oracle_lib.Graph(*host_graph(g))
    ref = oracle_lib.sample_neighbors(O, seeds(3000, 8).cpu().numpy(), [10, 5], batch_size=1024, rng_key=9)
    a = gs.sample_neighbors(Gh, seeds(3000, 8), [10, 5], batch_size=1024, rng_key=9).to_host()
    compare_all(a, ref, f"uva cache {budget_frac} vs oracle")


def test_uva_cache_rejects_hbm_graph(gs, graphs):
    g, Gd, Gh = graphs
    with pytest.raises(gs.GSError):
        Gd.cache_hot(1 << 20)

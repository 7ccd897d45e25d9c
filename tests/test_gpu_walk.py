"""GPU parity: DeepWalk / Node2Vec walks vs the oracle (bit-exact traces)."""
import numpy as np
import pytest
import torch

import synth
from tests.parity import host_graph

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def gs():
    from paper_conf_sosp_gonglmc0lwl23_b200 import gs as _gs
    _gs.load_library()
    _gs.use_torch_allocator()
    return _gs


@pytest.fixture(params=["index", "plain"], autouse=True)
def walk_layout(request, monkeypatch):
    """Every walk test runs on the walk index (one random 16-byte record per
    step) and on the plain CSC (GS_WALK_INDEX=0): identical traces."""
    monkeypatch.setenv("GS_WALK_INDEX", "1" if request.param == "index" else "0")
    return request.param


@pytest.fixture(scope="module")
def graph(gs, oracle_lib):
    g = synth.small_graph(100_000, 1_500_000, undirected=True, weights=None, seed=9, device="cuda")
    return g, gs.Graph(g["indptr"], g["indices"]), oracle_lib.Graph(*host_graph(g))


@pytest.mark.parametrize("pq,force", [((1.0, 1.0), False), ((2.0, 0.5), False),
                                      ((1.0, 1.0), True), ((0.25, 4.0), False)])
def test_walk_parity(gs, oracle_lib, graph, pq, force):
    g, G, O = graph
    starts = torch.arange(0, 100_000, 3, dtype=torch.int32)
    tr = gs.random_walk(G, starts.cuda(), 40, p=pq[0], q=pq[1], rng_key=123, walker_index_base=7,
                        force_node2vec=force).cpu().numpy()
    ref = oracle_lib.random_walk(O, starts.numpy(), 40, p=pq[0], q=pq[1], rng_key=123,
                                 walker_index_base=7, force_node2vec=force)
    assert np.array_equal(tr, ref), f"{(tr != ref).sum()} trace entries differ"


def test_walk_dead_ends_and_range(gs, oracle_lib):
    ip = torch.tensor([0, 2, 3, 3, 4], dtype=torch.int64)
    ix = torch.tensor([1, 3, 0, 2], dtype=torch.int32)
    G = gs.Graph(ip.cuda(), ix.cuda())
    O = oracle_lib.Graph(ip.numpy(), ix.numpy())
    starts = torch.tensor([0, 1, 2, 3, 0], dtype=torch.int32)
    tr = gs.random_walk(G, starts.cuda(), 6, p=2.0, q=0.5).cpu().numpy()
    assert np.array_equal(tr, oracle_lib.random_walk(O, starts.numpy(), 6, p=2.0, q=0.5))
    assert (tr[2, 1:] == -1).all()
    gs.walk_check(G)
    gs.random_walk(G, torch.tensor([4], dtype=torch.int32, device="cuda"), 3)
    with pytest.raises(gs.GSError):
        gs.walk_check(G)
    # zero-length walks and zero walkers
    assert gs.random_walk(G, starts.cuda(), 0).shape == (5, 1)
    assert gs.random_walk(G, torch.empty(0, dtype=torch.int32, device="cuda"), 5).shape == (0, 6)


def test_node2vec_needs_sorted(gs):
    ip = torch.tensor([0, 2, 2, 2], dtype=torch.int64)
    ix = torch.tensor([2, 1], dtype=torch.int32)  # column 0 unsorted
    G = gs.Graph(ip.cuda(), ix.cuda())
    assert not G.sorted
    with pytest.raises(gs.GSError) as ei:
        gs.random_walk(G, torch.tensor([0], dtype=torch.int32, device="cuda"), 3, p=2.0, q=0.5)
    assert ei.value.status == 4
    gs.random_walk(G, torch.tensor([0], dtype=torch.int32, device="cuda"), 3)  # DeepWalk is fine

"""GPU parity: PinSAGE-style sampling (Table 2; DESIGN R27) through
gs_sample_pinsage vs the CPU oracle, element by element (integers bit-exact,
visit counts exact in fp32): several batches with a ragged tail, one to three
layers, chunked hash tables (many walks), restart 0 and 1, dead-end seeds,
global batch keying, out-of-range seeds, and the PD-shaped epoch the bench
times (sampled batches recomputed by the oracle)."""
import numpy as np
import pytest
import torch

import synth
from tests.parity import compare_all, compare_block, host_graph

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def gs():
    from paper_conf_sosp_gonglmc0lwl23_b200 import gs as _gs
    _gs.load_library()
    _gs.use_torch_allocator()
    return _gs


@pytest.fixture(scope="module")
def tiny(gs, oracle_lib):
    g = synth.make_graph("tiny", device="cuda")
    return g, gs.Graph(g["indptr"], g["indices"], g["weights"]), oracle_lib.Graph(*host_graph(g))


@pytest.fixture(scope="module")
def medium(gs, oracle_lib):
    g = synth.small_graph(200_000, 3_000_000, undirected=True, weights="uniform", seed=77,
                          device="cuda")
    return g, gs.Graph(g["indptr"], g["indices"], g["weights"]), oracle_lib.Graph(*host_graph(g))


@pytest.mark.parametrize("topk,W,T,rp,bs", [([5, 3], 10, 3, 0.5, 300), ([8], 1, 1, 0.0, 97),
                                            ([4, 4, 2], 6, 4, 0.3, 128), ([32], 64, 8, 0.1, 200),
                                            ([3, 3], 5, 2, 1.0, 256)])
def test_pinsage_tiny(gs, oracle_lib, tiny, topk, W, T, rp, bs):
    g, G, O = tiny
    seeds = synth.make_seeds("tiny", 1000)
    out = gs.sample_pinsage(G, seeds.cuda(), topk, W, T, rp, batch_size=bs, rng_key=0xB0B).to_host()
    ref = oracle_lib.pinsage(O, seeds.numpy(), topk, W, T, rp, batch_size=bs, rng_key=0xB0B)
    compare_all(out, ref, f"pinsage {topk} W={W} T={T} r={rp}")


def test_pinsage_dead_end_seeds(gs, oracle_lib, tiny):
    g, G, O = tiny
    ip = g["indptr"].cpu()
    dead = torch.nonzero(ip[1:] == ip[:-1]).flatten()[:40].to(torch.int32)
    seeds = torch.cat([dead, synth.make_seeds("tiny", 100)]).to(torch.int32)
    out = gs.sample_pinsage(G, seeds.cuda(), [6, 2], 8, 3, 0.25, batch_size=50, rng_key=2).to_host()
    ref = oracle_lib.pinsage(O, seeds.numpy(), [6, 2], 8, 3, 0.25, batch_size=50, rng_key=2)
    compare_all(out, ref, "pinsage dead ends")


def test_pinsage_medium(gs, oracle_lib, medium):
    g, G, O = medium
    seeds = synth.make_seeds(synth.GraphSpec("m", 200_000, 1, True, None, 6), 3000)
    out = gs.sample_pinsage(G, seeds.cuda(), [10, 10], 10, 3, 0.5, batch_size=1024,
                            rng_key=29).to_host()
    ref = oracle_lib.pinsage(O, seeds.numpy(), [10, 10], 10, 3, 0.5, batch_size=1024, rng_key=29)
    compare_all(out, ref, "pinsage medium")


def test_pinsage_batch_keying_and_reuse(gs, medium):
    """Global batch index keying; one Blocks object reused across calls and kinds."""
    g, G, O = medium
    seeds = synth.make_seeds(synth.GraphSpec("m", 200_000, 1, True, None, 8), 4000).cuda()
    out = gs.Blocks()
    gs.sample_neighbors(G, seeds, [5, 5], batch_size=1000, rng_key=3, out=out).sync()
    full = gs.sample_pinsage(G, seeds, [6, 4], 8, 3, 0.5, batch_size=1000, rng_key=3,
                             out=out).to_host()
    part = gs.sample_pinsage(G, seeds[2000:], [6, 4], 8, 3, 0.5, batch_size=1000,
                             batch_index_base=2, rng_key=3).to_host()
    for b in range(2):
        for l in range(2):
            for k in ["col_map", "row_map", "indptr", "row_local", "eid", "val"]:
                assert np.array_equal(part[b][l][k], full[b + 2][l][k])


def test_pinsage_bad_seed(gs, tiny):
    g, G, O = tiny
    seeds = torch.tensor([1, 2, 10_000, 3], dtype=torch.int32, device="cuda")
    with pytest.raises(gs.GSError) as e:
        gs.sample_pinsage(G, seeds, [3], 4, 2, 0.5, batch_size=2).sync()
    assert e.value.status == 5


def test_pinsage_pd_epoch(gs, oracle_lib):
    """The bench workload: PD-shaped, batch 1024, top-k [10, 10], 10 walks of at
    most 3 steps, restart 0.5, 196,615 seeds; sampled batches vs the oracle."""
    g = synth.make_graph("PD", device="cuda")
    G = gs.Graph(g["indptr"], g["indices"], g["weights"])
    O = oracle_lib.Graph(g["indptr"].cpu().numpy(), g["indices"].cpu().numpy(), None)
    seeds = synth.make_seeds("PD", 196_615, device="cuda")
    out = gs.sample_pinsage(G, seeds, [10, 10], 10, 3, 0.5, batch_size=1024, rng_key=0x915)
    out.sync()
    s = seeds.cpu().numpy()
    rng = np.random.default_rng(3)
    for b in sorted({0, 192} | set(rng.integers(0, 193, 3).tolist())):
        ref = oracle_lib.pinsage(O, s[b * 1024:(b + 1) * 1024], [10, 10], 10, 3, 0.5,
                                 batch_size=1024, batch_index_base=b, rng_key=0x915)[0]
        for l in range(2):
            v = out.view(b, l)
            compare_block({k: (None if x is None else x.cpu().numpy()) for k, x in v.items()},
                          ref[l], f"pinsage PD batch {b} layer {l}")


def test_pinsage_empty(gs, tiny):
    g, G, O = tiny
    out = gs.sample_pinsage(G, torch.zeros(0, dtype=torch.int32, device="cuda"), [3, 3], 4, 2, 0.5,
                            batch_size=10)
    assert out.to_host() == []

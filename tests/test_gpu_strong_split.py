"""SURVEY 8(e) strong split on the GPU: the shards bench.py --gpus N gives the
ranks (dist.shard_epoch: contiguous global batch ranges, or contiguous walker
ranges) reproduce the single-call epoch bit for bit -- node-wise, layer-wise
and walks (the union over ranks is the one-GPU epoch)."""
import numpy as np
import pytest
import torch

import synth
from paper_conf_sosp_gonglmc0lwl23_b200 import dist as gdist
from tests.parity import compare_all

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def gs():
    from paper_conf_sosp_gonglmc0lwl23_b200 import gs as _gs
    _gs.load_library()
    _gs.use_torch_allocator()
    return _gs


@pytest.fixture(scope="module")
def medium(gs):
    g = synth.small_graph(200_000, 3_000_000, undirected=True, weights="uniform", seed=77, device="cuda")
    return g, gs.Graph(g["indptr"], g["indices"], g["weights"])


@pytest.mark.parametrize("world", [2, 3, 8])
def test_nodewise_and_layerwise_strong_split(gs, medium, world):
    g, G = medium
    seeds = (torch.arange(0, 7000, dtype=torch.int32, device="cuda") * 13) % 200_000
    bs = 500
    full = gs.sample_neighbors(G, seeds, [10, 5], batch_size=bs, rng_key=3).to_host()
    fl = gs.sample_layerwise(G, seeds, [64, 64], batch_size=bs, prob_mode=0, rng_key=4).to_host()
    for r in range(world):
        s0, s1, base = gdist.shard_epoch(seeds.numel(), bs, world, r)
        if s1 == s0:
            continue
        nb0, nb1 = base, base + (s1 - s0 + bs - 1) // bs
        part = gs.sample_neighbors(G, seeds[s0:s1], [10, 5], batch_size=bs, batch_index_base=base,
                                   rng_key=3).to_host()
        compare_all(part, full[nb0:nb1], f"node-wise rank {r}/{world}")
        lw = gs.sample_layerwise(G, seeds[s0:s1], [64, 64], batch_size=bs, batch_index_base=base,
                                 prob_mode=0, rng_key=4).to_host()
        compare_all(lw, fl[nb0:nb1], f"layer-wise rank {r}/{world}")


@pytest.mark.parametrize("pq", [(1.0, 1.0), (2.0, 0.5)])
def test_walk_strong_split(gs, medium, pq):
    g, G = medium
    starts = torch.arange(0, 20_000, dtype=torch.int32, device="cuda") * 7 % 200_000
    full = gs.random_walk(G, starts, 12, p=pq[0], q=pq[1], rng_key=9).cpu().numpy()
    world = 4
    parts = []
    for r in range(world):
        s0, s1, base = gdist.shard_epoch(starts.numel(), None, world, r)
        parts.append(gs.random_walk(G, starts[s0:s1], 12, p=pq[0], q=pq[1], walker_index_base=base,
                                    rng_key=9).cpu().numpy())
    assert np.array_equal(np.concatenate(parts), full)

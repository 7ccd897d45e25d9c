"""GPU parity of the ragged-batch and standalone-induce entry points (VERDICT
r1 item 5): gs_sample_neighbors_ragged (batch b = seeds
[batch_ptr[b], batch_ptr[b+1]), keyed by batch_index_base + b) and
gs_induce_subgraph over a node-wise result (R12), both
against the CPU oracle run batch by batch."""
import numpy as np
import pytest
import torch

import synth
from tests.parity import compare_all, host_graph

pytestmark = pytest.mark.gpu

RAGGED = [0, 100, 100, 357, 358, 512]  # an empty batch, a 1-seed batch, uneven sizes


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


def _oracle_ragged(oracle_lib, O, seeds, bp, fan, fn, **kw):
    ref = []
    for b in range(len(bp) - 1):
        s = seeds[bp[b]:bp[b + 1]]
        if len(s) == 0:
            ref.append(None)
            continue
        ref.extend(fn(O, s, fan, batch_size=len(s), batch_index_base=7 + b, **kw))
    return ref


@pytest.mark.parametrize("mode", ["uniform", "replace", "edge", "pass"])
def test_ragged_matches_per_batch_oracle(gs, oracle_lib, tiny, mode):
    g, G, O = tiny
    seeds = synth.make_seeds("tiny", 512)
    kw = dict(replace=mode == "replace", bias_mode={"uniform": 0, "replace": 0, "edge": 1, "pass": 2}[mode])
    out = gs.sample_neighbors(G, seeds.cuda(), [5, 3], batch_ptr=RAGGED, batch_index_base=7, rng_key=11,
                              **kw).to_host()
    ref = _oracle_ragged(oracle_lib, O, seeds.numpy(), RAGGED, [5, 3], oracle_lib.sample_neighbors,
                         rng_key=11, **kw)
    assert len(out) == len(ref)
    for b, r in enumerate(ref):
        if r is None:  # an empty batch: empty blocks
            for l in range(2):
                assert len(out[b][l]["row_map"]) == 0 and len(out[b][l]["eid"]) == 0
            continue
        compare_all([out[b]], [r], f"ragged {mode} batch {b}")


def test_ragged_fixed_equivalence(gs, tiny):
    """Equal-size batch_ptr == the fixed-batch call, byte for byte."""
    g, G, O = tiny
    seeds = synth.make_seeds("tiny", 512).cuda()
    a = gs.sample_neighbors(G, seeds, [4, 4], batch_size=128, rng_key=3).to_host()
    b = gs.sample_neighbors(G, seeds, [4, 4], batch_ptr=[0, 128, 256, 384, 512], rng_key=3).to_host()
    compare_all(a, b, "ragged == fixed")


@pytest.mark.parametrize("ragged", [False, True])
def test_induce_subgraph_matches_shadow_oracle(gs, oracle_lib, tiny, ragged):
    g, G, O = tiny
    seeds = synth.make_seeds("tiny", 512)
    if ragged:
        nw = gs.sample_neighbors(G, seeds.cuda(), [6, 3], batch_ptr=RAGGED, batch_index_base=7, rng_key=5)
    else:
        nw = gs.sample_neighbors(G, seeds.cuda(), [6, 3], batch_size=128, batch_index_base=7, rng_key=5)
    ind = gs.induce_subgraph(G, nw).to_host()
    if ragged:
        ref = []
        for b in range(len(RAGGED) - 1):
            s = seeds.numpy()[RAGGED[b]:RAGGED[b + 1]]
            ref.append(None if len(s) == 0 else
                       oracle_lib.shadow(O, s, [6, 3], batch_size=len(s), batch_index_base=7 + b, rng_key=5)[0])
    else:
        ref = oracle_lib.shadow(O, seeds.numpy(), [6, 3], batch_size=128, batch_index_base=7, rng_key=5)
    assert len(ind) == len(ref)
    for b, r in enumerate(ref):
        blk = ind[b][0]
        if r is None:
            assert len(blk["row_map"]) == 0 and len(blk["eid"]) == 0
            continue
        for k in ["row_map", "indptr", "row_local", "eid"]:
            assert np.array_equal(blk[k], r[k]), f"induce ragged={ragged} batch {b} {k}"

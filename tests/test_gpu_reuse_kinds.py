"""GPU parity: one gs_blocks object reused across sampler kinds.

The kinds share the blocks' workspace (row bitmaps, induce staging, hash
tables) and skip clearing it when the previous call's tag says it is already
zero; a stale tag would leave bits of the previous kind's rows behind and
surface as phantom rows.  Each call of the chain below runs on the SAME
Blocks object and is compared with the CPU oracle element by element:
node-wise -> ShaDow -> node-wise -> GraphSAINT-RW -> PinSAGE-style ->
LADIES -> node-wise -> FastGCN -> ShaDow -> node-wise."""
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
def medium(gs, oracle_lib):
    g = synth.small_graph(200_000, 3_000_000, undirected=True, weights="uniform", seed=91,
                          device="cuda")
    return g, gs.Graph(g["indptr"], g["indices"], g["weights"]), oracle_lib.Graph(*host_graph(g))


def test_blocks_reused_across_kinds(gs, oracle_lib, medium):
    g, G, O = medium
    seeds = synth.make_seeds(synth.GraphSpec("m", 200_000, 1, True, None, 12), 2500)
    s_np, s_cu = seeds.numpy(), seeds.cuda()
    out = gs.Blocks()

    def nodewise(key):
        got = gs.sample_neighbors(G, s_cu, [10, 5], batch_size=1000, rng_key=key, out=out).to_host()
        ref = oracle_lib.sample_neighbors(O, s_np, [10, 5], batch_size=1000, rng_key=key)
        compare_all(got, ref, f"node-wise key {key}")

    nodewise(1)
    got = gs.sample_shadow(G, s_cu, [6, 4], batch_size=1000, rng_key=2, out=out).to_host()
    ref = oracle_lib.shadow(O, s_np, [6, 4], batch_size=1000, rng_key=2)
    compare_all(got, [[r] for r in ref], "shadow after node-wise")
    nodewise(3)
    got = gs.sample_saint_rw(G, s_cu, 2, batch_size=1000, rng_key=4, out=out).to_host()
    ref = oracle_lib.saint_rw(O, s_np, 2, batch_size=1000, rng_key=4)
    compare_all(got, [[r] for r in ref], "saint after node-wise")
    got = gs.sample_pinsage(G, s_cu, [6, 4], 8, 3, 0.5, batch_size=1000, rng_key=5, out=out).to_host()
    ref = oracle_lib.pinsage(O, s_np, [6, 4], 8, 3, 0.5, batch_size=1000, rng_key=5)
    compare_all(got, ref, "pinsage after saint")
    got = gs.sample_layerwise(G, s_cu, [256, 256], batch_size=500, prob_mode=gs.LADIES, rng_key=6,
                              out=out).to_host()
    ref = oracle_lib.sample_layerwise(O, s_np, [256, 256], batch_size=500, prob_mode=gs.LADIES, rng_key=6)
    compare_all(got, ref, "ladies after pinsage")
    nodewise(7)
    got = gs.sample_layerwise(G, s_cu, [256, 256], batch_size=500, prob_mode=gs.DEGREE, rng_key=8,
                              out=out).to_host()
    ref = oracle_lib.sample_layerwise(O, s_np, [256, 256], batch_size=500, prob_mode=gs.DEGREE, rng_key=8)
    compare_all(got, ref, "fastgcn after node-wise")
    got = gs.sample_shadow(G, s_cu, [6, 4], batch_size=1000, rng_key=9, out=out).to_host()
    ref = oracle_lib.shadow(O, s_np, [6, 4], batch_size=1000, rng_key=9)
    compare_all(got, [[r] for r in ref], "shadow after fastgcn")
    nodewise(10)
    torch.cuda.synchronize()

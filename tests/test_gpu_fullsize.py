"""GPU parity at BASELINE.json's full sizes, in the launch configuration bench.py
times (whole epoch in one call), checked on sampled batches / walkers the CPU
oracle recomputes one by one (same global batch / walker index -> same
Philox counters).  Integers bit-exact, fp32 values within 1e-5 relative.

  configs[1]  GraphSAGE [25,10], batch 1024, PD-shaped, full epoch
  configs[2]  LADIES / FastGCN 512 x 3 layers, LJ-shaped, all nodes as seeds
  configs[3]  DeepWalk / Node2Vec (p=2, q=0.5), length 80, FS-shaped, one walker per node
  configs[4]  GraphSAGE [15,10,5] A-Res, PP-shaped
  + ShaDow [10,5] and PASS-style [10,10] on PD-shaped graphs (M6).
"""
import gc

import numpy as np
import pytest
import torch

import synth
from tests.parity import compare_block

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def gs():
    from paper_conf_sosp_gonglmc0lwl23_b200 import gs as _gs
    _gs.load_library()
    _gs.use_torch_allocator()
    return _gs


def _graph(name, oracle_lib, gs):
    g = synth.make_graph(name, device="cuda")
    G = gs.Graph(g["indptr"], g["indices"], g["weights"])
    O = oracle_lib.Graph(g["indptr"].cpu().numpy(), g["indices"].cpu().numpy(),
                         None if g["weights"] is None else g["weights"].cpu().numpy())
    return g, G, O


def _pick(nbatches, n=6, seed=0):
    rng = np.random.default_rng(seed)
    picks = {0, nbatches - 1} | set(rng.integers(0, nbatches, n).tolist())
    return sorted(picks)


def _check_batches(gs, oracle_lib, G, O, seeds, blocks, picks, bs, call):
    blocks.sync()
    s = seeds.cpu().numpy()
    for b in picks:
        ref = call(O, s[b * bs:(b + 1) * bs], b)
        for l, rb in enumerate(ref[0]):
            v = blocks.view(b, l)
            gb = {k: (None if x is None else x.cpu().numpy()) for k, x in v.items()}
            compare_block(gb, rb, f"batch {b} layer {l}")


def test_graphsage_pd_full_epoch(gs, oracle_lib):
    g, G, O = _graph("PD", oracle_lib, gs)
    seeds = synth.make_seeds("PD", 196_615, device="cuda")
    out = gs.sample_neighbors(G, seeds, [25, 10], batch_size=1024, rng_key=0x5EED)
    nb = (196_615 + 1023) // 1024
    _check_batches(gs, oracle_lib, G, O, seeds, out, _pick(nb), 1024,
                   lambda O_, s, b: oracle_lib.sample_neighbors(O_, s, [25, 10], batch_size=1024,
                                                                batch_index_base=b,
                                                                rng_key=0x5EED))
    # whole-epoch invariants: every edge exists, rows unique per block
    out.sync()
    meta = out.device_meta().cpu().numpy()
    assert meta[:, 0, 0].sum() == 196_615
    assert meta[:, :, 2].sum() > 25_000_000


@pytest.mark.parametrize("mode", [0, 2])
def test_pass_and_kgcn_pd(gs, oracle_lib, mode):
    g, G, O = _graph("PDw", oracle_lib, gs)
    seeds = synth.make_seeds("PDw", 196_615, device="cuda")
    if mode == 2:
        out = gs.sample_neighbors(G, seeds, [10, 10], batch_size=1024, bias_mode=2, rng_key=3)
        call = lambda O_, s, b: oracle_lib.sample_neighbors(O_, s, [10, 10], batch_size=1024,  # noqa
                                                            batch_index_base=b, bias_mode=2,
                                                            rng_key=3)
    else:
        out = gs.sample_neighbors(G, seeds, [8, 8], batch_size=1024, replace=True, rng_key=3)
        call = lambda O_, s, b: oracle_lib.sample_neighbors(O_, s, [8, 8], batch_size=1024,  # noqa
                                                            batch_index_base=b, replace=True,
                                                            rng_key=3)
    _check_batches(gs, oracle_lib, G, O, seeds, out, _pick(193, 4, 1), 1024, call)


def test_shadow_pd(gs, oracle_lib):
    g, G, O = _graph("PD", oracle_lib, gs)
    seeds = synth.make_seeds("PD", 196_615, device="cuda")
    out = gs.sample_shadow(G, seeds, [10, 5], batch_size=1024, rng_key=4)
    s = seeds.cpu().numpy()
    for b in _pick(193, 3, 2):
        ref = oracle_lib.shadow(O, s[b * 1024:(b + 1) * 1024], [10, 5], batch_size=1024,
                                batch_index_base=b, rng_key=4)[0]
        v = out.view(b, 0)
        compare_block({k: (None if x is None else x.cpu().numpy()) for k, x in v.items()}, ref,
                      f"shadow batch {b}")


@pytest.mark.parametrize("mode", [0, 1])
def test_layerwise_lj_full(gs, oracle_lib, mode):
    g, G, O = _graph("LJ", oracle_lib, gs)
    seeds = synth.make_seeds("LJ", None, device="cuda")
    out = gs.sample_layerwise(G, seeds, [512, 512, 512], batch_size=512, prob_mode=mode,
                              rng_key=6)
    nb = (seeds.numel() + 511) // 512
    _check_batches(gs, oracle_lib, G, O, seeds, out, _pick(nb, 4, 3), 512,
                   lambda O_, s, b: oracle_lib.sample_layerwise(O_, s, [512, 512, 512],
                                                                batch_size=512,
                                                                batch_index_base=b,
                                                                prob_mode=mode, rng_key=6))


def test_ares_pp(gs, oracle_lib):
    g, G, O = _graph("PP", oracle_lib, gs)
    seeds = synth.make_seeds("PP", 1_207_179, device="cuda")
    out = gs.sample_neighbors(G, seeds, [15, 10, 5], batch_size=1024, bias_mode=1, rng_key=8)
    nb = (1_207_179 + 1023) // 1024
    _check_batches(gs, oracle_lib, G, O, seeds, out, _pick(nb, 3, 4), 1024,
                   lambda O_, s, b: oracle_lib.sample_neighbors(O_, s, [15, 10, 5],
                                                                batch_size=1024,
                                                                batch_index_base=b, bias_mode=1,
                                                                rng_key=8))
    del g, G, O, out
    gc.collect()
    torch.cuda.empty_cache()


@pytest.mark.parametrize("pq", [(1.0, 1.0), (2.0, 0.5)])
def test_walks_fs(gs, oracle_lib, pq):
    g, G, O = _graph("FS", oracle_lib, gs)
    n = g["indptr"].numel() - 1
    starts = torch.arange(n, dtype=torch.int32, device="cuda")
    tr = gs.random_walk(G, starts, 80, p=pq[0], q=pq[1], rng_key=9)
    rng = np.random.default_rng(5)
    pick = np.unique(np.concatenate([np.arange(2000), rng.integers(0, n, 4000),
                                     np.arange(n - 1000, n)]))
    got = tr[torch.from_numpy(pick).cuda()].cpu().numpy()
    del tr
    torch.cuda.empty_cache()
    # the oracle walks the same walkers (global walker index = start node here)
    ref = np.concatenate([
        oracle_lib.random_walk(O, pick[i:i + 1].astype(np.int32), 80, p=pq[0], q=pq[1],
                               walker_index_base=int(pick[i]), rng_key=9)
        for i in range(len(pick))])
    assert np.array_equal(got, ref), f"{(got != ref).sum()} trace entries differ"
    del g, G, O
    gc.collect()
    torch.cuda.empty_cache()

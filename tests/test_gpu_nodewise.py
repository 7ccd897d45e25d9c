"""GPU parity: node-wise path (GraphSAGE, KGCN, weighted A-Res, PASS-style, ShaDow)
through the C ABI vs the CPU oracle, element by element (integers bit-exact,
fp32 values within 1e-5 relative)."""
import numpy as np
import pytest
import torch

import synth
from tests.parity import compare_all, host_graph

pytestmark = pytest.mark.gpu

cuda = pytest.mark.skipif(not torch.cuda.is_available(), reason="needs a CUDA device")


@pytest.fixture(scope="module")
def gs():
    from paper_conf_sosp_gonglmc0lwl23_b200 import gs as _gs
    _gs.load_library()
    _gs.use_torch_allocator()
    return _gs


@pytest.fixture(scope="module")
def tiny(gs, oracle_lib):
    g = synth.make_graph("tiny", device="cuda")
    G = gs.Graph(g["indptr"], g["indices"], g["weights"])
    O = oracle_lib.Graph(*host_graph(g))
    return g, G, O


@pytest.fixture(scope="module")
def medium(gs, oracle_lib):
    g = synth.small_graph(200_000, 3_000_000, undirected=True, weights="uniform", seed=77,
                          device="cuda")
    G = gs.Graph(g["indptr"], g["indices"], g["weights"])
    O = oracle_lib.Graph(*host_graph(g))
    return g, G, O


@pytest.mark.parametrize("batch", [512, 128, 100])
def test_graphsage_tiny(gs, oracle_lib, tiny, batch):
    """configs[0]: GraphSAGE [5,5], 512 seeds, 10k/100k R-MAT graph."""
    g, G, O = tiny
    seeds = synth.make_seeds("tiny", 512)
    out = gs.sample_neighbors(G, seeds.cuda(), [5, 5], batch_size=batch, rng_key=0x5EED).to_host()
    ref = oracle_lib.sample_neighbors(O, seeds.numpy(), [5, 5], batch_size=batch, rng_key=0x5EED)
    compare_all(out, ref, f"graphsage tiny bs={batch}")


@pytest.mark.parametrize("fan", [[25, 10], [1, 1, 1], [32, 2], [3, 7, 2]])
def test_graphsage_medium(gs, oracle_lib, medium, fan):
    g, G, O = medium
    seeds = torch.randperm(200_000, generator=torch.Generator().manual_seed(3))[:3000].int()
    out = gs.sample_neighbors(G, seeds.cuda(), fan, batch_size=1024, rng_key=99,
                              batch_index_base=5).to_host()
    ref = oracle_lib.sample_neighbors(O, seeds.numpy(), fan, batch_size=1024, rng_key=99,
                                      batch_index_base=5)
    compare_all(out, ref, f"graphsage medium {fan}")


def test_kgcn_replace(gs, oracle_lib, medium):
    g, G, O = medium
    seeds = synth.make_seeds(synth.GraphSpec("m", 200_000, 1, True, None, 4), 2048)
    out = gs.sample_neighbors(G, seeds.cuda(), [8, 8], batch_size=512, replace=True,
                              rng_key=7).to_host()
    ref = oracle_lib.sample_neighbors(O, seeds.numpy(), [8, 8], batch_size=512, replace=True,
                                      rng_key=7)
    compare_all(out, ref, "kgcn")


@pytest.mark.parametrize("mode,split,tau", [(1, "1", "0"), (2, "1", "0"), (1, "0", "0"),
                                            (1, "1", "1"), (1, "1", "2")])
def test_weighted_ares_and_pass(gs, oracle_lib, medium, mode, split, tau, monkeypatch):
    """A-Res / PASS-style.  GS_ARES_SPLIT: 1 heavy columns (d > 64) in their
    own kernel (default), 0 inside the select kernel; GS_ARES_TAU 1 / 2 start
    the heavy-column threshold too tight / too loose so that every widen and
    narrow step of the search runs."""
    monkeypatch.setenv("GS_ARES_SPLIT", split)
    monkeypatch.setenv("GS_ARES_TAU", tau)
    g, G, O = medium
    seeds = synth.make_seeds(synth.GraphSpec("m", 200_000, 1, True, None, 5), 2048)
    out = gs.sample_neighbors(G, seeds.cuda(), [10, 10], batch_size=1024, bias_mode=mode,
                              rng_key=11).to_host()
    ref = oracle_lib.sample_neighbors(O, seeds.numpy(), [10, 10], batch_size=1024, bias_mode=mode,
                                      rng_key=11)
    compare_all(out, ref, f"ares mode {mode}")


def test_edge_cases(gs, oracle_lib, tiny):
    g, G, O = tiny
    ip = g["indptr"].cpu()
    zero_deg = torch.nonzero(ip[1:] == ip[:-1]).flatten()[:5].int()
    seeds = torch.cat([zero_deg, torch.tensor([3, 3, 3, 17], dtype=torch.int32), zero_deg])
    for fan in [[1], [32, 32], [4, 4, 4, 4]]:
        out = gs.sample_neighbors(G, seeds.cuda(), fan, batch_size=3, rng_key=1).to_host()
        ref = oracle_lib.sample_neighbors(O, seeds.numpy(), fan, batch_size=3, rng_key=1)
        compare_all(out, ref, f"edge {fan}")
    # empty seed list
    b = gs.sample_neighbors(G, torch.empty(0, dtype=torch.int32, device="cuda"), [5], batch_size=4)
    b.sync()
    assert b.num_batches == 0


def test_out_of_range_seed(gs, tiny):
    g, G, O = tiny
    seeds = torch.tensor([1, 2, 10_000, 5], dtype=torch.int32, device="cuda")
    b = gs.sample_neighbors(G, seeds, [3])
    with pytest.raises(gs.GSError) as ei:
        b.sync()
    assert ei.value.status == 5


def test_reuse_and_determinism(gs, medium):
    g, G, O = medium
    seeds = torch.arange(0, 4096, dtype=torch.int32, device="cuda") * 37 % 200_000
    a = gs.sample_neighbors(G, seeds, [25, 10], batch_size=1024, rng_key=5)
    ha = a.to_host()
    # the same object reused 300 times: generation tags wrap (255) and tables are cleared
    for i in range(300):
        gs.sample_neighbors(G, seeds, [25, 10], batch_size=1024, rng_key=5, out=a)
    hb = a.to_host()
    compare_all(hb, ha, "reuse")


def test_shard_invariance(gs, medium):
    """Union of per-rank shards (batch_index_base) == single call, bit-exact (8(e))."""
    g, G, O = medium
    seeds = torch.arange(0, 5000, dtype=torch.int32, device="cuda") * 13 % 200_000
    full = gs.sample_neighbors(G, seeds, [10, 5], batch_size=500, rng_key=3).to_host()
    for lo in range(0, 5000, 1500):
        hi = min(5000, lo + 1500)
        part = gs.sample_neighbors(G, seeds[lo:hi], [10, 5], batch_size=500, rng_key=3,
                                   batch_index_base=lo // 500).to_host()
        compare_all(part, full[lo // 500: hi // 500 + (1 if hi % 500 else 0)], "shard")


@pytest.mark.parametrize("cs", [None, "2", "4"])
@pytest.mark.parametrize("wcap", [None, "40"])
@pytest.mark.parametrize("mode", [0, 1])
def test_shadow(gs, oracle_lib, medium, mode, wcap, cs, monkeypatch):
    """ShaDow vs the oracle; wcap = 40 shrinks the induce kernel's per-warp
    staging so that most columns take the re-stream path; cs forces a 2- or
    4-CTA cluster (the U bitmap split across peers' shared memory)."""
    if wcap:
        monkeypatch.setenv("GS_SH_WCAP", wcap)
    if cs:
        monkeypatch.setenv("GS_SH_CS", cs)
    g, G, O = medium
    seeds = synth.make_seeds(synth.GraphSpec("m", 200_000, 1, True, None, 6), 1000)
    out = gs.sample_shadow(G, seeds.cuda(), [10, 5], batch_size=256, bias_mode=mode,
                           rng_key=21).to_host()
    ref = oracle_lib.shadow(O, seeds.numpy(), [10, 5], batch_size=256, bias_mode=mode, rng_key=21)
    compare_all(out, [[r] for r in ref], f"shadow {mode}")


@pytest.mark.parametrize("narrow", [False, True])
@pytest.mark.parametrize("kind", ["nodewise", "layerwise"])
def test_pack_matches_views(gs, medium, kind, narrow):
    """gs_blocks_pack (and gs_blocks_pack_narrow, int32 ids): every batch's
    block, packed densely in batch order, is exactly its view (indptr
    block-relative), and `totals` are the sums."""
    g, G, O = medium
    seeds = synth.make_seeds(synth.GraphSpec("m", 200_000, 1, False, None, 12), 5000).cuda()
    if kind == "nodewise":
        out = gs.sample_neighbors(G, seeds, [7, 3], batch_size=700, rng_key=21)
    else:
        out = gs.sample_layerwise(G, seeds, [300, 300], batch_size=700, prob_mode=1, rng_key=21)
    out.sync()
    for l in range(2):
        pk = out.pack(l, narrow=narrow)
        torch.cuda.synchronize()
        if narrow:
            pk = {k: (v.long() if k in ("eid", "indptr") else v) for k, v in pk.items()}
        tot = pk["totals"].cpu().tolist()
        e = i = r = 0
        for b in range(out.num_batches):
            v = out.view(b, l)
            ne, nc, nr = v["eid"].numel(), v["indptr"].numel(), v["row_map"].numel()
            assert torch.equal(pk["row_local"][e:e + ne], v["row_local"])
            assert torch.equal(pk["eid"][e:e + ne], v["eid"])
            assert torch.equal(pk["indptr"][i:i + nc], v["indptr"])
            assert torch.equal(pk["row_map"][r:r + nr], v["row_map"])
            e, i, r = e + ne, i + nc, r + nr
        assert tot == [e, i, r]


@pytest.mark.parametrize("rowmode", ["auto", "GS_HOP_SPARSE", "GS_HOP_DENSE"])
@pytest.mark.parametrize("layout", ["0", "1"])
@pytest.mark.parametrize("fan", [[25, 10], [15, 10, 5]])
def test_row_bitmap_layouts(gs, oracle_lib, medium, fan, layout, rowmode, monkeypatch):
    """Both row-bitmap layouts of the node-wise engine (GS_HOP_LAYOUT: 1 = the
    rank inside each 96-node group, the default below 2^24 nodes; 0 = bits
    only with a rank per 128 nodes beside them, the default above), each with
    row() chosen by density or forced to the summary (sparse) or dense scan,
    uniform and weighted, against the oracle."""
    monkeypatch.setenv("GS_HOP_LAYOUT", layout)
    if rowmode != "auto":
        monkeypatch.setenv(rowmode, "1")
    g, G, O = medium
    seeds = synth.make_seeds(synth.GraphSpec("m", g["indptr"].numel() - 1, 1, True, None, 31), 3000)
    for bias in (0, 1):
        out = gs.sample_neighbors(G, seeds.cuda(), fan, batch_size=512, bias_mode=bias, rng_key=12).to_host()
        ref = oracle_lib.sample_neighbors(O, seeds.numpy(), fan, batch_size=512, bias_mode=bias, rng_key=12)
        compare_all(out, ref, f"layout {layout} bias {bias} fan {fan}")

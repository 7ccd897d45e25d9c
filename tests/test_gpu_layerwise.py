"""GPU parity: layer-wise path (LADIES / FastGCN / COUNT) vs the oracle.
Integers (row_map = S, indptr, row_local, eid) bit-exact; val and row_prob
within 1e-5 relative (north_star)."""
import numpy as np
import pytest
import torch

import synth
from tests.graphs_small import B, E, fig1_graph
from tests.parity import compare_all, host_graph

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def gs():
    from paper_conf_sosp_gonglmc0lwl23_b200 import gs as _gs
    _gs.load_library()
    _gs.use_torch_allocator()
    return _gs


@pytest.fixture(params=["sm", "bm", "old"], autouse=True)
def lw_path(request, monkeypatch):
    """Every test runs through every layer-wise kernel: the shared-memory
    kernel (layerwise_sm.cu, LADIES / COUNT default), the candidate-bitmap
    kernel (layerwise_bm.cu, FastGCN default) and the global hash-table kernel
    (layerwise.cu, the fallback)."""
    monkeypatch.setenv("GS_LW_PATH", request.param)
    return request.param


@pytest.fixture(scope="module")
def ljlike(gs, oracle_lib):
    # LiveJournal-shaped (directed, GCN-normalised weights) at reduced size
    g = synth.small_graph(300_000, 4_300_000, undirected=False, weights="gcn", seed=17,
                          device="cuda")
    return g, gs.Graph(g["indptr"], g["indices"], g["weights"]), oracle_lib.Graph(*host_graph(g))


@pytest.mark.parametrize("mode", [0, 1, 2])
def test_layerwise_parity(gs, oracle_lib, ljlike, mode):
    g, G, O = ljlike
    seeds = synth.make_seeds(synth.GraphSpec("lj", 300_000, 1, False, None, 8), 4000)
    out = gs.sample_layerwise(G, seeds.cuda(), [512, 512, 512], batch_size=512, prob_mode=mode,
                              rng_key=33, batch_index_base=2).to_host()
    ref = oracle_lib.sample_layerwise(O, seeds.numpy(), [512, 512, 512], batch_size=512,
                                      prob_mode=mode, rng_key=33, batch_index_base=2)
    compare_all(out, ref, f"layerwise mode {mode}")


@pytest.mark.parametrize("K", [1, 7, 64, 4096])
def test_layerwise_K(gs, oracle_lib, ljlike, K):
    g, G, O = ljlike
    seeds = torch.arange(0, 300_000, 997, dtype=torch.int32)
    out = gs.sample_layerwise(G, seeds.cuda(), [K, K], batch_size=100, prob_mode=0,
                              rng_key=4).to_host()
    ref = oracle_lib.sample_layerwise(O, seeds.numpy(), [K, K], batch_size=100, prob_mode=0,
                                      rng_key=4)
    compare_all(out, ref, f"layerwise K={K}")


def test_fig1_toy(gs, oracle_lib):
    ip, ix, w = fig1_graph()
    G = gs.Graph(torch.from_numpy(ip).cuda(), torch.from_numpy(ix).cuda(), torch.from_numpy(w).cuda())
    O = oracle_lib.Graph(ip, ix, w)
    seeds = np.array([B, E] * 50, np.int32)
    for K in [2, 4, 5]:
        out = gs.sample_layerwise(G, torch.from_numpy(seeds).cuda(), [K], batch_size=2,
                                  rng_key=K).to_host()
        ref = oracle_lib.sample_layerwise(O, seeds, [K], batch_size=2, rng_key=K)
        compare_all(out, ref, f"fig1 K={K}")
        if K == 5:  # B_f = 0.58; p(f) = 0.58 / 2.08
            assert out[0][0]["row_prob"][2] == pytest.approx(0.58 / 2.08, rel=1e-6)


def test_unit_weights_count_identity(gs, ljlike):
    g, G, O = ljlike
    G1 = gs.Graph(g["indptr"], g["indices"], torch.ones_like(g["weights"]))
    seeds = torch.arange(0, 300_000, 211, dtype=torch.int32, device="cuda")
    a = gs.sample_layerwise(G1, seeds, [256, 256], batch_size=300, prob_mode=0, rng_key=5).to_host()
    b = gs.sample_layerwise(G1, seeds, [256, 256], batch_size=300, prob_mode=2, rng_key=5).to_host()
    compare_all(a, b, "ladies(w=1) == count")


def test_capacity_retry(gs, oracle_lib, ljlike):
    """A tiny initial edge capacity overflows; the binding grows it and re-runs."""
    g, G, O = ljlike
    seeds = synth.make_seeds(synth.GraphSpec("lj", 300_000, 1, False, None, 9), 2048)
    out = gs.sample_layerwise(G, seeds.cuda(), [2048], batch_size=2048, prob_mode=1, rng_key=1)
    ref = oracle_lib.sample_layerwise(O, seeds.numpy(), [2048], batch_size=2048, prob_mode=1,
                                      rng_key=1)
    compare_all(out.to_host(), ref, "fastgcn big")


def test_ladies_bias_capacity_retry(gs, oracle_lib, ljlike):
    """LADIES batch-layers with more candidates than the initial b(u) capacity
    (32 Ki) overflow once; the binding grows the workspace and re-runs."""
    g, G, O = ljlike
    seeds = synth.make_seeds(synth.GraphSpec("lj", 300_000, 1, False, None, 10), 6000)
    out = gs.sample_layerwise(G, seeds.cuda(), [3000, 3000], batch_size=3000, prob_mode=0, rng_key=2)
    ref = oracle_lib.sample_layerwise(O, seeds.numpy(), [3000, 3000], batch_size=3000, prob_mode=0,
                                      rng_key=2)
    compare_all(out.to_host(), ref, "ladies big")


@pytest.mark.parametrize("ccap", [None, "3", "0"])
def test_fastgcn_threshold_reuse(gs, oracle_lib, ljlike, monkeypatch, lw_path, ccap):
    """One CTA walks every batch, so from the second batch on the bitmap
    kernel's extract filters against the previous batch's threshold (the
    fused select) and stages the candidate rows' edges for the finalize; the
    result must not depend on it (ccap 3: most warps overflow their staging and
    stream A[:, F] again; 0: no staging)."""
    if lw_path != "bm":
        pytest.skip("bitmap-kernel path")
    monkeypatch.setenv("GS_LW_CTAS", "1")
    if ccap is not None:
        monkeypatch.setenv("GS_LW_CCAP", ccap)
    g, G, O = ljlike
    seeds = synth.make_seeds(synth.GraphSpec("lj", 300_000, 1, False, None, 11), 512 * 12)
    for K in (64, 512):
        out = gs.sample_layerwise(G, seeds.cuda(), [K, K, K], batch_size=512, prob_mode=1, rng_key=K)
        ref = oracle_lib.sample_layerwise(O, seeds.numpy(), [K, K, K], batch_size=512, prob_mode=1,
                                          rng_key=K)
        compare_all(out.to_host(), ref, f"fastgcn one CTA K={K}")


def test_fastgcn_emit_restream(gs, oracle_lib, ljlike, monkeypatch, lw_path):
    """The bitmap kernel copies the kept edges its L5a pass staged; with a
    staging capacity of 2 edges per warp every batch-layer takes the
    re-stream emit instead -- same blocks."""
    if lw_path != "bm":
        pytest.skip("bitmap-kernel path")
    monkeypatch.setenv("GS_LW_SCAP", "2")
    g, G, O = ljlike
    seeds = synth.make_seeds(synth.GraphSpec("lj", 300_000, 1, False, None, 14), 2048)
    for mode in (1, 0):
        out = gs.sample_layerwise(G, seeds.cuda(), [512, 512], batch_size=512, prob_mode=mode, rng_key=5)
        ref = oracle_lib.sample_layerwise(O, seeds.numpy(), [512, 512], batch_size=512, prob_mode=mode,
                                          rng_key=5)
        compare_all(out.to_host(), ref, f"restream emit mode {mode}")


def test_sm_big_frontier(gs, oracle_lib, ljlike, lw_path):
    """Shared-memory kernel (layerwise_sm.cu) with 1024-column frontiers and
    K = 1024: batch-layers of more than one register chunk (re-streamed per
    pass) and several hash partitions, besides the one-chunk / one-partition
    common case."""
    if lw_path != "sm":
        pytest.skip("shared-memory kernel path")
    cfg = "1024x12"
    g, G, O = ljlike
    seeds = synth.make_seeds(synth.GraphSpec("lj", 300_000, 1, False, None, 21), 1024 * 5 + 300)
    for mode in (0, 2):
        out = gs.sample_layerwise(G, seeds.cuda(), [1024, 1024], batch_size=1024, prob_mode=mode,
                                  rng_key=77)
        ref = oracle_lib.sample_layerwise(O, seeds.numpy(), [1024, 1024], batch_size=1024,
                                          prob_mode=mode, rng_key=77)
        compare_all(out.to_host(), ref, f"sm cfg {cfg} mode {mode}")


@pytest.fixture(scope="module")
def hubby(gs, oracle_lib):
    # undirected power-law graph: LADIES frontiers pick hubs, so the later
    # layers extract tens of thousands of edges per batch (many chunks and
    # partitions in the shared-memory kernel)
    g = synth.small_graph(100_000, 3_000_000, undirected=True, weights="gcn", seed=23, device="cuda")
    return g, gs.Graph(g["indptr"], g["indices"], g["weights"]), oracle_lib.Graph(*host_graph(g))


def test_ladies_hub_frontiers(gs, oracle_lib, hubby, lw_path):
    if lw_path == "bm":
        pytest.skip("LADIES on the bitmap kernel is covered above")
    g, G, O = hubby
    seeds = synth.make_seeds(synth.GraphSpec("pd", 100_000, 1, True, None, 5), 512 * 4 + 17)
    out = gs.sample_layerwise(G, seeds.cuda(), [512, 256, 512], batch_size=512, prob_mode=0, rng_key=8)
    ref = oracle_lib.sample_layerwise(O, seeds.numpy(), [512, 256, 512], batch_size=512, prob_mode=0,
                                      rng_key=8)
    compare_all(out.to_host(), ref, "ladies hub frontiers")


def test_ladies_zero_weights(gs, oracle_lib, ljlike):
    """A third of the edge weights set to zero: rows whose b(u) = sum w^2 is 0
    are ineligible (R6, R24), rows mixing zero and non-zero edges keep their
    positive b -- every kernel against the oracle."""
    g, G, O = ljlike
    w = g["weights"].clone()
    w[torch.arange(w.numel(), device=w.device) % 3 == 0] = 0.0
    Gz = gs.Graph(g["indptr"], g["indices"], w)
    Oz = oracle_lib.Graph(g["indptr"].cpu().numpy(), g["indices"].cpu().numpy(), w.cpu().numpy())
    seeds = synth.make_seeds(synth.GraphSpec("lj", 300_000, 1, False, None, 41), 2500)
    for K in (64, 512):
        out = gs.sample_layerwise(Gz, seeds.cuda(), [K, K], batch_size=500, prob_mode=0, rng_key=K + 1)
        ref = oracle_lib.sample_layerwise(Oz, seeds.numpy(), [K, K], batch_size=500, prob_mode=0, rng_key=K + 1)
        compare_all(out.to_host(), ref, f"ladies zero weights K={K}")

"""GPU parity: GraphSAINT-RW (Table 2; DESIGN R26) through
gs_sample_saint_rw (walk kernel + cluster induce kernel) vs the CPU oracle,
element by element (integers bit-exact): several batches with a ragged tail,
walk_length 0, dead-end roots, the re-stream fallback of the induce kernel,
global batch keying, out-of-range roots, and the full PD-shaped epoch the bench
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


@pytest.mark.parametrize("L,bs", [(2, 300), (4, 128), (0, 97), (1, 1000)])
def test_saint_tiny(gs, oracle_lib, tiny, L, bs):
    g, G, O = tiny
    roots = synth.make_seeds("tiny", 1000)   # ragged last batch for bs 300 / 128 / 97
    out = gs.sample_saint_rw(G, roots.cuda(), L, batch_size=bs, rng_key=0xA11).to_host()
    ref = oracle_lib.saint_rw(O, roots.numpy(), L, batch_size=bs, rng_key=0xA11)
    compare_all(out, [[r] for r in ref], f"saint L={L} bs={bs}")


def test_saint_dead_end_roots(gs, oracle_lib, tiny):
    g, G, O = tiny
    ip = g["indptr"].cpu()
    dead = torch.nonzero(ip[1:] == ip[:-1]).flatten()[:50].to(torch.int32)
    assert dead.numel() > 0
    roots = torch.cat([dead, synth.make_seeds("tiny", 150)]).to(torch.int32)
    out = gs.sample_saint_rw(G, roots.cuda(), 3, batch_size=64, rng_key=5).to_host()
    ref = oracle_lib.saint_rw(O, roots.numpy(), 3, batch_size=64, rng_key=5)
    compare_all(out, [[r] for r in ref], "saint dead ends")


@pytest.mark.parametrize("cs", [None, "2"])
@pytest.mark.parametrize("wcap", [None, "40"])
def test_saint_medium(gs, oracle_lib, medium, wcap, cs, monkeypatch):
    """wcap = 40 shrinks the induce kernel's per-warp staging so that most
    columns take the re-stream path; cs = 2 forces a 2-CTA cluster."""
    if wcap:
        monkeypatch.setenv("GS_SH_WCAP", wcap)
    if cs:
        monkeypatch.setenv("GS_SH_CS", cs)
    g, G, O = medium
    roots = synth.make_seeds(synth.GraphSpec("m", 200_000, 1, True, None, 6), 7000)
    out = gs.sample_saint_rw(G, roots.cuda(), 3, batch_size=3000, rng_key=23).to_host()
    ref = oracle_lib.saint_rw(O, roots.numpy(), 3, batch_size=3000, rng_key=23)
    compare_all(out, [[r] for r in ref], "saint medium")


def test_saint_batch_keying(gs, medium):
    """Results depend on the global batch index only (shard invariance)."""
    g, G, O = medium
    roots = synth.make_seeds(synth.GraphSpec("m", 200_000, 1, True, None, 8), 4000).cuda()
    full = gs.sample_saint_rw(G, roots, 2, batch_size=1000, rng_key=3).to_host()
    part = gs.sample_saint_rw(G, roots[2000:], 2, batch_size=1000, batch_index_base=2,
                              rng_key=3).to_host()
    for b in range(2):
        for k in ["row_map", "indptr", "row_local", "eid"]:
            assert np.array_equal(part[b][0][k], full[b + 2][0][k])


def test_saint_bad_root(gs, tiny):
    g, G, O = tiny
    roots = torch.tensor([1, 2, 10_000, 3], dtype=torch.int32, device="cuda")
    with pytest.raises(gs.GSError) as e:
        gs.sample_saint_rw(G, roots, 2, batch_size=2)
    assert e.value.status == 5


def test_saint_pd_full_epoch(gs, oracle_lib):
    """The bench workload: every PD node a root once, 3000 roots per subgraph,
    walk length 2 (817 subgraphs in one call); sampled batches vs the oracle."""
    g = synth.make_graph("PD", device="cuda")
    G = gs.Graph(g["indptr"], g["indices"], g["weights"])
    O = oracle_lib.Graph(g["indptr"].cpu().numpy(), g["indices"].cpu().numpy(), None)
    roots = synth.make_seeds("PD", None, device="cuda")
    bs = 3000
    nb = (roots.numel() + bs - 1) // bs
    out = gs.sample_saint_rw(G, roots, 2, batch_size=bs, rng_key=0x5A1)
    s = roots.cpu().numpy()
    rng = np.random.default_rng(1)
    for b in sorted({0, nb - 1} | set(rng.integers(0, nb, 3).tolist())):
        ref = oracle_lib.saint_rw(O, s[b * bs:(b + 1) * bs], 2, batch_size=bs,
                                  batch_index_base=b, rng_key=0x5A1)[0]
        v = out.view(b, 0)
        compare_block({k: (None if x is None else x.cpu().numpy()) for k, x in v.items()}, ref,
                      f"saint PD batch {b}")


def test_saint_empty(gs, tiny):
    g, G, O = tiny
    out = gs.sample_saint_rw(G, torch.zeros(0, dtype=torch.int32, device="cuda"), 3, batch_size=10)
    assert out.to_host() == []

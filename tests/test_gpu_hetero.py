"""GPU parity: heterogeneous node-wise sampling (gs_sample_neighbors_hetero,
P:351: one CSC per edge type sampled by the homogeneous workflow; SURVEY 8(f)
f4) against oracle/ops.py hetero_sample_neighbors, bit-exact: every block
(columns, indptr, rows, eids) and every per-type frontier."""
import numpy as np
import pytest
import torch

import synth
from oracle import ops as oops

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def gs():
    from paper_conf_sosp_gonglmc0lwl23_b200 import gs as _gs
    _gs.load_library()
    _gs.use_torch_allocator()
    return _gs


def _relation(seed, n_src, n_dst, nnz):
    """A bipartite edge type: CSC with max(n_src, n_dst) columns, rows < n_src,
    only the first n_dst columns non-empty (R-MAT pairs folded into range)."""
    n = max(n_src, n_dst)
    g = synth.small_graph(n, nnz, undirected=False, weights=None, seed=seed)
    ip, ix = g["indptr"].numpy(), g["indices"].numpy()
    cols, rows = [], []
    for v in range(min(n, n_dst)):
        r = ix[ip[v]:ip[v + 1]] % n_src
        r = np.unique(r)
        rows.append(r.astype(np.int32))
    indptr = np.zeros(n + 1, np.int64)
    indptr[1:len(rows) + 1] = np.cumsum([len(r) for r in rows])
    indptr[len(rows) + 1:] = indptr[len(rows)]
    indices = np.concatenate(rows) if rows else np.zeros(0, np.int32)
    return indptr, indices


@pytest.fixture(scope="module")
def academic(gs):
    # node types: 0 author (30k), 1 paper (50k), 2 field (2k); edge types:
    # writes (author -> paper), cites (paper -> paper), has_topic (field -> paper),
    # written_by (paper -> author)
    nn = [30_000, 50_000, 2_000]
    spec = [(0, 1, 11, 400_000), (1, 1, 12, 600_000), (2, 1, 13, 150_000), (1, 0, 14, 400_000)]
    rels_h, rels_d = [], []
    for st, dt, seed, nnz in spec:
        ip, ix = _relation(seed, nn[st], nn[dt], nnz)
        rels_h.append((st, dt, ip, ix))
        rels_d.append((st, dt, gs.Graph(torch.from_numpy(ip).cuda(), torch.from_numpy(ix).cuda())))
    return nn, rels_h, rels_d


@pytest.mark.parametrize("fanouts", [[[5, 5, 3, 4], [3, 2, 0, 2]], [[10, 0, 0, 0]], [[2, 2, 2, 2]] * 3])
def test_hetero_matches_oracle(gs, academic, fanouts):
    nn, rels_h, rels_d = academic
    seeds = [np.zeros(0, np.int32), np.random.default_rng(3).choice(nn[1], 600, replace=False).astype(np.int32),
             np.zeros(0, np.int32)]
    got = gs.sample_neighbors_hetero(rels_d, nn, [torch.from_numpy(s).cuda() for s in seeds], fanouts, rng_key=99)
    blocks, fr = oops.hetero_sample_neighbors(rels_h, nn, seeds, fanouts, rng_key=99)
    for l in range(len(fanouts)):
        for r in range(len(rels_h)):
            a, b = got.blocks[l][r], blocks[l][r]
            assert (a is None) == (b is None), (l, r)
            if b is None:
                continue
            for k in ("cols", "indptr", "row", "eid"):
                assert np.array_equal(a[k].cpu().numpy(), b[k]), (l, r, k)
    for l in range(len(fanouts) + 1):
        for t in range(3):
            assert np.array_equal(got.frontiers[l][t].cpu().numpy(), fr[l][t]), (l, t)


def test_hetero_rejects_bad_relation(gs, academic):
    nn, rels_h, rels_d = academic
    bad = [(0, 1, rels_d[0][2]), (1, 5, rels_d[1][2])]
    with pytest.raises(gs.GSError):
        gs.sample_neighbors_hetero(bad, nn, [torch.zeros(0, dtype=torch.int32, device="cuda")] * 3, [[1, 1]])

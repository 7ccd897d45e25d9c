"""N>1 host path on CPU: world_size-2 gloo process group.

Rank 0 generates the graph and broadcasts it (dist.broadcast_graph); each rank
samples its shard of the epoch keyed by GLOBAL batch ids; the union over ranks
must equal a single-process run bit for bit (shard invariance).
The sampler here is the CPU oracle standing in for the kernels (no GPU in this
container); the GPU shard-invariance test is tests/test_gpu_nodewise.py.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_sosp_gonglmc0lwl23_b200 import dist as gdist


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out_dir):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import oracle
    import synth
    g = synth.make_graph("tiny") if rank == 0 else None
    g = gdist.broadcast_graph(g, torch.device("cpu"))
    seeds = synth.make_seeds("tiny", 600)  # same on every rank (deterministic)
    bs = 64
    nb = (600 + bs - 1) // bs
    s0, s1, lo = gdist.shard_epoch(600, bs, world, rank)  # the split bench.py uses
    hi = (s1 + bs - 1) // bs
    O = oracle.Graph(g["indptr"].numpy(), g["indices"].numpy(), g["weights"].numpy())
    res = oracle.sample_neighbors(O, seeds[s0:s1].numpy(), [5, 3], batch_size=bs,
                                  batch_index_base=lo, rng_key=77)
    # GraphSAINT-RW and PinSAGE-style shard the same way (global batch ids)
    sa = oracle.saint_rw(O, seeds[s0:s1].numpy(), 3, batch_size=bs, batch_index_base=lo,
                         rng_key=78)
    np.save(os.path.join(out_dir, f"saint_{rank}.npy"), np.concatenate([b["eid"] for b in sa]))
    ps = oracle.pinsage(O, seeds[s0:s1].numpy(), [4, 2], 6, 3, 0.4, batch_size=bs,
                        batch_index_base=lo, rng_key=79)
    np.save(os.path.join(out_dir, f"pinsage_{rank}.npy"),
            np.concatenate([blk["row_map"][blk["row_local"]] for layers in ps for blk in layers]))
    # layer-wise shards by batches, walks by contiguous walker ranges (shard_epoch)
    lw = oracle.sample_layerwise(O, seeds[s0:s1].numpy(), [16, 16], batch_size=bs, batch_index_base=lo,
                                 prob_mode=0, rng_key=81)
    np.save(os.path.join(out_dir, f"lw_{rank}.npy"), np.concatenate([blk["eid"] for layers in lw for blk in layers]))
    w0, w1, wbase = gdist.shard_epoch(600, None, world, rank)
    tr = oracle.random_walk(O, seeds[w0:w1].numpy(), 6, p=2.0, q=0.5, walker_index_base=wbase, rng_key=80)
    np.save(os.path.join(out_dir, f"walk_{rank}.npy"), tr)
    edges = sum(len(blk["eid"]) for layers in res for blk in layers)
    tot_edges, max_ms = gdist.reduce_measurement(edges, 10.0 + rank, torch.device("cpu"))
    np.save(os.path.join(out_dir, f"eids_{rank}.npy"),
            np.concatenate([blk["eid"] for layers in res for blk in layers]))
    np.save(os.path.join(out_dir, f"meta_{rank}.npy"), np.array([lo, hi, tot_edges, max_ms]))
    np.save(os.path.join(out_dir, f"graph_{rank}.npy"), g["indices"].numpy()[:1000])
    dist.barrier()
    dist.destroy_process_group()


def test_shard_ranges():
    for nb in [1, 7, 193, 1000]:
        for w in [1, 2, 3, 8]:
            rs = [gdist.shard_range(nb, w, r) for r in range(w)]
            assert rs[0][0] == 0 and rs[-1][1] == nb
            assert all(a[1] == b[0] for a, b in zip(rs, rs[1:]))
            sizes = [h - l for l, h in rs]
            assert max(sizes) - min(sizes) <= 1
    assert gdist.weak_batch_base(3, 193) == 579
    # shard_epoch: batch slices cover the epoch in order; walker slices likewise
    for n, bs in [(600, 64), (196615, 1024), (5, 8)]:
        parts = [gdist.shard_epoch(n, bs, 3, r) for r in range(3)]
        assert parts[0][0] == 0 and parts[-1][1] == n and all(a[1] == b[0] for a, b in zip(parts, parts[1:]))
        assert all(p[0] == min(n, p[2] * bs) for p in parts)
    parts = [gdist.shard_epoch(10, None, 4, r) for r in range(4)]
    assert [p[:2] for p in parts] == [(0, 3), (3, 6), (6, 8), (8, 10)] and all(p[0] == p[2] for p in parts)


def test_two_rank_gloo_shard_invariance(tmp_path, oracle_lib):
    import synth
    world = 2
    mp.spawn(_worker, args=(world, _free_port(), str(tmp_path)), nprocs=world, join=True)
    g = synth.make_graph("tiny")
    seeds = synth.make_seeds("tiny", 600).numpy()
    O = oracle_lib.Graph(g["indptr"].numpy(), g["indices"].numpy(), g["weights"].numpy())
    full = oracle_lib.sample_neighbors(O, seeds, [5, 3], batch_size=64, rng_key=77)
    want = np.concatenate([blk["eid"] for layers in full for blk in layers])
    got = np.concatenate([np.load(tmp_path / f"eids_{r}.npy") for r in range(world)])
    assert np.array_equal(got, want)
    sa = oracle_lib.saint_rw(O, seeds, 3, batch_size=64, rng_key=78)
    got = np.concatenate([np.load(tmp_path / f"saint_{r}.npy") for r in range(world)])
    assert np.array_equal(got, np.concatenate([b["eid"] for b in sa]))
    ps = oracle_lib.pinsage(O, seeds, [4, 2], 6, 3, 0.4, batch_size=64, rng_key=79)
    got = np.concatenate([np.load(tmp_path / f"pinsage_{r}.npy") for r in range(world)])
    assert np.array_equal(got, np.concatenate([blk["row_map"][blk["row_local"]]
                                               for layers in ps for blk in layers]))
    lw = oracle_lib.sample_layerwise(O, seeds, [16, 16], batch_size=64, prob_mode=0, rng_key=81)
    got = np.concatenate([np.load(tmp_path / f"lw_{r}.npy") for r in range(world)])
    assert np.array_equal(got, np.concatenate([blk["eid"] for layers in lw for blk in layers]))
    tr = oracle_lib.random_walk(O, seeds, 6, p=2.0, q=0.5, rng_key=80)
    got = np.concatenate([np.load(tmp_path / f"walk_{r}.npy") for r in range(world)])
    assert np.array_equal(got, tr)
    m0, m1 = np.load(tmp_path / "meta_0.npy"), np.load(tmp_path / "meta_1.npy")
    assert m0[2] == m1[2] == len(want)          # all-reduce SUM of edges
    assert m0[3] == m1[3] == 11.0               # all-reduce MAX of time
    # the broadcast graph is identical on both ranks
    assert np.array_equal(np.load(tmp_path / "graph_0.npy"), np.load(tmp_path / "graph_1.npy"))

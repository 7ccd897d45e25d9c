"""Multi-GPU plumbing for the data-parallel ECSF path.

One process per GPU (torchrun); torch.distributed carries only
  * the graph broadcast at load time (rank 0 generates or loads it), and
  * one reduction of counts / times per measurement.
Mini-batches are independent (super-batch semantics), so the sampling
itself needs no collective: every rank samples its own batches, keyed by their
GLOBAL batch index so the union over ranks equals a single-process run.
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def shard_range(num_batches: int, world: int, rank: int) -> tuple[int, int]:
    """Contiguous batch range [lo, hi) of `rank` for a strong-scaling split of
    one epoch (sizes differ by at most one batch)."""
    base, extra = divmod(num_batches, world)
    lo = rank * base + min(rank, extra)
    hi = lo + base + (1 if rank < extra else 0)
    return lo, hi


def seed_slice(num_seeds: int, batch_size: int, lo_batch: int, hi_batch: int) -> tuple[int, int]:
    """Seed index range covered by batches [lo_batch, hi_batch)."""
    return min(num_seeds, lo_batch * batch_size), min(num_seeds, hi_batch * batch_size)


def shard_epoch(num_inputs: int, batch_size: int | None, world: int, rank: int) -> tuple[int, int, int]:
    """Strong-scaling split of ONE epoch: returns (s0, s1, base):
    this rank's slice [s0, s1) of the epoch's inputs and the global index of its
    first unit, which keys the RNG so that the union over ranks equals a
    single-process run.  batch_size > 0: the units are mini-batches (contiguous
    batch ranges, base = first global batch index); batch_size None: the units
    are walkers (contiguous walker ranges, base = first global walker index)."""
    if batch_size:
        nb = (num_inputs + batch_size - 1) // batch_size
        lo, hi = shard_range(nb, world, rank)
        s0, s1 = seed_slice(num_inputs, batch_size, lo, hi)
        return s0, s1, lo
    lo, hi = shard_range(num_inputs, world, rank)
    return lo, hi, lo


def weak_batch_base(rank: int, num_batches: int) -> int:
    """Weak scaling (bench.py --scaling weak only): rank r samples a whole
    epoch with global batch ids r * num_batches + b (a different epoch per rank)."""
    return rank * num_batches


def broadcast_graph(g: dict | None, device, src: int = 0, group=None) -> dict:
    """Broadcasts a CSC graph dict (indptr int64, indices int32, weights fp32 or
    None) from `src` to every rank of the group.  Works with NCCL (CUDA
    tensors) and gloo (CPU tensors)."""
    rank = dist.get_rank(group)
    if rank == src:
        sizes = torch.tensor([g["indptr"].numel(), g["indices"].numel(),
                              -1 if g["weights"] is None else g["weights"].numel()],
                             dtype=torch.int64, device=device)
    else:
        sizes = torch.zeros(3, dtype=torch.int64, device=device)
    dist.broadcast(sizes, src, group=group)
    n_ip, n_ix, n_w = (int(x) for x in sizes.tolist())
    if rank != src:
        g = {"indptr": torch.empty(n_ip, dtype=torch.int64, device=device),
             "indices": torch.empty(n_ix, dtype=torch.int32, device=device),
             "weights": None if n_w < 0 else torch.empty(n_w, dtype=torch.float32, device=device),
             "spec": None}
    dist.broadcast(g["indptr"], src, group=group)
    dist.broadcast(g["indices"], src, group=group)
    if g["weights"] is not None:
        dist.broadcast(g["weights"], src, group=group)
    return g


def reduce_measurement(edges: float, elapsed_ms: float, device, group=None) -> tuple[float, float]:
    """(sum of sampled edges over ranks, max elapsed over ranks)."""
    t = torch.tensor([elapsed_ms], dtype=torch.float64, device=device)
    c = torch.tensor([edges], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    dist.all_reduce(c, op=dist.ReduceOp.SUM, group=group)
    return float(c.item()), float(t.item())

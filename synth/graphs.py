"""Deterministic R-MAT CSC graphs shaped like the paper's datasets (Table 6).

Recipe (readings Q16, Q20, Q21, Q8):
  * R-MAT (a, b, c, d) = (0.45, 0.22, 0.22, 0.11) at scale ceil(log2 N); node
    ids >= N rejected; ids permuted by a keyed hash; self loops dropped;
    duplicates removed; trimmed deterministically (smallest keyed hash kept)
    to the exact target edge count.
  * undirected graphs (PD, FS): target = undirected pairs, then symmetrised
    (two directed edges per pair); directed graphs (LJ, PP, tiny):
    target = directed edges.
  * CSC: column v lists the in-neighbours u of v, ascending, no duplicates.
  * weights: "uniform" w = fp32(((r >> 8) + 1) * 2^-24) in (0, 1] keyed by edge
    id (R21); "gcn" w_uv = fp32(1 / sqrt(max(1, dout(u)) * max(1, din(v)))) (R8).
All randomness is a splitmix64 counter hash evaluated with torch int64 ops, so
the same graph comes out on CPU and GPU.  Nothing here is part of the method.
"""
from __future__ import annotations

import dataclasses
import math

import numpy as np
import torch

RMAT = (0.45, 0.22, 0.22, 0.11)
_M64 = (1 << 64)


def _c(x: int) -> int:
    """Python int -> int64 two's complement value."""
    x &= _M64 - 1
    return x - _M64 if x >= (1 << 63) else x


_GOLDEN = _c(0x9E3779B97F4A7C15)
_MUL1 = _c(0xBF58476D1CE4E5B9)
_MUL2 = _c(0x94D049BB133111EB)


def _srl(x: torch.Tensor, s: int) -> torch.Tensor:
    """Logical right shift of int64 bit patterns."""
    return (x >> s) & ((1 << (64 - s)) - 1)


def hash64(stream: int, x: torch.Tensor) -> torch.Tensor:
    """splitmix64(x + stream * golden) on int64 bit patterns (wrapping)."""
    z = x.to(torch.int64) + _c(stream * 0x9E3779B97F4A7C15)
    z = z + _GOLDEN
    z = (z ^ _srl(z, 30)) * _MUL1
    z = (z ^ _srl(z, 27)) * _MUL2
    return z ^ _srl(z, 31)


def hash_u32(stream: int, x: torch.Tensor) -> torch.Tensor:
    """Uniform 32-bit values (as int64 in [0, 2^32))."""
    return _srl(hash64(stream, x), 32)


@dataclasses.dataclass(frozen=True)
class GraphSpec:
    name: str
    num_nodes: int
    num_edges: int          # undirected pairs if undirected else directed edges
    undirected: bool
    weights: str | None     # None | "uniform" | "gcn"
    seed: int = 0x5EED


CONFIGS = {
    # configs[0]: tiny 10k-node / 100k-edge graph (oracle in seconds)
    "tiny": GraphSpec("tiny", 10_000, 100_000, False, "uniform", 0x5EED),
    # configs[1]: Ogbn-Products-shaped (2.4M nodes, 62M undirected edges)
    "PD": GraphSpec("PD", 2_449_029, 61_859_140, True, None, 0x50D),
    "PDw": GraphSpec("PDw", 2_449_029, 61_859_140, True, "uniform", 0x50D),
    # configs[2]: LiveJournal-shaped (4.8M nodes, 69M directed edges)
    "LJ": GraphSpec("LJ", 4_847_571, 68_993_773, False, "gcn", 0x17),
    # configs[3]: Friendster-shaped (65.6M nodes, 1.8B undirected edges)
    "FS": GraphSpec("FS", 65_608_366, 1_806_067_135, True, None, 0xF5),
    # configs[4]: Papers100M-shaped (111M nodes, 1.6B directed edges)
    "PP": GraphSpec("PP", 111_059_956, 1_615_685_872, False, "uniform", 0x99),
}


def _rmat_pairs(spec: GraphSpec, n_gen: int, salt: int, device, chunk: int = 1 << 26,
                first: int = 0):
    """R-MAT (src, dst) pairs number first .. first + n_gen - 1 with ids < N
    (rejected ones dropped)."""
    N = spec.num_nodes
    scale = max(1, math.ceil(math.log2(N)))
    a, b, c, _ = RMAT
    ta = int(a * 2 ** 32)
    tb = int((a + b) * 2 ** 32)
    tc = int((a + b + c) * 2 ** 32)
    srcs, dsts = [], []
    for start in range(first, first + n_gen, chunk):
        e = torch.arange(start, min(first + n_gen, start + chunk), device=device, dtype=torch.int64)
        src = torch.zeros_like(e)
        dst = torch.zeros_like(e)
        base = e * 64
        for lvl in range(scale):
            r = hash_u32(spec.seed * 131 + salt, base + lvl)
            bs = (r >= tb).to(torch.int64)
            bd = (((r >= ta) & (r < tb)) | (r >= tc)).to(torch.int64)
            src = src * 2 + bs
            dst = dst * 2 + bd
        keep = (src < N) & (dst < N)
        srcs.append(src[keep])
        dsts.append(dst[keep])
        del e, src, dst, base, keep
    return torch.cat(srcs), torch.cat(dsts)


def _permutation(stream: int, n: int, device) -> torch.Tensor:
    """new_id[old_id]: a keyed pseudo-random permutation of range(n)."""
    h = hash64(stream, torch.arange(n, device=device, dtype=torch.int64))
    order = torch.argsort(h)
    new_id = torch.empty(n, dtype=torch.int64, device=device)
    new_id[order] = torch.arange(n, device=device, dtype=torch.int64)
    return new_id


_CHUNK = 1 << 29  # elements per torch sort/unique call (CUB handles < 2^31)


def _range_parts(x: torch.Tensor, parts: int, salt: int) -> list:
    """Value boundaries splitting x into ~equal ranges (quantiles of a keyed sample)."""
    if parts <= 1:
        return []
    n = x.numel()
    idx = hash64(salt, torch.arange(min(n, 1 << 22), device=x.device)) % n
    sample = torch.sort(x[idx]).values
    q = torch.linspace(0, sample.numel() - 1, parts + 1, device=x.device)[1:-1].long()
    return torch.unique(sample[q]).tolist()


def _sorted_unique(x: torch.Tensor, unique: bool, salt: int) -> torch.Tensor:
    """torch.unique / torch.sort for tensors of any length (range-partitioned)."""
    if x.numel() <= _CHUNK:
        return torch.unique(x) if unique else torch.sort(x).values
    bounds = _range_parts(x, (x.numel() + _CHUNK - 1) // _CHUNK * 2, salt)
    out, lo = [], None
    for hi in bounds + [None]:
        m = torch.ones_like(x, dtype=torch.bool)
        if lo is not None:
            m &= x > lo
        if hi is not None:
            m &= x <= hi
        part = x[m]
        del m
        out.append(torch.unique(part) if unique else torch.sort(part).values)
        del part
        lo = hi
    return torch.cat(out)


def _trim(key: torch.Tensor, target: int, salt: int) -> torch.Tensor:
    """Keeps exactly `target` keys: those with the smallest keyed 32-bit hash
    (ties by key), chosen with a 16-bit histogram; order of `key` preserved."""
    h = hash_u32(salt, key)
    hist = torch.bincount(_srl(h, 16), minlength=1 << 16).cumsum(0)
    cut = int(torch.searchsorted(hist, torch.tensor(target, device=key.device)))
    below = int(hist[cut - 1]) if cut > 0 else 0
    keep = _srl(h, 16) < cut
    border = torch.nonzero(_srl(h, 16) == cut).flatten()
    order = torch.argsort(h[border] * (1 << 31) + (border % (1 << 31)))
    keep[border[order[:target - below]]] = True
    return key[keep]


def _unique_keys(spec: GraphSpec, device) -> torch.Tensor:
    """Exactly spec.num_edges unique edge keys, sorted (undirected: lo*N+hi;
    directed: dst*N+src)."""
    N = spec.num_nodes
    target = spec.num_edges
    perm = _permutation(spec.seed * 7 + 1, N, device)
    factor = 1.25
    for attempt in range(8):
        n_gen = int(target * factor) + 1024
        chunks = []
        for start in range(0, n_gen, 1 << 28):
            src, dst = _rmat_pairs(spec, min(n_gen, start + (1 << 28)) - start, attempt, device,
                                   first=start)
            src = perm[src]
            dst = perm[dst]
            keep = src != dst
            src, dst = src[keep], dst[keep]
            if spec.undirected:
                chunks.append(torch.minimum(src, dst) * N + torch.maximum(src, dst))
            else:
                chunks.append(dst * N + src)
            del src, dst, keep
        key = torch.cat(chunks)
        del chunks
        key = _sorted_unique(key, True, spec.seed * 7 + 11)
        if key.numel() >= target:
            if key.numel() > target:
                key = _trim(key, target, spec.seed * 7 + 3)
            return key
        factor *= 1.25 * target / max(1, key.numel())
    raise RuntimeError(f"R-MAT generator could not reach {target} unique edges")


def make_graph(spec: GraphSpec | str, device="cpu"):
    """Returns dict(indptr int64[N+1], indices int32[nnz], weights fp32[nnz] | None)."""
    if isinstance(spec, str):
        spec = CONFIGS[spec]
    N = spec.num_nodes
    key = _unique_keys(spec, device)
    if spec.undirected:
        lo = torch.div(key, N, rounding_mode="floor")
        hi = key - lo * N
        del key
        # column v, row u: both directions of every pair
        ckey = torch.cat([hi * N + lo, lo * N + hi])
        del lo, hi
        ckey = _sorted_unique(ckey, False, spec.seed * 7 + 13)
    else:
        ckey = key
    nnz = ckey.numel()
    indices = torch.empty(nnz, dtype=torch.int32, device=device)
    counts = torch.zeros(N, dtype=torch.int64, device=device)
    for a in range(0, nnz, _CHUNK):
        c = ckey[a:a + _CHUNK]
        col = torch.div(c, N, rounding_mode="floor")
        indices[a:a + _CHUNK] = (c - col * N).to(torch.int32)
        counts += torch.bincount(col, minlength=N)
        del c, col
    del ckey
    indptr = torch.zeros(N + 1, dtype=torch.int64, device=device)
    indptr[1:] = torch.cumsum(counts, 0)
    weights = None
    if spec.weights == "uniform":
        weights = torch.empty(nnz, dtype=torch.float32, device=device)
        for a in range(0, nnz, _CHUNK):
            r = hash_u32(spec.seed * 7 + 5,
                         torch.arange(a, min(nnz, a + _CHUNK), device=device, dtype=torch.int64))
            weights[a:a + _CHUNK] = ((_srl(r, 8) + 1).to(torch.float64) * 2.0 ** -24).to(torch.float32)
    elif spec.weights == "gcn":
        din = counts.to(torch.float64).clamp_min(1.0)
        dout = torch.bincount(indices.to(torch.int64), minlength=N).to(torch.float64).clamp_min(1.0)
        col_of = torch.repeat_interleave(torch.arange(N, device=device), counts)
        weights = (1.0 / torch.sqrt(dout[indices.to(torch.int64)] * din[col_of])).to(torch.float32)
        del col_of
    return {"indptr": indptr, "indices": indices, "weights": weights, "spec": spec}


def make_seeds(spec: GraphSpec | str, count: int | None = None, device="cpu") -> torch.Tensor:
    """The first `count` nodes of a keyed permutation (R17), int32."""
    if isinstance(spec, str):
        spec = CONFIGS[spec]
    N = spec.num_nodes
    h = hash64(spec.seed * 7 + 9, torch.arange(N, device=device, dtype=torch.int64))
    order = torch.argsort(h)
    if count is not None:
        order = order[:count]
    return order.to(torch.int32)


def small_graph(num_nodes: int, num_edges: int, undirected=False, weights="uniform",
                seed=1234, device="cpu"):
    """Small R-MAT graph for tests."""
    spec = GraphSpec(f"small{num_nodes}_{num_edges}", num_nodes, num_edges, undirected,
                     weights, seed)
    return make_graph(spec, device)


def degree_stats(indptr) -> dict:
    d = (indptr[1:] - indptr[:-1])
    d = d.cpu().numpy() if isinstance(d, torch.Tensor) else np.asarray(d)
    return {
        "nodes": int(d.size), "nnz": int(d.sum()),
        "zero_in_degree_frac": float((d == 0).mean()),
        "median": float(np.median(d)), "p90": float(np.percentile(d, 90)),
        "p99": float(np.percentile(d, 99)), "max": int(d.max()) if d.size else 0,
    }


def make_grid_matrix(stream: int, rows: int, cols: int, levels: int = 4, device="cpu") -> torch.Tensor:
    """Seeded synthetic dense matrix (PASS features X and projections W1, W2),
    bf16 with values on the grid {-levels..levels} / levels: every product of two
    entries is a multiple of 1/levels^2 and every sum the path forms stays exactly
    representable (R29), so results do not depend on summation order."""
    idx = torch.arange(rows * cols, device=device, dtype=torch.int64)
    q = (hash_u32(stream, idx) % (2 * levels + 1)) - levels
    return (q.to(torch.float32) / levels).to(torch.bfloat16).reshape(rows, cols)


def make_feature_matrix(stream: int, rows: int, cols: int, device="cpu") -> torch.Tensor:
    """Seeded synthetic dense matrix with GENERAL bf16 values (no grid): roughly
    standard normal (sum of 4 uniforms, centred and scaled), rounded to bf16.
    The PASS projections of such inputs depend on the summation order in fp32,
    so GPU and oracle agree within the magnitude-scaled bound of DESIGN.md R29."""
    idx = torch.arange(rows * cols, device=device, dtype=torch.int64)
    acc = torch.zeros(rows * cols, device=device, dtype=torch.float32)
    for j in range(4):
        acc += (hash_u32(stream * 4 + j, idx).to(torch.float32) + 0.5) * (1.0 / 4294967296.0)
    return ((acc - 2.0) * 1.7320508).to(torch.bfloat16).reshape(rows, cols)

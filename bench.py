#!/usr/bin/env python
"""Benchmark of the B200 ECSF sampling hot path (BASELINE.json metric:
"sampled edges/s & epoch sampling time at 1/2/4/8 B200; % HBM roofline").

Default workload (BASELINE.json configs[1]): GraphSAGE [25,10] uniform
neighbour sampling, batch 1024, one full epoch of seeds (196,615 = the
ogbn-products train-split size, 193 mini-batches) on an Ogbn-Products-shaped
R-MAT graph (2,449,029 nodes, 61,859,140 undirected edges -> 123,718,280 CSC
entries).  One step = one epoch (every batch, every hop: Extract, Select,
Finalize) = one call of the node-wise engine (the hop-synchronous kernels of
nodewise_hop.cu, one CUDA graph).  Other configs of BASELINE.json are
selectable with --workload (parity cases / extra lines).

Contract: python bench.py --gpus N --steps K --warmup W [--impl reference]
Multi-GPU (torchrun): one process per GPU; rank 0 generates the graph and
broadcasts it over NCCL (load time, not timed); ONE epoch is split across the
ranks (dist.shard_epoch: contiguous batch ranges keyed by their global batch
index, or contiguous walker ranges), so the union over ranks is exactly the
single-GPU epoch ("scaling": "strong"); time = max over ranks (all-reduce),
edges = sum.  --scaling weak gives every rank its own full epoch instead.
Each timed epoch is a CUDA graph replay (captured per step key during warm-up;
--no-graph runs the calls eagerly).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402,F401
import torch  # noqa: E402

METRIC = "sampled edges/s & epoch sampling time at 1/2/4/8 B200; % HBM roofline"
# process-group backend: NCCL (one GPU per rank); GS_BENCH_BACKEND=gloo is a
# plumbing test only (several ranks sharing one GPU, collectives through host memory)
BACKEND = os.environ.get("GS_BENCH_BACKEND", "nccl")
UNIT = "sampled edges/s"
# Random-access ceiling of this B200's HBM (profiles/r01_random_access_probe.md,
# tools/microbench_l2fetch*.cu): every random load that misses L2 moves a
# 128-byte line, ~36.9 G random loads/s on an 8 GB working set = 1181 GB/s of
# useful 32-byte sectors.  The byte model counts 32 B per random sector, so a
# gather-bound kernel's roofline.frac against the streaming peak cannot exceed
# ~0.18; frac_of_random_sector_ceiling compares against this ceiling instead.
RANDOM_SECTOR_GBS = 36.9e9 * 32 / 1e9

WORKLOADS = {
    "graphsage_pd": dict(kind="nodewise", graph="PD", fanouts=[25, 10], batch=1024,
                         seeds=196_615, replace=False, bias=0,
                         desc="GraphSAGE [25,10] uniform, batch 1024, full epoch (196,615 seeds, "
                              "193 batches), Ogbn-Products-shaped R-MAT graph (2,449,029 nodes, "
                              "61,859,140 undirected edges)"),
    "graphsage_pd_uva": dict(kind="nodewise", graph="PD", fanouts=[25, 10], batch=1024,
                             seeds=196_615, replace=False, bias=0, host_mapped=True,
                             desc="GraphSAGE [25,10] as graphsage_pd with the CSC index array in "
                                  "pinned host memory read over the host link (UVA, P:415; "
                                  "SURVEY 8(f) f4)"),
    "graphsage_pd_uva_cache": dict(kind="nodewise", graph="PD", fanouts=[25, 10], batch=1024,
                                   seeds=196_615, replace=False, bias=0, host_mapped=True,
                                   cache_frac=0.25,
                                   desc="GraphSAGE [25,10] as graphsage_pd_uva with the hottest quarter "
                                        "of the index array cached in HBM (gs_graph_cache_hot, P:490; "
                                        "SURVEY 8(f) f4)"),
    "graphsage_tiny": dict(kind="nodewise", graph="tiny", fanouts=[5, 5], batch=512, seeds=512,
                           replace=False, bias=0,
                           desc="GraphSAGE [5,5] uniform, 512 seeds, 10k-node/100k-edge R-MAT"),
    "kgcn_pd": dict(kind="nodewise", graph="PD", fanouts=[8, 8], batch=1024, seeds=196_615,
                    replace=True, bias=0, desc="KGCN [8,8] with replacement, PD-shaped"),
    "pass_pd": dict(kind="nodewise", graph="PDw", fanouts=[10, 10], batch=1024, seeds=196_615,
                    replace=False, bias=2, desc="PASS-style A3 [10,10], PD-shaped weighted"),
    "ares_pp": dict(kind="nodewise", graph="PP", fanouts=[15, 10, 5], batch=1024,
                    seeds=1_207_179, replace=False, bias=1,
                    desc="GraphSAGE [15,10,5] weighted A-Res, Papers100M-shaped"),
    "shadow_pd": dict(kind="shadow", graph="PD", fanouts=[10, 5], batch=1024, seeds=196_615,
                      bias=0, desc="ShaDow [10,5] uniform + induce, PD-shaped"),
    "saint_pd": dict(kind="saint", graph="PD", walk_length=2, batch=3000, seeds=None,
                     desc="GraphSAINT-RW 3000 roots x walk length 2 + induce per subgraph, every "
                          "node a root once per epoch (817 subgraphs), PD-shaped"),
    "pass_full_pd": dict(kind="pass_full", graph="PDw", fanouts=[10, 10], batch=1024,
                         seeds=196_615, F=128, H=32, W3=[0.2, -0.4, 0.9],
                         desc="PASS full bias (A1, A2 SDDMM of 128-d features projected to 32-d, "
                              "A3, softmax(W3) mix, relu) for every edge + weighted A-Res [10,10], "
                              "batch 1024, full epoch, PD-shaped weighted"),
    "pinsage_pd": dict(kind="pinsage", graph="PD", topk=[10, 10], num_walks=10, walk_length=3,
                       restart=0.5, batch=1024, seeds=196_615,
                       desc="PinSAGE-style top-k [10,10] of 10 restart walks (<= 3 steps, restart "
                            "0.5), batch 1024, full epoch (196,615 seeds), PD-shaped"),
    "ladies_lj": dict(kind="layerwise", graph="LJ", n_per_layer=[512, 512, 512], batch=512,
                      seeds=None, mode=0, desc="LADIES 512x3, LJ-shaped, all nodes as seeds"),
    "fastgcn_lj": dict(kind="layerwise", graph="LJ", n_per_layer=[512, 512, 512], batch=512,
                       seeds=None, mode=1, desc="FastGCN 512x3, LJ-shaped, all nodes as seeds"),
    "deepwalk_fs": dict(kind="walk", graph="FS", length=80, p=1.0, q=1.0,
                        desc="DeepWalk length 80, one walker per node, Friendster-shaped"),
    "node2vec_fs": dict(kind="walk", graph="FS", length=80, p=2.0, q=0.5,
                        desc="Node2Vec p=2 q=0.5 length 80, one walker per node, FS-shaped"),
}


# ---------------------------------------------------------------------------
# helpers
# ---------------------------------------------------------------------------
def measured_peak_hbm():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(path) as f:
            return float(json.load(f)["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


class ClockSampler:
    """Samples SM clocks and throttle reasons through NVML during the timed region."""

    REASONS = {0x2: "applications_clocks_setting", 0x4: "sw_power_cap", 0x8: "hw_slowdown",
               0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown",
               0x80: "hw_power_brake_slowdown"}

    def __init__(self, device_index):
        self.samples, self.reasons = [], set()
        self._stop = threading.Event()
        self.max_mhz = None
        try:
            import pynvml
            pynvml.nvmlInit()
            self._nv = pynvml
            self._h = pynvml.nvmlDeviceGetHandleByIndex(device_index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self._h, pynvml.NVML_CLOCK_SM)
        except Exception:
            self._nv = None

    def _run(self):
        nv = self._nv
        while not self._stop.is_set():
            try:
                self.samples.append(nv.nvmlDeviceGetClockInfo(self._h, nv.NVML_CLOCK_SM))
                r = nv.nvmlDeviceGetCurrentClocksEventReasons(self._h)
                for bit, name in self.REASONS.items():
                    if r & bit:
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(0.002)

    def __enter__(self):
        if self._nv is not None:
            self._t = threading.Thread(target=self._run, daemon=True)
            self._t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self._nv is not None:
            self._t.join()

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons),
                    "samples": 0}
        return {"sm_mhz": statistics.median(self.samples), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


def dist_env():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


def make_graph_dist(name, world, rank, device):
    """Rank 0 generates the graph; NCCL broadcasts it to the other ranks (load time)."""
    import synth
    from paper_conf_sosp_gonglmc0lwl23_b200 import dist as gdist
    spec = synth.CONFIGS[name]
    if world == 1:
        return synth.make_graph(spec, device=device)
    if BACKEND == "gloo":  # plumbing test (several ranks on one GPU): broadcast through host memory
        g = synth.make_graph(spec, device="cpu") if rank == 0 else None
        g = gdist.broadcast_graph(g, torch.device("cpu"))
        g = {k: (v.to(device) if torch.is_tensor(v) else v) for k, v in g.items()}
    else:
        g = synth.make_graph(spec, device=device) if rank == 0 else None
        g = gdist.broadcast_graph(g, device)
    g["spec"] = spec
    return g


def _layer_arrays(blocks, l):
    import ctypes
    from paper_conf_sosp_gonglmc0lwl23_b200 import gs
    lb = gs._LayerBuffers()
    gs._check(gs._lib.gs_blocks_layer(blocks._h, l, ctypes.byref(lb)))
    t = gs._dev_tensor
    d = {"col_map": t(lb.col_map, lb.col_capacity, torch.int32, blocks),
         "row_map": t(lb.row_map, lb.row_capacity, torch.int32, blocks),
         "indptr": t(lb.indptr, lb.indptr_capacity, torch.int64, blocks),
         "row_local": t(lb.row_local, lb.edge_capacity, torch.int32, blocks),
         "eid": t(lb.eid, lb.edge_capacity, torch.int64, blocks)}
    if lb.val:
        d["val"] = t(lb.val, lb.edge_capacity, torch.float32, blocks)
    return d


def _secs(off, d):
    """32-byte int32 sectors spanned by [off, off + d) (0 when d == 0)."""
    return torch.where(d > 0, ((off + d - 1) >> 3) - (off >> 3) + 1, torch.zeros_like(d))


def _blocks_byte_model(blocks, g, kind, weighted, L, weighted_select=False):
    """Algorithmic bytes of one step (SURVEY.md 8(d) byte model).
    node-wise, per column: 4 (frontier id) + 32*(1 + [v%4==3]) (int64 indptr pair)
      + 32 * distinct sectors of the sampled positions (the column when d <= k)
      + 8 (block indptr); per edge 12 (row_local + eid); per row 4 (row_map).
    weighted node-wise (A-Res / PASS): + 32 * sectors of the column's weights.
    shadow: per U node the whole column streamed once (4 + 32(1+straddle) +
      32 secs(off, d)) + 12 per induced edge + 4 per node.
    layer-wise: every frontier column streamed twice (indices, + weights for
      LADIES) + 32(1+straddle) + 4; per block edge 16; per row 8.
    Also returns the number of those 32-byte sectors that are RANDOM accesses
    (indptr pairs, sampled positions, the first sector of a streamed column):
    on this B200 each moves a 128-byte HBM line (the line model)."""
    indptr = g["indptr"]
    meta = blocks.device_meta()
    total, edges, rnd = 0, 0, 0
    sel = 0  # node-wise: the select kernels' share (frontier ids, sampled sectors, eid + row id)
    for l in range(L):
        view = _layer_arrays(blocks, l)
        m = meta[:, l, :].cpu()
        cols_all, e_all = [], []
        for b in range(m.shape[0]):
            T, R, E = int(m[b, 0]), int(m[b, 1]), int(m[b, 2])
            if T == 0:
                continue
            co, io, eo = int(m[b, 3]), int(m[b, 5]), int(m[b, 6])
            cols_all.append(view["col_map"][co:co + T].to(torch.int64))
            ip = view["indptr"][io:io + T + 1]
            e_all.append((view["eid"][eo:eo + E], ip[1:] - ip[:-1]))
            total += E * (12 if kind != "layerwise" else 16) + R * (4 if kind != "layerwise" else 8)
            edges += E
        if not cols_all:
            continue
        cols = torch.cat(cols_all)
        off = indptr[cols]
        d = indptr[cols + 1] - off
        straddle = int(((cols & 3) == 3).sum())
        ncols = cols.numel()
        if kind == "nodewise":
            sec = 0
            for eids, cnt in e_all:
                cid = torch.repeat_interleave(torch.arange(cnt.numel(), device=cnt.device), cnt)
                sec += torch.unique(cid * (1 << 40) + (eids >> 3)).numel()
            total += ncols * 12 + 32 * (ncols + straddle) + 32 * sec
            rnd += ncols + straddle + sec
            sel += ncols * 4 + 32 * sec + 12 * sum(int(c.sum()) for _, c in e_all)
            if weighted_select:  # A-Res streams every weight of the column
                total += 32 * int(_secs(off, d).sum())
                sel += 32 * int(_secs(off, d).sum())
                rnd += int((d > 0).sum())
        elif kind == "shadow":
            total += ncols * 4 + 32 * (ncols + straddle) + 32 * int(_secs(off, d).sum())
            rnd += ncols + straddle + int((d > 0).sum())
        else:
            s = int(_secs(off, d).sum())
            total += 2 * (ncols * 4 + 32 * (ncols + straddle) + 32 * s * (2 if weighted else 1))
            rnd += 2 * (ncols + straddle + int((d > 0).sum()) * (2 if weighted else 1))
    _blocks_byte_model.sel = sel
    return total, edges, rnd


# ---------------------------------------------------------------------------
# Oracle (CPU baseline / reference arm): the oracle as it stands
# ---------------------------------------------------------------------------
def oracle_rate(g, inputs, wl, budget_s=15.0):
    import oracle
    O = oracle.Graph(g["indptr"].cpu().numpy(), g["indices"].cpu().numpy(),
                     None if g["weights"] is None else g["weights"].cpu().numpy())
    cores = len(os.sched_getaffinity(0))
    s = inputs.cpu().numpy()
    kind = wl["kind"]
    if kind == "walk":
        n1 = min(len(s), 4096)
        t0 = time.perf_counter()
        oracle.random_walk(O, s[:n1], wl["length"], p=wl["p"], q=wl["q"], num_threads=1)
        t1 = (time.perf_counter() - t0) / n1
        n = int(max(1024, min(len(s), budget_s * cores / max(t1, 1e-9))))
        t0 = time.perf_counter()
        tr = oracle.random_walk(O, s[:n], wl["length"], p=wl["p"], q=wl["q"], num_threads=cores)
        dt = time.perf_counter() - t0
        edges = int((tr[:, 1:] >= 0).sum())
        return {"value": edges / dt, "unit": UNIT, "cores": cores, "kind": "oracle",
                "sample": f"first {n} of {len(s)} walkers ({edges} transitions, {dt:.2f} s on "
                          f"{cores} threads)"}, edges, dt
    bs = wl["batch"]
    nb_total = (len(s) + bs - 1) // bs

    def run(nbat, threads):
        if kind == "nodewise":
            return oracle.sample_neighbors(O, s[:nbat * bs], wl["fanouts"], batch_size=bs,
                                           replace=wl["replace"], bias_mode=wl["bias"], rng_key=1,
                                           num_threads=threads)
        if kind == "pinsage":
            return oracle.pinsage(O, s[:nbat * bs], wl["topk"], wl["num_walks"], wl["walk_length"],
                                  wl["restart"], batch_size=bs, rng_key=1, num_threads=threads)
        if kind == "saint":
            return [[x] for x in oracle.saint_rw(O, s[:nbat * bs], wl["walk_length"],
                                                 batch_size=bs, rng_key=1, num_threads=threads)]
        if kind == "shadow":
            return [[x] for x in oracle.shadow(O, s[:nbat * bs], wl["fanouts"], batch_size=bs,
                                               bias_mode=wl["bias"], rng_key=1,
                                               num_threads=threads)]
        return oracle.sample_layerwise(O, s[:nbat * bs], wl["n_per_layer"], batch_size=bs,
                                       prob_mode=wl["mode"], rng_key=1, num_threads=threads)

    t0 = time.perf_counter()
    run(1, 1)
    t1 = time.perf_counter() - t0
    nb = int(max(1, min(nb_total, budget_s * cores / max(t1, 1e-4))))
    t0 = time.perf_counter()
    r = run(nb, cores)
    dt = time.perf_counter() - t0
    edges = sum(len(blk["eid"]) for layers in r for blk in layers)
    return {"value": edges / dt, "unit": UNIT, "cores": cores, "kind": "oracle",
            "sample": f"first {nb} of {nb_total} batches of the workload ({edges} sampled edges, "
                      f"{dt:.2f} s wall on {cores} threads)"}, edges, dt


def workload_inputs(wl, g, device):
    import synth
    if wl["kind"] == "walk":
        return torch.arange(g["indptr"].numel() - 1, dtype=torch.int32, device=device)
    return synth.make_seeds(wl["graph"], wl["seeds"], device=device)


def run_reference(args, wl):
    world, rank, _ = dist_env()
    if rank != 0:
        return
    import synth
    dev = "cuda" if torch.cuda.is_available() else "cpu"
    g = synth.make_graph(wl["graph"], device=dev)
    inputs = workload_inputs(wl, g, dev)
    total_edges, total_t, cb = 0, 0.0, None
    for i in range(args.warmup + args.steps):
        cb, e, dt = oracle_rate(g, inputs, wl, budget_s=3.0)
        if i >= args.warmup:
            total_edges += e
            total_t += dt
    value = total_edges / total_t
    line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": 1000 * total_t / args.steps, "higher_is_better": True,
            "scaling": args.scaling, "vs_baseline": None, "dtype": "int64",
            "data": "synthetic (deterministic R-MAT, DESIGN.md input recipe)", "impl": "reference",
            "config": {"workload": wl["desc"],
                       "reference": "CPU oracle oracle/gso.cpp as it stands (no reference "
                                    "implementation exists; DESIGN.md section 10)",
                       "step": "a bounded sample of the workload (see cpu_baseline.sample)"},
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": cb["cores"], "kind": "oracle",
                             "sample": cb["sample"]},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------------------
# GPU arm
# ---------------------------------------------------------------------------
def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return None


GRAPH_KINDS = ("nodewise", "walk", "pinsage", "shadow", "saint", "layerwise")


def run_gpu(args, wl, world, rank, device):
    from paper_conf_sosp_gonglmc0lwl23_b200 import dist as gdist
    from paper_conf_sosp_gonglmc0lwl23_b200 import gs
    import torch.distributed as dist
    gs.use_torch_allocator()
    kind = wl["kind"]
    t0 = time.time()
    g = make_graph_dist(wl["graph"], world, rank, device)
    gen_s = time.time() - t0
    G = gs.Graph(g["indptr"], g["indices"], g["weights"], host_mapped=wl.get("host_mapped", False))
    if wl.get("cache_frac"):
        G.cache_hot(int(wl["cache_frac"] * g["indices"].numel() * (8 if g["weights"] is not None else 4)))
    all_inputs = workload_inputs(wl, g, device)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=device)  # > 126 MB L2
    out = gs.Blocks()
    base_key = 0x5EED
    bs = wl.get("batch")
    strong = args.scaling == "strong"
    # this rank's share of the epoch: strong = a contiguous slice
    # of ONE epoch keyed by global indices; weak = a whole epoch per rank
    if kind == "walk":
        n_all = all_inputs.numel()
        if strong:
            s0, s1, wbase = gdist.shard_epoch(n_all, None, world, rank)
        else:
            s0, s1, wbase = 0, n_all, rank * n_all
        inputs = all_inputs[s0:s1]
        nunits = inputs.numel()
        traces = torch.empty((nunits, wl["length"] + 1), dtype=torch.int32, device=device)
        L = 1
    else:
        nb_all = (all_inputs.numel() + bs - 1) // bs
        if strong:
            s0, s1, wbase = gdist.shard_epoch(all_inputs.numel(), bs, world, rank)
        else:
            s0, s1, wbase = 0, all_inputs.numel(), gdist.weak_batch_base(rank, nb_all)
        inputs = all_inputs[s0:s1]
        nunits = (inputs.numel() + bs - 1) // bs
        L = 1 if kind in ("shadow", "saint") else len(wl.get("fanouts") or wl.get("n_per_layer")
                                                       or wl.get("topk"))
    if kind == "pass_full":
        import synth
        N = g["indptr"].numel() - 1
        PX = synth.make_grid_matrix(21, N, wl["F"], device=device)
        PW1 = synth.make_grid_matrix(22, wl["F"], wl["H"], device=device)
        PW2 = synth.make_grid_matrix(23, wl["F"], wl["H"], device=device)
        att = torch.empty(g["indices"].numel(), dtype=torch.float32, device=device)
        Ga = gs.Graph(g["indptr"], g["indices"], g["weights"])

    def step(i, x=None):
        x = inputs if x is None else x
        stream = torch.cuda.current_stream()
        key = base_key + 7919 * i
        if kind == "nodewise":
            gs.sample_neighbors(G, x, wl["fanouts"], batch_size=bs, batch_index_base=wbase,
                                replace=wl["replace"], bias_mode=wl["bias"], rng_key=key,
                                stream=stream, out=out)
        elif kind == "shadow":
            gs.sample_shadow(G, x, wl["fanouts"], batch_size=bs, batch_index_base=wbase,
                             bias_mode=wl["bias"], rng_key=key, stream=stream, out=out,
                             retry=False)
        elif kind == "pass_full":
            # Fig. 3(c): the learned bias of every edge (W1..W3 change per
            # training step, so it is recomputed every epoch), then line 10
            gs.pass_attention(G, PX, PW1, PW2, wl["W3"], stream=stream, out=att)
            Ga.set_weights(att, stream=stream)
            gs.sample_neighbors(Ga, x, wl["fanouts"], batch_size=bs, batch_index_base=wbase,
                                bias_mode=1, rng_key=key, stream=stream, out=out)
        elif kind == "pinsage":
            gs.sample_pinsage(G, x, wl["topk"], wl["num_walks"], wl["walk_length"], wl["restart"],
                              batch_size=bs, batch_index_base=wbase, rng_key=key, stream=stream,
                              out=out)
        elif kind == "saint":
            gs.sample_saint_rw(G, x, wl["walk_length"], batch_size=bs, batch_index_base=wbase,
                               rng_key=key, stream=stream, out=out, retry=False)
        elif kind == "layerwise":
            gs.sample_layerwise(G, x, wl["n_per_layer"], batch_size=bs, batch_index_base=wbase,
                                prob_mode=wl["mode"], rng_key=key, stream=stream, out=out,
                                retry=False)
        else:
            gs.random_walk(G, x, wl["length"], p=wl["p"], q=wl["q"], walker_index_base=wbase,
                           rng_key=key, stream=stream, out=traces)

    cur = [0]  # the step index account() describes

    def grow_until_fits():
        # layer-wise / ShaDow outputs are sized on the device: every rng key the
        # run will use is tried (and the buffers grown) before anything is timed
        for i in range(args.warmup + args.steps):
            for _ in range(6):
                step(i)
                try:
                    out.sync()
                    break
                except gs.GSError as e:
                    if e.status != 7:
                        raise

    def account():
        if kind == "walk":
            # walk index (walk_kernel): per step one 32-byte sector
            # holding the 16-byte record of the chosen neighbour + 4 bytes of
            # trace; per walker the start's indptr pair (32(1+straddle)) and
            # its trace entry.  Node2Vec's extra trials and membership probes
            # are not counted (a lower bound).
            nxt = traces[:, 1:]
            edges = int((nxt >= 0).sum())
            st = traces[:, 0].to(torch.int64)
            walkers = int((st >= 0).sum())
            straddle = int(((st & 3) == 3).sum())
            return (edges * (32 + 4) + walkers * (32 + 4) + 32 * straddle, edges,
                    edges + walkers + straddle)
        out.sync()
        if kind == "pass_full":
            # sampling as weighted node-wise (att streamed by the A-Res select) +
            # the bias: per edge 4 (index) + 4 (w) + 4 (att written) + 8H (the
            # projected row of u, 2H fp32, a random gather); per node 8H (its own
            # row) + 16 (indptr pair) + 4 (colsum); the GEMM reads X (2F per
            # node) and writes the projections (8H per node)
            tot, e, rnd = _blocks_byte_model(out, g, "nodewise", False, L, weighted_select=True)
            N = g["indptr"].numel() - 1
            nnz = g["indices"].numel()
            H = wl["H"]
            tot += nnz * (12 + 8 * H) + N * (8 * H + 20) + N * (2 * wl["F"] + 8 * H)
            return tot, e, rnd + N
        if kind == "pinsage":
            # per frontier column: 4 (id) + its walks' steps, each one random
            # indptr-pair sector + one random index sector (32 + 32); the steps
            # are counted by their expectation W * sum_t (1-r)^t (the restart
            # law); per selected neighbour 16 (row_local + val + eid) + 8
            # (indptr); per row 4
            meta = out.device_meta().cpu()
            cols = int(meta[:, :, 0].sum())
            rows = int(meta[:, :, 1].sum())
            e = int(meta[:, :, 2].sum())
            r = wl["restart"]
            steps = cols * wl["num_walks"] * sum((1 - r) ** t for t in range(1, wl["walk_length"] + 1))
            tot = cols * (4 + 8) + int(steps * 64) + e * 16 + rows * 4
            return tot, e, int(2 * steps)
        if kind == "saint":
            # induce as ShaDow (per U node its column streamed once, 12 per
            # induced edge, 4 per node) + the walks: per root 32(1+straddle) + 4,
            # per step one 32-B record sector + 4 written + 4 read back (the
            # traces, recomputed here outside the timed region for the count)
            tot, e, rnd = _blocks_byte_model(out, g, "shadow", False, 1)
            tr = gs.random_walk(G, inputs, wl["walk_length"], walker_index_base=wbase * bs,
                                rng_key=base_key + 7919 * cur[0])
            steps = int((tr[:, 1:] >= 0).sum())
            st = inputs.to(torch.int64)
            straddle = int(((st & 3) == 3).sum())
            tot += steps * 40 + st.numel() * 36 + 32 * straddle
            return tot, e, rnd + steps + st.numel() + straddle
        return _blocks_byte_model(out, g, kind, g["weights"] is not None and wl.get("mode") == 0,
                                  L, weighted_select=kind == "nodewise" and wl.get("bias", 0) != 0)

    if kind in ("shadow", "saint", "layerwise"):
        grow_until_fits()
    for i in range(args.warmup):
        step(i)
    if kind != "walk":
        out.sync()
    torch.cuda.synchronize()
    # CUDA graphs: one captured epoch per timed step key (the library call is
    # stream-ordered with no host sync and allocates nothing on reuse)
    graphs = None
    use_graph = args.graph and kind in GRAPH_KINDS
    k0 = gs.kernel_launches()
    step(args.warmup)  # one eager step: the library's kernel launches per step
    launches_per_step = gs.kernel_launches() - k0
    if kind != "walk":
        out.sync()
    torch.cuda.synchronize()
    if use_graph:
        try:
            graphs = []
            cs = torch.cuda.Stream()
            for i in range(args.steps):
                gr = torch.cuda.CUDAGraph()
                with torch.cuda.graph(gr, stream=cs):
                    step(args.warmup + i)
                graphs.append(gr)
            torch.cuda.synchronize()
        except Exception as e:  # capture unsupported for this call: eager timing
            print(f"# CUDA graph capture failed ({e}); timing eager calls", file=sys.stderr)
            graphs = None
            torch.cuda.synchronize()
    times, edges, model_bytes, rnd_secs, sel_bytes = [], 0, 0, 0, 0
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    stream = torch.cuda.current_stream()
    with ClockSampler(torch.cuda.current_device()) as clk:
        for i in range(args.steps):
            flush.zero_()
            ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            ev0.record(stream)
            cur[0] = args.warmup + i
            if graphs is not None:
                graphs[i].replay()
            else:
                step(args.warmup + i)
            ev1.record(stream)
            ev1.synchronize()
            times.append(ev0.elapsed_time(ev1))
            _blocks_byte_model.sel = 0
            mb, e, rs = account()
            model_bytes += mb
            edges += e
            rnd_secs += rs
            sel_bytes += _blocks_byte_model.sel
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    t_total_ms = sum(times)
    peak_mem = torch.cuda.max_memory_allocated(device)

    # per-kernel durations (profiling pass after the timed region: the
    # node-wise sampler records a CUDA event after each kernel on its stream)
    kernel_ms = {}
    if kind == "nodewise":
        gs.set_profiling(True)
        nprof = 3
        for i in range(nprof):
            step(args.warmup + i)
            for name, ms in gs.blocks_profile(out):
                kernel_ms[name] = kernel_ms.get(name, 0.0) + ms / nprof
        gs.set_profiling(False)
        torch.cuda.synchronize()

    # e2e: the same step through the C ABI with HOST buffers: pinned host
    # inputs copied in; the sampled blocks packed densely on the device
    # (gs_blocks_pack), their sizes read, and exactly the sampled data copied
    # back -- all inside the timed region
    host_in = inputs.cpu().pin_memory()
    dev_in = torch.empty_like(inputs)
    h2d = host_in.numel() * host_in.element_size()
    if kind == "walk":
        host_tr = torch.empty(traces.shape, dtype=traces.dtype).pin_memory()
    else:
        # int32 edge ids / block offsets when the graph allows (< 2^31 entries):
        # the host copy is the e2e bound (PCIe), so its bytes are what count
        narrow = g["indices"].numel() < (1 << 31)
        packs = [out.pack(l, narrow=narrow) for l in range(L)]
        meta_dev = out.device_meta()
        host_meta = torch.empty(meta_dev.shape, dtype=meta_dev.dtype).pin_memory()
        host_tot = torch.empty((L, 3), dtype=torch.int64).pin_memory()
        host_pk = [{k2: torch.empty(v.shape, dtype=v.dtype).pin_memory() for k2, v in pk.items()
                    if k2 != "totals"} for pk in packs]
    e2e_times, d2h_all = [], []
    copy_side = torch.cuda.Stream()
    # node-wise: the epoch's batches in E2E_CHUNKS contiguous chunks (each its
    # own call with batch_index_base = its first global batch, so the union is
    # the same epoch), every chunk's host copies issued on two copy streams as
    # soon as its sizes are known while the next chunks sample: the link, not
    # the sampler, bounds the step
    chunked = kind == "nodewise" and inputs.numel() > 0
    if chunked:
        nbat = (inputs.numel() + bs - 1) // bs
        nch = max(1, min(E2E_CHUNKS, nbat))
        # a small first chunk: the link starts as early as possible, the
        # later chunks sample while it drains
        first = nbat // E2E_FIRST if E2E_FIRST > 0 and nch > 1 else 0
        if first >= 1:
            cb = [0] + [first + (nbat - first) * c // (nch - 1) for c in range(nch)]
        else:
            cb = [nbat * c // nch for c in range(nch + 1)]
        souts = [gs.Blocks() for _ in range(nch)]
        cstreams = tuple(torch.cuda.Stream() for _ in range(E2E_STREAMS))
        mstream = torch.cuda.Stream()

        def step_chunk(i, c, x, st=stream):
            key = base_key + 7919 * i
            lo, hi = cb[c] * bs, min(cb[c + 1] * bs, x.numel())
            gs.sample_neighbors(G, x[lo:hi], wl["fanouts"], batch_size=bs, batch_index_base=wbase + cb[c],
                                replace=wl["replace"], bias_mode=wl["bias"], rng_key=key,
                                stream=st, out=souts[c])

        for c in range(nch):  # sizes the chunk results before the pack buffers
            step_chunk(args.warmup, c, inputs)
        torch.cuda.synchronize()
        cpacks = [[so.pack(l, narrow=narrow) for l in range(L)] for so in souts]
        cmeta = [so.device_meta() for so in souts]
        chost_meta = [torch.empty(m.shape, dtype=m.dtype).pin_memory() for m in cmeta]
        chost_tot = [torch.empty((L, 3), dtype=torch.int64).pin_memory() for _ in range(nch)]
        chost_pk = [[{k2: torch.empty(v.shape, dtype=v.dtype).pin_memory() for k2, v in pk.items()
                      if k2 != "totals"} for pk in cp] for cp in cpacks]
    n_e2e = max(2, min(args.steps, 5)) + (1 if chunked else 0)
    cgraphs = None
    if chunked and args.graph and E2E_GRAPH:
        # each chunk's public calls (sample + pack) captured once per step key,
        # as the device-timed epoch is: one launch per chunk instead of the
        # per-call host work between the link's chunks
        try:
            gcs = torch.cuda.Stream()
            cgraphs = []
            for i in range(n_e2e):
                row = []
                for c in range(nch):
                    gr = torch.cuda.CUDAGraph()
                    with torch.cuda.graph(gr, stream=gcs):
                        step_chunk(args.warmup + i, c, dev_in, st=gcs)
                        for l in range(L):
                            souts[c].pack(l, cpacks[c][l], stream=gcs, narrow=narrow)
                    row.append(gr)
                cgraphs.append(row)
            torch.cuda.synchronize()
        except Exception as e:
            print(f"# e2e chunk capture failed ({e}); eager chunks", file=sys.stderr)
            cgraphs = None
            torch.cuda.synchronize()
    for i in range(n_e2e):
        if chunked:
            flush.zero_()
            torch.cuda.synchronize()
            ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            ev0.record(stream)
            dev_in.copy_(host_in, non_blocking=True)
            ready, packs_ev = [], []
            for c in range(nch):
                if cgraphs is not None:
                    cgraphs[i][c].replay()
                else:
                    step_chunk(args.warmup + i, c, dev_in)
                    for l in range(L):
                        souts[c].pack(l, cpacks[c][l], stream=stream, narrow=narrow)
                # the chunk's sizes and batch offsets come back on a stream of
                # their own: a D2H copy on the sampling stream would queue
                # behind the previous chunks' bulk copies in the copy engine
                # and hold the next chunk's sampling back until they drain
                packed = torch.cuda.Event(enable_timing=E2E_DEBUG)
                packed.record(stream)
                packs_ev.append(packed)
                mstream.wait_event(packed)
                with torch.cuda.stream(mstream):
                    for l in range(L):
                        chost_tot[c][l].copy_(cpacks[c][l]["totals"], non_blocking=True)
                    chost_meta[c].copy_(cmeta[c], non_blocking=True)
                e = torch.cuda.Event(enable_timing=E2E_DEBUG)
                e.record(mstream)
                ready.append(e)
            d2h = 0
            queued = [0] * len(cstreams)  # bytes queued per copy stream (greedy balance)
            for c in range(nch):
                ready[c].synchronize()  # this chunk's sizes (the later chunks keep sampling)
                d2h += chost_tot[c].numel() * 8 + chost_meta[c].numel() * 8
                for cs_ in cstreams:
                    cs_.wait_event(ready[c])
                tot = chost_tot[c].tolist()
                for l in range(L):
                    ne, ni, nr = tot[l]
                    for k2, n in (("row_local", ne), ("eid", ne), ("indptr", ni), ("row_map", nr)):
                        nb = n * cpacks[c][l][k2].element_size()
                        si = min(range(len(cstreams)), key=lambda j: queued[j])
                        queued[si] += nb
                        with torch.cuda.stream(cstreams[si]):
                            chost_pk[c][l][k2][:n].copy_(cpacks[c][l][k2][:n], non_blocking=True)
                        d2h += nb
            for cs_ in cstreams + (mstream,):
                stream.wait_stream(cs_)
            ev1.record(stream)
            ev1.synchronize()
            if E2E_DEBUG:
                print(f"e2e step {i}: chunks packed at " + ", ".join(f"{ev0.elapsed_time(r):.3f}" for r in packs_ev)
                      + "; ready at " + ", ".join(f"{ev0.elapsed_time(r):.3f}" for r in ready)
                      + f" ms, end {ev0.elapsed_time(ev1):.3f} ms, {d2h / 1e6:.1f} MB", file=sys.stderr)
            if i > 0:  # the first pass warms the chunked path
                e2e_times.append(ev0.elapsed_time(ev1))
                d2h_all.append(d2h)
            continue
        flush.zero_()
        torch.cuda.synchronize()
        ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        ev0.record(stream)
        dev_in.copy_(host_in, non_blocking=True)
        step(args.warmup + i, dev_in)
        if kind == "walk":
            host_tr.copy_(traces, non_blocking=True)
            d2h = host_tr.numel() * 4
        else:
            for l in range(L):
                out.pack(l, packs[l], stream=stream, narrow=narrow)
                host_tot[l].copy_(packs[l]["totals"], non_blocking=True)
            host_meta.copy_(meta_dev, non_blocking=True)
            stream.synchronize()
            d2h = host_tot.numel() * 8 + host_meta.numel() * 8
            # the arrays split over two copy streams (both D2H copy engines busy)
            side = copy_side
            side.wait_stream(stream)
            for l in range(L):
                ne, ni, nr = (int(x) for x in host_tot[l])
                for k2, n in (("row_local", ne), ("eid", ne), ("indptr", ni), ("row_map", nr)):
                    with torch.cuda.stream(side if k2 == "eid" else stream):
                        host_pk[l][k2][:n].copy_(packs[l][k2][:n], non_blocking=True)
                    d2h += n * packs[l][k2].element_size()
            stream.wait_stream(side)
        ev1.record(stream)
        ev1.synchronize()
        e2e_times.append(ev0.elapsed_time(ev1))
        d2h_all.append(d2h)
    d2h = int(statistics.mean(d2h_all))
    e2e_ms = statistics.mean(e2e_times)

    # single-batch latency (first batch of this rank's share, eager call; after
    # e2e, whose pack buffers are sized by the full epoch's result)
    lat_ms = None
    if kind != "walk" and inputs.numel() > 0:
        one = inputs[:bs]
        lat = []
        for i in range(5):
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            step(args.warmup + i, one)
            e1.record(stream)
            e1.synchronize()
            lat.append(e0.elapsed_time(e1))
        lat_ms = statistics.median(lat[1:])

    t_min, t_max = min(times), max(times)
    if world > 1:
        rdev = torch.device("cpu") if BACKEND == "gloo" else device
        t = torch.tensor([t_total_ms, e2e_ms, t_max], dtype=torch.float64, device=rdev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        c = torch.tensor([edges, model_bytes, h2d, d2h], dtype=torch.float64, device=rdev)
        dist.all_reduce(c, op=dist.ReduceOp.SUM)
        mn = torch.tensor([t_min], dtype=torch.float64, device=rdev)
        dist.all_reduce(mn, op=dist.ReduceOp.MAX)
        t_total_ms, e2e_ms, t_max = float(t[0]), float(t[1]), float(t[2])
        t_min = float(mn[0])
        edges_all = float(c[0])
        h2d_all, d2h_all_r = int(c[2]), int(c[3])
    else:
        edges_all = float(edges)
        h2d_all, d2h_all_r = h2d, d2h
    peak, peak_src = measured_peak_hbm()
    bytes_per_launch = model_bytes / args.steps  # this rank, one step
    achieved = bytes_per_launch / (statistics.mean(times) / 1000.0) / 1e9
    line_bytes = (model_bytes + 96 * rnd_secs) / args.steps  # random 32-B sectors as 128-B lines
    line_achieved = line_bytes / (statistics.mean(times) / 1000.0) / 1e9
    # the Extract+Select stage: hop_select (+ hop_ares_big, which takes the
    # weighted heavy columns' filter, select and gather off it)
    sel_ms = sum(v for k, v in kernel_ms.items() if k.startswith("hop_select") or k.startswith("hop_ares"))
    has_ares = any(k.startswith("hop_ares") for k in kernel_ms)
    dom = None
    if sel_ms > 0:
        prof_total = sum(kernel_ms.values())
        dom = {"kernel": ("gsb::hop_select_kernel + gsb::hop_ares_big_kernel" if has_ares else
                          "gsb::hop_select_kernel") +
                         " (every hop; Extract+Select+gather: frontier ids, sampled sectors"
                         + (", weights streamed" if has_ares else "") + ", eid + row id written)",
               "bytes_per_step": sel_bytes / args.steps, "ms_per_step": sel_ms,
               "achieved": sel_bytes / args.steps / (sel_ms / 1000.0) / 1e9,
               "share_of_step": sel_ms / prof_total if prof_total > 0 else None,
               "kernels_ms": {k: round(v, 4) for k, v in kernel_ms.items()}}
    return {"value": edges_all / (t_total_ms / 1000.0), "ms_per_step": t_total_ms / args.steps, "dominant": dom,
            "edges_per_step": edges_all / args.steps,
            "e2e_value": (edges_all / args.steps) / (e2e_ms / 1000.0), "h2d": h2d_all, "d2h": d2h_all_r,
            "e2e_ms": e2e_ms,
            "achieved": achieved, "peak": peak, "peak_src": peak_src,
            "bytes_per_launch": bytes_per_launch, "line_bytes": line_bytes,
            "line_achieved": line_achieved, "clocks": clk.summary(), "gen_s": gen_s,
            "units": nunits, "graph": g, "inputs": all_inputs, "epoch_min_ms": t_min, "epoch_max_ms": t_max,
            "peak_mem": peak_mem, "lat_ms": lat_ms, "graphs": graphs is not None,
            "launches_per_step": launches_per_step}


E2E_CHUNKS = int(os.environ.get("GS_E2E_CHUNKS", 4))  # node-wise e2e: the epoch sampled and copied back in this many pipelined chunks
E2E_FIRST = int(os.environ.get("GS_E2E_FIRST", 16))  # the first chunk holds 1/E2E_FIRST of the batches (0: even chunks)
E2E_GRAPH = int(os.environ.get("GS_E2E_GRAPH", 1))  # chunk calls replayed from CUDA graphs
E2E_DEBUG = bool(os.environ.get("GS_E2E_DEBUG"))
E2E_STREAMS = int(os.environ.get("GS_E2E_STREAMS", 2))  # copy streams, bytes balanced greedily

KERNEL_OF = {"nodewise": "node-wise engine (nodewise_hop.cu: nprep / select / rows / relabel / clear per hop)",
             "shadow": "gsb::shadow_induce_kernel",
             "saint": "gsb::shadow_induce_kernel", "pinsage": "gsb::pinsage_kernel",
             "pass_full": "gsb::pass_att_kernel + gsb::nodewise_wave_kernel<1>",
             "layerwise": "gsb::layerwise_kernel", "walk": "gsb::walk_kernel"}


def kernel_name(kind, wl):
    if kind == "layerwise":  # layerwise.cu run_layerwise: which kernel takes the call
        if wl.get("mode", 0) == 1:
            return "gsb::layerwise_bm_kernel (FastGCN: candidate bitmaps)"
        if max(wl["n_per_layer"]) <= 1024 and wl["batch"] <= 1024:
            return "gsb::layerwise_sm_kernel<1024, 12> (LADIES / COUNT: shared-memory tables)"
    return KERNEL_OF[kind]


def ncu_traffic(workload):
    """DRAM bytes per launch of the dominant kernel from the committed ncu --set full capture."""
    try:
        with open(os.path.join(ROOT, "profiles", "ncu_traffic.json")) as f:
            return json.load(f).get(workload)
    except Exception:
        return None


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--workload", default="graphsage_pd", choices=sorted(WORKLOADS))
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--scaling", default="strong", choices=["strong", "weak"])
    ap.add_argument("--graph", dest="graph", action="store_true", default=True)
    ap.add_argument("--no-graph", dest="graph", action="store_false")
    args = ap.parse_args()
    wl = WORKLOADS[args.workload]
    world, rank, local = dist_env()
    if args.impl == "reference":
        run_reference(args, wl)
        return
    assert torch.cuda.is_available(), "bench.py needs a CUDA device"
    local = local % torch.cuda.device_count() if BACKEND == "gloo" else local
    torch.cuda.set_device(local)
    device = torch.device("cuda", local)
    if world > 1:
        import torch.distributed as dist
        if BACKEND == "gloo":
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=device)
    import __graft_entry__
    __graft_entry__.build()
    r = run_gpu(args, wl, world, rank, device)
    if rank == 0:
        cpu = None
        if not args.no_cpu_baseline and world == 1 and wl["kind"] != "pass_full":
            cpu, _, _ = oracle_rate(r["graph"], r["inputs"], wl)
        kind = wl["kind"]
        line = {
            "metric": METRIC, "value": r["value"], "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": r["ms_per_step"],
            "higher_is_better": True, "scaling": args.scaling, "vs_baseline": None, "dtype": "int64",
            "data": "synthetic (deterministic R-MAT, DESIGN.md input recipe)",
            "config": {"workload": wl["desc"], "graph": wl["graph"],
                       "units_per_rank": r["units"],
                       "sampled_edges_per_step": r["edges_per_step"],
                       "epoch_ms": r["ms_per_step"],
                       "epoch_min_ms": r["epoch_min_ms"], "epoch_max_ms": r["epoch_max_ms"],
                       "single_batch_latency_ms": r["lat_ms"],
                       "peak_device_memory_bytes": r["peak_mem"],
                       "cuda_graph": r["graphs"],
                       "l2": "flushed between timed steps (256 MiB write)",
                       "parallelism": (f"dp{world}: one epoch split across ranks (contiguous global batch / "
                                       f"walker ranges), graph replicated" if args.scaling == "strong" else
                                       f"dp{world}: one epoch per rank, graph replicated"),
                       "graph_gen_s": round(r["gen_s"], 2)},
            "roofline": {"bound": "hbm", "achieved": r["achieved"], "peak": r["peak"],
                         "unit": "GB/s", "frac": r["achieved"] / r["peak"],
                         "traffic": ncu_traffic(args.workload), "peak_source": r["peak_src"],
                         "kernel": kernel_name(kind, wl),
                         "algorithmic_bytes_per_launch": r["bytes_per_launch"],
                         "random_sector_ceiling_gbs": RANDOM_SECTOR_GBS,
                         "frac_of_random_sector_ceiling": r["achieved"] / RANDOM_SECTOR_GBS,
                         "line_model": {
                             "bytes_per_launch": r["line_bytes"], "achieved": r["line_achieved"],
                             "frac": r["line_achieved"] / r["peak"],
                             "note": "the same accesses with every random 32-B sector counted as "
                                     "the 128-B HBM line this B200 moves per random access "
                                     "(profiles/r01_random_access_probe.md)"}},
            "e2e": {"value": r["e2e_value"], "unit": UNIT, "h2d_bytes_per_step": r["h2d"],
                    "d2h_bytes_per_step": r["d2h"], "ms_per_step": r["e2e_ms"],
                    "d2h_gbs_over_step": r["d2h"] / (r["e2e_ms"] / 1000.0) / 1e9,
                    "note": "host copies (pinned) inside the timed region; sampled blocks packed densely "
                            "(int32 ids when the graph has < 2^31 entries) so exactly the sampled data "
                            "crosses the host link, which bounds this number"
                            + (f"; node-wise: the epoch in {E2E_CHUNKS} pipelined chunks (public calls with "
                               "batch_index_base = the chunk's first batch; the first chunk "
                               f"1/{E2E_FIRST} of the batches; each chunk's sample + pack calls replayed "
                               "from a CUDA graph per step key when graphs are on), each chunk's sizes "
                               f"read back on a stream of their own and its arrays on {E2E_STREAMS} copy "
                               "streams while the next chunks sample" if kind == "nodewise" else "")},
            "gpu_launches": args.steps * r["launches_per_step"],
            "clocks": r["clocks"],
        }
        if r["dominant"] is not None:
            # the contract's roofline is the dominant kernel's: its algorithmic
            # bytes / its duration (events after each kernel, profiling pass);
            # the whole-step numbers stay under roofline.step
            d = r["dominant"]
            step_roof = {k: line["roofline"][k] for k in ("achieved", "frac", "kernel",
                                                          "algorithmic_bytes_per_launch")}
            step_roof["note"] = "whole step (every kernel of the epoch): algorithmic bytes / step time"
            line["roofline"].update({"achieved": d["achieved"], "frac": d["achieved"] / r["peak"],
                                     "kernel": d["kernel"], "algorithmic_bytes_per_launch": d["bytes_per_step"],
                                     "kernel_ms_per_step": d["ms_per_step"], "share_of_step": d["share_of_step"],
                                     "kernels_ms": d["kernels_ms"], "step": step_roof})
        if kind == "nodewise":
            line["config"]["fanouts"] = wl["fanouts"]
            line["config"]["batch_size"] = wl["batch"]
        if cpu is not None:
            cpu["cpu_model"] = cpu_model()
            line["cpu_baseline"] = cpu
        print(json.dumps(line), flush=True)
    if world > 1:
        import torch.distributed as dist
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()

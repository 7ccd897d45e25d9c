#!/usr/bin/env python
"""Benchmark of the B200 ECSF sampling hot path (BASELINE.json metric:
"sampled edges/s & epoch sampling time at 1/2/4/8 B200; % HBM roofline").

Default workload (BASELINE.json configs[1]): GraphSAGE [25,10] uniform
neighbour sampling, batch 1024, one full epoch of seeds (196,615 = the
ogbn-products train-split size, 193 mini-batches) on an Ogbn-Products-shaped
R-MAT graph (2,449,029 nodes, 61,859,140 undirected edges -> 123,718,280 CSC
entries).  One step = one epoch (every batch, every hop: Extract, Select,
Finalize) = one launch of the cluster kernel.

Contract: python bench.py --gpus N --steps K --warmup W [--impl reference]
Multi-GPU (torchrun): one process per GPU; rank 0 generates the graph and
broadcasts it over NCCL; every rank samples its own epoch (global batch ids
rank*num_batches + b), no data-path collective ("scaling": "weak").
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

METRIC = "sampled edges/s & epoch sampling time at 1/2/4/8 B200; % HBM roofline"
UNIT = "sampled edges/s"

WORKLOADS = {
    "graphsage_pd": dict(kind="nodewise", graph="PD", fanouts=[25, 10], batch=1024,
                         seeds=196_615, replace=False, bias=0,
                         desc="GraphSAGE [25,10] uniform, batch 1024, full epoch (196,615 seeds, "
                              "193 batches), Ogbn-Products-shaped R-MAT graph"),
    "graphsage_tiny": dict(kind="nodewise", graph="tiny", fanouts=[5, 5], batch=512, seeds=512,
                           replace=False, bias=0,
                           desc="GraphSAGE [5,5] uniform, 512 seeds, 10k-node/100k-edge R-MAT"),
    "kgcn_pd": dict(kind="nodewise", graph="PD", fanouts=[8, 8], batch=1024, seeds=196_615,
                    replace=True, bias=0, desc="KGCN [8,8] with replacement, PD-shaped"),
    "pass_pd": dict(kind="nodewise", graph="PDw", fanouts=[10, 10], batch=1024, seeds=196_615,
                    replace=False, bias=2, desc="PASS-style A3 [10,10], PD-shaped weighted"),
    "shadow_pd": dict(kind="shadow", graph="PD", fanouts=[10, 5], batch=1024, seeds=196_615,
                      bias=0, desc="ShaDow [10,5] uniform + induce, PD-shaped"),
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

    REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap",
               0x8: "hw_slowdown", 0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown",
               0x80: "hw_power_brake_slowdown", 0x100: "display_clocks_setting"}

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
                    if r & bit and name != "gpu_idle":
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
    g = synth.make_graph(spec, device=device) if rank == 0 else None
    g = gdist.broadcast_graph(g, device)
    g["spec"] = spec
    return g


def nodewise_model_bytes(blocks, indptr, fanouts, L):
    """Algorithmic bytes of one node-wise step (SURVEY.md 8(d) byte model):
    per column 4 (frontier id) + 32*(1 + [v % 4 == 3]) (int64 indptr pair sector(s))
    + 32 * |distinct 32-byte sectors of the sampled positions| + 8 (block indptr);
    per sampled edge 4 (row_local) + 8 (eid); per new row 4 (row_map)."""
    meta = blocks.device_meta()            # [B, L, 8]
    total = 0
    edges = 0
    import ctypes
    from paper_conf_sosp_gonglmc0lwl23_b200 import gs
    for l in range(L):
        lb = gs._lib  # noqa
        m = meta[:, l, :]
        n_cols, n_rows, n_edges = m[:, 0], m[:, 1], m[:, 2]
        col_off, ind_off, e_off = m[:, 3], m[:, 5], m[:, 6]
        view = _layer_arrays(blocks, l)
        # per-edge column ids: from each batch's block indptr
        ecount = int(n_edges.sum())
        edges += ecount
        colv_all, sec_all = [], []
        for b in range(m.shape[0]):
            T = int(n_cols[b])
            if T == 0:
                continue
            ip = view["indptr"][int(ind_off[b]): int(ind_off[b]) + T + 1]
            E = int(n_edges[b])
            eids = view["eid"][int(e_off[b]): int(e_off[b]) + E]
            cols = view["col_map"][int(col_off[b]): int(col_off[b]) + T].to(torch.int64)
            cnt = ip[1:] - ip[:-1]
            cid = torch.repeat_interleave(torch.arange(T, device=ip.device), cnt)
            key = cid * (1 << 40) + (eids >> 3)
            sec_all.append(torch.unique(key).numel())
            colv_all.append(cols)
        cols = torch.cat(colv_all) if colv_all else torch.empty(0, dtype=torch.int64)
        ncols = cols.numel()
        straddle = int(((cols & 3) == 3).sum()) if ncols else 0
        total += ncols * (4 + 8) + 32 * (ncols + straddle) + 32 * sum(sec_all)
        total += ecount * 12 + int(n_rows.sum()) * 4
    return total, edges


def _layer_arrays(blocks, l):
    import ctypes
    from paper_conf_sosp_gonglmc0lwl23_b200 import gs

    class LB(ctypes.Structure):
        _fields_ = [("col_map", ctypes.c_void_p), ("col_capacity", ctypes.c_int64),
                    ("row_map", ctypes.c_void_p), ("row_capacity", ctypes.c_int64),
                    ("indptr", ctypes.c_void_p), ("indptr_capacity", ctypes.c_int64),
                    ("row_local", ctypes.c_void_p), ("eid", ctypes.c_void_p),
                    ("val", ctypes.c_void_p), ("edge_capacity", ctypes.c_int64),
                    ("row_prob", ctypes.c_void_p)]
    lb = LB()
    gs._lib.gs_blocks_layer.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.POINTER(LB)]
    gs._check(gs._lib.gs_blocks_layer(blocks._h, l, ctypes.byref(lb)))
    t = gs._dev_tensor
    return {"col_map": t(lb.col_map, lb.col_capacity, torch.int32, blocks),
            "row_map": t(lb.row_map, lb.row_capacity, torch.int32, blocks),
            "indptr": t(lb.indptr, lb.indptr_capacity, torch.int64, blocks),
            "row_local": t(lb.row_local, lb.edge_capacity, torch.int32, blocks),
            "eid": t(lb.eid, lb.edge_capacity, torch.int64, blocks)}


def ncu_traffic(workload):
    """DRAM bytes per launch of the dominant kernel from the committed ncu --set full capture."""
    path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        with open(path) as f:
            d = json.load(f)
        return d.get(workload)
    except Exception:
        return None


# ---------------------------------------------------------------------------
# CPU baseline / reference arm: the oracle as it stands
# ---------------------------------------------------------------------------
def oracle_nodewise_rate(g, seeds, wl, budget_s=15.0):
    import oracle
    O = oracle.Graph(g["indptr"].cpu().numpy(), g["indices"].cpu().numpy(),
                     None if g["weights"] is None else g["weights"].cpu().numpy())
    cores = len(os.sched_getaffinity(0))
    s = seeds.cpu().numpy()
    bs = wl["batch"]
    nb_total = (len(s) + bs - 1) // bs
    # calibrate on one batch, one thread
    t0 = time.perf_counter()
    r = oracle.sample_neighbors(O, s[:bs], wl["fanouts"], batch_size=bs, replace=wl["replace"],
                                bias_mode=wl["bias"], rng_key=1, num_threads=1)
    t1 = time.perf_counter() - t0
    nb = int(max(1, min(nb_total, budget_s * cores / max(t1, 1e-4))))
    t0 = time.perf_counter()
    r = oracle.sample_neighbors(O, s[:nb * bs], wl["fanouts"], batch_size=bs,
                                replace=wl["replace"], bias_mode=wl["bias"], rng_key=1,
                                num_threads=cores)
    dt = time.perf_counter() - t0
    edges = sum(len(blk["eid"]) for layers in r for blk in layers)
    return {"value": edges / dt, "unit": UNIT, "cores": cores, "kind": "oracle",
            "sample": f"first {nb} of {nb_total} batches of the workload ({edges} sampled edges, "
                      f"{dt:.2f} s wall on {cores} threads)"}, edges, dt


def run_reference(args, wl):
    world, rank, _ = dist_env()
    if rank != 0:
        return
    import synth
    g = synth.make_graph(wl["graph"], device="cuda" if torch.cuda.is_available() else "cpu")
    seeds = synth.make_seeds(wl["graph"], wl["seeds"])
    rates, total_edges, total_t = [], 0, 0.0
    for i in range(args.warmup + args.steps):
        cb, e, dt = oracle_nodewise_rate(g, seeds, wl, budget_s=3.0)
        if i >= args.warmup:
            rates.append(cb["value"])
            total_edges += e
            total_t += dt
    value = total_edges / total_t
    line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": 1000 * total_t / args.steps, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "int64", "data": "synthetic",
            "impl": "reference",
            "config": {"workload": wl["desc"], "oracle": "oracle/gso.cpp (CPU, OpenMP over batches)"},
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": cb["cores"], "kind": "oracle",
                             "sample": cb["sample"]},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------------------
# GPU arm
# ---------------------------------------------------------------------------
def run_nodewise(args, wl, world, rank, device):
    import synth
    from paper_conf_sosp_gonglmc0lwl23_b200 import dist as gdist
    from paper_conf_sosp_gonglmc0lwl23_b200 import gs
    import torch.distributed as dist
    gs.use_torch_allocator()
    t0 = time.time()
    g = make_graph_dist(wl["graph"], world, rank, device)
    gen_s = time.time() - t0
    G = gs.Graph(g["indptr"], g["indices"], g["weights"])
    seeds = synth.make_seeds(wl["graph"], wl["seeds"], device=device)
    bs = wl["batch"]
    nb = (seeds.numel() + bs - 1) // bs
    fan = wl["fanouts"]
    stream = torch.cuda.current_stream()
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=device)  # > 126 MB L2
    out = gs.Blocks()
    base_key = 0x5EED

    def step(i, blocks):
        return gs.sample_neighbors(G, seeds, fan, batch_size=bs, batch_index_base=gdist.weak_batch_base(rank, nb),
                                   replace=wl["replace"], bias_mode=wl["bias"],
                                   rng_key=base_key + 7919 * i, stream=stream, out=blocks)

    for i in range(args.warmup):
        step(i, out)
    out.sync()
    torch.cuda.synchronize()
    times, edges, model_bytes = [], 0, 0
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    with ClockSampler(torch.cuda.current_device()) as clk:
        for i in range(args.steps):
            flush.zero_()
            ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            ev0.record(stream)
            step(args.warmup + i, out)
            ev1.record(stream)
            ev1.synchronize()
            times.append(ev0.elapsed_time(ev1))
            out.sync()
            mb, e = nodewise_model_bytes(out, g["indptr"], fan, len(fan))
            model_bytes += mb
            edges += e
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    t_total_ms = sum(times)
    # e2e: the same step through the C ABI with HOST buffers (pinned), copies inside
    host_seeds = seeds.cpu().pin_memory()
    lay = [_layer_arrays(out, l) for l in range(len(fan))]
    host_out = [{k: torch.empty_like(v, device="cpu").pin_memory() for k, v in la.items()
                 if k in ("row_map", "indptr", "row_local", "eid")} for la in lay]
    meta_h = torch.empty_like(out.device_meta(), device="cpu").pin_memory()
    dev_seeds = torch.empty_like(seeds)
    h2d = host_seeds.numel() * 4
    d2h = meta_h.numel() * 8 + sum(t.numel() * t.element_size() for ho in host_out for t in ho.values())
    e2e_times = []
    for i in range(max(2, min(args.steps, 5))):
        flush.zero_()
        torch.cuda.synchronize()
        ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        ev0.record(stream)
        dev_seeds.copy_(host_seeds, non_blocking=True)
        gs.sample_neighbors(G, dev_seeds, fan, batch_size=bs, batch_index_base=gdist.weak_batch_base(rank, nb),
                            replace=wl["replace"], bias_mode=wl["bias"], rng_key=base_key + i,
                            stream=stream, out=out)
        meta_h.copy_(out.device_meta(), non_blocking=True)
        for la, ho in zip(lay, host_out):
            for k, t in ho.items():
                t.copy_(la[k], non_blocking=True)
        ev1.record(stream)
        ev1.synchronize()
        e2e_times.append(ev0.elapsed_time(ev1))
    e2e_ms = statistics.mean(e2e_times)
    if world > 1:
        t = torch.tensor([t_total_ms, e2e_ms], dtype=torch.float64, device=device)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        c = torch.tensor([edges, model_bytes], dtype=torch.float64, device=device)
        dist.all_reduce(c, op=dist.ReduceOp.SUM)
        t_total_ms, e2e_ms = float(t[0]), float(t[1])
        edges_all, bytes_all = float(c[0]), float(c[1])
    else:
        edges_all, bytes_all = float(edges), float(model_bytes)
    ms_per_step = t_total_ms / args.steps
    value = edges_all / (t_total_ms / 1000.0)
    peak, peak_src = measured_peak_hbm()
    bytes_per_launch = model_bytes / args.steps           # this rank, one launch = one epoch
    achieved = bytes_per_launch / (statistics.mean(times) / 1000.0) / 1e9
    res = {"value": value, "ms_per_step": ms_per_step, "edges_per_step": edges_all / args.steps,
           "e2e_value": edges_all / args.steps * world / (e2e_ms / 1000.0) if False else
           (edges / args.steps) * world / (e2e_ms / 1000.0),
           "h2d": h2d, "d2h": d2h, "achieved": achieved, "peak": peak, "peak_src": peak_src,
           "bytes_per_launch": bytes_per_launch, "clocks": clk.summary(), "gen_s": gen_s,
           "num_batches": nb, "times": times, "graph": g, "seeds": seeds}
    return res


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--workload", default="graphsage_pd", choices=sorted(WORKLOADS))
    ap.add_argument("--no-cpu-baseline", action="store_true")
    args = ap.parse_args()
    wl = WORKLOADS[args.workload]
    world, rank, local = dist_env()
    if args.impl == "reference":
        if world > 1:
            import torch.distributed as dist
            if rank != 0:
                return
        run_reference(args, wl)
        return
    assert torch.cuda.is_available(), "bench.py needs a CUDA device"
    torch.cuda.set_device(local)
    device = torch.device("cuda", local)
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl", device_id=device)
    import __graft_entry__
    __graft_entry__.build()
    if wl["kind"] != "nodewise":
        raise SystemExit(f"workload kind {wl['kind']} not wired into bench.py yet")
    r = run_nodewise(args, wl, world, rank, device)
    if rank == 0:
        cpu = None
        if not args.no_cpu_baseline and world == 1:
            cpu, _, _ = oracle_nodewise_rate(r["graph"], r["seeds"], wl)
        traffic = ncu_traffic(args.workload)
        line = {
            "metric": METRIC, "value": r["value"], "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": r["ms_per_step"],
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "int64",
            "data": "synthetic (deterministic R-MAT, DESIGN.md input recipe)",
            "config": {"workload": wl["desc"], "graph": wl["graph"],
                       "fanouts": wl.get("fanouts"), "batch_size": wl["batch"],
                       "num_batches_per_rank": r["num_batches"],
                       "sampled_edges_per_step": r["edges_per_step"],
                       "epoch_ms": r["ms_per_step"],
                       "l2": "flushed between timed steps (256 MiB write), graph 0.5 GB > L2",
                       "parallelism": f"dp{world} (epoch per rank, graph replicated)",
                       "graph_gen_s": round(r["gen_s"], 2)},
            "roofline": {"bound": "hbm", "achieved": r["achieved"], "peak": r["peak"],
                         "unit": "GB/s", "frac": r["achieved"] / r["peak"],
                         "traffic": traffic, "peak_source": r["peak_src"],
                         "kernel": "gsb::nodewise_kernel<8> (1 launch = 1 epoch)",
                         "algorithmic_bytes_per_launch": r["bytes_per_launch"]},
            "e2e": {"value": r["e2e_value"], "unit": UNIT, "h2d_bytes_per_step": r["h2d"],
                    "d2h_bytes_per_step": r["d2h"]},
            "gpu_launches": args.steps,
            "clocks": r["clocks"],
        }
        if cpu is not None:
            line["cpu_baseline"] = cpu
        print(json.dumps(line), flush=True)
    if world > 1:
        import torch.distributed as dist
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()

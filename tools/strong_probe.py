"""Strong-scaling probe on one GPU: the device time of 1/N of the PD GraphSAGE
epoch (rank 0's contiguous batch range, as bench.py --gpus N gives it),
CUDA-graph replayed, for N = 1, 2, 4, 8 -- what each rank of an N-GPU run
computes.  Prints one line per N."""
import sys
import time

import torch

sys.path.insert(0, ".")
import synth  # noqa: E402
from paper_conf_sosp_gonglmc0lwl23_b200 import dist as gdist, gs  # noqa: E402


def main():
    gs.use_torch_allocator()
    g = synth.make_graph("PD", device="cuda")
    G = gs.Graph(g["indptr"], g["indices"], g["weights"])
    seeds = synth.make_seeds("PD", 196_615).cuda()
    bs = 1024
    for N in (1, 2, 4, 8):
        s0, s1, wbase = gdist.shard_epoch(seeds.numel(), bs, N, 0)
        x = seeds[s0:s1].contiguous()
        out = gs.Blocks()
        for i in range(3):
            gs.sample_neighbors(G, x, [25, 10], batch_size=bs, batch_index_base=wbase, rng_key=7 + i, out=out)
        torch.cuda.synchronize()
        cs = torch.cuda.Stream()
        gr = torch.cuda.CUDAGraph()
        with torch.cuda.graph(gr, stream=cs):
            gs.sample_neighbors(G, x, [25, 10], batch_size=bs, batch_index_base=wbase, rng_key=9, stream=cs,
                                out=out)
        torch.cuda.synchronize()
        flush = torch.empty(64 << 20, dtype=torch.int32, device="cuda")
        ts = []
        for i in range(10):
            flush.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            gr.replay()
            e1.record()
            e1.synchronize()
            ts.append(e0.elapsed_time(e1))
        t = sorted(ts)[len(ts) // 2]
        print(f"N={N}: rank 0 samples {s1 - s0} seeds ({(s1 - s0 + bs - 1) // bs} batches) in {t:.4f} ms "
              f"-> ideal-link speedup {globals()["ts_1"] / t if N > 1 else 1.0:.2f}x" if N > 1 else
              f"N=1: {s1 - s0} seeds in {t:.4f} ms")
        if N == 1:
            globals()["ts_1"] = t




def kernels(N=8):
    gs.use_torch_allocator()
    g = synth.make_graph("PD", device="cuda")
    G = gs.Graph(g["indptr"], g["indices"], g["weights"])
    seeds = synth.make_seeds("PD", 196_615).cuda()
    bs = 1024
    s0, s1, wbase = gdist.shard_epoch(seeds.numel(), bs, N, 0)
    x = seeds[s0:s1].contiguous()
    out = gs.Blocks()
    for i in range(3):
        gs.sample_neighbors(G, x, [25, 10], batch_size=bs, batch_index_base=wbase, rng_key=7 + i, out=out)
    gs.set_profiling(True)
    acc = {}
    for i in range(5):
        gs.sample_neighbors(G, x, [25, 10], batch_size=bs, batch_index_base=wbase, rng_key=7 + i, out=out)
        for name, ms in gs.blocks_profile(out):
            acc[name] = acc.get(name, 0.0) + ms / 5
    gs.set_profiling(False)
    print(f"N={N} per-kernel ms:", {k: round(v, 4) for k, v in acc.items()}, "sum", round(sum(acc.values()), 4))


if __name__ == "__main__":
    ts_1 = None
    main()
    kernels(8)
    kernels(1)

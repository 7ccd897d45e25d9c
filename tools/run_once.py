"""Runs a workload a few times (for ncu / nsys-style captures): python tools/run_once.py <workload> [reps]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import synth  # noqa: E402
from paper_conf_sosp_gonglmc0lwl23_b200 import gs  # noqa: E402

wl_name = sys.argv[1] if len(sys.argv) > 1 else "graphsage_pd"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 2
wl = bench.WORKLOADS[wl_name]
gs.use_torch_allocator()
g = synth.make_graph(wl["graph"], device="cuda")
G = gs.Graph(g["indptr"], g["indices"], g["weights"])
out = gs.Blocks()
if wl["kind"] in ("nodewise", "shadow"):
    seeds = synth.make_seeds(wl["graph"], wl["seeds"], device="cuda")
    for i in range(reps):
        if wl["kind"] == "nodewise":
            gs.sample_neighbors(G, seeds, wl["fanouts"], batch_size=wl["batch"], replace=wl["replace"],
                                bias_mode=wl["bias"], rng_key=i, out=out)
        else:
            gs.sample_shadow(G, seeds, wl["fanouts"], batch_size=wl["batch"], bias_mode=wl["bias"],
                             rng_key=i, out=out)
elif wl["kind"] == "pass_full":
    N = g["indptr"].numel() - 1
    X = synth.make_grid_matrix(21, N, wl["F"], device="cuda")
    W1 = synth.make_grid_matrix(22, wl["F"], wl["H"], device="cuda")
    W2 = synth.make_grid_matrix(23, wl["F"], wl["H"], device="cuda")
    Ga = gs.Graph(g["indptr"], g["indices"], g["weights"])
    seeds = synth.make_seeds(wl["graph"], wl["seeds"], device="cuda")
    for i in range(reps):
        att = gs.pass_attention(G, X, W1, W2, wl["W3"])
        Ga.set_weights(att)
        gs.sample_neighbors(Ga, seeds, wl["fanouts"], batch_size=wl["batch"], bias_mode=1, rng_key=i, out=out)
elif wl["kind"] == "pinsage":
    seeds = synth.make_seeds(wl["graph"], wl["seeds"], device="cuda")
    for i in range(reps):
        gs.sample_pinsage(G, seeds, wl["topk"], wl["num_walks"], wl["walk_length"], wl["restart"],
                          batch_size=wl["batch"], rng_key=i, out=out)
elif wl["kind"] == "saint":
    roots = synth.make_seeds(wl["graph"], wl["seeds"], device="cuda")
    for i in range(reps):
        gs.sample_saint_rw(G, roots, wl["walk_length"], batch_size=wl["batch"], rng_key=i, out=out)
elif wl["kind"] == "layerwise":
    seeds = synth.make_seeds(wl["graph"], wl["seeds"], device="cuda")
    for i in range(reps):
        gs.sample_layerwise(G, seeds, wl["n_per_layer"], batch_size=wl["batch"],
                            prob_mode=wl["mode"], rng_key=i, out=out)
else:
    starts = torch.arange(g["indptr"].numel() - 1, dtype=torch.int32, device="cuda")
    tr = torch.empty((starts.numel(), wl["length"] + 1), dtype=torch.int32, device="cuda")
    for i in range(reps):
        gs.random_walk(G, starts, wl["length"], p=wl["p"], q=wl["q"], rng_key=i, out=tr)
torch.cuda.synchronize()
print("done", wl_name)

"""Per-kernel device times of one node-wise epoch (the library's event
profile): python tools/kernel_profile.py <graph> <fanouts> <bias> [seeds]
e.g. PDw 10,10 2  (PASS-style) / PD 25,10 0 (GraphSAGE) / PD 8,8 0 replace."""
import sys

import torch

sys.path.insert(0, ".")
import synth  # noqa: E402
from paper_conf_sosp_gonglmc0lwl23_b200 import gs  # noqa: E402


def main():
    graph, fan, bias = sys.argv[1], [int(x) for x in sys.argv[2].split(",")], int(sys.argv[3])
    replace = len(sys.argv) > 4 and sys.argv[4] == "replace"
    gs.use_torch_allocator()
    g = synth.make_graph(graph, device="cuda")
    G = gs.Graph(g["indptr"], g["indices"], g["weights"])
    n = {"PD": 196_615, "PDw": 196_615, "PP": 1_207_179}.get(graph, 100_000)
    seeds = synth.make_seeds(graph, n).cuda()
    out = gs.Blocks()
    for i in range(2):
        gs.sample_neighbors(G, seeds, fan, batch_size=1024, replace=replace, bias_mode=bias, rng_key=7 + i, out=out)
    gs.set_profiling(True)
    acc = {}
    for i in range(3):
        gs.sample_neighbors(G, seeds, fan, batch_size=1024, replace=replace, bias_mode=bias, rng_key=9 + i, out=out)
        for name, ms in gs.blocks_profile(out):
            acc[name] = acc.get(name, 0.0) + ms / 3
    gs.set_profiling(False)
    torch.cuda.synchronize()
    print(graph, fan, bias, {k: round(v, 4) for k, v in acc.items()}, "sum", round(sum(acc.values()), 4))


if __name__ == "__main__":
    main()

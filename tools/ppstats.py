"""Degree statistics of the node-wise frontiers (which A-Res select path each column takes)."""
import sys, torch
sys.path.insert(0, ".")
import synth
from paper_conf_sosp_gonglmc0lwl23_b200 import gs
name = sys.argv[1] if len(sys.argv) > 1 else "PP"
fan = [15, 10, 5]
g = synth.make_graph(name, device="cuda")
G = gs.Graph(g["indptr"], g["indices"], g["weights"])
seeds = synth.make_seeds(name, 8 * 1024, device="cuda")
b = gs.sample_neighbors(G, seeds, fan, batch_size=1024, bias_mode=1, rng_key=3).sync()
deg = (g["indptr"][1:] - g["indptr"][:-1])
edges = [0, 5, 10, 15, 32, 64, 128, 256, 1024, 4096, 1 << 40]
for l in range(len(fan)):
    cols = torch.cat([b.view(i, l)["col_map"] if l == 0 else b.view(i, l - 1)["row_map"] for i in range(8)]).long()
    d = deg[cols].double()
    print(f"hop {l} k={fan[l]}: cols {cols.numel()/8:.0f}/batch mean d {d.mean():.1f} sum d {d.sum()/8:.3g}/batch")
    for a, c in zip(edges[:-1], edges[1:]):
        m = (d > a) & (d <= c)
        print(f"   ({a},{c}]: cols {m.double().mean()*100:5.1f}%  sum d {d[m].sum()/d.sum()*100:5.1f}%")

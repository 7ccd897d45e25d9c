"""A-Res on PP: how much of the heavy-column (d > 64) work repeats across the
batches of one group -- sum of d over (batch, heavy column) pairs vs over the
distinct heavy columns of each 64-batch group -- plus the per-kernel profile."""
import sys

import torch

sys.path.insert(0, ".")
import synth  # noqa: E402
from paper_conf_sosp_gonglmc0lwl23_b200 import gs  # noqa: E402


def main():
    gs.use_torch_allocator()
    g = synth.make_graph("PP", device="cuda")
    G = gs.Graph(g["indptr"], g["indices"], g["weights"])
    deg = (g["indptr"][1:] - g["indptr"][:-1])
    seeds = synth.make_seeds("PP", 1_207_179).cuda()
    bs, fo = 1024, [15, 10, 5]
    out = gs.Blocks()
    gs.sample_neighbors(G, seeds, fo, batch_size=bs, rng_key=7, bias_mode=1, out=out)
    gs.set_profiling(True)
    gs.sample_neighbors(G, seeds, fo, batch_size=bs, rng_key=8, bias_mode=1, out=out)
    prof = {n: round(ms, 3) for n, ms in gs.blocks_profile(out)}
    gs.set_profiling(False)
    print("per-kernel ms:", prof, "sum", round(sum(prof.values()), 2))
    out.sync()
    for l in range(3):
        for WB in (16, 64):
            pairs = sd = sdu = 0
            for b0 in range(0, out.num_batches, WB):
                cols = []
                for b in range(b0, min(b0 + WB, out.num_batches)):
                    c = out.view(b, l)["col_map"].long()
                    cols.append(c[deg[c] > 64])
                c = torch.cat(cols)
                pairs += c.numel()
                sd += int(deg[c].sum())
                u = torch.unique(c)
                sdu += int(deg[u].sum())
            print(f"hop {l} WB={WB}: heavy pairs {pairs}, sum d {sd:.3e}, distinct-per-group sum d {sdu:.3e}, "
                  f"ratio {sd / max(sdu, 1):.2f}")


if __name__ == "__main__":
    main()

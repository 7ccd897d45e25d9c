"""Times the Table-4 operator kernels (ops.cu) on the PD-shaped graph, CUDA
events on the launching stream, L2 flushed between reps, and prints achieved
GB/s against their algorithmic bytes:
  A[:, F]        F = 1,000,000 columns: per column 4 (id) + 16 (indptr pair, twice:
                 degree pass and copy pass) + 8 (out indptr, written + scanned);
                 per entry 4 (index read) + 4 (row) + 8 (eid) + 4 (val) written
  A.sum(axis=0)  per entry 4 read; per column 16 (indptr) + 4
  A <op> v       per entry 4 read + 4 written
  A.sum(axis=1)  per entry 8 read (row, val) + an 8-byte fp64 atomic."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_sosp_gonglmc0lwl23_b200 import gs  # noqa: E402

gs.load_library()
gs.use_torch_allocator()
g = synth.make_graph("PD", device="cuda")
G = gs.Graph(g["indptr"], g["indices"], g["weights"])
f = synth.make_seeds("PD", 1_000_000, device="cuda")
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
peak = json.load(open(os.path.join(os.path.dirname(__file__), "..", "MEASURED_PEAKS.json")))["hbm_gbs"]


def timed(fn, reps=10):
    ts = []
    for _ in range(reps):
        flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        b.synchronize()
        ts.append(a.elapsed_time(b))
    ts.sort()
    return ts[len(ts) // 2]


M = gs.Matrix.slice_columns(G, f)
nnz = M.view()["row"].numel()
n = f.numel()
res = {}
ms = timed(lambda: gs.Matrix.slice_columns(G, f))
res["slice_columns"] = (ms, n * (4 + 16 + 16 + 16) + nnz * 20)
out0 = torch.empty(n, dtype=torch.float32, device="cuda")
ms = timed(lambda: M.sum(0))
res["sum_axis0"] = (ms, n * 20 + nnz * 4)
ms = timed(lambda: M.elementwise_(2, 1.0))
res["elementwise"] = (ms, nnz * 8)
ms = timed(lambda: M.sum(1))
res["sum_axis1"] = (ms, nnz * 8 + g["indptr"].numel() * 12)
for k, (ms, by) in res.items():
    print(json.dumps({"op": k, "ms": ms, "bytes": by, "GBps": by / ms / 1e6, "frac": by / ms / 1e6 / peak,
                      "nnz": nnz, "n_cols": n}))

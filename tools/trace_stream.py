"""Analyse a GS_TRACE file of the node-wise stream kernel.
usage: python tools/trace_stream.py trace.bin"""
import sys
import numpy as np
raw = np.fromfile(sys.argv[1], dtype=np.uint64).astype(np.int64)
ntk = len(raw) // 12
a = raw[:ntk * 8].reshape(-1, 8)
s2 = raw[ntk * 8:].reshape(-1, 4)
ok = (a[:, 0] > 0) & (a[:, 6] > 0)
a, s2 = a[ok], s2[ok]
t0 = a[:, 0].min()
l = (a[:, 7] >> 12) & 0xF
print("tiles", len(a), "span us", (a[:, 6].max() - t0) / 1e3)
names = ["claim->start", "select", "wait_sel", "flag", "lookback", "emit+"]
for hop in sorted(set(l.tolist())):
    m = l == hop
    d = np.diff(a[m][:, [0, 1, 2, 3, 4, 5, 6]], axis=1) / 1e3
    print(f"hop {hop}: tiles {m.sum()}")
    for i, n in enumerate(names):
        print(f"   {n:12s} mean {d[:, i].mean():8.2f} us  p90 {np.percentile(d[:, i], 90):8.2f}")
    w = s2[m]
    good = w[:, 2] > 0
    if good.sum():
        w = w[good]
        st = a[m][good][:, 1]
        print(f"   warp0: indptr {(w[:,0]-st).mean()/1e3:.2f}  positions {(w[:,1]-w[:,0]).mean()/1e3:.2f}"
              f"  gather+insert {(w[:,2]-w[:,1]).mean()/1e3:.2f}  (warp0 done -> all done {(a[m][good][:,2]-w[:,2]).mean()/1e3:.2f})")
busy = (a[:, 6] - a[:, 0]).sum() / 1e3
print("sum of tile durations us", round(busy), "-> avg concurrency", busy / ((a[:, 6].max() - t0) / 1e3))

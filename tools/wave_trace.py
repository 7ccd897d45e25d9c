"""Phase breakdown of the wave kernel from a GS_TRACE file: python tools/wave_trace.py trace.txt"""
import sys
import numpy as np
rows = np.loadtxt(sys.argv[1], dtype=np.int64).reshape(-1, 5)
# keep the last launch (super-step indices restart at 0)
starts = np.nonzero(rows[:, 0] == 0)[0]
r = rows[starts[-1]:]
t = r[:, 1:]
prev = np.concatenate([[t[0, 0]], t[:-1, 3]])
ph0 = (t[:, 0] - prev) / 1e3
ph1 = (t[:, 1] - t[:, 0]) / 1e3
ph2 = (t[:, 2] - t[:, 1]) / 1e3
ph3 = (t[:, 3] - t[:, 2]) / 1e3
print(f"steps {len(r)} span {(t[-1, 3] - t[0, 0]) / 1e3:.1f} us")
print(f"segments(us) sum {ph0.sum():.1f}  phase1 sum {ph1.sum():.1f}  phase2 sum {ph2.sum():.1f}  phase3 sum {ph3.sum():.1f}")
for i in range(len(r)):
    print(f"{i:4d} seg {ph0[i]:7.1f} p1 {ph1[i]:7.1f} p2 {ph2[i]:7.1f} p3 {ph3[i]:7.1f}")

import os
tf = sys.argv[1] + ".tasks"
if os.path.exists(tf):
    a = np.fromfile(tf, dtype=np.uint64).astype(np.int64).reshape(-1, 4096, 3)
    names = {0: "A", 1: "C", 2: "B", 3: "Z"}
    S = a.shape[0]
    for s in range(S):
        e = a[s]
        e = e[e[:, 0] > 0]
        if len(e) == 0:
            continue
        st = e[:, 2] & 0xFF
        hop = (e[:, 2] >> 8) & 0xFF
        dur = (e[:, 1] - e[:, 0]) / 1e3
        t0 = e[:, 0].min()
        parts = []
        for k in sorted(set(zip(st.tolist(), hop.tolist()))):
            m = (st == k[0]) & (hop == k[1])
            parts.append(f"{names[k[0]]}{k[1]}: n={m.sum()} mean={dur[m].mean():.1f} max={dur[m].max():.1f} end={((e[m, 1] - t0).max()) / 1e3:.1f}")
        print(f"step {s}: " + " | ".join(parts))

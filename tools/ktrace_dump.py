"""Per-k-block clocks of the traced task (OOO_KTASK) from an engine_trace npz:
producer issue, MMA wait start / passed, MMAs + commit issued (cycles from
the first producer issue).  python tools/ktrace_dump.py NPZ"""
import sys

import numpy as np

d = np.load(sys.argv[1], allow_pickle=True)
raw = d["raw"]
base = 2 * 200000 * 8
k = raw[base + 150000 * 8: base + (150000 + 1024) * 8].reshape(-1, 8).astype(np.int64)
n = int((k[:, 0] > 0).sum())
k = k[:n]
t0 = k[0, 0]
print("kb  issue   wait0   pass    mma_done  wait  issue->pass  mma_span  gap_from_prev_mma")
prev = None
for i, r in enumerate(k):
    gap = r[3] - prev if prev is not None else 0
    print(f"{i:2d} {r[0]-t0:7d} {r[2]-t0:7d} {r[3]-t0:7d} {r[4]-t0:8d} {r[3]-r[2]:6d} {r[3]-r[0]:8d} {r[4]-r[3]:8d} {gap:8d}")
    prev = r[4]

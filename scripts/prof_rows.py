"""Summarise per-row phase timestamps written with SPGEMM_PROF_GROUP / SPGEMM_PROF_OUT."""
import sys
import numpy as np
d = np.fromfile(sys.argv[1], dtype=np.uint64).reshape(-1, 4)
d = d[d[:, 3] > 0]
sm = (d[:, 0] >> 32).astype(np.int64)
t1, t2, t3 = d[:, 1].astype(np.int64), d[:, 2].astype(np.int64), d[:, 3].astype(np.int64)
t0 = t1.min()
acc, rank, tot = (t2 - t1) / 1e3, (t3 - t2) / 1e3, (t3 - t1) / 1e3
print(f"rows {len(d)}  kernel span {(t3.max() - t0) / 1e3:.1f} us")
for name, x in (("accumulate", acc), ("gather+rank+write", rank), ("row total", tot)):
    print(f"{name:20s} mean {x.mean():8.2f} us  p50 {np.median(x):8.2f}  p99 {np.percentile(x, 99):8.2f}  max {x.max():8.2f}")
busy = np.bincount(sm, weights=tot)
print(f"per-SM busy (sum of row times / concurrency) max {busy.max():.0f} us mean {busy.mean():.0f} us")
late = np.argsort(t3)[-5:]
print("last rows to finish (start us, dur us):", [(int((t1[i] - t0) / 1e3), round(tot[i], 1)) for i in late])

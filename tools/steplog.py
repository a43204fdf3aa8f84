"""Per-step durations from gpurun_out/steplog.txt (-DSAFARA_STEPLOG build):
per lockstep k-part, the median time of each step since the launch's first
step, and the median per-step duration."""
import sys

import numpy as np

ncol = int(sys.argv[2]) if len(sys.argv) > 2 else 70
rows = [[int(v) for v in l.split()] for l in open(sys.argv[1]) if l.strip()]
d = np.array([r[1:] for r in rows], dtype=np.float64)
c = np.array([r[0] for r in rows])
t0 = d[d > 0].min()
for p in range(2):
    m = (c >= p * ncol) & (c < (p + 1) * ncol)
    x = d[m][:, 2:]
    n = int((x > 0).sum(axis=1).max())
    med = [np.median((x[:, s][x[:, s] > 0] - t0) / 1e3) for s in range(n)]
    dur = np.diff(med)
    print(f"part {p}: {n} steps; step starts (us):", " ".join(f"{v:.1f}" for v in med))
    print(f"   step durations (us):", " ".join(f"{v:.2f}" for v in dur))

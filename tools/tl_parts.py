"""Per-part end times of the last launch in gpurun_out/timeline.txt (lockstep:
CTA c -> column tile c % ncol, k-part c // ncol; faces = the last --nface)."""
import argparse
from collections import defaultdict

import numpy as np

ap = argparse.ArgumentParser()
ap.add_argument("file")
ap.add_argument("--ncol", type=int, default=70)
ap.add_argument("--nface", type=int, default=8)
a = ap.parse_args()
by = defaultdict(list)
for l in open(a.file):
    x = [int(v) for v in l.split()]
    by[x[0]].append(x[1:])
for L in sorted(by)[-2:]:
    d = np.array(by[L], dtype=np.float64)
    t0 = d[:, 1].min()
    e = (d[:, 2] - t0) / 1e3
    n = len(d)
    nc = n - a.nface
    c = d[:, 0].astype(int)
    print(f"launch {L}: span {e.max():.1f} us")
    for p in range(nc // a.ncol):
        m = (c >= p * a.ncol) & (c < (p + 1) * a.ncol)
        print(f"  part {p}: end min {e[m].min():6.1f} med {np.median(e[m]):6.1f} max {e[m].max():6.1f}")
    m = c >= nc
    if m.any():
        print(f"  faces : end min {e[m].min():6.1f} med {np.median(e[m]):6.1f} max {e[m].max():6.1f}")

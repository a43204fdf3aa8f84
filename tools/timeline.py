"""Summarise gpurun_out/timeline.txt of a -DSAFARA_TIMELINE build: per-CTA
start/end/smid of the last 4 launches ("launch cta start end smid|cyc<<16").
Per launch: compute and boundary-face CTAs (the last --nface CTAs) separately,
and the idle gap between consecutive launches (last CTA end -> first CTA
start of the next launch)."""
import argparse
from collections import defaultdict

ap = argparse.ArgumentParser()
ap.add_argument("file")
ap.add_argument("--nface", type=int, default=8)
a = ap.parse_args()
by = defaultdict(list)
for l in open(a.file):
    if l.strip():
        x = [int(v) for v in l.split()]
        by[x[0]].append(tuple(x[1:]))
launches = sorted(by)
t0 = min(r[1] for r in by[launches[0]] if r[1])


def summ(name, rs):
    if not rs:
        return
    st = sorted((r[1] - t0) / 1e3 for r in rs)
    en = sorted((r[2] - t0) / 1e3 for r in rs)
    du = sorted((r[2] - r[1]) / 1e3 for r in rs)
    cy = sorted((r[3] >> 16) / 1e3 for r in rs)
    print(f"  {name:8s} n={len(rs):3d} start min {st[0]:7.1f} max {st[-1]:7.1f} | "
          f"end min {en[0]:7.1f} med {en[len(en)//2]:7.1f} max {en[-1]:7.1f} | "
          f"dur med {du[len(du)//2]:6.1f} max {du[-1]:6.1f} us | "
          f"kcyc med {cy[len(cy)//2]:7.1f} (clk {cy[len(cy)//2] / du[len(du)//2]:.3f} GHz)")


prev_end = None
for L in launches:
    rs = by[L]
    n = len(rs)
    first = min(r[1] for r in rs)
    last = max(r[2] for r in rs)
    gap = "" if prev_end is None else f"  gap from previous launch {(first - prev_end) / 1e3:.2f} us"
    print(f"launch {L}: span {(last - first) / 1e3:.1f} us{gap}")
    summ("compute", rs[:n - a.nface])
    summ("faces", rs[n - a.nface:])
    prev_end = last

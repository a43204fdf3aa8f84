"""Summarise gpurun_out/timeline.txt (per-CTA start/end/smid of the LAST
launch of a -DSAFARA_TIMELINE build).  Compute CTAs and boundary-face CTAs
(the last `nface` CTAs, --nface) are reported separately."""
import argparse

ap = argparse.ArgumentParser()
ap.add_argument("file")
ap.add_argument("--nface", type=int, default=8)
a = ap.parse_args()
rows = [tuple(int(x) for x in l.split()) for l in open(a.file) if l.strip()]
t0 = min(r[1] for r in rows if r[1])
n = len(rows)


def summ(name, rs):
    if not rs:
        return
    st = sorted((r[1] - t0) / 1e3 for r in rs)
    en = sorted((r[2] - t0) / 1e3 for r in rs)
    du = sorted((r[2] - r[1]) / 1e3 for r in rs)
    cy = sorted((r[3] >> 16) / 1e3 for r in rs)
    print(f"{name:8s} n={len(rs):3d} start med {st[len(st)//2]:6.1f} max {st[-1]:6.1f} | "
          f"end min {en[0]:6.1f} med {en[len(en)//2]:6.1f} max {en[-1]:6.1f} | "
          f"dur min {du[0]:6.1f} med {du[len(du)//2]:6.1f} max {du[-1]:6.1f} us | "
          f"kcycles med {cy[len(cy)//2]:7.1f} max {cy[-1]:7.1f} (clk {cy[len(cy)//2] / du[len(du)//2]:.3f} GHz)")


summ("compute", rows[:n - a.nface])
summ("faces", rows[n - a.nface:])

"""Summarise gpurun_out/timeline.txt (per-CTA start/end/smid of the LAST launch)."""
import sys
rows = [tuple(int(x) for x in l.split()) for l in open(sys.argv[1]) if l.strip()]
t0 = min(r[1] for r in rows if r[1])
st = sorted((r[1] - t0) / 1e3 for r in rows)
en = sorted((r[2] - t0) / 1e3 for r in rows)
dur = sorted((r[2] - r[1]) / 1e3 for r in rows)
print(f"CTAs {len(rows)}  start: min {st[0]:.1f} med {st[len(st)//2]:.1f} max {st[-1]:.1f} us")
print(f"end: min {en[0]:.1f} med {en[len(en)//2]:.1f} max {en[-1]:.1f} us; duration min {dur[0]:.1f} med {dur[len(dur)//2]:.1f} max {dur[-1]:.1f}")
sms = {}
for r in rows:
    sms.setdefault(r[3], []).append(r[0])
multi = {k: v for k, v in sms.items() if len(v) > 1}
print(f"distinct SMs {len(sms)}; SMs hosting >1 CTA: {len(multi)} e.g. {list(multi.items())[:5]}")
late = sorted(rows, key=lambda r: r[1])[-5:]
print("latest starters (cta, start_us, end_us, sm):", [(r[0], round((r[1]-t0)/1e3,1), round((r[2]-t0)/1e3,1), r[3]) for r in late])

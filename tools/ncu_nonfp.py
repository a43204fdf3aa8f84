"""Non-FP64 executed instructions per CUDA source line (cuda,sass view)."""
import csv
import io
import subprocess
import sys
from collections import defaultdict, Counter

rep = sys.argv[1]
npts = float(sys.argv[2]) if len(sys.argv) > 2 else 4251528
txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(txt)))
agg = defaultdict(Counter)
fname = ix = line = None
for r in rows:
    if not r:
        continue
    if r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if r[0] == "Line No":
        ix = {h: i for i, h in enumerate(r)}
        continue
    if ix is None or len(r) < 6:
        continue
    if r[0]:
        line = (fname, r[0], r[1][:70])
    sass = r[ix["Source"] + 2] if False else r[3]
    try:
        n = int(r[ix["Instructions Executed"]] or 0)
    except (ValueError, KeyError):
        continue
    op = sass.strip().split()
    if not op or op[0] == "-":
        continue
    o = op[1] if op[0].startswith("@") else op[0]
    o = o.split(".")[0]
    if o in ("DFMA", "DMUL", "DADD"):
        continue
    agg[line][o] += n
tot = sum(sum(c.values()) for c in agg.values())
print(f"non-FP64 warp-instr per point: {tot * 32 / npts:.1f}")
for (f, ln, src), c in sorted(agg.items(), key=lambda x: -sum(x[1].values()))[:30]:
    s = sum(c.values())
    print(f"{s * 32 / npts:6.1f}/pt {f}:{ln:>4} {src.strip()[:60]:60s} {dict(c.most_common(4))}")

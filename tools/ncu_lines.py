"""Per-CUDA-source-line stall samples and executed instructions from an ncu report
(--print-source cuda,sass).  usage: python tools/ncu_lines.py rep [topN]"""
import csv
import io
import subprocess
import sys
from collections import defaultdict

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(txt)))
agg = defaultdict(lambda: [0, 0, 0, ""])
fname = None
ix = None
line = None
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
        line = (fname, r[0], r[1][:80])
    if line is None:
        continue
    try:
        s = int(r[ix["Warp Stall Sampling (All Samples)"]] or 0)
        n = int(r[ix["Instructions Executed"]] or 0)
    except (ValueError, KeyError):
        continue
    a = agg[line]
    a[0] += s
    a[1] += n
tot_s = sum(v[0] for v in agg.values())
tot_n = sum(v[1] for v in agg.values())
print(f"samples {tot_s}  warp-instr {tot_n}")
for (f, ln, src), (s, n, _, _) in sorted(agg.items(), key=lambda x: -x[1][0])[:top]:
    print(f"{s / tot_s * 100:5.1f}% smp {n / tot_n * 100:5.1f}% ins  {f}:{ln:>4}  {src.strip()}")

"""Top SASS instructions of an ncu report by stall samples, with the
preceding instructions for context (which barrier / load a spin is on).
usage: python tools/ncu_hot.py REP [N]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 8
txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(txt)))
hdr = rows[1]
data = rows[2:]
ia, isrc, ismp, iex = hdr.index("Address"), hdr.index("Source"), hdr.index(
    "Warp Stall Sampling (All Samples)"), hdr.index("Instructions Executed")
tot = sum(int(r[ismp] or 0) for r in data)
order = sorted(range(len(data)), key=lambda i: -int(data[i][ismp] or 0))
for i in order[:n]:
    print(f"--- {int(data[i][ismp])} samples ({100*int(data[i][ismp])/tot:.1f}%) exec {data[i][iex]}")
    for j in range(max(0, i - 6), min(len(data), i + 2)):
        print(f"   {data[j][ia][-5:]} {int(data[j][ismp] or 0):6d} {data[j][isrc].strip()[:90]}")

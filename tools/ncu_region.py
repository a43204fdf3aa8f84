"""Stall reasons summed per loop of an ncu report's SASS (source page).
Loops are found from backward branches; each loop's address range gets its
samples, executed warp-instructions and stall breakdown, so the consumer
k-march can be separated from producer / spin loops.
usage: python tools/ncu_region.py REP [min_samples]"""
import csv
import io
import re
import subprocess
import sys

rep = sys.argv[1]
mins = int(sys.argv[2]) if len(sys.argv) > 2 else 200
txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(txt)))
hdr, data = rows[1], rows[2:]
ia, isrc, ismp, iex = (hdr.index(h) for h in ("Address", "Source",
                                              "Warp Stall Sampling (All Samples)",
                                              "Instructions Executed"))
stall_cols = [i for i, h in enumerate(hdr) if h.startswith("stall_") and "Not Issued" not in h]
addr = [int(r[ia], 16) for r in data]
base = addr[0]
loops = []
for r, a in zip(data, addr):
    m = re.search(r"BRA(?:\.\w+)? 0x([0-9a-f]+)", r[isrc])
    if m:
        t = int(m.group(1), 16)
        if t < a:
            loops.append((t, a))
# keep outermost-ish distinct ranges with many samples
res = []
for lo, hi in set(loops):
    sel = [r for r, a in zip(data, addr) if lo <= a <= hi]
    smp = sum(int(r[ismp] or 0) for r in sel)
    if smp < mins:
        continue
    ex = sum(int(r[iex] or 0) for r in sel)
    st = {hdr[i][6:]: sum(int(r[i] or 0) for r in sel) for i in stall_cols}
    res.append((smp, lo - base, hi - base, ex, st))
tot = sum(int(r[ismp] or 0) for r in data)
print(f"total samples {tot}")
for smp, lo, hi, ex, st in sorted(res, key=lambda x: -x[0])[:8]:
    top = sorted(st.items(), key=lambda kv: -kv[1])[:7]
    print(f"loop [{lo:#x},{hi:#x}] {hi-lo:>6} B  samples {smp} ({100*smp/tot:.0f}%)  exec {ex}  " +
          " ".join(f"{k}={v}" for k, v in top))

"""Summarise an ncu --set full report (raw page + per-instruction stalls)."""
import csv
import io
import subprocess
import sys
from collections import Counter

rep = sys.argv[1]
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
hdr, units, vals = rows[0], rows[1], rows[2]
KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "launch__registers_per_thread",
        "sm__warps_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_issued.avg.per_cycle_active", "lts__t_sector_hit_rate.pct",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "smsp__inst_executed.sum",
        "sm__cycles_elapsed.avg.per_second", "l1tex__t_bytes_pipe_lsu_mem_local_op_ld.sum",
        "l1tex__t_bytes_pipe_lsu_mem_local_op_st.sum", "lts__t_bytes.sum",
        "launch__grid_size", "launch__block_size", "launch__occupancy_limit_registers"]
out = {}
for h, u, v in zip(hdr, units, vals):
    if h in KEYS or h.startswith("smsp__average_warps_issue_stalled_") and h.endswith("per_issue_active.ratio"):
        out[h] = (v, u)
for k in KEYS:
    if k in out:
        print(f"{k:75s} {out[k][0]:>16s} {out[k][1]}")
st = sorted(((float(v[0] or 0), k) for k, v in out.items() if "stalled" in k), reverse=True)
print("stalls per issue:", ", ".join(f"{k.split('stalled_')[1].split('_per')[0]}={v:.2f}" for v, k in st[:10]))
sass = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=sass"],
                      capture_output=True, text=True).stdout
srows = list(csv.reader(io.StringIO(sass)))
shdr = srows[1]
ix = {h: i for i, h in enumerate(shdr)}
c, tot = Counter(), 0
top = []
for r in srows[2:]:
    try:
        s = int(r[ix["Warp Stall Sampling (All Samples)"]] or 0)
    except (ValueError, IndexError):
        continue
    src = r[ix["Source"]].strip()
    op = src.split()[0]
    if op.startswith("@"):
        op = src.split()[1]
    c[op.split(".")[0]] += s
    tot += s
    top.append((s, src[:70], {k[6:]: r[ix[k]] for k in shdr if k.startswith("stall_") and "Not" not in k and r[ix[k]] not in ("0", "")}))
print("samples", tot, "by opcode:", ", ".join(f"{k}={v}" for k, v in c.most_common(14)))
for s, src, d in sorted(top, key=lambda x: -x[0])[:12]:
    print(f"{s:6d} {src:70s} {d}")

# executed-instruction mix by opcode (warp-level)
ex = Counter()
for r in srows[2:]:
    try:
        n = int(r[ix["Instructions Executed"]] or 0)
    except (ValueError, IndexError):
        continue
    src = r[ix["Source"]].strip()
    if not src:
        continue
    op = src.split()[0]
    if op.startswith("@"):
        op = src.split()[1]
    ex[op.split(".")[0]] += n
totex = sum(ex.values())
print("executed warp-instr", totex, "mix:", ", ".join(f"{k}={v / totex * 100:.1f}%" for k, v in ex.most_common(24)))

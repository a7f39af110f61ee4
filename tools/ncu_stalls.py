"""Summarise an ncu report: SOL numbers + stall reasons + top SASS lines (usage: report [N])."""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
ntop = int(sys.argv[2]) if len(sys.argv) > 2 else 25
det = subprocess.run(["ncu", "-i", rep, "--page", "details"], capture_output=True, text=True).stdout
keys = ["Duration", "DRAM Throughput", "Memory Throughput", "Executed Ipc Active", "Issue Slots Busy",
        "Active Warps Per Scheduler", "Eligible Warps Per Scheduler", "Registers Per Thread",
        "Grid Size", "Block Size", "L2 Hit Rate", "Dynamic Shared Memory Per Block"]
for line in det.splitlines():
    if any(line.strip().startswith(k) for k in keys):
        print(line.rstrip())
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
if len(rows) > 2:
    h = rows[0]
    for name in ["dram__bytes_read.sum", "dram__bytes_write.sum", "gpu__time_duration.sum"]:
        if name in h:
            i = h.index(name)
            print(name, rows[1][i], rows[2][i])
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(src)))
hdr = rows[1]
data = rows[2:]
iS = hdr.index("Warp Stall Sampling (All Samples)")
ie = hdr.index("Instructions Executed")
cols = [c for c in hdr if c.startswith("stall_") and "Not Issued" not in c]
agg = {c: 0 for c in cols}
for r in data:
    for c in cols:
        v = r[hdr.index(c)]
        if v.isdigit():
            agg[c] += int(v)
tot = sum(agg.values())
print("samples", tot, "warp-instr", sum(int(r[ie]) for r in data if r[ie].isdigit()))
print(" ".join(f"{k[6:]}={v/tot:.1%}" for k, v in sorted(agg.items(), key=lambda x: -x[1])[:9]))
top = sorted(range(len(data)), key=lambda i: -int(data[i][iS]) if data[i][iS].isdigit() else 0)[:ntop]
for i in sorted(top):
    r = data[i]
    st = {c: int(r[hdr.index(c)]) for c in cols if r[hdr.index(c)].isdigit() and int(r[hdr.index(c)]) > 0}
    best = sorted(st.items(), key=lambda x: -x[1])[:2]
    print(f"{i:5d} {int(r[iS])/tot:6.1%} {r[1].strip()[:58]:58s} {[(b[0][6:], b[1]) for b in best]}")

"""Opcode histogram (executed warp instructions and stall samples) of an ncu report."""
import collections
import csv
import io
import re
import subprocess
import sys

src = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(src)))
hdr = rows[1]
data = rows[2:]
ie = hdr.index("Instructions Executed")
iS = hdr.index("Warp Stall Sampling (All Samples)")
agg, smp = collections.Counter(), collections.Counter()
for r in data:
    src_ = r[1].strip()
    op = re.sub(r"^@!?U?P\w+\s+", "", src_).split()[0] if src_ else "?"
    op = op.split(".")[0]
    if r[ie].isdigit():
        agg[op] += int(r[ie])
    if r[iS].isdigit():
        smp[op] += int(r[iS])
tot = sum(agg.values())
for op, c in agg.most_common(int(sys.argv[2]) if len(sys.argv) > 2 else 25):
    print(f"{op:10s} {c/1e6:9.1f}M {c/tot:6.1%}  stall-samples {smp[op]}")

"""Warp instructions executed per CUDA source line (and per SASS opcode) from an ncu report.
usage: ncu_inst_lines.py report [N] [n_keys]"""
import csv
import io
import subprocess
import sys
from collections import Counter

rep = sys.argv[1]
ntop = int(sys.argv[2]) if len(sys.argv) > 2 else 40
nkeys = float(sys.argv[3]) if len(sys.argv) > 3 else 1 << 30
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(src)))
hdr_i = next(i for i, r in enumerate(rows) if r and r[0] == "Line No")
hdr = rows[hdr_i]
iI = hdr.index("Instructions Executed")
per_line, per_op = Counter(), Counter()
cur = None
for r in rows[hdr_i + 1:]:
    if not r:
        continue
    if r[0]:
        cur = (int(r[0]), r[1].strip()[:90]) if r[0].isdigit() else None
        continue
    if cur is None or not r[iI].replace(",", "").isdigit():
        continue
    v = int(r[iI].replace(",", ""))
    per_line[cur] += v
    sass = r[3].strip()
    op = sass.split()[0] if sass else "?"
    if op.startswith("@"):
        op = sass.split()[1]
    per_op[op.split(".")[0]] += v
tot = sum(per_line.values())
print("total warp-inst %.3e = %.2f per key" % (tot, tot / nkeys))
for (ln, s), v in per_line.most_common(ntop):
    print("%5d %6.3f/key %5.1f%%  %s" % (ln, v / nkeys, 100 * v / tot, s))
print("--- by opcode")
for op, v in per_op.most_common(30):
    print("%-12s %6.3f/key %5.1f%%" % (op, v / nkeys, 100 * v / tot))

"""Per-CUDA-source-line stall samples from an ncu report (cuda,sass view).  usage: report [N]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
ntop = int(sys.argv[2]) if len(sys.argv) > 2 else 30
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(src)))
hdr_i = next(i for i, r in enumerate(rows) if r and r[0] == "Line No")
hdr = rows[hdr_i]
iS = hdr.index("Warp Stall Sampling (All Samples)")
cols = [i for i, c in enumerate(hdr) if c.startswith("stall_") and "Not Issued" not in c]
agg = {}
cur = None
for r in rows[hdr_i + 1:]:
    if not r:
        continue
    if r[0]:
        cur = (int(r[0]), r[1].strip()[:80]) if r[0].isdigit() else None
        continue
    if cur is None or not r[iS].isdigit():
        continue
    a = agg.setdefault(cur, [0, {}])
    a[0] += int(r[iS])
    for i in cols:
        if r[i].isdigit() and int(r[i]):
            a[1][hdr[i][6:]] = a[1].get(hdr[i][6:], 0) + int(r[i])
tot = sum(v[0] for v in agg.values())
for (ln, text), (s, st) in sorted(agg.items(), key=lambda x: -x[1][0])[:ntop]:
    best = sorted(st.items(), key=lambda x: -x[1])[:2]
    print(f"{ln:5d} {s/tot:6.1%} {text[:70]:70s} {best}")

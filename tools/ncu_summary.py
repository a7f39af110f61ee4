"""Summarise a gpu__time_duration launch list (+ optional --set full reports) into markdown/JSON.

usage: ncu_summary.py launches.csv [full_report.ncu-rep ...] --n N --out-md F --out-json F
"""
import argparse
import csv
import io
import json
import re
import subprocess
from collections import OrderedDict


def short(name):
    m = re.search(r"::(k_[a-z0-9_]+)(<[^>]*>)?", name)
    if m:
        return m.group(1) + (m.group(2) or "")
    return name[:60]


def launches(path):
    rows = []
    with open(path) as f:
        lines = [l for l in f if l.startswith('"')]
    for r in csv.DictReader(io.StringIO("".join(lines))):
        if r.get("Metric Name") == "gpu__time_duration.sum":
            v = float(r["Metric Value"].replace(",", ""))
            unit = r["Metric Unit"]
            ns = v * {"ns": 1, "us": 1e3, "usecond": 1e3, "ms": 1e6, "msecond": 1e6, "nsecond": 1}.get(unit, 1)
            rows.append((short(r["Kernel Name"]), ns, r["Grid Size"], r["Block Size"]))
    return rows


def full_metrics(rep):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    h, units, vals = rows[0], rows[1], rows[2]
    out = {}
    for name in ["Kernel Name", "dram__bytes_read.sum", "dram__bytes_write.sum", "gpu__time_duration.sum",
                 "dram__throughput.avg.pct_of_peak_sustained_elapsed", "sm__warps_active.avg.pct_of_peak_sustained_active",
                 "launch__registers_per_thread", "smsp__inst_executed.sum", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum"]:
        if name in h:
            i = h.index(name)
            out[name] = (vals[i], units[i])
    return out


def to_bytes(v, unit):
    v = float(v.replace(",", ""))
    return v * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}.get(unit, 1)


ap = argparse.ArgumentParser()
ap.add_argument("csv")
ap.add_argument("reports", nargs="*")
ap.add_argument("--n", type=int, required=True)
ap.add_argument("--out-md", required=True)
ap.add_argument("--out-json", default=None)
ap.add_argument("--steps", type=int, default=0,
                help="keep only the first S device-sort steps (a step starts at a K1 launch on the "
                     "first K1's grid; the elision's outlier sort runs its own smaller K1)")
a = ap.parse_args()
rows = launches(a.csv)
if a.steps:
    k1 = next((r for r in rows if r[0].startswith("k_hist")), None)
    seen, keep = 0, []
    for r in rows:
        if k1 and r[0].startswith("k_hist") and r[2] == k1[2]:
            seen += 1
            if seen > a.steps:
                break
        keep.append(r)
    rows = keep
# the library's own kernels (k_*); torch kernels (bench input copies, the output guard outside
# the timed steps) are listed separately and excluded from the shares
ours = [r for r in rows if r[0].startswith("k_")]
other = [r for r in rows if not r[0].startswith("k_")]
rows = ours
agg = OrderedDict()
for k, ns, g, b in rows:
    e = agg.setdefault((k, g), [0, 0.0, g, b])
    e[0] += 1
    e[1] += ns
tot = sum(e[1] for e in agg.values())
md = ["# ncu launch list summary", "", f"source: `{a.csv}` (gpu__time_duration.sum, --clock-control none; "
      "cold-cache, serialised launches: compare shares, not absolutes)"
      + (f"; first {a.steps} device-sort steps of the bench command (warm-up + timed)" if a.steps else ""), "",
      "| kernel | launches | total ms | mean ms | share | grid | block |", "|---|---|---|---|---|---|---|"]
for (k, _), (c, ns, g, b) in sorted(agg.items(), key=lambda x: -x[1][1]):
    md.append(f"| `{k}` | {c} | {ns/1e6:.3f} | {ns/1e6/c:.3f} | {ns/tot:.1%} | {g} | {b} |")
if other:
    md += ["", f"Not ours (torch; excluded from the shares): {len(other)} launches, "
           f"{sum(r[1] for r in other)/1e6:.3f} ms (bench input copies and the output guard)."]
js = {"n": a.n}
for rep in a.reports:
    m = full_metrics(rep)
    md += ["", f"## `--set full` capture: `{rep.split('/')[-1]}`", ""]
    for k, (v, u) in m.items():
        md.append(f"- {k}: {v} {u}")
    if "dram__bytes_read.sum" in m:
        rd = to_bytes(*m["dram__bytes_read.sum"])
        wr = to_bytes(*m["dram__bytes_write.sum"])
        kn = m["Kernel Name"][0]
        md.append(f"- dram read+write per launch: {(rd+wr)/1e9:.3f} GB "
                  f"({(rd+wr)/a.n:.2f} B/key over n={a.n})")
        if "onesweep" in kn:
            js["onesweep_dram_bytes_per_launch"] = rd + wr
            js["onesweep_alg_bytes_per_launch"] = 16 * a.n
        if "hist" in kn:
            js["hist_dram_bytes_per_launch"] = rd + wr
open(a.out_md, "w").write("\n".join(md) + "\n")
if a.out_json:
    json.dump(js, open(a.out_json, "w"), indent=1)
print("\n".join(md))

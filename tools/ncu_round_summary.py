"""Round ncu summary from tools/gpurun_profile.sh outputs: launch list of the bench command (shares
of our kernels) + --set full metrics of the K3 / K5 / K1 captures.  usage: ncu_round_summary.py <tag>
Writes profiles/<tag>_ncu_summary.md and profiles/ncu_traffic.json."""
import csv
import io
import json
import re
import subprocess
import sys
from collections import OrderedDict

tag = sys.argv[1]
G = "gpurun_out"
try:  # HBM peak of this pool (driver-written)
    PEAK = float(json.load(open("MEASURED_PEAKS.json"))["hbm_gbs"])
except Exception:
    PEAK = 6464.0


def short(name):
    m = re.search(r"(k_[a-z0-9_]+)(<[^>]*>)?", name)
    return (m.group(1) + (m.group(2) or "")) if m else name[:60]


rows = []
lines = [l for l in open(f"{G}/{tag}_launches.csv") if l.startswith('"')]
for r in csv.DictReader(io.StringIO("".join(lines))):
    if r.get("Metric Name") == "gpu__time_duration.sum":
        v = float(r["Metric Value"].replace(",", ""))
        ns = v * {"ns": 1, "us": 1e3, "usecond": 1e3, "ms": 1e6, "msecond": 1e6, "nsecond": 1}.get(r["Metric Unit"], 1)
        rows.append((short(r["Kernel Name"]), ns, r["Grid Size"], r["Block Size"]))
ours = [r for r in rows if r[0].startswith("k_")]
other = [r for r in rows if not r[0].startswith("k_")]
agg = OrderedDict()
for k, ns, g, b in ours:
    e = agg.setdefault((k, g), [0, 0.0, g, b])
    e[0] += 1
    e[1] += ns
tot = sum(e[1] for e in agg.values())
md = [f"# ncu summary `{tag}` (B200, `--clock-control none`)", "",
      "## Launch list of the bench command", "",
      "`ncu --metrics gpu__time_duration.sum --clock-control none -c 5000 --csv python bench.py --steps 2 "
      "--warmup 3 --no-cpu-baseline --no-extras` (`profiles/" + tag + "_launches.csv`; cold-cache, serialised "
      "launches: compare shares, not absolutes).  5 host->host calls (12 resident batch sorts of 2^27 keys "
      "+ halving tail, 16 merge chunks of 2^26 keys: K4 coarse + fine and K5 each) and 5 device GPUSorts "
      "of 2^30 keys (K1, K2, 7 passes with the elision, the outlier sort).", "",
      "| kernel | launches | total ms | mean ms | share | grid | block |", "|---|---|---|---|---|---|---|"]
for (k, _), (c, ns, g, b) in sorted(agg.items(), key=lambda x: -x[1][1]):
    if ns / tot >= 0.0005:
        md.append(f"| `{k}` | {c} | {ns/1e6:.3f} | {ns/1e6/c:.3f} | {ns/tot:.1%} | {g} | {b} |")
by = OrderedDict()
for k, ns, g, b in ours:
    e = by.setdefault(k.split("<")[0], [0, 0.0])
    e[0] += 1
    e[1] += ns
md += ["", f"Not ours (torch: input copies, link probe, guards outside the timed steps): {len(other)} launches, "
       f"{sum(r[1] for r in other)/1e6:.1f} ms.", "",
       "By kernel family: " + ", ".join(f"`{k}` {ns/tot:.1%}" for k, (c, ns) in
                                       sorted(by.items(), key=lambda x: -x[1][1]) if ns / tot > 0.001) + ".", ""]


def full(rep):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rr = list(csv.reader(io.StringIO(raw)))
    h, u, v = rr[0], rr[1], rr[2]
    want = ["Kernel Name", "Grid Size", "Block Size", "gpu__time_duration.sum", "dram__bytes_read.sum",
            "dram__bytes_write.sum", "dram__throughput.avg.pct_of_peak_sustained_elapsed",
            "l1tex__throughput.avg.pct_of_peak_sustained_active",
            "smsp__issue_active.avg.pct_of_peak_sustained_active",
            "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__warps_eligible.avg.per_cycle_active",
            "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "launch__registers_per_thread",
            "smsp__inst_executed.sum"]
    return {w: (v[h.index(w)], u[h.index(w)]) for w in want if w in h}


def tob(v, u):
    return float(v.replace(",", "")) * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u, 1)


caps = [(f"{G}/{tag}_onesweep_full.ncu-rep", "K3 `k_onesweep_ws` (raw-key pass, DM = 0), device arm, 2^30 keys (`--device-only --no-dde`)", 1 << 30, 16, "onesweep"),
        (f"{G}/{tag}_merge_full.ncu-rep", "K5 `k_merge_tile`, one 2^26-key merge chunk of the host->host arm (k = 12 resident runs)", 1 << 26, 16, "merge"),
        (f"{G}/{tag}_hist_full.ncu-rep", "K1 `k_hist3`, device arm, 2^30 keys", 1 << 30, 8, "hist")]
traffic = {}
for rep, what, n, bpk, key in caps:
    m = full(rep)
    md += [f"## `--set full`: {what}", "", f"report `{rep.split('/')[-1]}` (not committed, ~10 MB)", ""]
    for k, (v, u) in m.items():
        md.append(f"- {k}: {short(v) if k == 'Kernel Name' else v} {u}")
    rd, wr = tob(*m["dram__bytes_read.sum"]), tob(*m["dram__bytes_write.sum"])
    t = float(m["gpu__time_duration.sum"][0].replace(",", "")) * (1e-3 if m["gpu__time_duration.sum"][1] in ("us", "usecond") else 1)
    md.append(f"- DRAM read+write: {(rd+wr)/1e9:.3f} GB = {(rd+wr)/n:.2f} B/key (algorithmic {bpk} B/key: "
              f"{(rd+wr)/(bpk*n):.3f}x); algorithmic {bpk*n/(t*1e-3)/1e9:.0f} GB/s = {bpk*n/(t*1e-3)/1e9/PEAK:.1%} of {PEAK:.0f} GB/s")
    md.append("")
    traffic[f"{key}_dram_bytes_per_launch"] = rd + wr
    traffic[f"{key}_n"] = n
traffic["n"] = 1 << 30
traffic["onesweep_alg_bytes_per_launch"] = 16 << 30
open(f"profiles/{tag}_ncu_summary.md", "w").write("\n".join(md) + "\n")
json.dump(traffic, open("profiles/ncu_traffic.json", "w"), indent=1)
print("\n".join(md))

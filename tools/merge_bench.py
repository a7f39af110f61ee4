"""Time the GPU merge (K4 co-ranks + K5 tile merge) of k device-resident sorted runs.

usage: python tools/merge_bench.py [n_log2=30] [k,k,...] [dist]
For each k: n uniform float64 keys are split into k runs of ragged lengths, each run sorted into
transformed uint64 keys (hsort_sort_device_keys), then hsort_device_corank (K4 alone) and
hsort_device_merge (K4 + K5) are timed with CUDA events on one stream.  Algorithmic bytes of K5:
16 per key (each key read once, written once).  The merged output is checked bit-exactly against
the library's own sort of the whole array (tests/ hold the oracle parity).
"""
import json, os, statistics, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import hsort_inputs
import paper_conf_ipps_gowanlockk18a_b200 as hs

if os.environ.get("HSORT_LIB"):  # A/B: an alternative build of the library
    hs.LIB_PATH = os.path.abspath(os.environ["HSORT_LIB"])

nlog = int(sys.argv[1]) if len(sys.argv) > 1 else 30
ks = [int(x) for x in sys.argv[2].split(",")] if len(sys.argv) > 2 else [2, 4, 8, 12, 32, 128]
dist = sys.argv[3] if len(sys.argv) > 3 else "uniform"
n = 1 << nlog
peak = None
try:
    peak = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                       "MEASURED_PEAKS.json")))["hbm_gbs"]
except Exception:
    pass

hs.hsort_init()
A = hsort_inputs.generate(dist, n, seed=7)
d_a = torch.from_numpy(A).cuda()
d_runs = torch.empty(n, dtype=torch.int64, device="cuda")
d_out = torch.empty_like(d_runs)
want = torch.empty_like(d_runs)
hs.hsort_sort_device_keys(d_a, want, True, False)
torch.cuda.synchronize()
st = torch.cuda.current_stream()
rng = np.random.default_rng(1)
for k in ks:
    w = rng.uniform(0.5, 1.5, size=k)
    cuts = np.concatenate([[0], np.floor(np.cumsum(w) / w.sum() * n).astype(np.uint64)])
    cuts[-1] = n
    for j in range(k):
        a, b = int(cuts[j]), int(cuts[j + 1])
        if b > a:
            hs.hsort_sort_device_keys(d_a[a:b], d_runs[a:b], True, False)
    mt = int(os.environ.get("MERGE_TILE", "4096"))  # the build's kMergeTile (A/B builds)
    tiles = (n + mt - 1) // mt
    d_ranks = torch.empty((tiles + 1) * k, dtype=torch.int64, device="cuda")
    for _ in range(2):
        hs.hsort_device_merge(d_runs, cuts, d_out, False)
    ok = bool(torch.equal(d_out, want))
    tc, tm = [], []
    for _ in range(5):
        e = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
        e[0].record(st)
        hs.hsort_device_corank(d_runs, cuts, mt, tiles + 1, d_ranks)
        e[1].record(st)
        e[2].record(st)
        hs.hsort_device_merge(d_runs, cuts, d_out, False)
        e[3].record(st)
        torch.cuda.synchronize()
        tc.append(e[0].elapsed_time(e[1]))
        tm.append(e[2].elapsed_time(e[3]))
    c, m = statistics.median(tc), statistics.median(tm)
    k5 = max(m - c, 1e-6)
    rec = {"k": k, "n": n, "dist": dist, "ok": ok, "corank_ms": c, "merge_ms": m, "k5_ms": k5,
           "k5_gbs": 16 * n / k5 / 1e6, "merge_keys_per_s": n / m * 1e3}
    if peak:
        rec["k5_frac"] = rec["k5_gbs"] / peak
        rec["merge_frac"] = 16 * n / m / 1e6 / peak
    print(json.dumps(rec), flush=True)
hs.hsort_finalize()

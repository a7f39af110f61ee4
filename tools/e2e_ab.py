"""Interleaved A/B of the host->host sort (pinned A/B, 2^30 uniform, auto plan) over an option."""
import json, os, statistics, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import hsort_inputs
import paper_conf_ipps_gowanlockk18a_b200 as hs
opt, vals = sys.argv[1], [int(v) for v in sys.argv[2].split(",")]
pageable = len(sys.argv) > 3 and sys.argv[3] == "pageable"
n = 1 << 30
hs.hsort_init()
if pageable:  # the paper's setting: staged through the pinned ring
    import numpy as np
    A = hsort_inputs.generate("uniform", n, seed=2)
    B = np.empty_like(A)
    B[::512] = 0
else:
    A = torch.empty(n, dtype=torch.float64).pin_memory()
    hsort_inputs.generate("uniform", n, seed=2, out=A.numpy())
    B = torch.empty(n, dtype=torch.float64).pin_memory()
hs.hsort_sort(A, B)
res = {v: [] for v in vals}
for r in range(4):
    for v in vals:
        hs.hsort_set_option(opt, v)
        t = time.perf_counter()
        hs.hsort_sort(A, B)
        res[v].append(time.perf_counter() - t)
for v in vals:
    print(json.dumps({opt: v, "pageable": pageable, "median_ms": 1e3 * statistics.median(res[v]), "min_ms": 1e3 * min(res[v]),
                      "keys_per_s": n / statistics.median(res[v])}))

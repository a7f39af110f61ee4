"""A/B of the two RESIDENT finishes at n = 2^30 on one B200: the merge path (K4/K5 over resident
runs) vs the MSD-first split (option "msd": bucket partition per batch, gather, LSD per bucket).
Host->host through hsort_sort on pinned A/B, interleaved rounds; prints one JSON line per run."""
import json
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import hsort_inputs  # noqa: E402
import paper_conf_ipps_gowanlockk18a_b200 as hs  # noqa: E402

n = int(float(sys.argv[1])) if len(sys.argv) > 1 else 1 << 30
hs.hsort_init()
A = torch.empty(n, dtype=torch.float64, pin_memory=True)
B = torch.empty(n, dtype=torch.float64, pin_memory=True)
variants = [("merge", {"msd": 0}), ("msd_2^24", {"msd": 1, "msd_bucket_keys": 1 << 24}),
            ("msd_2^23", {"msd": 1, "msd_bucket_keys": 1 << 23}),
            ("msd_2^25", {"msd": 1, "msd_bucket_keys": 1 << 25})]
for dist, seed in (("uniform", 2), ("zipf_dup", 5)):
    hsort_inputs.generate(dist, n, seed=seed, out=A.numpy())
    res = {v: [] for v, _ in variants}
    for rnd in range(3):
        for name, opts in variants:
            for k, v in opts.items():
                hs.hsort_set_option(k, v)
            hs.hsort_sort(A, B)
            t = time.perf_counter()
            hs.hsort_sort(A, B)
            res[name].append(time.perf_counter() - t)
            st = hs.hsort_get_stats()
            if rnd == 2:
                Bv = B.numpy()
                ok = bool(np.all(Bv[1:] >= Bv[:-1]))
                print(json.dumps({"dist": dist, "variant": name, "s": statistics.median(res[name]),
                                  "all_s": res[name], "sorted": ok,
                                  **{k: st[k] for k in ("n_b", "msd_buckets", "t_sort_phase",
                                                         "t_merge_phase", "t_gpu_sort", "t_merge_gpu",
                                                         "t_h2d", "t_d2h", "passes_run")}}), flush=True)
    hs.hsort_set_option("msd", 0)
hs.hsort_finalize()

"""CPU merge (H2, hsort_host_merge: loser trees over exact co-rank ranges) vs the CPU-merge
reference (__gnu_parallel::multiway_merge, the paper's merge) on the same runs."""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import oracle
import paper_conf_ipps_gowanlockk18a_b200 as hs
try:
    import psutil
    cores = psutil.cpu_count(logical=False) or os.cpu_count()
except Exception:
    cores = os.cpu_count()
n = int(float(sys.argv[1])) if len(sys.argv) > 1 else 1 << 28
rng = np.random.default_rng(1)
keys_all = rng.integers(0, 2**64, size=n, dtype=np.uint64)
w = np.sort(keys_all[: 1 << 20])  # warm both thread pools
hs.hsort_host_merge(w, np.array([0, w.size], dtype=np.uint64), False, cores)
oracle.par_multiway_merge_u64(w, np.array([0, w.size], dtype=np.uint64), cores)
for k in (8, 32, 120):
    cuts = np.linspace(0, n, k + 1).astype(np.uint64)
    keys = keys_all.copy()
    for j in range(k):
        keys[cuts[j]:cuts[j + 1]].sort()
    t = time.perf_counter(); ours = hs.hsort_host_merge(keys, cuts, False, cores); t_ours = time.perf_counter() - t
    t = time.perf_counter(); ref = oracle.par_multiway_merge_u64(keys, cuts, cores); t_ref = time.perf_counter() - t
    print(json.dumps({"n": n, "k": k, "threads": cores, "h2_s": t_ours, "gnu_multiway_merge_s": t_ref,
                      "h2_keys_per_s": n / t_ours, "gnu_keys_per_s": n / t_ref,
                      "equal": bool(np.array_equal(ours, ref))}), flush=True)

"""STREAM sort-phase staging vs the pinned chunk size p_s (and ring depth): n = 4.3e9 pageable,
2 GB batches, auto split; one JSON line per (p_s, n_ring).  usage: ooc_ps_probe.py <p_s MB> <n_ring>"""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import hsort_inputs
import paper_conf_ipps_gowanlockk18a_b200 as hs
ps, nr = int(sys.argv[1]), int(sys.argv[2])
hs.hsort_set_option("p_s", ps << 20)
hs.hsort_set_option("n_ring", nr)
hs.hsort_init()
n = int(4.3e9)
A = hsort_inputs.generate("uniform", n, seed=3)
B = np.empty_like(A)
hs.hsort_set_option("resident", 0); hs.hsort_set_option("pin_w", 1)
hs.hsort_sort(A, B, batch_elems=250_000_000)
ts = []
for _ in range(3):
    t = time.perf_counter(); hs.hsort_sort(A, B, batch_elems=250_000_000); ts.append(time.perf_counter() - t)
s = hs.hsort_get_stats()
print(json.dumps({"p_s_mb": ps, "n_ring": nr, "s": round(min(ts), 3), "sort_phase": round(s["t_sort_phase"], 3),
                  "merge_phase": round(s["t_merge_phase"], 3), "stage": round(s["t_stage"], 3),
                  "f": round(s["merge_gpu_fraction"], 3)}), flush=True)

import json, os, sys, time
sys.path.insert(0, os.getcwd())
import numpy as np
import hsort_inputs
import paper_conf_ipps_gowanlockk18a_b200 as hs
n = int(4.3e9)
hs.hsort_init()
A = hsort_inputs.generate("uniform", n, seed=3)
B = np.empty_like(A)
hs.hsort_set_option("resident", 0); hs.hsort_set_option("pin_w", 1)
hs.hsort_sort(A, B, batch_elems=250_000_000)
for st_threads in (2, 4, 8, 12):
    for fp in (800, 900, -1):
        hs.hsort_set_option("merge_stage_threads", st_threads)
        hs.hsort_set_option("merge_gpu_permille", fp)
        ts = []
        for _ in range(2):
            t = time.perf_counter(); hs.hsort_sort(A, B, batch_elems=250_000_000); ts.append(time.perf_counter() - t)
        s = hs.hsort_get_stats()
        print(json.dumps({"stage_threads": st_threads, "f": round(s["merge_gpu_fraction"], 3), "s": round(min(ts), 3),
                          "merge_phase": round(s["t_merge_phase"], 3), "cpu": round(s["t_merge_cpu"], 3), "gpu": round(s["t_merge_gpu"], 3)}), flush=True)

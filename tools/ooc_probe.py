"""Out-of-core STREAM probe (the bench's out_of_core block): n keys, pageable A/B, 2 GB batches,
page-locked cached W.  Auto merge split over consecutive calls (f adapts to the measured rates),
then fixed splits.  One JSON line per call."""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import hsort_inputs
import paper_conf_ipps_gowanlockk18a_b200 as hs
if os.environ.get("HSORT_LIB"):  # A/B: an alternative build of the library
    hs.LIB_PATH = os.path.abspath(os.environ["HSORT_LIB"])

n = int(float(sys.argv[1])) if len(sys.argv) > 1 else int(4.3e9)
for kv in os.environ.get("OOC_OPTS", "").split(","):  # e.g. merge_stage_threads=12,merge_gpu_permille=1000
    if kv:
        k_, v_ = kv.split("=")
        hs.hsort_set_option(k_, int(v_))
hs.hsort_init()
A = hsort_inputs.generate("uniform", n, seed=3)
B = np.empty_like(A)
hs.hsort_set_option("resident", 0)
hs.hsort_set_option("pin_w", 1)
runs = [("auto", -1)] * 5 + [("f600", 600), ("f700", 700), ("f800", 800)]
if os.environ.get("OOC_AUTO_ONLY"):
    runs = [("auto", -1)] * int(os.environ["OOC_AUTO_ONLY"])
if os.environ.get("OOC_FIXED"):  # e.g. 1000,1000,950: fixed merge splits (per mille)
    runs = [("f" + x, int(x)) for x in os.environ["OOC_FIXED"].split(",")]
for name, fp in runs:
    hs.hsort_set_option("merge_gpu_permille", fp)
    t = time.perf_counter()
    hs.hsort_sort(A, B, batch_elems=250_000_000)
    dt = time.perf_counter() - t
    st = hs.hsort_get_stats()
    print(json.dumps({"lib": os.environ.get("HSORT_LIB", "default"), "run": name, "s": round(dt, 3), "keys_per_s": n / dt, "f": round(st["merge_gpu_fraction"], 3),
                      "sort_phase": round(st["t_sort_phase"], 3), "merge_phase": round(st["t_merge_phase"], 3),
                      "merge_cpu": round(st["t_merge_cpu"], 3), "merge_gpu": round(st["t_merge_gpu"], 3),
                      "stage": round(st["t_stage"], 3), "alloc": round(st["t_host_alloc"], 3)}), flush=True)

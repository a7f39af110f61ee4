"""Per-pass kernel times of the 2^30 uniform device sort with the dominant-digit elision on/off."""
import json, os, statistics, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_gowanlockk18a_b200 as hs
if os.environ.get("HSORT_LIB"):
    hs.LIB_PATH = os.path.abspath(os.environ["HSORT_LIB"])
import torch
import hsort_inputs
n = 1 << 30
hs.hsort_set_option("kernel_timing", 1)
hs.hsort_init()
A = hsort_inputs.generate("uniform", n, seed=2)
d_in = torch.from_numpy(A).cuda(); d_out = torch.empty_like(d_in)
for rnd in range(2):
    for dde in (1, 0):
        hs.hsort_set_option("dde", dde)
        for _ in range(3): hs.hsort_sort_device(d_in, d_out)
        torch.cuda.synchronize()
        tot, per = [], []
        for _ in range(5):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(); hs.hsort_sort_device(d_in, d_out); e1.record(); e1.synchronize()
            tot.append(e0.elapsed_time(e1))
            kt = hs.hsort_get_kernel_times(); per.append(kt)
        na = per[-1]["num_active"]
        print(json.dumps({"dde": dde, "sort_ms": statistics.median(tot), "num_active": na,
                          "hist": round(per[-1]["hist"], 3), "passes": [round(x, 3) for x in per[-1]["passes"]],
                          "copy_tail": round(per[-1]["copy"], 3)}), flush=True)
ok = bool((d_out[1:] >= d_out[:-1]).all().item())
print("sorted", ok)

"""Key/value GPUSort of 2^30 (uniform float64 key, index) pairs: sort time and per-pass times."""
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
d = torch.from_numpy(hsort_inputs.generate("uniform", n, seed=2)).cuda()
v = torch.arange(n, dtype=torch.int64, device="cuda")
ko, vo = torch.empty_like(d), torch.empty_like(v)
hs.hsort_sort_device_pairs(d, v, ko, vo, True)
ts, ps = [], []
for _ in range(4):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(); hs.hsort_sort_device_pairs(d, v, ko, vo, True); e1.record(); e1.synchronize()
    ts.append(e0.elapsed_time(e1)); kt = hs.hsort_get_kernel_times(); ps += kt["passes"][:kt["num_active"]]
ok = bool((ko[1:] >= ko[:-1]).all()) and bool(torch.equal(d[vo], ko))
print(json.dumps({"lib": os.environ.get("HSORT_LIB", "default"), "sort_ms": statistics.median(ts), "pass_ms": statistics.mean(ps), "ok": ok}))

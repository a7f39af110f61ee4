"""float32 device sorts of 2^30 U[0,1) keys (native 32-bit path): whole-sort ms and per-kernel times
(HSORT_LIB = an alternative build for A/B)."""
import os, sys, json, statistics
sys.path.insert(0, os.getcwd())
import torch, numpy as np
import hsort_inputs
import paper_conf_ipps_gowanlockk18a_b200 as hs
if os.environ.get("HSORT_LIB"):
    hs.LIB_PATH = os.path.abspath(os.environ["HSORT_LIB"])
hs.hsort_set_option("kernel_timing", 1)
hs.hsort_init()
n = 1 << 30
A = hsort_inputs.generate("uniform", n, seed=2).astype(np.float32)
d = torch.from_numpy(A).cuda(); o = torch.empty_like(d)
st = torch.cuda.current_stream()
for desc in (False, True):
    for _ in range(2): hs.hsort_sort_device_typed(d, o, desc)
    ts = []
    for _ in range(5):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st); hs.hsort_sort_device_typed(d, o, desc); e1.record(st); e1.synchronize()
        ts.append(e0.elapsed_time(e1))
    kt = hs.hsort_get_kernel_times()
    ok = bool((o[1:] >= o[:-1]).all()) if not desc else bool((o[1:] <= o[:-1]).all())
    print(json.dumps({"lib": os.environ.get("HSORT_LIB", "default"), "desc": desc, "ms": statistics.median(ts), "hist": kt["hist"], "passes": kt["passes"][:4], "active": kt["num_active"], "sorted": ok}))

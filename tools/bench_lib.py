"""Time the device sort with an alternative libhsort build (argv[1] = .so path), 2^30 keys of
distribution argv[2] (default uniform)."""
import json, os, statistics, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_gowanlockk18a_b200 as hs
hs.LIB_PATH = os.path.abspath(sys.argv[1])
import torch
import hsort_inputs
n = 1 << 30
hs.hsort_set_option("kernel_timing", 1)
if os.environ.get("HSORT_AB_NO_DDE"): hs.hsort_set_option("dde", 0)
hs.hsort_init()
dist = sys.argv[2] if len(sys.argv) > 2 else "uniform"
A = hsort_inputs.generate(dist, n, seed=2)
d_in = torch.from_numpy(A).cuda(); d_out = torch.empty_like(d_in)
for _ in range(3): hs.hsort_sort_device(d_in, d_out)
torch.cuda.synchronize()
ps = []
for _ in range(5):
    hs.hsort_sort_device(d_in, d_out); torch.cuda.synchronize()
    kt = hs.hsort_get_kernel_times(); ps += kt["passes"][:kt["num_active"]]
ok = bool((d_out[1:] >= d_out[:-1]).all().item()) and torch.equal(torch.sort(d_in)[0], d_out)
print(json.dumps({"lib": sys.argv[1], "dist": dist, "pass_ms": statistics.mean(ps), "sort_ms": sum(kt["passes"][:kt["num_active"]]) + kt["hist"], "ok": ok, "per_pass": [round(x, 3) for x in kt["passes"]]}))

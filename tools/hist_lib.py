"""Time K1 (device histograms) with an alternative libhsort build (argv[1]), 2^30 uniform f64."""
import json, os, statistics, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_gowanlockk18a_b200 as hs
hs.LIB_PATH = os.path.abspath(sys.argv[1])
import torch
import hsort_inputs
n = 1 << 30
hs.hsort_set_option("kernel_timing", 1)
hs.hsort_init()
A = hsort_inputs.generate("uniform", n, seed=2)
d_in = torch.from_numpy(A).cuda(); d_out = torch.empty_like(d_in)
for _ in range(3): hs.hsort_sort_device(d_in, d_out)
torch.cuda.synchronize()
h = []
for _ in range(5):
    hs.hsort_sort_device(d_in, d_out); torch.cuda.synchronize()
    h.append(hs.hsort_get_kernel_times()["hist"])
ref = torch.zeros(8 * 256, dtype=torch.uint64, device="cuda")
hs.hsort_device_histograms(d_in, True, ref)
k = d_in.view(torch.int64)
key = torch.where(k < 0, ~k, k | (-(1 << 63)))  # to_key: negative -> ~u, else u | 2^63
ok = True
for p in range(8):
    dig = ((key >> (8 * p)) & 255)
    ok &= torch.equal(torch.bincount(dig, minlength=256).to(torch.int64), ref[p * 256:(p + 1) * 256].view(torch.int64))
print(json.dumps({"lib": sys.argv[1], "hist_ms": statistics.mean(h), "hist_ok": bool(ok)}))

"""Time the device sort of 2^30 uniform float64 for the kernel variant selected by env vars
(HSORT_PASS_VARIANT, HSORT_HIST_VARIANT); checks the result against torch.sort (library)."""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import hsort_inputs  # noqa: E402
import paper_conf_ipps_gowanlockk18a_b200 as hs  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 1 << 30
dist = sys.argv[2] if len(sys.argv) > 2 else "uniform"
hs.hsort_set_option("kernel_timing", 1)
hs.hsort_init()
A = hsort_inputs.generate(dist, n, seed=2)
d_in = torch.from_numpy(A).cuda()
d_out = torch.empty_like(d_in)
for _ in range(3):
    hs.hsort_sort_device(d_in, d_out)
torch.cuda.synchronize()
ok = bool(torch.equal(d_out.view(torch.int64), torch.sort(d_in).values.view(torch.int64))) \
    if dist in ("uniform", "normal") else None
passes, hists, steps = [], [], []
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
for _ in range(10):
    e0.record()
    hs.hsort_sort_device(d_in, d_out)
    e1.record()
    e1.synchronize()
    steps.append(e0.elapsed_time(e1))
    kt = hs.hsort_get_kernel_times()
    passes += kt["passes"][:kt["num_active"]]
    hists.append(kt["hist"])
pm = statistics.mean(passes)
print(json.dumps({"pass_variant": os.environ.get("HSORT_PASS_VARIANT"),
                  "hist_variant": os.environ.get("HSORT_HIST_VARIANT"), "n": n, "dist": dist,
                  "ok": ok, "step_ms": statistics.mean(steps), "pass_ms": pm,
                  "pass_GBps": 16 * n / pm / 1e6, "hist_ms": statistics.mean(hists),
                  "hist_GBps": 8 * n / statistics.mean(hists) / 1e6,
                  "keys_per_s": n / statistics.mean(steps) * 1e3}), flush=True)
hs.hsort_finalize()

"""Device GPUSort of 2^30 normal / zipf-dup keys: per-step event time vs the library's per-kernel
times (why bench's skewed device rows read ~200 ms)."""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import hsort_inputs
import paper_conf_ipps_gowanlockk18a_b200 as hs
n = 1 << 30
hs.hsort_set_option("kernel_timing", int(sys.argv[1]) if len(sys.argv) > 1 else 1)
hs.hsort_init()
A = torch.empty(n, dtype=torch.float64, pin_memory=True)
st = torch.cuda.current_stream()
for dist, seed in (("uniform", 2), ("normal", 4), ("zipf_dup", 5), ("uniform_pm1", 6)):
    hsort_inputs.generate(dist, n, seed=seed, out=A.numpy())
    d_in = A.cuda(); d_out = torch.empty_like(d_in)
    for _ in range(2):
        hs.hsort_sort_device(d_in, d_out, st)
    torch.cuda.synchronize()
    for _ in range(3):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        t = time.perf_counter()
        e0.record(st); hs.hsort_sort_device(d_in, d_out, st); e1.record(st); e1.synchronize()
        w = time.perf_counter() - t
        kt = hs.hsort_get_kernel_times(); pl = hs.hsort_get_last_plan()
        rec = {"dist": dist, "ev_ms": round(e0.elapsed_time(e1), 2), "wall_ms": round(w * 1e3, 2), "plan": pl}
        if "hist" in kt:
            rec.update(hist=round(kt["hist"], 3), passes=[round(x, 3) for x in kt["passes"]])
        print(json.dumps(rec), flush=True)
    del d_in, d_out

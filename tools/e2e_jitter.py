"""Per-call phase times of hsort_sort(A pinned, B pinned, 2^30, 0, 1) over 30 calls, with and
without an NVML clock sampler running, to locate the slow outlier calls of the e2e arm."""
import gc, json, os, sys, threading, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import hsort_inputs
import paper_conf_ipps_gowanlockk18a_b200 as hs
import bench

n = 1 << 30
hs.hsort_init()
A = torch.empty(n, dtype=torch.float64, pin_memory=True)
B = torch.empty(n, dtype=torch.float64, pin_memory=True)
hsort_inputs.generate("uniform", n, seed=2, out=A.numpy())
for _ in range(3):
    hs.hsort_sort(A, B)
for sampler, nogc in ((False, False), (True, False), (False, True), (True, True)):
    cs = bench.ClockSampler([0]) if sampler else None
    if nogc:
        gc.collect()
        gc.disable()
    if cs: cs.__enter__()
    rows = []
    for i in range(15):
        t = time.perf_counter()
        hs.hsort_sort(A, B)
        dt = time.perf_counter() - t
        st = hs.hsort_get_stats()
        rows.append((round(dt * 1e3, 1), round(st["t_total"] * 1e3, 1), round(st["t_setup"] * 1e3, 2), round(st["t_sort_phase"] * 1e3, 1), round(st["t_merge_phase"] * 1e3, 1),
                     round(st["t_h2d"] * 1e3, 1), round(st["t_d2h"] * 1e3, 1)))
    if cs: cs.__exit__()
    gc.enable()
    print(json.dumps({"sampler": sampler, "gc_disabled": nogc, "calls_ms(py,lib_total,sort,merge,h2d,d2h)": rows}), flush=True)

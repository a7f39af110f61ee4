"""Cycle breakdown of one forced onesweep pass (instrumented libhsort_timing.so) on 2^30 uint64
keys: digit 0 of random keys (high entropy) and digit 7 of keys whose top byte is constant."""
import ctypes
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_ipps_gowanlockk18a_b200 as hs  # noqa: E402

hs.LIB_PATH = os.environ.get("HSORT_LIB", os.path.join(ROOT, "paper_conf_ipps_gowanlockk18a_b200", "libhsort_timing.so"))
import torch  # noqa: E402

n = 1 << 30
hs.hsort_init()
L = hs.lib()
L.hsort_debug_phase_counters.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_int]
g = torch.Generator(device="cuda").manual_seed(1)
src = torch.randint(-(1 << 62), 1 << 62, (n,), device="cuda", dtype=torch.int64, generator=g)
src = src.view(torch.uint64)
dst = torch.empty_like(src)
buf = (ctypes.c_ulonglong * 256)()
for name, digit, fix in [("random digit 0", 0, False), ("constant digit 7", 7, True)]:
    if fix:
        src.view(torch.int64).bitwise_and_(0x00FFFFFFFFFFFFFF).bitwise_or_(0x3F00000000000000)
    hs.hsort_device_radix_pass(src, dst, digit)
    torch.cuda.synchronize()
    L.hsort_debug_phase_counters(buf, 256, 1)
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    hs.hsort_device_radix_pass(src, dst, digit)
    e.record()
    torch.cuda.synchronize()
    L.hsort_debug_phase_counters(buf, 256, 1)
    T = max(1, buf[213])
    res = {"pass": name, "ms(incl hist)": round(s.elapsed_time(e), 3), "tiles": T,
           "compute_total": buf[212] / T, "wait_tma": buf[211] / T, "count+publish": buf[219] / T,
           "rank+scatter": buf[218] / T, "  of which peers": buf[221] / T, "writeout(incl wait)": buf[220] / T, "wait_lookback": buf[210] / T,
           "lb_idle": buf[214] / max(1, buf[217]), "lb_time": buf[215] / max(1, buf[217]),
           "lb_rounds": buf[216] / max(1, buf[217])}
    print(json.dumps({k: round(v, 1) if isinstance(v, float) else v for k, v in res.items()}))

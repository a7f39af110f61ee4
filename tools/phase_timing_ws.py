"""Cycle breakdown of the warp-specialised onesweep pass (instrumented libhsort_timing.so).

Compute side (thread 0 of warp 0): waits for TMA, count+publish, rank+scatter, write-out of the
previous tile (incl. the wait for its look-back), barriers.  Look-back warp (lane 0): idle wait
for the next tile, look-back time, rounds.  Per tile averages over all passes of one 2^30 sort."""
import ctypes
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_ipps_gowanlockk18a_b200 as hs  # noqa: E402

hs.LIB_PATH = os.environ.get("HSORT_LIB", os.path.join(ROOT, "paper_conf_ipps_gowanlockk18a_b200", "libhsort_timing.so"))
import torch  # noqa: E402

import hsort_inputs  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 1 << 30
hs.hsort_init()
L = hs.lib()
L.hsort_debug_phase_counters.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_int]
A = hsort_inputs.generate("uniform", n, seed=2)
d_in = torch.from_numpy(A).cuda()
d_out = torch.empty_like(d_in)
hs.hsort_sort_device(d_in, d_out)
torch.cuda.synchronize()
buf = (ctypes.c_ulonglong * 256)()
L.hsort_debug_phase_counters(buf, 256, 1)
hs.hsort_sort_device(d_in, d_out)
torch.cuda.synchronize()
L.hsort_debug_phase_counters(buf, 256, 1)
T = max(1, buf[213])
res = {"tiles": T,
       "compute_total": buf[212] / T, "wait_tma": buf[211] / T, "count+publish": buf[219] / T,
       "rank+scatter": buf[218] / T, "  of which peers": buf[221] / T, "writeout(incl wait)": buf[220] / T, "wait_lookback": buf[210] / T,
       "lb_idle": buf[214] / max(1, buf[217]), "lb_time": buf[215] / max(1, buf[217]),
       "lb_rounds": buf[216] / max(1, buf[217]),
       "warp0(digit): bar1_wait": buf[224] / max(1, buf[227]), "warp0: reduce+scan+bases": buf[225] / max(1, buf[227]),
       "warp0: bar2_wait": buf[226] / max(1, buf[227]),
       "warp17: bar1_wait": buf[228] / max(1, buf[231]), "warp17: scan window": buf[229] / max(1, buf[231]),
       "warp17: bar2_wait": buf[230] / max(1, buf[231])}
print(json.dumps({k: round(v, 1) if isinstance(v, float) else v for k, v in res.items()}))

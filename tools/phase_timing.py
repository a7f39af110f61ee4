"""Per-phase cycle breakdown of the TMA onesweep pass (instrumented libhsort_timing.so)."""
import ctypes
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_ipps_gowanlockk18a_b200 as hs  # noqa: E402

hs.LIB_PATH = os.path.join(ROOT, "paper_conf_ipps_gowanlockk18a_b200", "libhsort_timing.so")
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
names = {0: "wait+claim", 2: "keys+earlycount+scan+bases", 3: "rank", 4: "scatter+lookback",
         5: "writeout"}
res = {}
for p in range(8):
    tiles = buf[p * 16 + 8]
    if tiles:
        res[p] = {nm: round(buf[p * 16 + i] / tiles) for i, nm in names.items()}
        res[p]["tiles"] = tiles
print(json.dumps(res))
T = max(1, sum(buf[p * 16 + 8] for p in range(8)))
print("lookback rounds (digit 0) per tile:", buf[200] / T, " rounds whose nearest window tile was unpublished:",
      buf[201] / T, " rounds whose nearest tile had P:", buf[202] / T)

"""Probe host->host hsort_sort configurations at full size and print per-stage stats."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import hsort_inputs  # noqa: E402
import paper_conf_ipps_gowanlockk18a_b200 as hs  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 1 << 30
batches = [int(x) for x in sys.argv[2].split(",")] if len(sys.argv) > 2 else [0, 1 << 28, 1 << 27]
hs.hsort_init()
A = torch.empty(n, dtype=torch.float64).pin_memory()
hsort_inputs.generate("uniform", n, seed=2, out=A.numpy())
B = torch.empty(n, dtype=torch.float64).pin_memory()
for b in batches:
    hs.hsort_sort(A, B, batch_elems=b)  # warm
    ts = []
    for _ in range(3):
        t = time.perf_counter()
        hs.hsort_sort(A, B, batch_elems=b)
        ts.append(time.perf_counter() - t)
    st = hs.hsort_get_stats()
    v = B.numpy()[:: 1 << 10]
    ok = bool((v[1:] >= v[:-1]).all())
    print(json.dumps({"batch": b, "best_s": min(ts), "keys_per_s": n / min(ts), "sorted_sample": ok,
                      **{k: (round(v, 5) if isinstance(v, float) else v) for k, v in st.items()}}),
          flush=True)
hs.hsort_finalize()

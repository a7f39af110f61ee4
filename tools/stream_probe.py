"""Probe the STREAM (paper PIPEDATA / BLINEMULTI) path: pageable vs pinned, CPU merge."""
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
b = int(sys.argv[2]) if len(sys.argv) > 2 else 1 << 27
hs.hsort_init()
A = hsort_inputs.generate("uniform", n, seed=3)
B = np.empty_like(A)
B[::4096] = 0  # touch
Ap = torch.empty(n, dtype=torch.float64).pin_memory()
Bp = torch.empty(n, dtype=torch.float64).pin_memory()
Ap.numpy()[:] = A
for label, aa, bb, opts in [
    ("stream_pageable", A, B, {"resident": 0, "pipeline": 1}),
    ("stream_pinned", Ap, Bp, {"resident": 0, "pipeline": 1}),
    ("blinemulti_pageable", A, B, {"resident": 0, "pipeline": 0}),
    ("resident_pageable", A, B, {"resident": 1, "pipeline": 1}),
    ("auto_pageable", A, B, {"resident": -1, "pipeline": 1}),
]:
    for k, v in opts.items():
        hs.hsort_set_option(k, v)
    bs = 0 if label.startswith("auto") else b
    hs.hsort_sort(aa, bb, batch_elems=bs)
    t = time.perf_counter()
    hs.hsort_sort(aa, bb, batch_elems=bs)
    dt = time.perf_counter() - t
    st = hs.hsort_get_stats()
    out = bb.numpy() if hasattr(bb, "numpy") else bb
    v = out[:: 1 << 12]
    print(json.dumps({"label": label, "s": dt, "keys_per_s": n / dt,
                      "sorted_sample": bool((v[1:] >= v[:-1]).all()),
                      **{k: (round(x, 4) if isinstance(x, float) else x) for k, x in st.items()}}), flush=True)
hs.hsort_set_option("resident", -1)
hs.hsort_set_option("pipeline", 1)
hs.hsort_finalize()

import os, sys, time, json
sys.path.insert(0, os.getcwd())
import torch, hsort_inputs
import paper_conf_ipps_gowanlockk18a_b200 as hs
n = 1 << 30
hs.hsort_init()
A = torch.empty(n, dtype=torch.float64).pin_memory()
hsort_inputs.generate("uniform", n, seed=2, out=A.numpy())
B = torch.empty(n, dtype=torch.float64).pin_memory()
hs.hsort_sort(A, B)
for _ in range(3):
    t = time.perf_counter(); hs.hsort_sort(A, B); dt = time.perf_counter() - t
    st = hs.hsort_get_stats()
    print(json.dumps({"wall_ms": dt * 1e3, **{k: (round(v * 1e3, 2) if isinstance(v, float) else v) for k, v in st.items() if k.startswith("t_") or k in ("n_b", "mode_name")}}))

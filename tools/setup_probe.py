import os, sys, time, json, ctypes
sys.path.insert(0, os.getcwd())
import torch
import hsort_inputs
import paper_conf_ipps_gowanlockk18a_b200 as hs
n = 1 << 30
hs.hsort_init()
A = torch.empty(n, dtype=torch.float64, pin_memory=True)
B = torch.empty(n, dtype=torch.float64, pin_memory=True)
hsort_inputs.generate("uniform", n, seed=2, out=A.numpy())
cudart = ctypes.CDLL("libcudart.so.12") if False else None
for _ in range(2): hs.hsort_sort(A, B)
rows = []
for i in range(20):
    hs.hsort_sort(A, B)
    st = hs.hsort_get_stats()
    t = time.perf_counter(); torch.cuda.mem_get_info(); t1 = time.perf_counter() - t
    time.sleep(0.0)
    t = time.perf_counter(); torch.cuda.mem_get_info(); t2 = time.perf_counter() - t
    rows.append((round(st["t_setup"]*1e3, 2), round(t1*1e3, 3), round(t2*1e3, 3)))
print(json.dumps(rows))
# after an idle pause
for i in range(5):
    time.sleep(0.5)
    t = time.perf_counter(); torch.cuda.mem_get_info(); print("idle memgetinfo ms", (time.perf_counter()-t)*1e3)

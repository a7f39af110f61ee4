import torch, time, os, subprocess
print(torch.cuda.get_device_name(0), torch.cuda.get_device_properties(0))
free, total = torch.cuda.mem_get_info()
print("mem", free/2**30, total/2**30)
n = 1<<30
h = torch.empty(n, dtype=torch.uint8).pin_memory()
d = torch.empty(n, dtype=torch.uint8, device='cuda')
for name, fn in [("h2d", lambda: d.copy_(h, non_blocking=True)), ("d2h", lambda: h.copy_(d, non_blocking=True))]:
    fn(); torch.cuda.synchronize()
    e0=torch.cuda.Event(enable_timing=True); e1=torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(5): fn()
    e1.record(); torch.cuda.synchronize()
    print(name, 5*n/(e0.elapsed_time(e1)/1e3)/1e9, "GB/s")
# bidir
h2 = torch.empty(n, dtype=torch.uint8).pin_memory(); d2 = torch.empty(n, dtype=torch.uint8, device='cuda')
s1=torch.cuda.Stream(); s2=torch.cuda.Stream()
torch.cuda.synchronize(); t=time.perf_counter()
for _ in range(5):
    with torch.cuda.stream(s1): d.copy_(h, non_blocking=True)
    with torch.cuda.stream(s2): h2.copy_(d2, non_blocking=True)
torch.cuda.synchronize(); dt=time.perf_counter()-t
print("bidir total", 10*n/dt/1e9, "GB/s")
# pageable
p = torch.empty(n, dtype=torch.uint8)
p.fill_(1)
torch.cuda.synchronize(); t=time.perf_counter()
for _ in range(3): d.copy_(p)
torch.cuda.synchronize(); print("pageable h2d", 3*n/(time.perf_counter()-t)/1e9)
t=time.perf_counter()
for _ in range(3): p.copy_(d)
torch.cuda.synchronize(); print("pageable d2h", 3*n/(time.perf_counter()-t)/1e9)
# host memcpy single thread
import numpy as np
a = np.ones(n, dtype=np.uint8); b = np.empty_like(a)
t=time.perf_counter(); np.copyto(b,a); print("np memcpy 1 thread", n/(time.perf_counter()-t)/1e9)
t=time.perf_counter(); np.copyto(b,a); print("np memcpy 1 thread", n/(time.perf_counter()-t)/1e9)
# device sort reference (library context)
x = torch.rand(1<<28, dtype=torch.float64, device='cuda')
torch.sort(x); torch.cuda.synchronize()
e0.record(); torch.sort(x); e1.record(); torch.cuda.synchronize()
print("torch.sort f64 2^28 ms", e0.elapsed_time(e1))

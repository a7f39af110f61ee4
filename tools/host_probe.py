"""Host-side roofline probe for the out-of-core (STREAM) regime (SURVEY §8(d) roofline 3).

Measures on the GPU box: CPU/NUMA layout, host memcpy bandwidth of PARMEMCPY (hsort_par_memcpy)
by thread count and store kind, cudaHostRegister / cudaHostAlloc cost per GB, and pinned link
bandwidth.  Prints one JSON line per measurement.
"""
import ctypes
import json
import os
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_gowanlockk18a_b200 as hs  # noqa: E402


def emit(**kw):
    print(json.dumps(kw), flush=True)


def sh(cmd):
    try:
        return subprocess.run(cmd, shell=True, capture_output=True, text=True, timeout=30).stdout
    except Exception as e:  # noqa: BLE001
        return str(e)


emit(kind="lscpu", text=sh("lscpu | head -30"))
emit(kind="numa", text=sh("numactl -H 2>/dev/null | head -20; cat /sys/devices/system/node/online"))
emit(kind="meminfo", text=sh("grep -E 'MemTotal|MemAvailable|Hugepage|AnonHuge' /proc/meminfo"))
emit(kind="topo", text=sh("nvidia-smi topo -m"))
emit(kind="thp", text=sh("cat /sys/kernel/mm/transparent_hugepage/enabled"))

GB = 1 << 30
nbytes = 8 * GB
a = np.empty(nbytes // 8, dtype=np.uint64)
b = np.empty_like(a)
a.fill(1)
b.fill(2)
for nt in (1, 0):
    hs.hsort_set_option("memcpy_nt", nt)
    for th in (1, 2, 4, 8, 12, 16, 24, 32):
        if th > os.cpu_count():
            continue
        hs.hsort_par_memcpy(b, a, th)
        t = time.perf_counter()
        for _ in range(2):
            hs.hsort_par_memcpy(b, a, th)
        dt = (time.perf_counter() - t) / 2
        emit(kind="par_memcpy", nt=nt, threads=th, GBps_copy=nbytes / dt / 1e9,
             GBps_traffic=(2 if nt else 3) * nbytes / dt / 1e9)
hs.hsort_set_option("memcpy_nt", 1)

# pinning costs
cudart = torch.cuda.cudart()
for gb in (4, 16):
    x = np.empty(gb * GB // 8, dtype=np.uint64)
    x.fill(3)
    t = time.perf_counter()
    r = cudart.cudaHostRegister(x.ctypes.data, x.nbytes, 0)
    dt = time.perf_counter() - t
    emit(kind="cudaHostRegister", GB=gb, seconds=dt, GBps=gb / dt, rc=int(r))
    t = time.perf_counter()
    cudart.cudaHostUnregister(x.ctypes.data)
    emit(kind="cudaHostUnregister", GB=gb, seconds=time.perf_counter() - t)
    del x
    t = time.perf_counter()
    y = torch.empty(gb * GB // 8, dtype=torch.float64).pin_memory()
    emit(kind="pin_memory(alloc)", GB=gb, seconds=time.perf_counter() - t)
    del y

# H2D / D2H into pageable vs pinned (driver-staged pageable copies for context)
d = torch.empty(nbytes // 8, dtype=torch.float64, device="cuda")
ta = torch.from_numpy(a.view(np.float64))
for name, fn in (("h2d_pageable", lambda: d.copy_(ta)), ("d2h_pageable", lambda: ta.copy_(d))):
    fn()
    torch.cuda.synchronize()
    t = time.perf_counter()
    fn()
    torch.cuda.synchronize()
    emit(kind=name, GBps=nbytes / (time.perf_counter() - t) / 1e9)

"""Throughput of concurrent host->host sorts on one B200 (hsort_sort_lane): L lanes (GPU contexts
of the same device, option virtual_gpus), each sorting its own pinned 2^30-key array K times;
keys/s = L K 2^30 / wall time.  One sort cannot overlap its HtoD with its DtoH; two can."""
import json, os, sys, threading, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import hsort_inputs
import paper_conf_ipps_gowanlockk18a_b200 as hs

n = 1 << 30
L = int(sys.argv[1]) if len(sys.argv) > 1 else 2
K = int(sys.argv[2]) if len(sys.argv) > 2 else 6
hs.hsort_set_option("virtual_gpus", L)
hs.hsort_init()
A = [torch.empty(n, dtype=torch.float64, pin_memory=True) for _ in range(L)]
B = [torch.empty(n, dtype=torch.float64, pin_memory=True) for _ in range(L)]
for i in range(L):
    hsort_inputs.generate("uniform", n, seed=2 + i, out=A[i].numpy())
for i in range(L):
    hs.hsort_sort_lane(i, A[i], B[i])  # warm (buffers)
for lanes in range(1, L + 1):
    bar = threading.Barrier(lanes + 1)
    done = []
    phases = []
    t_start = [time.perf_counter()]
    def work(l):
        bar.wait()
        for _ in range(K):
            t = time.perf_counter()
            hs.hsort_sort_lane(l, A[l], B[l])
            st = hs.hsort_get_stats()
            phases.append({"lane": l, "t0": round(t - t_start[0], 3), "s": round(time.perf_counter() - t, 3),
                           "sort_phase": round(st["t_sort_phase"], 3), "merge_phase": round(st["t_merge_phase"], 3)})
        done.append(time.perf_counter())
    th = [threading.Thread(target=work, args=(l,)) for l in range(lanes)]
    for t in th: t.start()
    bar.wait()
    t0 = time.perf_counter()
    t_start[0] = t0
    for t in th: t.join()
    dt = max(done) - t0
    ok = all(bool(np.all(B[l].numpy()[1:] >= B[l].numpy()[:-1])) for l in range(lanes))
    print(json.dumps({"lanes": lanes, "sorts": lanes * K, "s": dt, "keys_per_s": lanes * K * n / dt,
                      "ms_per_sort": 1e3 * dt / K, "sorted": ok}), flush=True)
    if os.environ.get("LANES_PHASES"):
        for ph in sorted(phases, key=lambda x: x["t0"]): print(json.dumps(ph))
hs.hsort_finalize()

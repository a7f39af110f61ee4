"""Small invocations of every kernel path, for compute-sanitizer (memcheck / racecheck /
synccheck / initcheck): K1/K2/K3 (f64, u64, elision with a lowered threshold; the elision's K1
outlier count on normal data), key/value, typed float32 descending, K4 two-level + K5, host
RESIDENT and STREAM modes, and (round 2) the multi-GPU RESIDENT merge through the run-pointer
table, the MSD-first split (K6a-d), multi-GPU STREAM on 3 virtual GPUs, the key/value RESIDENT
plan (key/value K5), the native float32 GPUSort and two concurrent lanes.  Checks results against
the oracle so a silent corruption also fails."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import hsort_inputs
import oracle
import paper_conf_ipps_gowanlockk18a_b200 as hs

hs.hsort_init()
hs.hsort_set_option("dde_min_n", 1 << 16)
bits = lambda a: np.ascontiguousarray(a).view(np.uint64)

A = hsort_inputs.generate("salted", 100_003, seed=1)
d = torch.from_numpy(A).cuda(); o = torch.empty_like(d)
hs.hsort_sort_device(d, o); torch.cuda.synchronize()
assert np.array_equal(bits(o.cpu().numpy()), bits(oracle.sort_f64(A))), "device f64"

U = hsort_inputs.generate("uniform", 1 << 17, seed=2)       # elision: ~4 outliers, cap 4096
d = torch.from_numpy(U).cuda(); o = torch.empty_like(d)
hs.hsort_sort_device(d, o); torch.cuda.synchronize()
assert hs.hsort_get_last_plan()["elided"], "elision not triggered"
assert np.array_equal(bits(o.cpu().numpy()), bits(oracle.sort_f64(U))), "elision"

V = np.arange(50_001, dtype=np.uint64)
B, VB = hs.hsort_sort_pairs(A[:50_001], V)
wB, wV = oracle.sort_pairs_f64(A[:50_001], V)
assert np.array_equal(bits(B), bits(wB)) and np.array_equal(VB, wV), "pairs"

A32 = A.astype(np.float32)
assert np.array_equal(hs.hsort_sort_typed(A32, descending=True).view(np.uint32),
                      oracle.sort_f32(A32, True).view(np.uint32)), "typed"

rng = np.random.default_rng(3)
runs = [np.sort(rng.integers(0, 2**64, size=int(rng.integers(50_000, 70_000)), dtype=np.uint64)) for _ in range(5)]
off = np.cumsum([0] + [r.size for r in runs]).astype(np.uint64)
dk = torch.from_numpy(np.concatenate(runs).view(np.int64)).cuda(); dm = torch.empty_like(dk)
hs.hsort_device_merge(dk, off, dm, False); torch.cuda.synchronize()
assert np.array_equal(dm.cpu().numpy().view(np.uint64), oracle.merge_runs(runs)), "K4/K5"

want = bits(oracle.sort_f64(A))
assert np.array_equal(bits(hs.hsort_sort(A, batch_elems=30_001)), want), "RESIDENT"
hs.hsort_set_option("resident", 0)
assert np.array_equal(bits(hs.hsort_sort(A, batch_elems=30_001)), want), "STREAM"
N = hsort_inputs.generate("normal", 1 << 17, seed=5)  # elision K1 with a wrong guess (shared count)
d = torch.from_numpy(N).cuda(); o = torch.empty_like(d)
hs.hsort_sort_device(d, o); torch.cuda.synchronize()
assert np.array_equal(bits(o.cpu().numpy()), bits(oracle.sort_f64(N))), "elision K1, normal data"
hs.hsort_finalize()

hs.hsort_set_option("resident", -1)
hs.hsort_set_option("virtual_gpus", 3)
hs.hsort_init()
assert np.array_equal(bits(hs.hsort_sort(A, batch_elems=20_000, n_gpus=3)), want), "multi RESIDENT"
hs.hsort_set_option("msd", 1)
hs.hsort_set_option("msd_bucket_keys", 1 << 16)
assert np.array_equal(bits(hs.hsort_sort(A, batch_elems=20_000, n_gpus=3)), want), "MSD split"
hs.hsort_set_option("msd", 0)
hs.hsort_set_option("resident", 0)
hs.hsort_set_option("merge_gpu_permille", 500)
assert np.array_equal(bits(hs.hsort_sort(A, batch_elems=20_000, n_gpus=3)), want), "multi STREAM"
hs.hsort_set_option("resident", -1)
# key/value RESIDENT plan over 2 GPU contexts (key/value K5, value run-pointer tables)
Vp = np.arange(A.size, dtype=np.uint64)
wB, wV = oracle.sort_pairs_f64(A, Vp)
B2, VB2 = hs.hsort_sort_pairs_ex(A, Vp, batch_elems=20_000, n_gpus=2)
assert np.array_equal(bits(B2), bits(wB)) and np.array_equal(VB2, wV), "pairs RESIDENT multi"
# native float32 GPUSort
F = A.astype(np.float32)
assert np.array_equal(hs.hsort_sort_typed(F).view(np.uint32), oracle.sort_f32(F, False).view(np.uint32)), "f32 native"
# two lanes at once
import threading
res = {}
def lane(l):
    res[l] = hs.hsort_sort_lane(l, A, batch_elems=30_000 if l else 0)
th = [threading.Thread(target=lane, args=(l,)) for l in (0, 1)]
for t in th: t.start()
for t in th: t.join()
assert all(np.array_equal(bits(res[l]), want) for l in (0, 1)), "lanes"
hs.hsort_finalize()
print("sanitize_run ok")

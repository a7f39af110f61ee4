#!/usr/bin/env python
"""bench.py — headline benchmark of the B200-native heterogeneous float64 sort.

Metric (BASELINE.json): end-to-end keys/s host->host (float64) at 1/2/4/8 B200; radix GB/s vs HBM.

One step = one call of the public C ABI  hsort_sort(A, B, n, batch_elems=0, n_gpus=N)  on pinned
host buffers: HtoD of A, the batched GPUSort (§III-B), the merge of the sorted batches
(§III-A; K4/K5 on the GPUs) and the DtoH into B are all inside the timed region.  At N = 1 the
workload is BASELINE.json configs[1]: n = 2^30 uniform float64 (8 GiB); the auto plan runs it as
the pipelined RESIDENT schedule (12 batches: 2^27-key batches + a halving tail, merged on the GPU,
merged chunks DtoH'd while the next is merged).  ``value`` is that host->host rate (the metric);
``e2e`` repeats it with the bytes copied per step.

At N > 1 (torchrun, one process per GPU) rank 0 drives all N GPUs through ONE library call on
N x 2^30 keys (the multi-GPU method inside the library: every GPU sorts a shard resident in HBM and
merges one range of B from all GPUs' runs by peer loads) -- the other ranks only
join the control barriers (gloo: no data-path collective exists, and an idle NCCL kernel would sit
on a GPU that rank 0 is sorting on).  Total work grows with N: "weak" scaling.

Also reported (outside the timed region, rank 0): ``device_value`` -- the GPUSort alone on 2^30
keys already in HBM, whose dominant kernel gives ``roofline`` (K3 onesweep pass, algorithmic
16 B/key over its CUDA-event launch time); ``stages`` (K1, K3, key/value pass, typed sorts, K4/K5
merge); ``skewed`` (C4's normal and zipf-dup data: host->host and device sorts); ``out_of_core``
(the paper's STREAM workflow at the largest n this host fits: 2 GB batches, runs to W, CPU/GPU
merge split, with its own link / host-DRAM roofline); the CPU oracle and a 16-thread GNU parallel
sort on the host cores.

``--impl reference`` times the CPU oracle (oracle/, serial std::sort under IEEE totalOrder) on the
host cores, on a bounded sample of the same workload per step.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "end-to-end keys/s host->host (float64) at 1/2/4/8 B200; radix GB/s vs HBM"
N_PER_GPU = 1 << 30
SEED = 2
WORKLOAD = ("C2: n=2^30 uniform float64 (8 GiB) per GPU, host->host through hsort_sort "
            "(auto plan: pipelined RESIDENT batches, GPU merge)")
ALG_BYTES_PER_KEY_PASS = 16  # one onesweep digit pass reads 8 B and writes 8 B per key
ORACLE_SAMPLE = 1 << 26      # cpu_baseline sample (~10 s of serial CPU work)
REF_STEP_SAMPLE = 1 << 24    # --impl reference: keys per step
OOC_BATCH = 250_000_000      # C3: 2 GB batches (reading A-7)
OOC_SEED = 3


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def load_traffic():
    """Per-launch DRAM bytes of the onesweep pass from the committed ncu --set full capture."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(p):
        try:
            d = json.load(open(p))
            return d.get("onesweep_dram_bytes_per_launch"), d.get("n")
        except Exception:
            return None, None
    return None, None


class ClockSampler:
    """Samples SM clocks and throttle reasons via NVML during the timed region (all devices used)."""

    def __init__(self, dev_indices):
        self.samples = []
        self.reasons = set()
        self.max_mhz = None
        self._stop = threading.Event()
        self._t = None
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.hs = [pynvml.nvmlDeviceGetHandleByIndex(i) for i in dev_indices]
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.hs[0], pynvml.NVML_CLOCK_SM)
        except Exception:
            self.nv = None

    def _run(self):
        nv = self.nv
        names = {
            getattr(nv, "nvmlClocksEventReasonHwSlowdown", 0x8): "hw_slowdown",
            getattr(nv, "nvmlClocksEventReasonHwThermalSlowdown", 0x40): "hw_thermal_slowdown",
            getattr(nv, "nvmlClocksEventReasonSwThermalSlowdown", 0x20): "sw_thermal_slowdown",
            getattr(nv, "nvmlClocksEventReasonSwPowerCap", 0x4): "sw_power_cap",
        }
        while not self._stop.is_set():
            try:
                for h in self.hs:
                    self.samples.append(nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM))
                    r = nv.nvmlDeviceGetCurrentClocksEventReasons(h)
                    for bit, name in names.items():
                        if r & bit:
                            self.reasons.add(name)
            except Exception:
                pass
            time.sleep(0.02)

    def __enter__(self):
        if self.nv:
            self._t = threading.Thread(target=self._run, daemon=True)
            self._t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self._t:
            self._t.join()

    def summary(self):
        return {
            "sm_mhz": statistics.median(self.samples) if self.samples else None,
            "sm_max_mhz": self.max_mhz,
            "reasons": sorted(self.reasons),
            "samples": len(self.samples),
        }


def dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


def mem_available():
    try:
        for line in open("/proc/meminfo"):
            if line.startswith("MemAvailable:"):
                return int(line.split()[1]) * 1024
    except OSError:
        pass
    return 64 << 30


# ---- output guards (outside the timed region; full size) --------------------------------------
def _chunks(n, chunk):
    return [(i, min(n, i + chunk)) for i in range(0, n, chunk)]


def _pmap(fn, items):
    from concurrent.futures import ThreadPoolExecutor
    with ThreadPoolExecutor(max_workers=os.cpu_count() or 8) as ex:  # numpy releases the GIL
        return list(ex.map(fn, items))


def multiset_sig(a: np.ndarray, chunk: int = 1 << 24):
    """Order-independent signature of the 64-bit patterns (two wrap-around sums of mixed bits)."""
    u = a.view(np.uint64)

    def part(r):
        x = u[r[0]:r[1]]
        with np.errstate(over="ignore"):
            m = (x ^ (x >> np.uint64(29))) * np.uint64(0x9E3779B97F4A7C15)
            return int(x.sum(dtype=np.uint64)), int((m ^ (m >> np.uint64(32))).sum(dtype=np.uint64))
    parts = _pmap(part, _chunks(u.size, chunk))
    return sum(p[0] for p in parts) % 2**64, sum(p[1] for p in parts) % 2**64


def is_sorted(b: np.ndarray, chunk: int = 1 << 24) -> bool:
    """Non-decreasing as float64 (NaN-free data); chunk seams included."""
    def part(r):
        x = b[r[0]:min(b.size, r[1] + 1)]
        return bool(np.all(x[1:] >= x[:-1]))
    return all(_pmap(part, _chunks(b.size, chunk)))


def guard(A, B, what):
    assert is_sorted(B), f"{what}: output not sorted"
    assert multiset_sig(A) == multiset_sig(B), f"{what}: output is not a permutation of the input"


def cpu_baseline_oracle(n_sample: int):
    import hsort_inputs
    import oracle
    A = hsort_inputs.generate("uniform", n_sample, seed=SEED)
    t = time.perf_counter()
    oracle.sort_f64(A)
    dt = time.perf_counter() - t
    return {
        "value": n_sample / dt, "unit": "keys/s", "cores": 1, "kind": "oracle",
        "sample": f"first {n_sample} keys of the C2 workload (uniform seed {SEED}), serial "
                  f"std::sort under IEEE totalOrder (oracle/oracle.cpp), {dt:.2f} s",
    }


PAR_SAMPLE = 1 << 27        # parallel-CPU baseline sample (~2-3 s on 16 cores)


def cpu_parallel_baseline(n_sample: int):
    """The paper's reference implementation: GNU parallel-mode sort (multiway
    mergesort) under the same totalOrder, on all physical host cores, 3 trials."""
    import hsort_inputs
    import oracle
    try:
        import psutil
        cores = psutil.cpu_count(logical=False) or os.cpu_count()
    except Exception:
        cores = os.cpu_count()
    A = hsort_inputs.generate("uniform", n_sample, seed=SEED)
    oracle.par_sort_f64(A[: 1 << 20], cores)  # warm (thread pool, library load)
    ts = []
    for _ in range(3):
        t = time.perf_counter()
        oracle.par_sort_f64(A, cores)
        ts.append(time.perf_counter() - t)
    dt = statistics.median(ts)
    return {
        "value": n_sample / dt, "unit": "keys/s", "cores": cores, "kind": "gnu_parallel_sort",
        "sample": f"first {n_sample} keys of the C2 workload (uniform seed {SEED}), "
                  f"__gnu_parallel::sort (multiway mergesort, exact splitting) under IEEE totalOrder, "
                  f"{cores} OpenMP threads, median of 3: {dt:.2f} s",
        "paper_context": "paper: up to 3.47x end-to-end over a 16-thread GNU parallel sort on "
                         "2x8-core Xeon E5-2620 v4 + 1x Quadro GP100, PCIe 3, n = 1e9 float64 "
                         "(P:907-910, P:499-504); context only",
    }


# ---- link probe -------------------------------------------------------------------------------
def link_probe(torch, h_a, h_b, d_a, d_b):
    """Pinned copy bandwidth per direction (best of 1 and 2 streams) and both directions at once
    (the aggregate when HtoD and DtoH overlap, as in the STREAM pipeline)."""
    n = min(h_a.numel(), d_a.numel(), 1 << 27)
    side = [torch.cuda.Stream(), torch.cuda.Stream()]

    def timed(jobs):
        best = 0.0
        for _ in range(2):
            torch.cuda.synchronize()
            e_a, e_b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e_a.record()
            for i, (dst, src) in enumerate(jobs):
                side[i % 2].wait_event(e_a)
                with torch.cuda.stream(side[i % 2]):
                    dst.copy_(src, non_blocking=True)
            for s in side:
                torch.cuda.current_stream().wait_stream(s)
            e_b.record()
            e_b.synchronize()
            nbytes = sum(src.numel() * 8 for _, src in jobs)
            best = max(best, nbytes / (e_a.elapsed_time(e_b) / 1e3))
        return best

    h = n // 2
    bw = {
        "h2d": max(timed([(d_a[:n], h_a[:n])]), timed([(d_a[:h], h_a[:h]), (d_a[h:n], h_a[h:n])])),
        "d2h": max(timed([(h_b[:n], d_b[:n])]), timed([(h_b[:h], d_b[:h]), (h_b[h:n], d_b[h:n])])),
        "both": timed([(d_a[:n], h_a[:n]), (h_b[:n], d_b[:n])]),
    }
    return bw


def host_copy_bw(hs):
    """Host-DRAM traffic rate: PARMEMCPY on 2 GiB prefaulted pageable buffers with all host threads,
    streaming stores (2 bytes of traffic per byte copied) and ordinary stores (3: the destination
    is read for ownership); the larger traffic rate is the host-DRAM peak for the roofline."""
    a = np.ones(1 << 28, dtype=np.uint64)
    b = np.zeros_like(a)
    best = 0.0
    old = hs.hsort_get_option("memcpy_nt")
    try:
        for nt, per_byte in ((1, 2), (0, 3)):
            hs.hsort_set_option("memcpy_nt", nt)
            hs.hsort_par_memcpy(b, a)
            t = time.perf_counter()
            for _ in range(3):
                hs.hsort_par_memcpy(b, a)
            best = max(best, per_byte * 3 * a.nbytes / (time.perf_counter() - t))
    finally:
        hs.hsort_set_option("memcpy_nt", old)
    return best


MERGE_K = 12  # runs of the RESIDENT auto plan at n = 2^30 (2^27-key batches + halving tail)


def stage_rooflines(hs, torch, d_in, d_out, n, peak, hist_ms, pass_ms, stream):
    """Per-stage HBM rooflines (outside the timed region): K1 and K3 from the timed device steps,
    the key/value pass, the typed sorts, and the GPU merge of k = MERGE_K device-resident sorted
    runs (K4 co-ranks + K5 tile merge, the RESIDENT mode's merge), timed with CUDA events on the
    launching stream.  Algorithmic bytes: K1 8 B/key, K3 16 B/key per pass, K5 16 B/key.
    Overwrites d_out (d_in is restored)."""
    vals = torch.arange(n, dtype=torch.int64, device=d_in.device)
    kout, vout = torch.empty_like(d_in), torch.empty_like(vals)
    hs.hsort_sort_device_pairs(d_in, vals, kout, vout, True, stream)  # warm
    kv_ms, kv_pass = [], []
    for _ in range(3):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        hs.hsort_sort_device_pairs(d_in, vals, kout, vout, True, stream)
        e1.record(stream)
        e1.synchronize()
        kv_ms.append(e0.elapsed_time(e1))
        kt = hs.hsort_get_kernel_times()
        kv_pass.extend(kt["passes"][:kt["num_active"]])
    assert bool((kout[1:] >= kout[:-1]).all()), "pairs output not sorted"
    del vals, kout, vout
    kv = statistics.median(kv_ms)
    kv_pass_ms = statistics.mean(kv_pass)

    def timed(fn):
        fn()
        ts = []
        for _ in range(3):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            fn()
            e1.record(stream)
            e1.synchronize()
            ts.append(e0.elapsed_time(e1))
        return statistics.median(ts)
    d32 = d_in.float()
    o32 = torch.empty_like(d32)
    f32_ms = timed(lambda: hs.hsort_sort_device_typed(d32, o32, False, stream))
    f32_passes = hs.hsort_get_kernel_times()["num_active"]
    assert bool((o32[1:] >= o32[:-1]).all()), "float32 output not sorted"
    del d32, o32
    desc_ms = timed(lambda: hs.hsort_sort_device_typed(d_in, d_out, True, stream))
    assert bool((d_out[1:] <= d_out[:-1]).all()), "descending output not sorted"
    types = {"f32_asc": {"sort_ms": f32_ms, "keys_per_s": n / (f32_ms / 1e3), "passes": f32_passes},
             "f64_desc": {"sort_ms": desc_ms, "keys_per_s": n / (desc_ms / 1e3)}}

    cuts = [n * j // MERGE_K for j in range(MERGE_K + 1)]
    for j in range(MERGE_K):
        hs.hsort_sort_device_keys(d_in[cuts[j]:cuts[j + 1]], d_out[cuts[j]:cuts[j + 1]], True, False,
                                  stream)
    tiles = (n + 4095) // 4096
    d_ranks = torch.empty((tiles + 1) * MERGE_K, dtype=torch.int64, device=d_in.device)
    merged = torch.empty_like(d_in)
    hs.hsort_device_merge(d_out, cuts, merged, True, stream)  # warm
    tc, tm = [], []
    for _ in range(3):
        e = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
        e[0].record(stream)
        hs.hsort_device_corank(d_out, cuts, 4096, tiles + 1, d_ranks, stream)
        e[1].record(stream)
        hs.hsort_device_merge(d_out, cuts, merged, True, stream)
        e[2].record(stream)
        e[2].synchronize()
        tc.append(e[0].elapsed_time(e[1]))
        tm.append(e[1].elapsed_time(e[2]))
    assert bool((merged[1:] >= merged[:-1]).all()), "merged output not sorted"
    del merged, d_ranks
    k4, merge = statistics.median(tc), statistics.median(tm)
    k5 = merge - k4

    def hbm(ms, bpk, what):
        gbs = bpk * n / (ms / 1e3) / 1e9
        return {"kernel": what, "bound": "hbm", "ms": ms, "alg_bytes_per_key": bpk,
                "achieved": gbs, "unit": "GB/s", "peak": peak, "frac": gbs / peak}

    return {
        "K1_hist": hbm(hist_ms, 8, "k_hist3 (8 digit histograms, one read)"),
        "K3_onesweep": hbm(pass_ms, 16, "k_onesweep_ws (one 8-bit LSD pass)"),
        "K3_kv_pass": dict(hbm(kv_pass_ms, 32, "k_onesweep_ws<KV> (one LSD pass over key/value pairs)"),
                           sort_ms=kv, pairs_per_s=n / (kv / 1e3)),
        "key_types": types,
        "K5_merge": dict(hbm(k5, 16, f"k_merge_tile (k = {MERGE_K} resident runs, 2^30 keys)"),
                         k4_corank_ms=k4, k4_k5_frac=16 * n / (merge / 1e3) / 1e9 / peak),
    }


def device_sort_timed(hs, torch, d_in, d_out, stream, steps):
    """K GPUSorts of d_in (in HBM) -> d_out, CUDA events on the launching stream; per-kernel
    times from the library's own events (option kernel_timing)."""
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    step_ms, pass_ms, hist_ms = [], [], []
    n_active, plan = 8, None
    for _ in range(steps):
        ev0.record(stream)
        hs.hsort_sort_device(d_in, d_out, stream)
        ev1.record(stream)
        ev1.synchronize()
        step_ms.append(ev0.elapsed_time(ev1))
        kt = hs.hsort_get_kernel_times()
        n_active = kt["num_active"]
        plan = hs.hsort_get_last_plan()
        pass_ms.extend(kt["passes"][:n_active])
        hist_ms.append(kt["hist"])
    return step_ms, pass_ms, hist_ms, n_active, plan


def host_sort_timed(hs, torch, A, B, n_gpus, steps, batch=0):
    """K synchronous hsort_sort calls, each bracketed by CUDA events on device 0's stream (the
    call returns when B is complete, so the event interval is the call's duration on the GPU
    clock) and by the host clock."""
    s = torch.cuda.current_stream(0)
    ev_ms, wall = [], []
    for _ in range(steps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        t = time.perf_counter()
        hs.hsort_sort(A, B, batch_elems=batch, n_gpus=n_gpus)
        wall.append(time.perf_counter() - t)
        e1.record(s)
        e1.synchronize()
        ev_ms.append(e0.elapsed_time(e1))
    return ev_ms, wall


def skewed_rows(hs, torch, A_h, B_h, d_in, d_out, stream, peak, n):
    """C4's distributions (normal N(0,1); zipf-dup: 50% from a 2^16-value Zipf hot set, 50%
    normal) at n = 2^30 on one GPU: host->host through hsort_sort and the device GPUSort (no
    dominant digit: 8 passes), each guarded against its input."""
    import hsort_inputs
    rows = {}
    for dist, seed in (("normal", 4), ("zipf_dup", 5)):
        hsort_inputs.generate(dist, n, seed=seed, out=A_h.numpy())
        hs.hsort_sort(A_h, B_h, batch_elems=0, n_gpus=1)  # warm
        ev_ms, _ = host_sort_timed(hs, torch, A_h, B_h, 1, 3)
        guard(A_h.numpy(), B_h.numpy(), f"{dist} host->host")
        st = hs.hsort_get_stats()
        d_in.copy_(A_h)
        hs.hsort_sort_device(d_in, d_out, stream)
        step_ms, pass_ms, _, n_active, plan = device_sort_timed(hs, torch, d_in, d_out, stream, 3)
        assert bool((d_out[1:] >= d_out[:-1]).all()), f"{dist}: device output not sorted"
        avg = statistics.mean(pass_ms)
        ach = ALG_BYTES_PER_KEY_PASS * n / (avg / 1e3) / 1e9
        rows[dist] = {
            "e2e_keys_per_s": n / (statistics.median(ev_ms) / 1e3), "e2e_ms": statistics.median(ev_ms),
            "mode": st["mode_name"], "n_b": st["n_b"],
            "device_keys_per_s": n / (statistics.median(step_ms) / 1e3),
            "device_ms": statistics.median(step_ms), "passes": n_active, "elided": plan["elided"],
            "K3_avg_pass_ms": avg, "K3_frac": ach / peak,
        }
    return rows


def pairs_e2e(hs, torch, A_h, B_h, n):
    """Key/value host->host (S§8(f) #3, the [5] workload of keys with 64-bit values): 2^30
    (uniform key, index) pairs through hsort_sort_pairs on pinned buffers -- the RESIDENT
    key/value plan (stable batch sorts in HBM + the key/value merge); 32 B/pair cross the link."""
    import hsort_inputs
    hsort_inputs.generate("uniform", n, seed=SEED, out=A_h.numpy())
    V = torch.arange(n, dtype=torch.int64).pin_memory()
    VB = torch.empty(n, dtype=torch.int64, pin_memory=True)
    Vn, VBn = V.numpy().view(np.uint64), VB.numpy().view(np.uint64)
    hs.hsort_sort_pairs(A_h.numpy(), Vn, B_h.numpy(), VBn)  # warm
    ts = []
    for _ in range(3):
        t = time.perf_counter()
        hs.hsort_sort_pairs(A_h.numpy(), Vn, B_h.numpy(), VBn)
        ts.append(time.perf_counter() - t)
    st = hs.hsort_get_stats()
    Bv = B_h.numpy()
    assert is_sorted(Bv), "pairs: keys not sorted"
    assert multiset_sig(A_h.numpy()) == multiset_sig(Bv), "pairs: keys not a permutation"
    # values: the stable argsort of A; spot-check the pairing on a sample (full pairing is pinned
    # against the oracle in tests/test_gpu_pairs.py)
    idx = np.random.default_rng(0).integers(0, n, size=1 << 16)
    assert np.array_equal(A_h.numpy()[VBn[idx].astype(np.int64)].view(np.uint64), Bv[idx].view(np.uint64))
    dt = statistics.median(ts)
    del V, VB
    return {"what": "hsort_sort_pairs(A, V = 0..n-1, B, VB) pinned, 2^30 pairs, RESIDENT key/value plan",
            "pairs_per_s": n / dt, "ms": 1e3 * dt, "mode": st["mode_name"], "n_b": st["n_b"],
            "t_h2d_s": st["t_h2d"], "t_d2h_s": st["t_d2h"], "t_gpu_sort_s": st["t_gpu_sort"],
            "t_merge_gpu_s": st["t_merge_gpu"], "link_bytes_per_pair": 32}


def lanes_row(hs, torch, A_h, B_h, n, sorts_per_lane=3):
    """Serving throughput: two host threads sort their own pinned 2^30-key arrays at the same time
    on lanes 0 and 1 (two GPU contexts of the same B200, hsort_sort_lane).  One sort cannot overlap
    its HtoD with its DtoH (its first output key depends on its last input key); two concurrent
    sorts use both link directions.  Not the headline: `value` is one sort at a time."""
    import hsort_inputs
    hsort_inputs.generate("uniform", n, seed=SEED, out=A_h.numpy())
    A2 = torch.empty(n, dtype=torch.float64, pin_memory=True)
    B2 = torch.empty(n, dtype=torch.float64, pin_memory=True)
    hsort_inputs.generate("uniform", n, seed=SEED + 1, out=A2.numpy())
    pairs = [(A_h, B_h), (A2, B2)]
    for lane in (0, 1):
        hs.hsort_sort_lane(lane, *pairs[lane])  # warm: the lane's buffers
    bar = threading.Barrier(3)
    ends = []

    def work(lane):
        bar.wait()
        for _ in range(sorts_per_lane):
            hs.hsort_sort_lane(lane, *pairs[lane])
        ends.append(time.perf_counter())
    th = [threading.Thread(target=work, args=(lane,)) for lane in (0, 1)]
    for t in th:
        t.start()
    bar.wait()
    t0 = time.perf_counter()
    for t in th:
        t.join()
    dt = max(ends) - t0
    for a, b in pairs:
        guard(a.numpy(), b.numpy(), "lanes")
    del A2, B2
    return {"what": "2 concurrent hsort_sort_lane calls (lanes 0/1 = 2 GPU contexts of one B200), "
                    f"{sorts_per_lane} sorts of 2^30 pinned keys each",
            "keys_per_s": 2 * sorts_per_lane * n / dt, "ms_per_sort_per_lane": 1e3 * dt / sorts_per_lane,
            "vs_one_at_a_time": None}


def out_of_core(hs, torch, bw, host_bw):
    """The paper's out-of-core workflow (STREAM: batches -> HtoD -> GPUSort -> DtoH -> W, then the
    CPU/GPU merge split W -> B, configs C3/C5) at the largest n this host fits with
    A, W and B in RAM (24 B/key), pageable A and B, 2 GB batches (C3).  W is allocated,
    prefaulted and page-locked once (warm-up call) and reused.  Roofline: T_roof = max(T_link,
    T_host) with T_link = max(8n/BW_h2d, 8n/BW_d2h, 16n/BW_both) (1 + f) (the merge share f
    crosses the link again) and T_host = host-DRAM bytes / measured host copy traffic rate, host
    bytes = (48 + 16 f) n."""
    import hsort_inputs
    n = int(min(6e9, 0.5 * mem_available() / 24) // 10**8 * 10**8)
    A = hsort_inputs.generate("uniform", n, seed=OOC_SEED)
    B = np.empty_like(A)
    B[::512] = 0  # prefault lightly; the first call faults the rest
    opts = {"resident": 0, "pin_w": 1}
    old = {k: hs.hsort_get_option(k) for k in opts}
    for k, v in opts.items():
        hs.hsort_set_option(k, v)
    try:
        t = time.perf_counter()
        hs.hsort_sort(A, B, batch_elems=OOC_BATCH, n_gpus=1)  # warm: W allocated + locked here
        warm_s = time.perf_counter() - t
        st0 = hs.hsort_get_stats()
        ev_ms, wall = host_sort_timed(hs, torch, A, B, 1, 2, batch=OOC_BATCH)
        st = hs.hsort_get_stats()
    finally:
        for k, v in old.items():
            hs.hsort_set_option(k, v)
    guard(A, B, "out-of-core")
    f = st["merge_gpu_fraction"]
    t_meas = statistics.median(ev_ms) / 1e3
    t_link = max(8 * n / bw["h2d"], 8 * n / bw["d2h"], 16 * n / bw["both"]) * (1 + f)
    host_bytes = (48 + 16 * f) * n
    t_host = host_bytes / host_bw
    t_roof = max(t_link, t_host)
    del A, B
    return {
        "workload": f"C3-shaped STREAM at the host's limit: n={n} uniform float64 (seed {OOC_SEED}), "
                    f"pageable A/B, b_s={OOC_BATCH} (2 GB batches), runs to page-locked W, "
                    f"CPU/GPU merge split (auto f), 1 B200",
        "n": n, "value": n / t_meas, "unit": "keys/s", "ms": 1e3 * t_meas,
        "steps_ms": [round(x, 1) for x in ev_ms], "warm_call_s": warm_s,
        "w_alloc_s": st0["t_host_alloc"], "mode": st["mode_name"], "n_b": st["n_b"],
        "merge_gpu_fraction": f, "t_sort_phase_s": st["t_sort_phase"],
        "t_merge_phase_s": st["t_merge_phase"], "t_stage_s": st["t_stage"],
        "t_merge_cpu_s": st["t_merge_cpu"], "t_merge_gpu_s": st["t_merge_gpu"],
        "t_h2d_s": st["t_h2d"], "t_d2h_s": st["t_d2h"],
        "roofline": {"bound": "host_link" if t_link >= t_host else "host_dram",
                     "t_link_s": t_link, "t_host_dram_s": t_host, "t_roof_s": t_roof,
                     "host_bytes_per_key": 48 + 16 * f, "host_copy_traffic_gbs": host_bw / 1e9,
                     "frac": t_roof / t_meas},
    }


def run_reference(args):
    ws, rank, _ = dist_env()
    if rank != 0:
        return 0
    import hsort_inputs
    import oracle
    n = REF_STEP_SAMPLE
    A = hsort_inputs.generate("uniform", n, seed=SEED)
    for _ in range(args.warmup):
        oracle.sort_f64(A[: n // 16])
    times = []
    for _ in range(args.steps):
        t = time.perf_counter()
        oracle.sort_f64(A)
        times.append(time.perf_counter() - t)
    tot = sum(times)
    value = n * args.steps / tot
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": "keys/s",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": 1e3 * tot / args.steps, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": WORKLOAD, "n": N_PER_GPU * max(1, args.gpus),
                   "reference_sample_per_step": n},
        "cpu_baseline": {"value": value, "unit": "keys/s", "cores": 1, "kind": "oracle",
                         "sample": f"{n} keys of the C2 workload per step (uniform seed {SEED})"},
        "e2e": {"value": value, "unit": "keys/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--keys-per-gpu", type=int, default=N_PER_GPU, help="keys per GPU (default 2^30, config C2)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-extras", action="store_true",
                    help="only the timed host->host and device steps (profiling runs)")
    ap.add_argument("--device-only", action="store_true",
                    help="profiling: skip the host->host arm (ncu captures of the device GPUSort)")
    ap.add_argument("--virtual-gpus", action="store_true",
                    help="testing on a box with fewer GPUs than --gpus: map N GPU contexts onto the "
                         "visible devices (library option virtual_gpus); not a scaling number")
    ap.add_argument("--no-dde", action="store_true",
                    help="profiling: dominant-digit elision off (every device pass is a full pass)")
    args = ap.parse_args()
    if args.impl == "reference":
        return run_reference(args)
    args.warmup = max(args.warmup, 3)

    import torch
    import torch.distributed as dist

    ws, rank, _ = dist_env()
    N = ws if ws > 1 else max(1, args.gpus)
    if ws > 1:
        # control plane only (barriers, the max over ranks): rank 0 drives all N GPUs through one
        # library call, so no data-path collective exists
        dist.init_process_group("gloo")

    def barrier():
        if ws > 1:
            dist.barrier()

    def max_over_ranks(x: float) -> float:
        if ws == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    if rank != 0:
        barrier()  # timed region starts
        barrier()  # timed region ends
        max_over_ranks(0.0)
        barrier()  # rank 0 done
        dist.destroy_process_group()
        return 0

    import hsort_inputs
    import paper_conf_ipps_gowanlockk18a_b200 as hs

    torch.cuda.set_device(0)
    virtual = torch.cuda.device_count() < N
    if virtual and not args.virtual_gpus:
        raise SystemExit(f"--gpus {N} but only {torch.cuda.device_count()} visible devices")
    if virtual:
        hs.hsort_set_option("virtual_gpus", N)
    # N x 2^30 keys of pinned A and B (16 B/key of host RAM): cap to 60% of the free RAM
    n_gpu = args.keys_per_gpu
    while N * n_gpu * 16 > 0.6 * mem_available() and n_gpu > (1 << 24):
        n_gpu //= 2
    n = N * n_gpu
    hs.hsort_set_option("kernel_timing", 1)
    if N == 1 and not args.no_extras:
        hs.hsort_set_option("virtual_gpus", 2)  # a second GPU context on the device: the lanes row
    if args.no_dde:
        hs.hsort_set_option("dde", 0)
    t0 = time.perf_counter()
    hs.hsort_init()
    t_init = time.perf_counter() - t0

    A_h = torch.empty(n, dtype=torch.float64, pin_memory=True)
    hsort_inputs.generate("uniform", n, seed=SEED, out=A_h.numpy())
    B_h = torch.empty(n, dtype=torch.float64, pin_memory=True)
    d_in = A_h[:n_gpu].to("cuda:0", non_blocking=False)
    d_out = torch.empty_like(d_in)
    stream = torch.cuda.current_stream()
    bw = link_probe(torch, A_h, B_h, d_out, d_in)

    # ---- host->host (value, e2e): one step = hsort_sort(A, B, n, 0, N) -------------------------
    cold_ms = None  # the first call after hsort_init: device buffers allocated inside
    for w in range(0 if args.device_only else args.warmup):
        t = time.perf_counter()
        hs.hsort_sort(A_h, B_h, batch_elems=0, n_gpus=N)
        if w == 0:
            cold_ms = 1e3 * (time.perf_counter() - t)
    if not args.device_only:
        guard(A_h.numpy(), B_h.numpy(), "host->host (warm-up)")
    devs = list(range(min(N, torch.cuda.device_count())))
    L0 = hs.hsort_get_launch_count()
    sampler = ClockSampler(devs)
    barrier()
    for d in devs:
        torch.cuda.synchronize(d)
    with sampler:
        ev_ms, wall = host_sort_timed(hs, torch, A_h, B_h, N, 0 if args.device_only else args.steps)
    if args.device_only:
        ev_ms, wall = [1.0], [1e-3]
    for d in devs:
        torch.cuda.synchronize(d)
    launches = hs.hsort_get_launch_count() - L0
    barrier()
    total_ms = max_over_ranks(sum(ev_ms))
    st = hs.hsort_get_stats()
    if not args.device_only:
        guard(A_h.numpy(), B_h.numpy(), "host->host (last timed step)")  # full size, outside timing
    ms_per_step = total_ms / args.steps
    value = n * args.steps / (total_ms / 1e3)
    link_floor_s = n_gpu * 8 / bw["h2d"] + n_gpu * 8 / bw["d2h"]

    # ---- device-resident GPUSort on GPU 0 (device_value, roofline of the dominant kernel) --------
    for _ in range(args.warmup):
        hs.hsort_sort_device(d_in, d_out, stream)
    torch.cuda.synchronize()
    dsampler = ClockSampler([0])
    with dsampler:
        step_ms, pass_ms, hist_ms, n_active, plan = device_sort_timed(hs, torch, d_in, d_out, stream,
                                                                       args.steps)
    torch.cuda.synchronize()
    assert bool((d_out[1:] >= d_out[:-1]).all()), "device output not sorted"

    def dsig(t):
        u = t.view(torch.int64)
        m = (u ^ (u >> 29)) * -7046029254386353131
        return int(u.sum()), int((m ^ (m >> 32)).sum())
    assert dsig(d_out) == dsig(d_in), "device output is not a permutation of the input"
    device_value = n_gpu * len(step_ms) / (sum(step_ms) / 1e3)
    peak, peak_src = load_peaks()
    avg_pass_ms = statistics.mean(pass_ms)
    achieved = ALG_BYTES_PER_KEY_PASS * n_gpu / (avg_pass_ms / 1e3) / 1e9
    traffic, traffic_n = load_traffic()
    if traffic is not None and traffic_n and traffic_n != n_gpu:
        traffic = traffic * n_gpu / traffic_n

    line = {
        "metric": METRIC,
        "value": value,
        "unit": "keys/s",
        "n_gpus": N,
        "steps": args.steps,
        "warmup": args.warmup,
        "ms_per_step": ms_per_step,
        "higher_is_better": True,
        "scaling": "weak",
        "vs_baseline": None,
        "dtype": "f64",
        "data": "synthetic",
        "config": {
            "workload": WORKLOAD if N == 1 else
            f"C4-shaped: n={N}x2^{n_gpu.bit_length() - 1} uniform float64 on {N} B200 in one "
            f"hsort_sort call (multi-GPU RESIDENT: per-GPU shards, range merge by peer loads)",
            "n": n,
            "api": f"hsort_sort(A pinned, B pinned, n, batch_elems=0 (auto plan), n_gpus={N})",
            "plan": {"mode": st["mode_name"], "n_b": st["n_b"], "b_s": st["b_s"],
                     "n_gpus": st["n_gpus"]},
            "distribution": f"uniform U[0,1) 53-bit, splitmix64 seed {SEED}",
            "parallelism": f"{N} GPU(s) driven by rank 0 through the library" +
                           (f"; {ws} torchrun ranks (control barriers over gloo)" if ws > 1 else ""),
            "l2": f"input {n_gpu * 8 / 2**30:.0f} GiB per GPU >> 126 MB L2: no flush needed between steps",
            "timing": "CUDA events on device 0's stream around each synchronous call (= call "
                      "duration); HtoD, sort, merge and DtoH all inside",
            "virtual_gpus": virtual,
        },
        "e2e": {
            "value": value,
            "unit": "keys/s",
            "h2d_bytes_per_step": n * 8,
            "d2h_bytes_per_step": n * 8,
            "api": f"hsort_sort(A pinned, B pinned, n, batch_elems=0, n_gpus={N})",
            "ms_per_step": ms_per_step,
            "wall_ms_per_step": 1e3 * sum(wall) / len(wall),
            "cold_first_call_ms": cold_ms,
            "cold_init_plus_first_call_ms": (cold_ms or 0) + 1e3 * t_init,
            "mode": st["mode_name"], "n_b": st["n_b"], "b_s": st["b_s"],
            "t_h2d_s": st["t_h2d"], "t_gpu_sort_s": st["t_gpu_sort"], "t_d2h_s": st["t_d2h"],
            "t_merge_gpu_s": st["t_merge_gpu"], "t_sort_phase_s": st["t_sort_phase"],
            "t_merge_phase_s": st["t_merge_phase"],
            "link_gbs": {k: v / 1e9 for k, v in bw.items()},
            "link_floor_ms": 1e3 * link_floor_s,
            "link_frac": link_floor_s / (ms_per_step / 1e3),
            "step_ms": [round(x, 2) for x in ev_ms],
        },
        "device_value": {
            "value": device_value, "unit": "keys/s", "n": n_gpu,
            "what": "hsort_sort_device: K1 + K2 + LSD passes (+ elision) on 2^30 keys already in HBM",
            "ms_per_step": statistics.mean(step_ms), "steps": len(step_ms),
            "clocks": dsampler.summary(),
        },
        "roofline": {
            "kernel": "k_onesweep_ws (one 8-bit LSD digit pass)",
            "bound": "hbm",
            "achieved": achieved,
            "peak": peak,
            "peak_source": peak_src,
            "unit": "GB/s",
            "frac": achieved / peak,
            "traffic": traffic,
            "alg_bytes_per_launch": ALG_BYTES_PER_KEY_PASS * n_gpu,
            "avg_launch_ms": avg_pass_ms,
            "launches_per_step": n_active,
            "share_of_device_step": sum(pass_ms) / sum(step_ms),
            "hist_ms": statistics.mean(hist_ms),
            "measured_in": "device_value steps (CUDA events recorded by the library on the sort's "
                           "stream around each kernel)",
            "dominant_digit_elision": plan,
        },
        "gpu_launches": launches,
        "gpu_launches_per_step": launches / args.steps,
        "clocks": sampler.summary(),
        "init_s": t_init,
    }
    if not args.no_extras and N == 1:
        stages = stage_rooflines(hs, torch, d_in, d_out, n_gpu, peak, statistics.mean(hist_ms),
                                 avg_pass_ms, stream)
        line["stages"] = stages
        line["skewed"] = skewed_rows(hs, torch, A_h, B_h, d_in, d_out, stream, peak, n_gpu)
        line["pairs_e2e"] = pairs_e2e(hs, torch, A_h, B_h, n_gpu)
        line["lanes"] = lanes_row(hs, torch, A_h, B_h, n_gpu)
        line["lanes"]["vs_one_at_a_time"] = line["lanes"]["keys_per_s"] / value
    del d_in, d_out
    torch.cuda.empty_cache()
    host_bw = None
    if not args.no_extras and N == 1:
        del A_h, B_h
        torch._C._host_emptyCache()
        host_bw = host_copy_bw(hs)
        line["out_of_core"] = out_of_core(hs, torch, bw, host_bw)
    if not args.no_cpu_baseline and N == 1:
        line["cpu_baseline"] = cpu_baseline_oracle(ORACLE_SAMPLE)
        par = cpu_parallel_baseline(PAR_SAMPLE)
        par["e2e_speedup"] = value / par["value"]  # our host->host rate / parallel CPU rate
        line["cpu_parallel_baseline"] = par
    print(json.dumps(line), flush=True)
    hs.hsort_finalize()
    if ws > 1:
        barrier()
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())

#!/usr/bin/env python
"""bench.py — headline benchmark of the B200-native heterogeneous float64 sort.

Metric (BASELINE.json): end-to-end keys/s host->host (float64) at 1/2/4/8 B200; radix GB/s vs HBM.
Workload at N=1: BASELINE.json configs[1] — n = 2^30 uniform float64 (8 GiB), one batch
(b_s = n), one B200.  A "step" is one whole GPUSort of that batch (K1 + K2 + 8 onesweep passes,
PAPER.md §III-B) with the input already resident in HBM -> ``value``; ``e2e`` is the same metric
through the public C ABI hsort_sort() with pinned HOST buffers (HtoD + GPUSort + DtoH inside the
timed region, BLINE workflow P:285-292).

Multi-GPU (torchrun, one process per GPU): every rank sorts its own 2^30-key batch — batches are
independent units, no data-path collective — so scaling is "weak" and
value = (N * n) / max-over-ranks time.

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
N_KEYS = 1 << 30
SEED = 2
WORKLOAD = "C2: n=2^30 uniform float64 (8 GiB), single batch b_s=n, 1 B200 per rank"
ALG_BYTES_PER_KEY_PASS = 16  # one onesweep digit pass reads 8 B and writes 8 B per key
ORACLE_SAMPLE = 1 << 26      # cpu_baseline sample (~15 s of serial CPU work)
REF_STEP_SAMPLE = 1 << 24    # --impl reference: keys per step


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
    """Samples SM clocks and throttle reasons via NVML during the timed region."""

    def __init__(self, dev_index: int):
        self.samples = []
        self.reasons = set()
        self.max_mhz = None
        self._stop = threading.Event()
        self._t = None
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(dev_index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
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
                self.samples.append(nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM))
                r = nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
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


MERGE_K = 12  # runs of the RESIDENT auto plan at n = 2^30 (2^27-key batches + halving tail)


def stage_rooflines(hs, torch, d_in, d_out, n, peak, hist_ms, pass_ms, stream):
    """Per-stage HBM rooflines (outside the timed region): K1 and K3 from the timed steps, and the
    GPU merge of k = MERGE_K device-resident sorted runs of the same workload (K4 co-ranks + K5
    tile merge, the RESIDENT mode's merge), timed with CUDA events on the launching stream.
    Algorithmic bytes: K1 8 B/key, K3 16 B/key per pass, K5 16 B/key (read once, write once).
    Overwrites d_in/d_out."""
    # key/value GPUSort (S§8(f) #3): 2^30 (key, index) pairs, 32 B/pair per pass
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

    # other key types / orders (S§8(f) #4): float32 (encode -> 4 LSD passes -> decode) and
    # float64 descending (encode -> 8 passes -> decode), 2^30 keys, whole-sort time
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
    hs.hsort_device_merge(d_out, cuts, d_in, True, stream)  # warm
    tc, tm = [], []
    for _ in range(3):
        e = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
        e[0].record(stream)
        hs.hsort_device_corank(d_out, cuts, 4096, tiles + 1, d_ranks, stream)
        e[1].record(stream)
        hs.hsort_device_merge(d_out, cuts, d_in, True, stream)
        e[2].record(stream)
        e[2].synchronize()
        tc.append(e[0].elapsed_time(e[1]))
        tm.append(e[1].elapsed_time(e[2]))
    o = d_in[:: max(1, n // (1 << 20))]
    assert bool((o[1:] >= o[:-1]).all()), "merged output not sorted"
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
        "config": {"workload": WORKLOAD, "n": N_KEYS, "batch_elems": N_KEYS,
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
    ap.add_argument("--n", type=int, default=N_KEYS, help="keys per rank (default 2^30, config C2)")
    ap.add_argument("--e2e-steps", type=int, default=None)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    args = ap.parse_args()
    if args.impl == "reference":
        return run_reference(args)
    args.warmup = max(args.warmup, 3)

    import torch
    import torch.distributed as dist

    import hsort_inputs
    import paper_conf_ipps_gowanlockk18a_b200 as hs

    ws, rank, local = dist_env()
    if ws > 1:
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    else:
        torch.cuda.set_device(0)
    dev = torch.cuda.current_device()

    def barrier():
        if ws > 1:
            dist.barrier()

    def max_over_ranks(x: float) -> float:
        if ws == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    n = args.n
    hs.hsort_set_option("kernel_timing", 1)
    t0 = time.perf_counter()
    hs.hsort_init()
    t_init = time.perf_counter() - t0

    # inputs: pinned host A (generated in place), device copy for the resident arm
    A_h = torch.empty(n, dtype=torch.float64).pin_memory()
    hsort_inputs.generate("uniform", n, seed=SEED + rank, out=A_h.numpy())
    B_h = torch.empty(n, dtype=torch.float64).pin_memory()
    d_in = A_h.to(f"cuda:{dev}", non_blocking=False)
    d_out = torch.empty_like(d_in)
    stream = torch.cuda.current_stream()

    # ---- device-resident arm (value): one step = one GPUSort of the whole batch ----------------
    for _ in range(args.warmup):
        hs.hsort_sort_device(d_in, d_out, stream)
    torch.cuda.synchronize()
    # sampled correctness guard on the benchmarked output (full parity lives in tests/)
    o = d_out[:: max(1, n // (1 << 20))]
    assert bool((o[1:] >= o[:-1]).all()), "device output not sorted"

    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    pass_ms, hist_ms, other_ms = [], [], []
    n_active = 8
    sampler = ClockSampler(dev)
    barrier()
    torch.cuda.synchronize()
    with sampler:
        step_ms = []
        for _ in range(args.steps):
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
            other_ms.append(kt["scan"] + kt["copy"] + sum(kt["passes"][n_active:]))
    torch.cuda.synchronize()
    barrier()
    total_ms = max_over_ranks(sum(step_ms))
    # full-size guard on the last timed output (outside the timed region): every adjacent pair
    # ordered, and the same multiset as the input (two order-independent 64-bit sums of mixed
    # bit patterns, wrap-around).  The unique answer is pinned against the oracle in tests/.
    assert bool((d_out[1:] >= d_out[:-1]).all()), "device output not sorted"

    def multiset_sig(t):
        u = t.view(torch.int64)
        m = (u ^ (u >> 29)) * -7046029254386353131  # odd multiplier (splitmix64 style)
        return int(u.sum()), int((m ^ (m >> 32)).sum())
    assert multiset_sig(d_out) == multiset_sig(d_in), "device output is not a permutation of the input"
    ms_per_step = total_ms / args.steps
    value = ws * n * args.steps / (total_ms / 1e3)

    # roofline of the dominant kernel (k_onesweep): algorithmic 16 B/key per pass
    peak, peak_src = load_peaks()
    avg_pass_ms = statistics.mean(pass_ms) if pass_ms else float("nan")
    achieved = ALG_BYTES_PER_KEY_PASS * n / (avg_pass_ms / 1e3) / 1e9
    traffic, traffic_n = load_traffic()
    if traffic is not None and traffic_n and traffic_n != n:
        traffic = traffic * n / traffic_n
    share = sum(pass_ms) / sum(step_ms) if step_ms else None

    # ---- end-to-end arm (e2e): public API, pinned host buffers, HtoD + sort + DtoH ------------
    # link floor: the first output key depends on the last input key, so HtoD and DtoH of the
    # whole array serialise: T_floor = n*8/BW_h2d + n*8/BW_d2h (measured here, pinned copies)
    # per direction: the better of one copy stream and two concurrent half copies (the library's
    # RESIDENT DtoH keeps two copies in flight; tools/link_probe.py)
    bw = {}
    side = [torch.cuda.Stream(), torch.cuda.Stream()]
    for name, dst_t, src_t in (("h2d", d_out, A_h), ("d2h", B_h, d_in)):
        best = 0.0
        for ns in (1, 2):
            for _ in range(2):
                torch.cuda.synchronize()
                e_a, e_b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e_a.record()
                h = n // ns
                for i in range(ns):
                    side[i].wait_event(e_a)
                    with torch.cuda.stream(side[i]):
                        dst_t[i * h:(i + 1) * h].copy_(src_t[i * h:(i + 1) * h], non_blocking=True)
                for i in range(ns):
                    torch.cuda.current_stream().wait_stream(side[i])
                e_b.record()
                e_b.synchronize()
                best = max(best, n * 8 / (e_a.elapsed_time(e_b) / 1e3))
        bw[name] = best
    link_floor_s = n * 8 / bw["h2d"] + n * 8 / bw["d2h"]
    e2e_steps = args.e2e_steps or max(3, min(args.steps, 5))
    hs.hsort_sort(A_h, B_h, batch_elems=0, n_gpus=1)  # warm (buffers cached)
    barrier()
    e2e_t = []
    for _ in range(e2e_steps):
        t = time.perf_counter()
        hs.hsort_sort(A_h, B_h, batch_elems=0, n_gpus=1)
        e2e_t.append(time.perf_counter() - t)
    st = hs.hsort_get_stats()
    Bv = B_h.numpy()[:: max(1, n // (1 << 20))]
    assert bool((Bv[1:] >= Bv[:-1]).all()), "host output not sorted"
    barrier()
    e2e_total = max_over_ranks(sum(e2e_t))
    e2e_value = ws * n * e2e_steps / e2e_total

    stages = stage_rooflines(hs, torch, d_in, d_out, n, peak, statistics.mean(hist_ms), avg_pass_ms,
                             stream)

    line = {
        "metric": METRIC,
        "value": value,
        "unit": "keys/s",
        "n_gpus": ws,
        "steps": args.steps,
        "warmup": args.warmup,
        "ms_per_step": ms_per_step,
        "higher_is_better": True,
        "scaling": "weak",
        "vs_baseline": None,
        "dtype": "f64",
        "data": "synthetic",
        "config": {
            "workload": WORKLOAD,
            "n": n,
            "batch_elems": n,
            "distribution": f"uniform U[0,1) 53-bit, splitmix64 seed {SEED}+rank",
            "parallelism": f"independent batches, {ws} rank(s) x 1 GPU",
            "l2": "input 8 GiB >> 126 MB L2: no flush needed between steps",
        },
        "roofline": {
            "kernel": "k_onesweep (one 8-bit LSD digit pass)",
            "bound": "hbm",
            "achieved": achieved,
            "peak": peak,
            "peak_source": peak_src,
            "unit": "GB/s",
            "frac": achieved / peak,
            "traffic": traffic,
            "alg_bytes_per_launch": ALG_BYTES_PER_KEY_PASS * n,
            "avg_launch_ms": avg_pass_ms,
            "launches_per_step": n_active,
            "share_of_step": share,
            "hist_ms": statistics.mean(hist_ms) if hist_ms else None,
            "dominant_digit_elision": plan,
        },
        "e2e": {
            "value": e2e_value,
            "unit": "keys/s",
            "h2d_bytes_per_step": n * 8,
            "d2h_bytes_per_step": n * 8,
            "api": "hsort_sort(A pinned, B pinned, n, batch_elems=0 (auto plan), n_gpus=1)",
            "ms_per_step": 1e3 * e2e_total / e2e_steps,
            "mode": st["mode_name"], "n_b": st["n_b"], "b_s": st["b_s"],
            "t_h2d_s": st["t_h2d"], "t_gpu_sort_s": st["t_gpu_sort"], "t_d2h_s": st["t_d2h"],
            "t_merge_gpu_s": st["t_merge_gpu"],
            "link_gbs": {"h2d": bw["h2d"] / 1e9, "d2h": bw["d2h"] / 1e9},
            "link_floor_ms": 1e3 * link_floor_s,
            "link_frac": link_floor_s / (e2e_total / e2e_steps),
            "step_ms": [round(1e3 * t, 2) for t in e2e_t],  # this rank's steps (value uses the sum)
        },
        "stages": stages,
        # per step: K1, K2, 8 pass launches (inactive ones return at once), final copy; with the
        # elision: K1, K2, the active passes, final copy, the outlier sort (11), the placement
        "gpu_launches": args.steps * ((n_active + 15) if plan["elided"] else 11),
        "clocks": sampler.summary(),
        "init_s": t_init,
    }
    if rank == 0 and ws == 1 and not args.no_cpu_baseline:
        line["cpu_baseline"] = cpu_baseline_oracle(ORACLE_SAMPLE)
        par = cpu_parallel_baseline(PAR_SAMPLE)
        par["e2e_speedup"] = e2e_value / par["value"]  # our host->host rate / parallel CPU rate
        line["cpu_parallel_baseline"] = par
    if rank == 0:
        print(json.dumps(line), flush=True)
    hs.hsort_finalize()
    if ws > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())

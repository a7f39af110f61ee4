"""Run BASELINE.json configs (scaled to the GPU box's 197 GB host RAM) through the public API.

C1: 2^20 uniform, one batch: bit-exact vs the oracle.
C3s: the paper's out-of-core workflow (STREAM: batches -> W -> CPU/GPU merge) with 2 GB batches
     (b_s = 2.5e8), pageable A/B, n = N3 (default 4e9 = 32 GB).
C4s: normal and zipf-dup skew, auto plan, n = N4.
C5s: fixed n = N5, sweep b_s and the merge split f in STREAM mode; reports end-to-end time next to
     the "GPU-only" sum (sum HtoD + sum DtoH + sum GPUSort) the paper criticises.
C6p: PIPEMERGE on/off in STREAM mode at n = N6 over several b_s, CPU-only merge and A12 split.
Large outputs are verified by sortedness + multiset hash (oracle verifiers; unique answer, A-4).
Prints one JSON line per run.
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402

import hsort_inputs  # noqa: E402
import oracle  # noqa: E402
import paper_conf_ipps_gowanlockk18a_b200 as hs  # noqa: E402


def emit(**kw):
    print(json.dumps(kw), flush=True)


def verify(A, B, full=False):
    if full:
        return bool(np.array_equal(oracle.sort_f64(A).view(np.uint64), B.view(np.uint64)))
    srt = bool(np.all(B[1:] >= B[:-1])) if not np.isnan(B[:: 1 << 16]).any() else oracle.is_sorted_f64(B)
    return srt and oracle.multiset_hash(A) == oracle.multiset_hash(B)


def run(label, A, B, batch, opts, full=False, reps=2):
    """min over reps calls (the first STREAM call of a size pays the one-off W allocation, which
    is reported as t_host_alloc of that call)"""
    old = {k: hs.hsort_get_option(k) for k in opts}
    for k, v in opts.items():
        hs.hsort_set_option(k, v)
    try:
        ts = []
        for _ in range(reps):
            t = time.perf_counter()
            hs.hsort_sort(A, B, batch_elems=batch)
            ts.append(time.perf_counter() - t)
        st = hs.hsort_get_stats()
    finally:
        for k, v in old.items():
            hs.hsort_set_option(k, v)
    ok = verify(A, B, full)
    gpu_only = st["t_h2d"] + st["t_d2h"] + st["t_gpu_sort"]
    emit(config=label, n=int(A.size), batch=batch, opts=opts, seconds=min(ts),
         keys_per_s=A.size / min(ts), verified=ok, gpu_only_s=gpu_only,
         e2e_over_gpu_only=min(ts) / gpu_only if gpu_only else None,
         **{k: (round(v, 5) if isinstance(v, float) else v) for k, v in st.items() if k != "n"})


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n3", type=float, default=4.3e9)
    ap.add_argument("--n4", type=float, default=4e9)
    ap.add_argument("--n5", type=float, default=2e9)
    ap.add_argument("--n6", type=float, default=2e9)
    ap.add_argument("--only", default="C1,C3s,C4s,C5s,C6p")
    a = ap.parse_args()
    which = set(a.only.split(","))
    hs.hsort_init()
    if "C1" in which:
        A = hsort_inputs.generate("uniform", 1 << 20, seed=1)
        B = np.empty_like(A)
        run("C1", A, B, 0, {}, full=True, reps=3)
    if "C3s" in which:
        n = int(a.n3)
        A = hsort_inputs.generate("uniform", n, seed=3)
        B = np.empty_like(A)
        run("C3s-stream-2GB-batches", A, B, 250_000_000, {"resident": 0})
        run("C3s-auto", A, B, 0, {})
        del A, B
    if "C4s" in which:
        n = int(a.n4)
        for dist, seed in (("normal", 4), ("zipf_dup", 5)):
            A = hsort_inputs.generate(dist, n, seed=seed)
            B = np.empty_like(A)
            run(f"C4s-{dist}-auto", A, B, 0, {})
            del A, B
    if "C5s" in which:
        n = int(a.n5)
        A = hsort_inputs.generate("uniform", n, seed=6)
        B = np.empty_like(A)
        for b in (1 << 26, 1 << 27, 1 << 28, 1 << 29):
            for pm in (0, 250, 500, 750, 1000, -1):
                run("C5s-sweep", A, B, b, {"resident": 0, "merge_gpu_permille": pm})
        run("C5s-auto", A, B, 0, {})
        del A, B
    if "C6p" in which:
        # PIPEMERGE ablation (S§8(f) #1, Fig. 6): pair-wise merges during the sort
        # phase on/off, with the paper's CPU-only merge (f = 0) and with the A12 split
        n = int(a.n6)
        A = hsort_inputs.generate("uniform", n, seed=7)
        B = np.empty_like(A)
        for b in (1 << 26, 1 << 27, 250_000_000):
            for pm in (0, 1):
                for f in (0, -1):
                    run("C6p-pipemerge", A, B, b, {"resident": 0, "pipemerge": pm, "merge_gpu_permille": f,
                                                   "pin_w_max_mb": 24576}, reps=2)
    hs.hsort_finalize()


if __name__ == "__main__":
    main()

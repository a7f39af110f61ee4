"""Host-native components of the product library against the oracle (CPU, no GPU needed).

H2 CPU multiway merge + co-rank (§III-A), PARMEMCPY, the planner
(Table I) and the PIPEMERGE count (Fig. 3).
"""
import os

import numpy as np
import pytest

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _runs(rng, k, maxlen, hi=2**64, allow_empty=True):
    runs = []
    for _ in range(k):
        m = int(rng.integers(0 if allow_empty else 1, maxlen + 1))
        runs.append(np.sort(rng.integers(0, hi, size=m, dtype=np.uint64)))
    return runs


def _pack(runs):
    off = np.zeros(len(runs) + 1, dtype=np.uint64)
    for j, r in enumerate(runs):
        off[j + 1] = off[j] + r.size
    keys = np.concatenate(runs) if runs else np.zeros(0, np.uint64)
    return np.ascontiguousarray(keys, dtype=np.uint64), off


@pytest.mark.parametrize("k", [1, 2, 3, 5, 16, 64, 130])
@pytest.mark.parametrize("hi", [2**64, 1000, 3])
def test_host_merge_equals_oracle(hs, oracle_mod, k, hi):
    rng = np.random.default_rng(k * 7 + (hi % 97))
    runs = _runs(rng, k, 40000 if k < 20 else 3000, hi)
    keys, off = _pack(runs)
    got = hs.hsort_host_merge(keys, off, out_f64=False, threads=8)
    assert np.array_equal(got, oracle_mod.merge_runs(runs))


def test_host_merge_inverse_transform_on_store(hs, oracle_mod, inputs_mod):
    A = inputs_mod.generate("special", 300_000, seed=3)
    K = oracle_mod.keys_from_f64(A)
    parts = np.array_split(K, 7)
    runs = [oracle_mod.sort_u64(p) for p in parts]
    keys, off = _pack(runs)
    got = hs.hsort_host_merge(keys, off, out_f64=True, threads=8)
    want = oracle_mod.sort_f64(A)
    assert np.array_equal(got.view(np.uint64), want.view(np.uint64))


def test_host_merge_offset_base_and_single_thread(hs, oracle_mod):
    rng = np.random.default_rng(1)
    runs = _runs(rng, 9, 5000, 50)
    keys, off = _pack(runs)
    pad = np.concatenate([np.full(13, 7, np.uint64), keys])
    off2 = off + np.uint64(13)
    got = hs.hsort_host_merge(pad, off2, threads=1)
    assert np.array_equal(got, oracle_mod.merge_runs(runs))


@pytest.mark.parametrize("k", [1, 2, 7, 40])
def test_host_corank_equals_oracle(hs, oracle_mod, k):
    rng = np.random.default_rng(100 + k)
    for hi in (2**64, 20):
        runs = _runs(rng, k, 200, hi)
        keys, off = _pack(runs)
        n = int(off[-1])
        for o in sorted({0, 1, n // 3, n // 2, max(n - 1, 0), n}):
            assert np.array_equal(hs.hsort_host_corank(keys, off, o), oracle_mod.corank(runs, o))


def test_par_memcpy(hs):
    rng = np.random.default_rng(0)
    src = rng.integers(0, 255, size=(64 << 20) + 77, dtype=np.uint8)
    for t in (1, 3, 8):
        dst = np.zeros_like(src)
        hs.hsort_par_memcpy(dst, src, threads=t)
        assert np.array_equal(dst, src)


def test_pipemerge_count_matches_fig3_golden(hs):
    rows = [l.split() for l in open(os.path.join(GOLDEN, "fig3_pipemerge.txt"))
            if l.strip() and not l.startswith("#")]
    for n_b, n_gpu, merges, final_lists in rows:
        assert hs.hsort_pipemerge_count(int(n_b), int(n_gpu)) == int(merges)
    for n_b in range(0, 50):
        for g in (1, 2, 4, 8):
            assert hs.hsort_pipemerge_count(n_b, g) <= max(0, (n_b - 1) // 2) if n_b else True


def test_planner_table1_identities(hs):
    rows = [l.split() for l in open(os.path.join(GOLDEN, "table1_identities.txt"))
            if l.strip() and not l.startswith("#")]
    old = hs.hsort_get_option("n_s")
    # the paper's streamed pipeline (runs through W): the multi-GPU RESIDENT plan would keep the
    # 2-GPU rows resident instead
    hs.hsort_set_option("resident", 0)
    try:
        for n, b_s, n_s, n_gpu, n_b, per_stream, gpu_bytes in rows:
            hs.hsort_set_option("n_s", int(n_s))
            # a GPU exactly as large as the paper's (16 GiB / 12 GiB)
            dev = 16 << 30 if int(b_s) == 500000000 else 12 << 30
            p = hs.hsort_plan(int(n), int(b_s), int(n_gpu), dev)
            assert p["b_s"] == int(b_s)
            assert p["n_b"] == int(n_b) == -(-int(n) // int(b_s))
            assert abs(p["batches_per_stream"] - float(per_stream)) < 1e-9
            if p["mode_name"] == "STREAM":
                # B200 design shares one alt buffer: (n_s + 1) b_s keys <= paper's 2 b_s n_s
                assert p["device_bytes_per_gpu"] <= int(gpu_bytes) + int(b_s)
    finally:
        hs.hsort_set_option("n_s", old)
        hs.hsort_set_option("resident", -1)


def test_planner_modes_and_ragged_batches(hs):
    G = 180 << 30
    # auto plan: pipelined RESIDENT schedule (b_s = 2^27 batches + halving tail)
    p = hs.hsort_plan(1 << 30, 0, 1, G)
    assert p["mode_name"] == "RESIDENT" and p["schedule"] == 1 and p["b_s"] == 1 << 27
    assert p["n_b"] == 12 and p["last_batch"] == 1 << 23
    p = hs.hsort_plan(10**9 + 7, 0, 1, G)
    assert p["mode_name"] == "RESIDENT" and p["schedule"] == 1 and p["n_b"] <= 1024
    assert p["last_batch"] <= (10**9 + 7) // 128
    hs.hsort_set_option("auto_pipeline_min", 0)
    try:
        p = hs.hsort_plan(1 << 30, 0, 1, G)  # the paper's auto rule: one batch if it fits
        assert p["mode_name"] == "BLINE" and p["n_b"] == 1 and p["b_s"] == 1 << 30
    finally:
        hs.hsort_set_option("auto_pipeline_min", 1 << 24)
    p = hs.hsort_plan((1 << 24) - 1, 0, 1, G)  # below the threshold: BLINE
    assert p["mode_name"] == "BLINE"
    p = hs.hsort_plan(10**9 + 7, 250_000_000, 1, G)
    assert p["n_b"] == 5 and p["last_batch"] == 7 and p["mode_name"] == "RESIDENT"
    p = hs.hsort_plan(3 * 10**10, 250_000_000, 1, G)  # 240 GB: runs cannot stay in HBM
    assert p["n_b"] == 120 and p["mode_name"] == "STREAM"
    p = hs.hsort_plan(3 * 10**10, 0, 1, G)  # auto b_s fills HBM with n_s + 1 buffers
    assert p["mode_name"] == "STREAM" and p["b_s"] % 4096 == 0
    assert p["device_bytes_per_gpu"] <= G
    p = hs.hsort_plan(10**9, 10**8, 4, G)  # multi-GPU RESIDENT: 4 tile-aligned shards of 1e8-key batches
    assert p["mode_name"] == "RESIDENT" and p["n_gpus"] == 4 and p["n_b"] == 12
    hs.hsort_set_option("resident", 0)
    try:
        assert hs.hsort_plan(10**9, 10**8, 1, G)["mode_name"] == "STREAM"
        p = hs.hsort_plan(10**9, 10**8, 4, G)
        assert p["mode_name"] == "STREAM" and p["n_gpus"] == 4 and p["n_b"] == 10
    finally:
        hs.hsort_set_option("resident", -1)


@pytest.mark.parametrize("N", [2, 4, 8])
def test_planner_multi_gpu_resident(hs, N):
    """A1 for n_gpus = N > 1: whenever N shards fit in N x HBM the plan is the
    multi-GPU RESIDENT one -- every GPU sorts its shard as resident batches and merges one range of
    B -- and asking for more GPUs never falls back to one GPU."""
    G = 180 << 30
    p = hs.hsort_plan(1 << 30, 0, N, G)
    assert p["mode_name"] == "RESIDENT" and p["n_gpus"] == N and p["schedule"] == 1
    assert p["n_b"] % N == 0 and p["n_b"] <= 1024  # equal shards, equal schedules
    assert abs(p["batches_per_stream"] - p["n_b"] / N) < 1e-9
    assert p["device_bytes_per_gpu"] < (1 << 30) * 8 // N + (3 << 30)
    p = hs.hsort_plan(3 * 10**10, 0, N, G)  # 240 GB over N x 180 GB
    if N >= 2 and 3 * 10**10 * 8 / N < G - (6 << 30):
        assert p["mode_name"] == "RESIDENT" and p["n_gpus"] == N
    p = hs.hsort_plan(1 << 20, 0, N, G)  # small: one GPU, one batch
    assert p["mode_name"] == "BLINE" and p["n_gpus"] == 1
    p = hs.hsort_plan(10**12, 0, N, G)  # 8 TB: streamed through W on all N GPUs
    assert p["mode_name"] == "STREAM" and p["n_gpus"] == N and p["b_s"] <= 1 << 30


def test_options_validation(hs):
    with pytest.raises(hs.HsortError):
        hs.hsort_set_option("no_such_option", 1)
    with pytest.raises(hs.HsortError):
        hs.hsort_set_option("resident", 5)
    with pytest.raises(hs.HsortError):
        hs.hsort_set_option("n_s", 0)


def test_sort_without_init_fails_cleanly(hs):
    A = np.zeros(10)
    with pytest.raises(hs.HsortError) as e:
        hs.hsort_sort(A)
    assert e.value.code == -2


def test_par_memcpy_streaming_stores(hs):
    """PARMEMCPY with non-temporal stores (option memcpy_nt): unaligned heads/tails, all sizes."""
    rng = np.random.default_rng(0)
    src = rng.integers(0, 256, size=(9 << 20) + 100, dtype=np.uint8)
    for nt in (1, 0):
        hs.hsort_set_option("memcpy_nt", nt)
        for size, so, do in ((0, 0, 0), (5, 1, 3), ((2 << 20) + 3, 7, 1), ((8 << 20) + 17, 3, 9)):
            dst = np.zeros(size + 16, dtype=np.uint8)
            hs.hsort_par_memcpy(dst[do:do + size], src[so:so + size], 4)
            assert np.array_equal(dst[do:do + size], src[so:so + size]), (nt, size, so, do)
            assert not dst[:do].any() and not dst[do + size:].any()
    hs.hsort_set_option("memcpy_nt", 1)


def test_splitter_arithmetic(hs):
    """A13 splitter arithmetic in the library: regular sample positions of a sorted run and the
    P-quantile splitters of the merged samples (used by dist.exchange_sorted_runs)."""
    for n, s in ((1, 5), (10, 3), (10**9 + 7, 64), (7, 7)):
        pos = hs.hsort_sample_positions(n, s)
        assert pos.size == s and int(pos.max()) <= n - 1
        assert np.all(np.diff(pos.astype(np.int64)) >= 0)  # non-decreasing
        if n > s:
            assert np.all(np.diff(pos.astype(np.int64)) > 0)  # distinct when the run is long enough
    samp = np.sort(np.random.default_rng(0).integers(0, 2**64, size=1000, dtype=np.uint64))
    for P in (1, 2, 3, 8):
        spl = hs.hsort_select_splitters(samp, P)
        assert spl.size == P - 1 and np.all(np.diff(spl.astype(np.float64)) >= 0)
        # each rank's share of the samples is within one sample of m / P
        cuts = [0] + [int(np.searchsorted(samp, v, side="right")) for v in spl] + [samp.size]
        assert all(abs((cuts[r + 1] - cuts[r]) - samp.size / P) <= 1 for r in range(P))
    assert np.array_equal(hs.hsort_select_splitters(np.zeros(0, np.uint64), 4), np.zeros(3, np.uint64))
    with pytest.raises(hs.HsortError):
        hs.hsort_sample_positions(0, 3)

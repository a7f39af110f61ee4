"""GPU parity of the multi-GPU method inside the C ABI, on virtual GPUs.

Option "virtual_gpus" = V maps V GPU contexts (own streams, pinned rings, radix scratch, runs)
round-robin onto the visible devices, so on a one-GPU pool every multi-GPU code path runs:
  * RESIDENT over N GPUs: A cut into N shards, each sorted as resident batches on its GPU; B cut
    into N ranges, each merged by its GPU from ALL runs through the run-pointer table (K4/K5 peer
    loads: the splitter exchange fused into the merge) and DMA'd to B[o_g, o_{g+1});
  * STREAM over N GPUs: one uploader/downloader pair per GPU on a shared batch queue, and the A12
    GPU merge share cut across all N GPUs.
Every output is compared bit-exactly with the oracle (oracle.sort_f64, serial std::sort under IEEE
totalOrder).  Paper: n_b/(n_s n_GPU) batches per stream, merging on the GPUs.
"""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu

V = 4


def _bits(a):
    return np.ascontiguousarray(a).view(np.uint64)


def _pinned(a):
    import torch
    return torch.from_numpy(a).pin_memory()


@pytest.fixture(scope="module")
def hv(hs_gpu):
    """The library re-initialised with V virtual GPU contexts on the visible device(s)."""
    hs_gpu.hsort_finalize()
    hs_gpu.hsort_set_option("virtual_gpus", V)
    hs_gpu.hsort_init()
    yield hs_gpu
    hs_gpu.hsort_finalize()
    hs_gpu.hsort_set_option("virtual_gpus", 0)
    hs_gpu.hsort_init()


def _with(hs, opts, fn):
    old = {k: hs.hsort_get_option(k) for k in opts}
    for k, v in opts.items():
        hs.hsort_set_option(k, v)
    try:
        return fn()
    finally:
        for k, v in old.items():
            hs.hsort_set_option(k, v)


def _runs_expected(n, N, b):
    """Run count of the multi-GPU RESIDENT plan: tile-aligned shards, uniform b-key batches."""
    sh = [0] + [(n * g // N) - (n * g // N) % 4096 for g in range(1, N)] + [n]
    for g in range(1, N):
        sh[g] = max(sh[g], sh[g - 1])
    return sum(-(-(sh[g + 1] - sh[g]) // b) for g in range(N))


@pytest.mark.parametrize("N", [2, 3, 4])
@pytest.mark.parametrize("dist", ["uniform", "zipf_dup", "special", "all_equal", "normal"])
def test_multi_resident_explicit_batches(hv, oracle_mod, inputs_mod, N, dist):
    n = 1_000_003
    b = 100_000
    A = inputs_mod.generate(dist, n, seed=N * 10 + len(dist))
    want = _bits(oracle_mod.sort_f64(A))
    B = _with(hv, {"merge_chunk": 1 << 17}, lambda: hv.hsort_sort(A, batch_elems=b, n_gpus=N))
    st = hv.hsort_get_stats()
    assert st["mode_name"] == "RESIDENT" and st["n_gpus"] == N
    assert st["n_b"] == _runs_expected(n, N, b)
    assert np.array_equal(_bits(B), want), (N, dist)


@pytest.mark.parametrize("N", [2, 4])
@pytest.mark.parametrize("dist", ["uniform", "zipf_dup", "special"])
def test_multi_resident_auto_plan_pinned(hv, oracle_mod, inputs_mod, N, dist):
    """The auto plan (batch_elems = 0) over N GPUs: per shard 2^27-capped batches + halving tail;
    pinned A/B are DMA'd directly; several merge chunks per GPU range."""
    n = 3_000_017
    A = inputs_mod.generate(dist, n, seed=N + 5)
    want = _bits(oracle_mod.sort_f64(A))
    At, Bt = _pinned(A.copy()), _pinned(np.zeros_like(A))
    opts = {"auto_pipeline_min": 1 << 20, "merge_chunk": 1 << 18}
    _with(hv, opts, lambda: hv.hsort_sort(At, Bt, batch_elems=0, n_gpus=N))
    st = hv.hsort_get_stats()
    assert st["mode_name"] == "RESIDENT" and st["n_gpus"] == N and st["n_b"] >= 2 * N
    assert st["direct_in"] == 1 and st["direct_out"] == 1
    assert np.array_equal(_bits(Bt.numpy()), want), (N, dist)
    B = _with(hv, opts, lambda: hv.hsort_sort(A, batch_elems=0, n_gpus=N))  # pageable: staged
    assert np.array_equal(_bits(B), want)


def test_multi_resident_all_visible_and_in_place(hv, oracle_mod, inputs_mod):
    """n_gpus = 0 -> every context (V); in-place B == A; raw uint64 keys."""
    A = inputs_mod.generate("salted", 777_777, seed=3)
    want = _bits(oracle_mod.sort_f64(A))
    X = A.copy()
    hv.hsort_sort(X, X, batch_elems=65_536, n_gpus=0)
    assert hv.hsort_get_stats()["n_gpus"] == V
    assert np.array_equal(_bits(X), want)
    K = np.random.default_rng(9).integers(0, 2**64, size=600_000, dtype=np.uint64)
    assert np.array_equal(hv.hsort_sort_u64(K, batch_elems=50_000, n_gpus=3), oracle_mod.sort_u64(K))


@pytest.mark.parametrize("n,b", [(5000, 1000), (4097, 4096), (12_289, 4096), (1, 1)])
def test_multi_resident_tiny_and_empty_shards(hv, oracle_mod, inputs_mod, n, b):
    """Shards are tile-aligned: small n leaves some GPUs without runs and some ranges empty."""
    A = inputs_mod.generate("special", n, seed=n)
    want = _bits(oracle_mod.sort_f64(A))
    B = hv.hsort_sort(A, batch_elems=b, n_gpus=4)
    assert np.array_equal(_bits(B), want)


@pytest.mark.parametrize("N", [2, 3])
@pytest.mark.parametrize("permille", [0, 500, -1, 1000])
def test_multi_stream_merge_split(hv, oracle_mod, inputs_mod, N, permille):
    """STREAM over N GPUs (shared batch queue) and the A12 merge share spread over the N GPUs."""
    n = 2_000_003
    A = inputs_mod.generate("zipf_dup" if permille % 2 else "normal", n, seed=N * 1000 + permille)
    want = _bits(oracle_mod.sort_f64(A))
    opts = {"resident": 0, "merge_gpu_permille": permille, "merge_chunk": 1 << 18}
    for pinned in (False, True):
        if pinned:
            Bt = _pinned(np.zeros_like(A))
            _with(hv, opts, lambda: hv.hsort_sort(_pinned(A.copy()), Bt, batch_elems=150_000, n_gpus=N))
            B = Bt.numpy()
        else:
            B = _with(hv, opts, lambda: hv.hsort_sort(A, batch_elems=150_000, n_gpus=N))
        st = hv.hsort_get_stats()
        assert st["mode_name"] == "STREAM" and st["n_gpus"] == N and st["n_b"] == -(-n // 150_000)
        assert np.array_equal(_bits(B), want), (N, permille, pinned)
        if permille >= 0:
            assert abs(st["merge_gpu_fraction"] - permille / 1000) < 1e-3


def test_multi_stream_pipemerge(hv, oracle_mod, inputs_mod):
    """PIPEMERGE with n_GPU = 3: hsort_pipemerge_count(n_b, 3) pair merges (reading A-9)."""
    n, b = 12 * 65_536 + 17, 65_536
    A = inputs_mod.generate("uniform", n, seed=41)
    want = _bits(oracle_mod.sort_f64(A))
    n_b = -(-n // b)
    opts = {"resident": 0, "pipemerge": 1, "merge_gpu_permille": 300}
    B = _with(hv, opts, lambda: hv.hsort_sort(A, batch_elems=b, n_gpus=3))
    st = hv.hsort_get_stats()
    assert np.array_equal(_bits(B), want)
    assert st["pipe_merges"] == oracle_mod.pipemerge_count(n_b, 3)


def test_multi_device_entry_points_still_work(hv, oracle_mod, inputs_mod):
    """Device entry points use the first context of the current device."""
    import torch
    A = inputs_mod.generate("uniform", 300_000, seed=2)
    d = torch.from_numpy(A).cuda()
    o = torch.empty_like(d)
    hv.hsort_sort_device(d, o)
    torch.cuda.synchronize()
    assert np.array_equal(_bits(o.cpu().numpy()), _bits(oracle_mod.sort_f64(A)))


# ---- N2: MSD-first split (option "msd", S§8(f) #2) ------------------------------------------------
MSD_DISTS = ["uniform", "zipf_dup", "special", "all_equal", "normal", "sorted", "few_distinct"]


@pytest.mark.parametrize("N", [1, 2, 3, 4])
@pytest.mark.parametrize("dist", MSD_DISTS)
def test_msd_split_matches_oracle(hv, oracle_mod, inputs_mod, N, dist):
    """Sampled splitters -> per-batch bucket partition (K6a-c) -> bucket gather from every GPU
    (K6d, peer loads) -> one LSD sort per bucket -> DtoH to B[sum of earlier buckets].  No merge.
    Heavy duplicates / all-equal keys put whole equal-key groups in one bucket."""
    n = 2_000_003
    A = inputs_mod.generate(dist, n, seed=N * 100 + len(dist))
    want = _bits(oracle_mod.sort_f64(A))
    opts = {"msd": 1, "msd_bucket_keys": 1 << 16, "auto_pipeline_min": 1 << 20}
    B = _with(hv, opts, lambda: hv.hsort_sort(A, batch_elems=0, n_gpus=N))
    st = hv.hsort_get_stats()
    assert st["mode_name"] == "RESIDENT" and st["n_gpus"] == N and st["msd_buckets"] >= 4 * N
    assert np.array_equal(_bits(B), want), (N, dist)


@pytest.mark.parametrize("N", [1, 3])
def test_msd_split_pinned_explicit_batches_u64(hv, oracle_mod, inputs_mod, N):
    A = inputs_mod.generate("salted", 1_500_001, seed=N)
    want = _bits(oracle_mod.sort_f64(A))
    opts = {"msd": 1, "msd_bucket_keys": 1 << 17}
    At, Bt = _pinned(A.copy()), _pinned(np.zeros_like(A))
    _with(hv, opts, lambda: hv.hsort_sort(At, Bt, batch_elems=200_000, n_gpus=N))
    st = hv.hsort_get_stats()
    assert st["msd_buckets"] > 0 and st["direct_in"] == 1 and st["direct_out"] == 1
    assert np.array_equal(_bits(Bt.numpy()), want)
    K = np.random.default_rng(N).integers(0, 2**64, size=700_001, dtype=np.uint64)
    got = _with(hv, opts, lambda: hv.hsort_sort_u64(K, batch_elems=100_000, n_gpus=N))
    assert np.array_equal(got, oracle_mod.sort_u64(K))


@pytest.mark.parametrize("n,b", [(5000, 1000), (12_289, 4096), (70_001, 8192)])
def test_msd_split_tiny(hv, oracle_mod, inputs_mod, n, b):
    A = inputs_mod.generate("special", n, seed=n)
    want = _bits(oracle_mod.sort_f64(A))
    B = _with(hv, {"msd": 1}, lambda: hv.hsort_sort(A, batch_elems=b, n_gpus=4))
    assert np.array_equal(_bits(B), want)


@pytest.mark.parametrize("N", [2, 3])
@pytest.mark.parametrize("dist", ["few_distinct", "uniform", "zipf_dup"])
def test_multi_pairs_resident(hv, oracle_mod, inputs_mod, N, dist):
    """Key/value RESIDENT plan over N GPUs: per-GPU stable batch sorts, then each GPU merges its
    range of B/VB from all GPUs' key and value runs (two run-pointer tables)."""
    n = 900_001
    A = inputs_mod.generate(dist, n, seed=N + len(dist))
    V = np.arange(n, dtype=np.uint64)[::-1].copy()
    wantB, wantV = oracle_mod.sort_pairs_f64(A, V)
    B, VB = _with(hv, {"merge_chunk": 1 << 17}, lambda: hv.hsort_sort_pairs_ex(A, V, batch_elems=65_536, n_gpus=N))
    st = hv.hsort_get_stats()
    assert st["mode_name"] == "RESIDENT" and st["n_gpus"] == N
    assert np.array_equal(_bits(B), _bits(wantB)) and np.array_equal(VB, wantV)


# ---- lanes: concurrent sorts on one GPU (hsort_sort_lane) -------------------------------------------
def test_lanes_concurrent_sorts(hv, oracle_mod, inputs_mod):
    """Two host threads sort different arrays at the same time on lanes 0 and 1 (two GPU contexts
    of the same device): every output bit-exact; a regular call meanwhile gets HSORT_ERR_BUSY."""
    import threading
    arrays = [inputs_mod.generate(d, 1_500_001 + i, seed=i) for i, d in enumerate(["uniform", "zipf_dup"])]
    wants = [_bits(oracle_mod.sort_f64(a)) for a in arrays]
    errors, busy_seen = [], []
    start = threading.Barrier(2)

    def worker(lane):
        try:
            start.wait()
            for rep in range(4):
                B = hv.hsort_sort_lane(lane, arrays[lane], batch_elems=200_000 if rep % 2 else 0)
                if not np.array_equal(_bits(B), wants[lane]):
                    errors.append((lane, rep))
                st = hv.hsort_get_stats()
                if st["n"] != arrays[lane].size:  # per-thread stats
                    errors.append(("stats", lane))
        except Exception as e:  # noqa: BLE001
            errors.append(repr(e))

    th = [threading.Thread(target=worker, args=(l,)) for l in (0, 1)]
    for t in th:
        t.start()
    try:
        hv.hsort_sort(arrays[0])
    except hv.HsortError as e:
        busy_seen.append(e.code)
    for t in th:
        t.join()
    assert not errors, errors
    assert all(c == -7 for c in busy_seen)
    with pytest.raises(hv.HsortError):
        hv.hsort_sort_lane(99, arrays[0])
    with pytest.raises(hv.HsortError):  # a STREAM plan is not per lane
        _with(hv, {"resident": 0}, lambda: hv.hsort_sort_lane(0, arrays[0], batch_elems=100_000))

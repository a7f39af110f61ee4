"""GPU parity: K4 co-ranks, K5 merge, and the host->host hsort_sort in every mode vs the oracle."""
import os

import numpy as np
import pytest

pytestmark = pytest.mark.gpu


def _bits(a):
    return np.ascontiguousarray(a).view(np.uint64)


def _runs(rng, k, maxlen, hi=2**64):
    runs = [np.sort(rng.integers(0, hi, size=int(rng.integers(0, maxlen + 1)), dtype=np.uint64))
            for _ in range(k)]
    off = np.zeros(k + 1, dtype=np.uint64)
    for j, r in enumerate(runs):
        off[j + 1] = off[j] + r.size
    return runs, np.concatenate(runs), off


@pytest.mark.parametrize("k", [1, 2, 3, 8, 17, 24, 32, 33, 64, 100, 128, 300, 600])
@pytest.mark.parametrize("hi", [2**64, 50, 7])
def test_corank_matches_oracle(hs_gpu, oracle_mod, k, hi):
    import torch
    rng = np.random.default_rng(k + hi % 1000)
    runs, keys, off = _runs(rng, k, 3000 if k < 50 else 400, hi)
    total = int(off[-1])
    step = max(1, total // 37)
    nb = total // step + 2
    d_keys = torch.from_numpy(keys).cuda()
    d_r = torch.zeros(nb * k, dtype=torch.uint64, device="cuda")
    hs_gpu.hsort_device_corank(d_keys, off, step, nb, d_r)
    got = d_r.cpu().numpy().reshape(nb, k)
    for b in range(nb):
        o = min(b * step, total)
        assert np.array_equal(got[b], oracle_mod.corank(runs, o)), (b, o)


@pytest.mark.parametrize("k", [2, 5, 17, 24, 32, 33, 64, 128, 200])
@pytest.mark.parametrize("hi", [2**64, 7, 3000])
def test_corank_two_level_matches_oracle(hs_gpu, oracle_mod, k, hi):
    """>= 64 bounds: coarse co-ranks every 16 steps, fine ones from the coarse windows (ties at
    the coarse cuts with hi = 7 / 3000 exercise the galloping bounds)."""
    import torch
    rng = np.random.default_rng(k * 7 + hi % 991)
    runs, keys, off = _runs(rng, k, 4000 if k < 50 else 300, hi)
    total = int(off[-1])
    step = 64
    nb = total // step + 2
    d_keys = torch.from_numpy(keys).cuda()
    d_r = torch.zeros(nb * k, dtype=torch.uint64, device="cuda")
    hs_gpu.hsort_device_corank(d_keys, off, step, nb, d_r)
    got = d_r.cpu().numpy().reshape(nb, k)
    for b in list(range(0, nb, 7)) + [nb - 2, nb - 1]:
        o = min(b * step, total)
        assert np.array_equal(got[b], oracle_mod.corank(runs, o)), (b, o)


@pytest.mark.parametrize("k", [32, 48, 128])
@pytest.mark.parametrize("hi", [2**64, 7])
def test_corank_three_level_matches_oracle(hs_gpu, oracle_mod, k, hi):
    """k >= 32 with >= 1024 bounds: the coarse level is itself computed from a coarser one (three
    levels, merge.cu corank_levels), windows entered by galloping at every level."""
    import torch
    rng = np.random.default_rng(k * 11 + hi % 997)
    runs, keys, off = _runs(rng, k, 3000, hi)
    total = int(off[-1])
    step = 16
    nb = total // step + 2
    assert nb >= 1024
    d_keys = torch.from_numpy(keys).cuda()
    d_r = torch.zeros(nb * k, dtype=torch.uint64, device="cuda")
    hs_gpu.hsort_device_corank(d_keys, off, step, nb, d_r)
    got = d_r.cpu().numpy().reshape(nb, k)
    for b in list(range(0, nb, 97)) + list(range(1, 40)) + [nb - 2, nb - 1]:
        o = min(b * step, total)
        assert np.array_equal(got[b], oracle_mod.corank(runs, o)), (b, o)


@pytest.mark.parametrize("k", [1, 2, 5, 16, 120, 1024])
@pytest.mark.parametrize("hi", [2**64, 7])
def test_device_merge_matches_oracle(hs_gpu, oracle_mod, k, hi):
    import torch
    rng = np.random.default_rng(3 * k + hi % 100)
    runs, keys, off = _runs(rng, k, 20000 if k <= 16 else 300, hi)
    d_keys = torch.from_numpy(keys).cuda()
    d_out = torch.empty_like(d_keys)
    hs_gpu.hsort_device_merge(d_keys, off, d_out, False)
    assert np.array_equal(d_out.cpu().numpy(), oracle_mod.merge_runs(runs))


@pytest.mark.parametrize("k", [31, 32, 33, 511, 512, 513])
@pytest.mark.parametrize("misaligned", [False, True])
def test_device_merge_slice_table_paths(hs_gpu, oracle_mod, k, misaligned):
    """K5 slice-table scan: one warp (k <= 32) vs block scan in chunks of 512 runs; 16-byte
    vector store vs the scalar store of a misaligned output; tiles with many empty slices."""
    import torch
    rng = np.random.default_rng(k + 1000 * misaligned)
    runs, keys, off = _runs(rng, k, 9000 if k <= 33 else 60)
    d_keys = torch.from_numpy(keys).cuda()
    d_buf = torch.zeros(keys.size + 1, dtype=torch.uint64, device="cuda")
    d_out = d_buf[1:] if misaligned else d_buf[:-1]
    hs_gpu.hsort_device_merge(d_keys, off, d_out, False)
    assert np.array_equal(d_out.cpu().numpy(), oracle_mod.merge_runs(runs))


def test_device_merge_inverse_transform(hs_gpu, oracle_mod, inputs_mod):
    import torch
    A = inputs_mod.generate("special", 200_000, seed=12)
    K = oracle_mod.keys_from_f64(A)
    parts = [oracle_mod.sort_u64(p) for p in np.array_split(K, 9)]
    off = np.cumsum([0] + [p.size for p in parts]).astype(np.uint64)
    d_keys = torch.from_numpy(np.concatenate(parts)).cuda()
    d_out = torch.empty_like(d_keys)
    hs_gpu.hsort_device_merge(d_keys, off, d_out, True)
    assert np.array_equal(d_out.cpu().numpy(), _bits(oracle_mod.sort_f64(A)))


@pytest.mark.parametrize("hi", [2**64, 40])
def test_device_upper_bounds_match_host(hs_gpu, hi):
    import torch
    rng = np.random.default_rng(hi % 1000)
    keys = np.sort(rng.integers(0, hi, size=100_003, dtype=np.uint64))
    vals = rng.integers(0, hi, size=1000, dtype=np.uint64)
    vals[:3] = [0, 2**64 - 1, keys[500]]
    d_out = torch.empty(vals.size, dtype=torch.uint64, device="cuda")
    hs_gpu.hsort_device_upper_bounds(torch.from_numpy(keys).cuda(), torch.from_numpy(vals).cuda(), d_out)
    want = np.searchsorted(keys, vals, side="right").astype(np.uint64)
    assert np.array_equal(d_out.cpu().numpy(), want)
    assert np.array_equal(hs_gpu.hsort_host_upper_bounds(keys, vals), want)


def test_exchange_single_rank_cuda_path(hs_gpu, oracle_mod, inputs_mod):
    """dist.exchange_sorted_runs on one NCCL rank (the P == 1 path + device merge)."""
    import torch
    import torch.distributed as dist
    from paper_conf_ipps_gowanlockk18a_b200 import dist as hd
    A = inputs_mod.generate("salted", 100_000, seed=5)
    K = oracle_mod.sort_u64(oracle_mod.keys_from_f64(A))
    if not dist.is_initialized():
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ.setdefault("MASTER_PORT", "29581")
        dist.init_process_group("nccl", rank=0, world_size=1)
    try:
        out = hd.exchange_sorted_runs(torch.from_numpy(K).cuda(), out_f64=True)
        assert np.array_equal(out.view(torch.uint64).cpu().numpy(), _bits(oracle_mod.sort_f64(A)))
    finally:
        dist.destroy_process_group()


# ---- host -> host ------------------------------------------------------------------------------
def _pinned(a):
    import torch
    t = torch.from_numpy(a).pin_memory()
    return t


CASES = [
    # (n, batch_elems, resident option, pipeline option, expected mode)
    (1 << 20, 0, -1, 1, "BLINE"),
    (1_000_003, 150_000, -1, 1, "RESIDENT"),
    (1_000_003, 150_000, 0, 1, "STREAM"),
    (1_000_003, 150_000, 0, 0, "STREAM"),
    (777_777, 4096, -1, 1, "RESIDENT"),
    (300_001, 1, 0, 1, None),  # b_s = 1 -> n_b > 1024: STREAM with huge k on the CPU merge
]


@pytest.mark.parametrize("n,b,res,pipe,mode", CASES)
@pytest.mark.parametrize("pinned", [False, True])
def test_hsort_sort_modes(hs_gpu, oracle_mod, inputs_mod, n, b, res, pipe, mode, pinned):
    if b == 1 and n > 5000:
        n, b = 5000, 1
    A = inputs_mod.generate("salted", n, seed=n + b)
    want = _bits(oracle_mod.sort_f64(A))
    hs_gpu.hsort_set_option("resident", res)
    hs_gpu.hsort_set_option("pipeline", pipe)
    try:
        if pinned:
            At, Bt = _pinned(A.copy()), _pinned(np.zeros_like(A))
            hs_gpu.hsort_sort(At, Bt, batch_elems=b, n_gpus=1)
            B = Bt.numpy()
        else:
            B = hs_gpu.hsort_sort(A, batch_elems=b, n_gpus=1)
        st = hs_gpu.hsort_get_stats()
    finally:
        hs_gpu.hsort_set_option("resident", -1)
        hs_gpu.hsort_set_option("pipeline", 1)
    assert np.array_equal(_bits(B), want)
    if mode:
        assert st["mode_name"] == mode
    assert st["direct_in"] == int(pinned) and st["direct_out"] == int(pinned)
    assert st["n"] == n and st["n_b"] == -(-n // (b or n))


@pytest.mark.parametrize("dist", ["uniform", "normal", "zipf_dup", "special", "all_equal",
                                  "closed_form", "reverse"])
def test_hsort_sort_distributions(hs_gpu, oracle_mod, inputs_mod, dist):
    A = inputs_mod.generate(dist, 2_000_003, seed=77)
    want = _bits(oracle_mod.sort_f64(A))
    for b in (0, 300_000):
        assert np.array_equal(_bits(hs_gpu.hsort_sort(A, batch_elems=b)), want), (dist, b)


@pytest.mark.parametrize("dist", ["special", "zipf_dup", "uniform"])
def test_hsort_sort_auto_pipelined_schedule(hs_gpu, oracle_mod, inputs_mod, dist):
    """auto plan at n >= 2^24: RESIDENT with b_s batches + halving tail, GPU merge, chunked DtoH."""
    n = (1 << 24) + 12345
    A = inputs_mod.generate(dist, n, seed=31)
    want = _bits(oracle_mod.sort_f64(A))
    hs_gpu.hsort_set_option("merge_chunk", 1 << 20)  # several merge/DtoH chunks
    try:
        B = hs_gpu.hsort_sort(A)
        st = hs_gpu.hsort_get_stats()
        Bp = _pinned(np.zeros_like(A))
        hs_gpu.hsort_sort(_pinned(A.copy()), Bp)
    finally:
        hs_gpu.hsort_set_option("merge_chunk", 1 << 26)
    assert st["mode_name"] == "RESIDENT" and st["n_b"] > 8
    assert np.array_equal(_bits(B), want)
    assert np.array_equal(_bits(Bp.numpy()), want)


@pytest.mark.parametrize("permille", [0, 300, 1000, -1])
@pytest.mark.parametrize("pin_w", [1, 0])
def test_stream_merge_split(hs_gpu, oracle_mod, inputs_mod, permille, pin_w):
    """A12: STREAM mode with a GPU share f of the merge streamed from W (K4/K5) and the rest on
    the CPU loser trees; every split point must give the same bytes."""
    n = 3_000_017
    A = inputs_mod.generate("zipf_dup", n, seed=permille + 7)
    want = _bits(oracle_mod.sort_f64(A))
    opts = {"resident": 0, "merge_gpu_permille": permille, "pin_w": pin_w, "merge_chunk": 1 << 19}
    old = {k: hs_gpu.hsort_get_option(k) for k in opts}
    for k, v in opts.items():
        hs_gpu.hsort_set_option(k, v)
    try:
        for pinned in (False, True):
            if pinned:
                Bp = _pinned(np.zeros_like(A))
                hs_gpu.hsort_sort(_pinned(A.copy()), Bp, batch_elems=400_000)
                B = Bp.numpy()
            else:
                B = hs_gpu.hsort_sort(A, batch_elems=400_000)
            st = hs_gpu.hsort_get_stats()
            assert st["mode_name"] == "STREAM" and st["n_b"] == 8
            assert np.array_equal(_bits(B), want), (permille, pin_w, pinned)
            if permille >= 0:
                assert abs(st["merge_gpu_fraction"] - permille / 1000) < 1e-3
    finally:
        for k, v in old.items():
            hs_gpu.hsort_set_option(k, v)


def test_hsort_sort_in_place_and_u64(hs_gpu, oracle_mod, inputs_mod):
    A = inputs_mod.generate("special", 500_001, seed=4)
    want = _bits(oracle_mod.sort_f64(A))
    for b in (0, 100_000):
        X = A.copy()
        hs_gpu.hsort_sort(X, X, batch_elems=b)
        assert np.array_equal(_bits(X), want)
    K = np.random.default_rng(3).integers(0, 2**64, size=400_000, dtype=np.uint64)
    for b in (0, 64_000):
        assert np.array_equal(hs_gpu.hsort_sort_u64(K, batch_elems=b), oracle_mod.sort_u64(K))


def test_hsort_sort_edge_cases(hs_gpu, oracle_mod):
    hs_gpu.hsort_sort(np.zeros(0))
    for n in (1, 2, 3):
        A = np.array([np.nan, -0.0, 0.0][:n])
        assert np.array_equal(_bits(hs_gpu.hsort_sort(A)), _bits(oracle_mod.sort_f64(A)))
    with pytest.raises(hs_gpu.HsortError) as e:
        hs_gpu.hsort_sort(np.zeros(10), n_gpus=99)
    assert e.value.code == -1
    buf = np.zeros(20)
    rc = hs_gpu.lib().hsort_sort(buf.ctypes.data, buf.ctypes.data + 40, 10, 0, 1)  # partial overlap
    assert rc == -1
    with pytest.raises(hs_gpu.HsortError):
        hs_gpu.hsort_init()  # second init -> BUSY


def test_stats_fields(hs_gpu, inputs_mod):
    A = inputs_mod.generate("uniform", 1 << 22, seed=1)
    hs_gpu.hsort_sort(A, batch_elems=1 << 20)
    st = hs_gpu.hsort_get_stats()
    assert st["n_b"] == 4 and st["passes_run"] >= 1
    assert st["bytes_h2d"] == A.nbytes and st["bytes_d2h"] == A.nbytes
    assert st["t_total"] > 0 and st["t_gpu_sort"] > 0 and st["t_h2d"] > 0


@pytest.mark.parametrize("n,b", [(3 * 100_000, 100_000), (4 * 100_000 - 7, 100_000),
                                 (5 * 65_536 + 1, 65_536), (6 * 100_000, 100_000),
                                 (9 * 50_000 + 123, 50_000)])
@pytest.mark.parametrize("permille,pin_w", [(0, 1), (500, 1), (-1, 0), (1000, 0)])
def test_stream_pipemerge(hs_gpu, oracle_mod, inputs_mod, n, b, permille, pin_w):
    """PIPEMERGE (S§8(f) #1): STREAM mode pre-merges pairs (0,1), (2,3), ... of sorted
    batches on the host threads during the sort phase, pipemerge_count(n_b, 1) of them (reading
    A-9, pinned by tests/golden/fig3_pipemerge.txt), and the final merge takes the merged pairs plus
    the remaining batches.  Output bit-exact vs the oracle for even/odd n_b and ragged last
    batches, with every merge split f."""
    A = inputs_mod.generate("normal" if n % 2 else "zipf_dup", n, seed=n + permille)
    want = _bits(oracle_mod.sort_f64(A))
    n_b = -(-n // b)
    m = oracle_mod.pipemerge_count(n_b, 1)
    opts = {"resident": 0, "merge_gpu_permille": permille, "pin_w": pin_w, "merge_chunk": 1 << 18}
    old = {k: hs_gpu.hsort_get_option(k) for k in list(opts) + ["pipemerge"]}
    for k, v in opts.items():
        hs_gpu.hsort_set_option(k, v)
    try:
        for pm in (1, 0):
            hs_gpu.hsort_set_option("pipemerge", pm)
            B = hs_gpu.hsort_sort(A, batch_elems=b)
            st = hs_gpu.hsort_get_stats()
            assert st["mode_name"] == "STREAM" and st["n_b"] == n_b
            assert np.array_equal(_bits(B), want), (n, b, permille, pm)
            assert st["pipe_merges"] == (m if pm else 0)
            assert st["merge_k"] == n_b - (m if pm else 0)
    finally:
        for k, v in old.items():
            hs_gpu.hsort_set_option(k, v)

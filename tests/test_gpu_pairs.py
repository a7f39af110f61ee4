"""GPU parity of the key/value sort against the oracle, through the C ABI.

Stable sort by key => unique result => bit-exact comparison of keys AND values.  Sizes span
several 4160-pair tiles and ragged tails; full size (2^30 pairs) is checked by properties that pin
the unique answer when V = 0..n-1: keys equal the (oracle-pinned) key sort, pairs are preserved
(A[VB] == B) and equal keys keep input order (VB increasing inside every run of equal keys).
"""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu

SIZES = [1, 2, 3, 4159, 4160, 4161, 3 * 4160 + 5, 100_003, (1 << 20) + 17]
DISTS = ["uniform", "few_distinct", "special", "salted", "all_equal", "sorted", "reverse", "normal"]


def _bits(a):
    return np.ascontiguousarray(a).view(np.uint64)


@pytest.mark.parametrize("dist", DISTS)
@pytest.mark.parametrize("n", SIZES)
def test_device_pairs_match_oracle(hs_gpu, oracle_mod, inputs_mod, dist, n):
    import torch
    A = inputs_mod.generate(dist, n, seed=n % 977 + 7)
    V = np.random.default_rng(n).integers(0, 2**64, size=n, dtype=np.uint64)
    wantB, wantV = oracle_mod.sort_pairs_f64(A, V)
    dA, dV = torch.from_numpy(A).cuda(), torch.from_numpy(V).cuda()
    dB, dVB = torch.empty_like(dA), torch.empty_like(dV)
    hs_gpu.hsort_sort_device_pairs(dA, dV, dB, dVB, True)
    torch.cuda.synchronize()
    assert np.array_equal(_bits(dB.cpu().numpy()), _bits(wantB))
    assert np.array_equal(dVB.cpu().numpy(), wantV)


@pytest.mark.parametrize("n", [4033, 250_001])
def test_device_pairs_in_place_and_u64(hs_gpu, oracle_mod, inputs_mod, n):
    import torch
    K = _bits(inputs_mod.generate("random_bits", n, seed=4)).copy()
    K[::3] = K[0]  # duplicates
    V = np.arange(n, dtype=np.uint64)
    wantB, wantV = oracle_mod.sort_pairs_u64(K, V)
    dK, dV = torch.from_numpy(K.view(np.int64)).cuda(), torch.from_numpy(V.view(np.int64)).cuda()
    hs_gpu.hsort_sort_device_pairs(dK, dV, dK, dV, False)
    torch.cuda.synchronize()
    assert np.array_equal(dK.cpu().numpy().view(np.uint64), wantB)
    assert np.array_equal(dV.cpu().numpy().view(np.uint64), wantV)


@pytest.mark.parametrize("pinned", [False, True])
@pytest.mark.parametrize("n", [1, 70_001, (1 << 21) + 3])
def test_host_pairs_match_oracle(hs_gpu, oracle_mod, inputs_mod, pinned, n):
    import torch
    A = inputs_mod.generate("salted", n, seed=n % 101)
    V = np.arange(n, dtype=np.uint64)[::-1].copy()
    wantB, wantV = oracle_mod.sort_pairs_f64(A, V)
    if pinned:
        tA, tV = torch.from_numpy(A).pin_memory(), torch.from_numpy(V.view(np.int64)).pin_memory()
        A, V = tA.numpy(), tV.numpy().view(np.uint64)
    B, VB = hs_gpu.hsort_sort_pairs(A, V)
    assert np.array_equal(_bits(B), _bits(wantB))
    assert np.array_equal(VB, wantV)
    st = hs_gpu.hsort_get_stats()
    assert st["mode_name"] == "BLINE" and st["n"] == n


def test_host_pairs_in_place_and_errors(hs_gpu, oracle_mod, inputs_mod):
    A = inputs_mod.generate("few_distinct", 33_333, seed=2)
    V = np.arange(A.size, dtype=np.uint64)
    wantB, wantV = oracle_mod.sort_pairs_f64(A, V)
    hs_gpu.hsort_sort_pairs(A, V, A, V)
    assert np.array_equal(_bits(A), _bits(wantB)) and np.array_equal(V, wantV)
    with pytest.raises(Exception):
        hs_gpu.hsort_sort_pairs(A, A.view(np.uint64))  # V aliases A


def test_device_pairs_misaligned_rejected(hs_gpu):
    import torch
    d = torch.zeros(1001, dtype=torch.float64, device="cuda")
    v = torch.zeros(1001, dtype=torch.int64, device="cuda")
    with pytest.raises(Exception):
        hs_gpu.hsort_sort_device_pairs(d[1:], v[1:], d[:-1].clone(), v[:-1].clone(), True)


def test_device_pairs_full_size_properties(hs_gpu, inputs_mod):
    """2^30 pairs (the bench size), V = 0..n-1: the unique stable answer, checked on the GPU."""
    import torch
    n = 1 << 30
    A = inputs_mod.generate("uniform", n, seed=2)
    dA = torch.from_numpy(A).cuda()
    del A
    dV = torch.arange(n, dtype=torch.int64, device="cuda")
    dB, dVB = torch.empty_like(dA), torch.empty_like(dV)
    hs_gpu.hsort_sort_device_pairs(dA, dV, dB, dVB, True)
    keys = torch.empty_like(dA)
    hs_gpu.hsort_sort_device(dA, keys)
    torch.cuda.synchronize()
    assert torch.equal(dB.view(torch.int64), keys.view(torch.int64))
    del keys, dV
    assert torch.equal(dA.view(torch.int64)[dVB], dB.view(torch.int64))  # pairs preserved
    eq = dB[1:] == dB[:-1]
    assert bool((dVB[1:][eq] > dVB[:-1][eq]).all())                       # stable
    assert bool((torch.bincount(dVB, minlength=n) == 1).all())            # a permutation


# ---- out-of-core key/value: the RESIDENT plan (batches sorted stably in HBM + key/value merge) ----
@pytest.mark.parametrize("dist", ["few_distinct", "zipf_dup", "all_equal", "special", "salted", "uniform"])
@pytest.mark.parametrize("pinned", [False, True])
def test_host_pairs_resident_batches(hs_gpu, oracle_mod, inputs_mod, dist, pinned):
    """hsort_sort_pairs_ex with b_s < n: each batch stably sorted by the key/value GPUSort, then
    K4 + the key/value K5 merge the runs with equal keys in run (= input) order: the unique stable
    sort, bit-exact on keys and values.  Heavy ties cross batch boundaries (few_distinct, all_equal)."""
    import torch
    n, b = 1_000_003, 100_000
    A = inputs_mod.generate(dist, n, seed=len(dist) + 3)
    V = np.arange(n, dtype=np.uint64)
    wantB, wantV = oracle_mod.sort_pairs_f64(A, V)
    if pinned:
        A = torch.from_numpy(A).pin_memory().numpy()
        V = torch.from_numpy(V.view(np.int64)).pin_memory().numpy().view(np.uint64)
    old = hs_gpu.hsort_get_option("merge_chunk")
    hs_gpu.hsort_set_option("merge_chunk", 1 << 17)  # several merge chunks
    try:
        B, VB = hs_gpu.hsort_sort_pairs_ex(A, V, batch_elems=b)
    finally:
        hs_gpu.hsort_set_option("merge_chunk", old)
    st = hs_gpu.hsort_get_stats()
    assert st["mode_name"] == "RESIDENT" and st["n_b"] == -(-n // b)
    assert np.array_equal(_bits(B), _bits(wantB))
    assert np.array_equal(VB, wantV)


def test_host_pairs_resident_auto_u64_in_place(hs_gpu, oracle_mod, inputs_mod):
    """The auto plan of hsort_sort_pairs from n >= auto_pipeline_min (lowered here): pipelined
    batches + halving tail; raw uint64 keys with duplicates; in place (B == A, VB == V)."""
    n = 3_000_017
    K = _bits(inputs_mod.generate("random_bits", n, seed=8)).copy()
    K[::5] = K[7]
    V = np.random.default_rng(1).integers(0, 2**64, size=n, dtype=np.uint64)
    wantB, wantV = oracle_mod.sort_pairs_u64(K, V)
    old = hs_gpu.hsort_get_option("auto_pipeline_min")
    hs_gpu.hsort_set_option("auto_pipeline_min", 1 << 20)
    try:
        hs_gpu.hsort_sort_pairs_u64(K, V, K, V)
        st = hs_gpu.hsort_get_stats()
    finally:
        hs_gpu.hsort_set_option("auto_pipeline_min", old)
    assert st["mode_name"] == "RESIDENT" and st["n_b"] > 8
    assert np.array_equal(K, wantB) and np.array_equal(V, wantV)

"""GPU parity of the dominant-digit elision against the oracle.

The top active digit L has a dominant value v; its pass is dropped, the outliers (digit L != v) are
diverted by the new last pass, sorted separately and placed at both ends.  Output-invisible: every
case is compared bit-exactly with the oracle, with the elision on and off, and the plan's pass
count shows whether it triggered.
"""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu

N = (1 << 22) + 77  # >= HSORT_DDE_MIN_N; side buffer cap = max(2^12, n >> 13) = 2^12


def _cap(n):
    return min(max(n >> 13, 1 << 12), 1 << 20)


def _keys(n, n_lo, n_hi, seed):
    """Random 64-bit keys whose top byte is 0x80, except n_lo below (0x10..) and n_hi above."""
    rng = np.random.default_rng(seed)
    K = rng.integers(0, 2**56, size=n, dtype=np.uint64) | np.uint64(0x80 << 56)
    idx = rng.permutation(n)
    lo, hi = idx[:n_lo], idx[n_lo:n_lo + n_hi]
    K[lo] = (K[lo] & np.uint64(2**56 - 1)) | (rng.integers(0, 0x80, size=n_lo, dtype=np.uint64) << np.uint64(56))
    K[hi] = (K[hi] & np.uint64(2**56 - 1)) | (rng.integers(0x81, 0x100, size=n_hi, dtype=np.uint64) << np.uint64(56))
    if n_lo:
        K[lo[:3]] = K[lo[0]]  # duplicates among outliers
    return K


def _sort_keys(hs, K, in_place=False, dde=True):
    import torch
    hs.hsort_set_option("dde", int(dde))
    try:
        d = torch.from_numpy(K.view(np.int64)).cuda()
        out = d if in_place else torch.empty_like(d)
        hs.hsort_sort_device_keys(d, out, False, False)
        torch.cuda.synchronize()
        na = hs.hsort_get_kernel_times()["num_active"]
        return out.cpu().numpy().view(np.uint64), na
    finally:
        hs.hsort_set_option("dde", 1)


@pytest.mark.parametrize("n_lo,n_hi", [(1, 0), (0, 1), (500, 700), (3, (1 << 12) - 3), ((1 << 12), 0)])
def test_dde_outliers_at_both_ends(hs_gpu, oracle_mod, n_lo, n_hi):
    K = _keys(N, n_lo, n_hi, seed=n_lo + 7 * n_hi)
    got, na = _sort_keys(hs_gpu, K)
    assert np.array_equal(got, oracle_mod.sort_u64(K))
    assert na == 7  # 8 active digits, the top one elided (n_out <= cap)


def test_dde_over_capacity_falls_back(hs_gpu, oracle_mod):
    K = _keys(N, _cap(N) + 1, 0, seed=5)
    got, na = _sort_keys(hs_gpu, K)
    assert np.array_equal(got, oracle_mod.sort_u64(K))
    assert na == 8


def test_dde_off_matches(hs_gpu, oracle_mod):
    K = _keys(N, 40, 40, seed=9)
    on, na_on = _sort_keys(hs_gpu, K, dde=True)
    off, na_off = _sort_keys(hs_gpu, K, dde=False)
    assert na_on == 7 and na_off == 8
    assert np.array_equal(on, off) and np.array_equal(on, oracle_mod.sort_u64(K))


def test_dde_not_in_place(hs_gpu, oracle_mod):
    """In place the remaining passes would end in the scratch buffer (an extra copy): no elision."""
    K = _keys(N, 10, 10, seed=2)
    got, na = _sort_keys(hs_gpu, K, in_place=True)
    assert np.array_equal(got, oracle_mod.sort_u64(K))
    assert na == 8
    K2 = K & ~np.uint64(0xFF)  # digit 0 trivial: 7 active digits, elided out of place -> 6
    got, na = _sort_keys(hs_gpu, K2)
    assert np.array_equal(got, oracle_mod.sort_u64(K2))
    assert na == 6


@pytest.mark.parametrize("n", [(1 << 22) + 1, (1 << 23) + 4097])
def test_dde_uniform_float64(hs_gpu, oracle_mod, inputs_mod, n):
    """The paper's workload: U[0,1) doubles; keys >= 2^-15 share the top byte 0xBF."""
    import torch
    A = inputs_mod.generate("uniform", n, seed=n)
    d = torch.from_numpy(A).cuda()
    out = torch.empty_like(d)
    hs_gpu.hsort_sort_device(d, out)
    torch.cuda.synchronize()
    assert hs_gpu.hsort_get_kernel_times()["num_active"] == 7
    assert np.array_equal(out.cpu().numpy().view(np.uint64), oracle_mod.sort_f64(A).view(np.uint64))


def test_dde_special_values_and_host_paths(hs_gpu, oracle_mod, inputs_mod):
    """Salted data (±0, NaNs) in the outlier set; host->host RESIDENT and typed (codec) paths."""
    A = inputs_mod.generate("uniform", N, seed=3)
    rng = np.random.default_rng(3)
    salt = rng.choice(N, 2000, replace=False)
    A[salt[:500]] = -0.0
    A[salt[500:1000]] = np.nan
    A[salt[1000:1500]] = -A[salt[1000:1500]]
    A[salt[1500:]] = np.float64(np.inf)
    want = oracle_mod.sort_f64(A).view(np.uint64)
    import torch
    d = torch.from_numpy(A).cuda()
    out = torch.empty_like(d)
    hs_gpu.hsort_sort_device(d, out)
    torch.cuda.synchronize()
    assert np.array_equal(out.cpu().numpy().view(np.uint64), want)
    B = hs_gpu.hsort_sort(A, batch_elems=N // 3 + 5)  # RESIDENT batches
    assert np.array_equal(B.view(np.uint64), want)
    B = hs_gpu.hsort_sort_typed(A, descending=True)
    assert np.array_equal(B.view(np.uint64), want[::-1])


def test_dde_pass0_count_fallbacks(hs_gpu, oracle_mod):
    """The outlier histogram is counted by pass 0 (not K1) when K1's guess (key 0's top byte) is an
    outlier, and when the elided digit is not the top byte (L = 6: digit 7 trivial)."""
    K = _keys(N, 300, 300, seed=11)
    lo = np.flatnonzero((K >> np.uint64(56)) < np.uint64(0x80))[0]
    K[[0, lo]] = K[[lo, 0]]  # an outlier first: wrong guess
    got, na = _sort_keys(hs_gpu, K)
    assert np.array_equal(got, oracle_mod.sort_u64(K)) and na == 7
    K6 = (K >> np.uint64(8)) | np.uint64(0x42 << 56)  # digit 7 constant, digit 6 dominant
    got, na = _sort_keys(hs_gpu, K6)
    assert np.array_equal(got, oracle_mod.sort_u64(K6)) and na == 6  # 7 active digits, L = 6 elided
    assert hs_gpu.hsort_get_last_plan()["elided"]

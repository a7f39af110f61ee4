"""GPU parity of the other key types / orders vs the oracle, via the C ABI.

float32 ascending/descending and float64 descending, device -> device and host -> host; sizes
across tile boundaries and ragged tails (incl. n % 4 != 0 for the 16-byte codec loads); float32
special values (NaN payloads, -0.0, denormals) bit-exact.
"""
import numpy as np
import pytest

from tests.ieee_total_order import SPECIAL32

pytestmark = pytest.mark.gpu

SIZES = [1, 2, 3, 5, 4097, 8641, 100_003, (1 << 20) + 3]


def _f32(inputs_mod, dist, n, seed):
    if dist == "special32":
        rng = np.random.default_rng(seed)
        a = rng.integers(0, 2**32, size=n, dtype=np.uint32)
        pick = rng.random(n) < 0.5
        a[pick] = np.array(SPECIAL32, dtype=np.uint32)[rng.integers(0, len(SPECIAL32), size=int(pick.sum()))]
        return a.view(np.float32)
    return inputs_mod.generate(dist, n, seed=seed).astype(np.float32)


@pytest.mark.parametrize("desc", [False, True])
@pytest.mark.parametrize("dist", ["uniform", "normal", "few_distinct", "special32"])
@pytest.mark.parametrize("n", SIZES)
def test_device_f32(hs_gpu, oracle_mod, inputs_mod, desc, dist, n):
    import torch
    A = _f32(inputs_mod, dist, n, seed=n % 1009)
    want = oracle_mod.sort_f32(A, desc).view(np.uint32)
    d = torch.from_numpy(A.view(np.int32)).cuda().view(torch.float32)
    out = torch.empty_like(d)
    hs_gpu.hsort_sort_device_typed(d, out, desc)
    torch.cuda.synchronize()
    assert np.array_equal(out.view(torch.int32).cpu().numpy().view(np.uint32), want)


@pytest.mark.parametrize("dist", ["uniform", "special", "salted", "all_equal"])
@pytest.mark.parametrize("n", SIZES)
def test_device_f64_descending(hs_gpu, oracle_mod, inputs_mod, dist, n):
    import torch
    A = inputs_mod.generate(dist, n, seed=n % 97)
    want = oracle_mod.sort_desc_f64(A).view(np.uint64)
    d = torch.from_numpy(A).cuda()
    hs_gpu.hsort_sort_device_typed(d, d, True)  # in place
    torch.cuda.synchronize()
    assert np.array_equal(d.cpu().numpy().view(np.uint64), want)


@pytest.mark.parametrize("pinned", [False, True])
@pytest.mark.parametrize("case", ["f32", "f32desc", "f64desc", "f64asc"])
def test_host_typed(hs_gpu, oracle_mod, inputs_mod, pinned, case):
    import torch
    n = (1 << 21) + 5
    if case.startswith("f32"):
        A = _f32(inputs_mod, "special32", n, seed=3)
        want = oracle_mod.sort_f32(A, case.endswith("desc")).view(np.uint32)
    else:
        A = inputs_mod.generate("salted", n, seed=3)
        want = (oracle_mod.sort_desc_f64(A) if case == "f64desc" else oracle_mod.sort_f64(A)).view(np.uint64)
    if pinned:
        A = torch.from_numpy(A.view(np.int32 if A.dtype == np.float32 else np.int64)).pin_memory().numpy().view(A.dtype)
    B = hs_gpu.hsort_sort_typed(A, descending=case.endswith("desc"))
    assert np.array_equal(B.view(want.dtype), want)
    hs_gpu.hsort_sort_typed(A, A, descending=case.endswith("desc"))  # in place
    assert np.array_equal(A.view(want.dtype), want)


@pytest.mark.parametrize("dist,n", [("salted", (1 << 20) + 7), ("special", (1 << 21) + 1),
                                    ("uniform", (1 << 22) + 3), ("all_equal", 1 << 20)])
def test_device_f64_descending_fused(hs_gpu, oracle_mod, inputs_mod, dist, n):
    """Out of place, n >= 2^20: the reverse transform fused into the GPUSort (U[0,1) at 2^22 also
    takes the dominant-digit elision in the complemented key space)."""
    import torch
    A = inputs_mod.generate(dist, n, seed=n % 89)
    want = oracle_mod.sort_desc_f64(A).view(np.uint64)
    d = torch.from_numpy(A).cuda()
    out = torch.empty_like(d)
    hs_gpu.hsort_sort_device_typed(d, out, True)
    torch.cuda.synchronize()
    assert np.array_equal(out.cpu().numpy().view(np.uint64), want)
    if dist == "uniform":
        assert hs_gpu.hsort_get_last_plan()["elided"]


@pytest.mark.parametrize("desc", [False, True])
@pytest.mark.parametrize("dist", ["uniform", "special32", "all_equal", "few_distinct"])
@pytest.mark.parametrize("n", [1, 3, 4, 7, 8641, 17_283, (1 << 22) + 3])
def test_device_f32_native_in_place_and_launches(hs_gpu, oracle_mod, inputs_mod, desc, dist, n):
    """The native 32-bit GPUSort (4-byte keys; K1 over 4 digits, <= 4 warp-specialised passes with
    the binary32 transform fused into the first and last pass): 7 launches (K1, K2,
    4 pass launches, final copy) instead of the codec path's encode/decode around a 64-bit sort;
    in place (odd active-pass counts end with the final copy) and all-equal keys (no active
    digit) included."""
    import torch
    A = _f32(inputs_mod, dist, n, seed=n % 1013)
    want = oracle_mod.sort_f32(A, desc).view(np.uint32)
    d = torch.from_numpy(A.view(np.int32).copy()).cuda().view(torch.float32)
    out = torch.empty_like(d)
    L0 = hs_gpu.hsort_get_launch_count()
    hs_gpu.hsort_sort_device_typed(d, out, desc)
    torch.cuda.synchronize()
    assert hs_gpu.hsort_get_launch_count() - L0 == 7
    assert np.array_equal(out.view(torch.int32).cpu().numpy().view(np.uint32), want)
    assert hs_gpu.hsort_get_last_plan()["num_active"] <= 4
    hs_gpu.hsort_sort_device_typed(d, d, desc)  # in place
    torch.cuda.synchronize()
    assert np.array_equal(d.view(torch.int32).cpu().numpy().view(np.uint32), want)


def test_device_typed_requires_16_byte_alignment(hs_gpu):
    """hsort_sort_device_typed's contract: 16-byte aligned device buffers (TMA tile loads)."""
    import torch
    buf = torch.zeros(1001, dtype=torch.float32, device="cuda")
    with pytest.raises(hs_gpu.HsortError) as e:
        hs_gpu.hsort_sort_device_typed(buf[1:], buf[1:].clone(), False)
    assert e.value.code == -1

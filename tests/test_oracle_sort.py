"""Pins for oracle_sort_f64 and the whole-result verifiers."""
import itertools

import numpy as np
import pytest

from tests.ieee_total_order import insertion_sort_bits


def _bits(a):
    return np.ascontiguousarray(a, dtype=np.float64).view(np.uint64)


def test_brute_force_all_permutations(oracle_mod, inputs_mod):
    alpha = [int(u) for u in inputs_mod.special_alphabet()]
    rng = np.random.default_rng(3)
    for n in range(0, 8):
        pool = [alpha[int(i)] for i in rng.permutation(len(alpha))[:n]]
        want = insertion_sort_bits(pool)
        perms = list(itertools.permutations(pool))
        if len(perms) > 800:
            perms = [perms[i] for i in rng.choice(len(perms), 800, replace=False)]
        for p in perms:
            A = np.array(p, dtype=np.uint64).view(np.float64)
            B = oracle_mod.sort_f64(A)
            assert [int(u) for u in _bits(B)] == want


def test_brute_force_all_short_sequences_over_alphabet(oracle_mod, inputs_mod):
    alpha = [int(u) for u in inputs_mod.special_alphabet()]
    for n in range(0, 4):
        for seq in itertools.product(alpha, repeat=n):
            A = np.array(seq, dtype=np.uint64).view(np.float64)
            B = oracle_mod.sort_f64(A)
            assert [int(u) for u in _bits(B)] == insertion_sort_bits(list(seq))


def test_random_length4_sequences_with_duplicates(oracle_mod, inputs_mod):
    alpha = [int(u) for u in inputs_mod.special_alphabet()]
    rng = np.random.default_rng(11)
    for _ in range(3000):
        seq = [alpha[i] for i in rng.integers(0, len(alpha), size=int(rng.integers(4, 9)))]
        A = np.array(seq, dtype=np.uint64).view(np.float64)
        assert [int(u) for u in _bits(oracle_mod.sort_f64(A))] == insertion_sort_bits(seq)


@pytest.mark.parametrize("dist", ["uniform", "normal", "zipf_dup", "uniform_pm1", "few_distinct"])
def test_matches_numpy_sort_on_nan_and_negzero_free_data(oracle_mod, inputs_mod, dist):
    A = inputs_mod.generate(dist, 200_003, seed=5)
    assert not np.isnan(A).any()
    A[A == 0] = 0.0  # canonical +0 only (numpy's < cannot order -0/+0)
    B = oracle_mod.sort_f64(A)
    assert np.array_equal(_bits(B), _bits(np.sort(A, kind="stable")))


@pytest.mark.parametrize("n", [1, 2, 3, 255, 256, 257, 4096, 65537, 1 << 18])
def test_closed_form_permutation_inputs(oracle_mod, inputs_mod, n):
    A = inputs_mod.generate("closed_form", n, seed=n)
    B = oracle_mod.sort_f64(A)
    want = (np.arange(n, dtype=np.int64) - n // 2).astype(np.float64)
    assert np.array_equal(_bits(B), _bits(want))


def test_key_route_equals_definition(oracle_mod, inputs_mod):
    # The GPU path sorts unsigned keys; the oracle's two routes must agree on every distribution,
    # including NaNs / signed zeros (where numpy cannot serve as a check).
    for dist in ["special", "random_bits", "salted", "zipf_dup"]:
        A = inputs_mod.generate(dist, 50_000, seed=9)
        B1 = oracle_mod.sort_f64(A)
        B2 = oracle_mod.f64_from_keys(oracle_mod.sort_u64(oracle_mod.keys_from_f64(A)))
        assert np.array_equal(_bits(B1), _bits(B2)), dist


def test_verifiers_detect_planted_faults(oracle_mod, inputs_mod):
    A = inputs_mod.generate("salted", 100_000, seed=2)
    B = oracle_mod.sort_f64(A)
    assert oracle_mod.is_sorted_f64(B)
    assert oracle_mod.multiset_hash(A) == oracle_mod.multiset_hash(B)
    # swap two distinct neighbours -> not sorted, same multiset
    i = int(np.nonzero(_bits(B)[1:] != _bits(B)[:-1])[0][500])
    C = B.copy()
    C[i], C[i + 1] = C[i + 1], C[i]
    assert not oracle_mod.is_sorted_f64(C)
    assert oracle_mod.multiset_hash(C) == oracle_mod.multiset_hash(A)
    # flip one low bit -> multiset differs
    D = B.copy()
    D.view(np.uint64)[777] ^= np.uint64(1)
    assert oracle_mod.multiset_hash(D) != oracle_mod.multiset_hash(A)
    # -0 <-> +0 swap is a different multiset
    E = np.array([0.0, -0.0, 1.0])
    F = np.array([0.0, 0.0, 1.0])
    assert oracle_mod.multiset_hash(E) != oracle_mod.multiset_hash(F)
    assert not oracle_mod.is_sorted_f64(np.array([0.0, -0.0]))
    assert oracle_mod.is_sorted_f64(np.array([-0.0, 0.0]))


def test_empty_and_single(oracle_mod):
    assert oracle_mod.sort_f64(np.zeros(0)).size == 0
    x = np.array([np.nan])
    assert _bits(oracle_mod.sort_f64(x))[0] == _bits(x)[0]


def test_parallel_cpu_baseline_equals_oracle(oracle_mod, inputs_mod):
    """The parallel-CPU baseline (GNU parallel sort, the paper's reference) is bit-identical to the
    oracle under totalOrder (the result is unique), incl. ±0 and NaN payloads."""
    for dist, n in (("special", 100_000), ("salted", 1_000_003), ("uniform", 777)):
        A = inputs_mod.generate(dist, n, seed=n)
        want = oracle_mod.sort_f64(A).view(np.uint64)
        for threads in (1, 4):
            assert np.array_equal(oracle_mod.par_sort_f64(A, threads).view(np.uint64), want)

"""Pins for the other key types / orders: oracle_sort_f32, oracle_sort_desc_f64.

Brute force over permutations of binary32 special values vs the IEEE clauses restated on binary32
fields (tests/ieee_total_order.py), numpy.sort on NaN/-0-free data, and descending = the exact
reverse of ascending (every totalOrder class is one bit pattern, so both results are unique).
"""
import itertools

import numpy as np

from tests.ieee_total_order import SPECIAL32, insertion_sort_bits, insertion_sort_bits32


def test_f32_brute_force_permutations(oracle_mod):
    rng = np.random.default_rng(2)
    for n in range(0, 7):
        pool = [SPECIAL32[int(i)] for i in rng.integers(0, len(SPECIAL32), size=n)]
        for desc in (False, True):
            want = insertion_sort_bits32(pool, desc)
            for perm in itertools.islice(itertools.permutations(pool), 300):
                A = np.array(perm, dtype=np.uint32).view(np.float32)
                B = oracle_mod.sort_f32(A, desc)
                assert [int(u) for u in B.view(np.uint32)] == want


def test_f32_matches_numpy_on_plain_data(oracle_mod):
    A = np.random.default_rng(4).standard_normal(100_000).astype(np.float32)
    A[A == 0] = 1.0
    assert np.array_equal(oracle_mod.sort_f32(A), np.sort(A))
    assert np.array_equal(oracle_mod.sort_f32(A, True), np.sort(A)[::-1])


def test_desc_is_reverse_of_asc(oracle_mod, inputs_mod):
    A = inputs_mod.generate("special", 30_000, seed=6)
    asc = oracle_mod.sort_f64(A).view(np.uint64)
    assert np.array_equal(oracle_mod.sort_desc_f64(A).view(np.uint64), asc[::-1])
    A32 = np.random.default_rng(1).integers(0, 2**32, size=30_000, dtype=np.uint32).view(np.float32)
    assert np.array_equal(oracle_mod.sort_f32(A32, True).view(np.uint32),
                          oracle_mod.sort_f32(A32).view(np.uint32)[::-1])


def test_desc_f64_brute_force(oracle_mod, inputs_mod):
    alpha = [int(u) for u in inputs_mod.special_alphabet()]
    rng = np.random.default_rng(8)
    for n in range(0, 6):
        pool = [alpha[int(i)] for i in rng.integers(0, len(alpha), size=n)]
        want = insertion_sort_bits(pool)[::-1]
        for perm in itertools.islice(itertools.permutations(pool), 200):
            B = oracle_mod.sort_desc_f64(np.array(perm, dtype=np.uint64).view(np.float64))
            assert [int(u) for u in B.view(np.uint64)] == want

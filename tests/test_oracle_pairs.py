"""Pins for the key/value oracle (oracle_sort_pairs_f64/_u64).

The definition is a STABLE sort of the pairs by key under IEEE totalOrder, so the result is
unique.  Pinned against: a textbook stable insertion sort over (key, value) pairs written here with
the clause-by-clause IEEE predicate (brute force over all permutations of small duplicate-heavy
inputs); numpy's stable argsort on NaN/-0-free keys; the pair multiset.
"""
import itertools

import numpy as np

from tests.ieee_total_order import total_order_less


def _stable_insertion_pairs(keys, vals):
    """Textbook insertion sort: an element moves left only past strictly greater keys (stable)."""
    out = []
    for k, v in zip(keys, vals):
        i = len(out)
        while i > 0 and total_order_less(k, out[i - 1][0]):
            i -= 1
        out.insert(i, (k, v))
    return [k for k, _ in out], [v for _, v in out]


def test_pairs_brute_force_permutations_with_duplicates(oracle_mod, inputs_mod):
    alpha = [int(u) for u in inputs_mod.special_alphabet()]
    rng = np.random.default_rng(21)
    for n in range(0, 7):
        # few distinct keys (incl. -0/+0 and NaNs) so equal keys exercise stability
        pool = [alpha[int(i)] for i in rng.integers(0, len(alpha), size=max(1, n // 2))]
        keys = [pool[int(i)] for i in rng.integers(0, len(pool), size=n)]
        for perm in itertools.permutations(range(n)):
            kk = [keys[i] for i in perm]
            vv = [1000 + i for i in range(n)]  # input position as payload
            want_k, want_v = _stable_insertion_pairs(kk, vv)
            B, VB = oracle_mod.sort_pairs_f64(np.array(kk, dtype=np.uint64).view(np.float64),
                                              np.array(vv, dtype=np.uint64))
            assert [int(u) for u in B.view(np.uint64)] == want_k
            assert [int(u) for u in VB] == want_v


def test_pairs_match_numpy_stable_argsort(oracle_mod, inputs_mod):
    rng = np.random.default_rng(5)
    A = inputs_mod.generate("few_distinct", 50_000, seed=3)  # heavy duplicates, no NaN/-0
    assert not np.isnan(A).any()
    A[A == 0] = 0.0  # +0 only
    V = rng.integers(0, 2**64, size=A.size, dtype=np.uint64)
    B, VB = oracle_mod.sort_pairs_f64(A, V)
    idx = np.argsort(A, kind="stable")
    assert np.array_equal(B, A[idx])
    assert np.array_equal(VB, V[idx])
    Bu, VBu = oracle_mod.sort_pairs_u64(A.view(np.uint64) ^ np.uint64(0x5555), V)
    idx = np.argsort(A.view(np.uint64) ^ np.uint64(0x5555), kind="stable")
    assert np.array_equal(VBu, V[idx])


def test_pairs_keys_equal_key_sort_and_pairs_preserved(oracle_mod, inputs_mod):
    A = inputs_mod.generate("special", 20_000, seed=9)
    V = np.arange(A.size, dtype=np.uint64)
    B, VB = oracle_mod.sort_pairs_f64(A, V)
    assert np.array_equal(B.view(np.uint64), oracle_mod.sort_f64(A).view(np.uint64))
    assert np.array_equal(np.sort(VB), V)                       # values are a permutation
    assert np.array_equal(A[VB.astype(np.int64)].view(np.uint64), B.view(np.uint64))  # pairs kept

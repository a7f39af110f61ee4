"""Pins for the oracle's radix-pass, merge, co-rank and PIPEMERGE functions."""
import heapq
import itertools
import os

import numpy as np
import pytest

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def test_histograms_closed_forms(oracle_mod):
    for d in range(8):
        K = (np.arange(256, dtype=np.uint64) << np.uint64(8 * d))
        h = oracle_mod.digit_histograms(K)
        assert np.all(h[d] == 1)
        for e in range(8):
            if e != d:
                assert h[e][0] == 256 and h[e][1:].sum() == 0
    K = np.full(1000, 0x0123456789ABCDEF, dtype=np.uint64)
    h = oracle_mod.digit_histograms(K)
    for d, v in enumerate([0xEF, 0xCD, 0xAB, 0x89, 0x67, 0x45, 0x23, 0x01]):
        assert h[d][v] == 1000 and h[d].sum() == 1000


def test_histograms_sum_to_n(oracle_mod):
    K = np.random.default_rng(1).integers(0, 2**64, size=12345, dtype=np.uint64)
    h = oracle_mod.digit_histograms(K)
    assert np.all(h.sum(axis=1) == 12345)


@pytest.mark.parametrize("d", range(8))
def test_counting_pass_is_stable_gather_by_digit(oracle_mod, d):
    rng = np.random.default_rng(d)
    K = rng.integers(0, 2**64, size=20000, dtype=np.uint64)
    K[::7] = K[3]  # duplicates
    digit = (K >> np.uint64(8 * d)) & np.uint64(255)
    want = K[np.argsort(digit, kind="stable")]
    got = oracle_mod.counting_sort_pass(K, d)
    assert np.array_equal(got, want)
    # stability stated directly: each digit-class subsequence keeps input order
    gd = (got >> np.uint64(8 * d)) & np.uint64(255)
    for v in rng.integers(0, 256, size=5):
        assert np.array_equal(got[gd == v], K[digit == v])


def test_lsd_composition_is_full_sort(oracle_mod, inputs_mod):
    A = inputs_mod.generate("special", 30011, seed=4)
    K = oracle_mod.keys_from_f64(A)
    cur = K
    for d in range(8):
        cur = oracle_mod.counting_sort_pass(cur, d)
    assert np.array_equal(cur, np.sort(K))
    assert np.array_equal(cur, oracle_mod.sort_u64(K))


def _random_runs(rng, k, maxlen, dup=False):
    runs = []
    for _ in range(k):
        m = int(rng.integers(0, maxlen + 1))
        hi = 50 if dup else 2**64
        runs.append(np.sort(rng.integers(0, hi, size=m, dtype=np.uint64)))
    return runs


@pytest.mark.parametrize("k", [1, 2, 3, 7, 16, 33])
def test_merge_runs_equals_heapq_merge(oracle_mod, k):
    rng = np.random.default_rng(k)
    for dup in (False, True):
        runs = _random_runs(rng, k, 300, dup)
        want = np.array(list(heapq.merge(*[r.tolist() for r in runs])), dtype=np.uint64)
        assert np.array_equal(oracle_mod.merge_runs(runs), want)


def _lex_ok(runs, ranks):
    """Co-rank invariant: every (key, run, index) left of the cut < every one right of it."""
    left_max, right_min = None, None
    for j, (r, i) in enumerate(zip(runs, ranks)):
        i = int(i)
        if i > 0:
            t = (int(r[i - 1]), j, i - 1)
            left_max = t if left_max is None or t > left_max else left_max
        if i < r.size:
            t = (int(r[i]), j, i)
            right_min = t if right_min is None or t < right_min else right_min
    return left_max is None or right_min is None or left_max < right_min


def test_corank_invariants_and_uniqueness_brute_force(oracle_mod):
    rng = np.random.default_rng(5)
    for trial in range(60):
        k = int(rng.integers(1, 4))
        runs = _random_runs(rng, k, 5, dup=True)
        n = sum(r.size for r in runs)
        for o in range(n + 1):
            ranks = oracle_mod.corank(runs, o)
            assert int(ranks.sum()) == o
            assert _lex_ok(runs, ranks)
            # brute force: exactly one rank vector with sum o satisfies the invariant
            sols = [c for c in itertools.product(*[range(r.size + 1) for r in runs])
                    if sum(c) == o and _lex_ok(runs, c)]
            assert sols == [tuple(int(x) for x in ranks)]


def test_corank_large_k_invariants(oracle_mod):
    rng = np.random.default_rng(8)
    runs = _random_runs(rng, 40, 200, dup=True)
    n = sum(r.size for r in runs)
    for o in [0, 1, n // 3, n // 2, n - 1, n]:
        ranks = oracle_mod.corank(runs, o)
        assert int(ranks.sum()) == o and _lex_ok(runs, ranks)


def test_pipemerge_fig3_golden(oracle_mod):
    rows = [l.split() for l in open(os.path.join(GOLDEN, "fig3_pipemerge.txt"))
            if l.strip() and not l.startswith("#")]
    for n_b, n_gpu, merges, final_lists in rows:
        m = oracle_mod.pipemerge_count(int(n_b), int(n_gpu))
        assert m == int(merges)
        assert int(n_b) - m == int(final_lists)


def test_pipemerge_parity_rule(oracle_mod):
    # even n_b -> the last two batches stay unmerged; odd -> the last batch does.
    for n_b in range(2, 40):
        m = oracle_mod.pipemerge_count(n_b, 1)
        unmerged = n_b - 2 * m
        assert unmerged == (2 if n_b % 2 == 0 else 1)
    # with 2+ GPUs fewer pair-wise merges happen than with one.
    for n_b in range(2, 40):
        assert oracle_mod.pipemerge_count(n_b, 2) <= oracle_mod.pipemerge_count(n_b, 1)


def test_gnu_multiway_merge_reference_equals_oracle(oracle_mod):
    """The CPU-merge reference (GNU parallel multiway_merge, the paper's merge) = oracle merge."""
    rng = np.random.default_rng(4)
    runs = [np.sort(rng.integers(0, 1000, size=int(rng.integers(0, 5000)), dtype=np.uint64))
            for _ in range(9)]
    off = np.cumsum([0] + [r.size for r in runs]).astype(np.uint64)
    keys = np.concatenate(runs)
    assert np.array_equal(oracle_mod.par_multiway_merge_u64(keys, off, 4), oracle_mod.merge_runs(runs))

"""Pins for the oracle's total order and key map (readings A-1..A-3).

oracle_total_order_cmp (std::strong_order) and oracle_key (unsigned key map) are checked against
tests/ieee_total_order.py, a clause-by-clause restatement of IEEE 754 §5.10 totalOrder.
"""
import itertools

import numpy as np

from tests.ieee_total_order import bits_to_f, total_order_le, total_order_less


def _alphabet(inputs_mod):
    return [int(u) for u in inputs_mod.special_alphabet()]


def test_alphabet_is_the_fifteen_specials(inputs_mod):
    a = _alphabet(inputs_mod)
    assert len(a) == 15 and len(set(a)) == 15


def test_total_order_cmp_matches_ieee_clauses_on_alphabet(oracle_mod, inputs_mod):
    a = _alphabet(inputs_mod)
    for ux, uy in itertools.product(a, a):
        want = -1 if total_order_less(ux, uy) else (1 if total_order_less(uy, ux) else 0)
        assert oracle_mod.total_order_cmp(bits_to_f(ux), bits_to_f(uy)) == want, (hex(ux), hex(uy))


def test_alphabet_listed_in_total_order(inputs_mod):
    # The alphabet is written in ascending totalOrder (−qNaN first ... +qNaN max payload last),
    # which is the order IEEE §5.10 fixes (reading A-2 for the payload tie only).
    a = _alphabet(inputs_mod)
    for i in range(len(a) - 1):
        assert total_order_less(a[i], a[i + 1]), (hex(a[i]), hex(a[i + 1]))


def test_key_order_isomorphic_on_alphabet(oracle_mod, inputs_mod):
    a = _alphabet(inputs_mod)
    for ux, uy in itertools.product(a, a):
        kx, ky = oracle_mod.key(ux), oracle_mod.key(uy)
        assert (kx < ky) == total_order_less(ux, uy)
        assert (kx == ky) == (ux == uy)


def test_key_order_isomorphic_random_pairs(oracle_mod):
    rng = np.random.default_rng(12345)
    # mix raw random bit patterns with patterns that share sign/exponent (close values)
    x = rng.integers(0, 2**64, size=20000, dtype=np.uint64)
    y = rng.integers(0, 2**64, size=20000, dtype=np.uint64)
    y[:10000] = x[:10000] ^ (rng.integers(0, 2**20, size=10000, dtype=np.uint64))
    kx = oracle_mod.keys_from_f64(x.view(np.float64))
    ky = oracle_mod.keys_from_f64(y.view(np.float64))
    for i in range(x.size):
        assert bool(kx[i] < ky[i]) == total_order_less(int(x[i]), int(y[i]))
        if i < 3000:
            c = oracle_mod.total_order_cmp(float(x[i].view(np.float64)), float(y[i].view(np.float64)))
            assert (c < 0) == total_order_less(int(x[i]), int(y[i]))


def test_key_is_bijection(oracle_mod):
    rng = np.random.default_rng(7)
    u = rng.integers(0, 2**64, size=200000, dtype=np.uint64)
    k = oracle_mod.keys_from_f64(u.view(np.float64))
    back = oracle_mod.f64_from_keys(k).view(np.uint64)
    assert np.array_equal(back, u)
    assert len(np.unique(k)) == len(np.unique(u))
    for v in [0, 1, 2**63, 2**64 - 1, 0x7FF8000000000000]:
        assert oracle_mod.key_inv(oracle_mod.key(v)) == v


def test_signed_zero_and_nan_placement(oracle_mod):
    # A-1: -0 strictly before +0.  A-2: negative NaNs first, positive NaNs last.
    m0, p0 = 0x8000000000000000, 0
    assert oracle_mod.key(m0) < oracle_mod.key(p0)
    assert total_order_less(m0, p0) and total_order_le(p0, p0)
    assert oracle_mod.key(0xFFF8000000000000) < oracle_mod.key(0xFFF0000000000000)  # -qNaN < -inf
    assert oracle_mod.key(0x7FF0000000000000) < oracle_mod.key(0x7FF0000000000001)  # +inf < +sNaN

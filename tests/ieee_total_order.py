"""IEEE 754-2008 §5.10 totalOrder, written clause by clause (test-side, independent of oracle/).

This is the pin for the oracle's order: the oracle uses C++20 ``std::strong_order`` (library) and
an unsigned-key map; this module restates the standard's clauses directly in Python with Python
float comparisons and bit-field reads, so a mistake in either oracle route shows up here.

totalOrder(x, y) is true iff x precedes or equals y:
  (a) x < y numerically                                 -> true;   x > y -> false
  (b) x == y numerically (incl. ±0):   -0 precedes +0; identical data -> true (equal)
  (c) x or y NaN:
      negative-signed NaN precedes every non-NaN; every non-NaN precedes positive-signed NaN;
      both NaN, different sign: the negative one precedes;
      both NaN, same sign: for positive sign sNaN precedes qNaN, for negative qNaN precedes sNaN;
      otherwise (same sign, same kind) the order is implementation-defined — DESIGN.md reading A-2
      fixes it as payload order (larger payload is later for +, earlier for -).
"""
from __future__ import annotations

import math
import struct


def bits_to_f(u: int) -> float:
    return struct.unpack("<d", struct.pack("<Q", u & 0xFFFFFFFFFFFFFFFF))[0]


def f_to_bits(x: float) -> int:
    return struct.unpack("<Q", struct.pack("<d", x))[0]


def _sign(u: int) -> int:
    return u >> 63


def _is_nan(u: int) -> bool:
    return ((u >> 52) & 0x7FF) == 0x7FF and (u & ((1 << 52) - 1)) != 0


def _is_quiet(u: int) -> bool:
    return bool((u >> 51) & 1)


def _payload(u: int) -> int:
    return u & ((1 << 51) - 1)


def total_order_le(ux: int, uy: int) -> bool:
    """totalOrder(x, y) for the float64 bit patterns ux, uy."""
    nx, ny = _is_nan(ux), _is_nan(uy)
    if not nx and not ny:
        x, y = bits_to_f(ux), bits_to_f(uy)
        if x < y:
            return True
        if x > y:
            return False
        # numerically equal: only ±0 can differ in bits
        if x == 0.0:
            if _sign(ux) == 1 and _sign(uy) == 0:
                return True
            if _sign(ux) == 0 and _sign(uy) == 1:
                return False
        return True
    if nx and not ny:
        return _sign(ux) == 1
    if ny and not nx:
        return _sign(uy) == 0
    # both NaN
    if _sign(ux) != _sign(uy):
        return _sign(ux) == 1
    neg = _sign(ux) == 1
    qx, qy = _is_quiet(ux), _is_quiet(uy)
    if qx != qy:
        # positive: sNaN precedes qNaN; negative: qNaN precedes sNaN
        return (not qx) if not neg else qx
    px, py = _payload(ux), _payload(uy)
    return px <= py if not neg else px >= py


def total_order_less(ux: int, uy: int) -> bool:
    return total_order_le(ux, uy) and not total_order_le(uy, ux)


def insertion_sort_bits(bits: list[int]) -> list[int]:
    out: list[int] = []
    for u in bits:
        i = len(out)
        while i > 0 and total_order_less(u, out[i - 1]):
            i -= 1
        out.insert(i, u)
    return out


# ---- binary32 (S§8(f) #4): the same clauses on 32-bit fields --------------------------------------
def bits32_to_f(u: int) -> float:
    return struct.unpack("<f", struct.pack("<I", u & 0xFFFFFFFF))[0]


def _is_nan32(u: int) -> bool:
    return ((u >> 23) & 0xFF) == 0xFF and (u & ((1 << 23) - 1)) != 0


def total_order_le32(ux: int, uy: int) -> bool:
    """totalOrder(x, y) for the binary32 bit patterns ux, uy (clauses as total_order_le)."""
    sx, sy = ux >> 31, uy >> 31
    nx, ny = _is_nan32(ux), _is_nan32(uy)
    if not nx and not ny:
        x, y = bits32_to_f(ux), bits32_to_f(uy)  # exact (binary32 -> double)
        if x < y:
            return True
        if x > y:
            return False
        if x == 0.0 and sx != sy:
            return sx == 1
        return True
    if nx and not ny:
        return sx == 1
    if ny and not nx:
        return sy == 0
    if sx != sy:
        return sx == 1
    neg = sx == 1
    qx, qy = bool((ux >> 22) & 1), bool((uy >> 22) & 1)
    if qx != qy:
        return (not qx) if not neg else qx
    px, py = ux & ((1 << 22) - 1), uy & ((1 << 22) - 1)
    return px <= py if not neg else px >= py


def insertion_sort_bits32(bits: list[int], descending: bool = False) -> list[int]:
    out: list[int] = []
    for u in bits:
        i = len(out)
        if descending:  # u moves left past elements it strictly follows in totalOrder
            while i > 0 and total_order_le32(out[i - 1], u) and not total_order_le32(u, out[i - 1]):
                i -= 1
        else:
            while i > 0 and total_order_le32(u, out[i - 1]) and not total_order_le32(out[i - 1], u):
                i -= 1
        out.insert(i, u)
    return out


SPECIAL32 = [0xFFC00000, 0xFF800001, 0xFF800000, 0xFF7FFFFF, 0xBF800000, 0x80000001, 0x80000000,
             0x00000000, 0x00000001, 0x3F800000, 0x7F7FFFFF, 0x7F800000, 0x7F800001, 0x7FC00000,
             0x7FFFFFFF]  # -qNaN -sNaN -inf -max -1 -denorm -0 +0 +denorm 1 max inf sNaN qNaN qNaN(max)

assert math.isnan(bits_to_f(0x7FF8000000000000))

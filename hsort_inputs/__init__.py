"""Seeded synthetic inputs for the heterogeneous float64 sort (tests + bench).

Shared by both sides of every parity check (the oracle in ``oracle/`` and the CUDA path in
``paper_conf_ipps_gowanlockk18a_b200/``) and holding none of the method's arithmetic: it only
produces input arrays A.  The recipe follows the paper's workload — uniformly
distributed 64-bit floats (§IV-A) — plus the normal / zipf-dup skew of
BASELINE.json configs[3] and edge-case mixes.  Generation is counter-based splitmix64, so it is
bit-reproducible for any thread count.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libhsort_inputs.so")
_SRC = os.path.join(_HERE, "gen.cpp")
_lock = threading.Lock()
_lib = None

DISTS = {
    "uniform": 0,
    "normal": 1,
    "zipf_dup": 2,
    "special": 3,
    "random_bits": 4,
    "sorted": 5,
    "reverse": 6,
    "all_equal": 7,
    "few_distinct": 8,
    "closed_form": 9,
    "salted": 10,
    "uniform_pm1": 11,
}


def build(force: bool = False) -> str:
    """Compile gen.cpp into libhsort_inputs.so (in-tree)."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        subprocess.check_call(
            ["g++", "-O3", "-std=c++17", "-shared", "-fPIC", "-pthread", _SRC, "-o", _SO + ".tmp"]
        )
        os.replace(_SO + ".tmp", _SO)
    return _SO


def _load():
    global _lib
    with _lock:
        if _lib is None:
            build()
            lib = ctypes.CDLL(_SO)
            lib.hsort_inputs_generate.argtypes = [
                ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int, ctypes.c_uint64, ctypes.c_int]
            lib.hsort_inputs_generate.restype = ctypes.c_int
            lib.hsort_inputs_special.argtypes = [ctypes.c_void_p]
            lib.hsort_inputs_num_special.restype = ctypes.c_int
            _lib = lib
    return _lib


def generate(dist: str, n: int, seed: int, out: np.ndarray | None = None, threads: int = 0) -> np.ndarray:
    """Return (or fill ``out`` with) n float64 values of distribution ``dist`` for ``seed``.

    ``out`` may be any writable C-contiguous float64 host buffer (numpy array, or the numpy
    view of a pinned torch tensor).
    """
    lib = _load()
    if out is None:
        out = np.empty(n, dtype=np.float64)
    assert out.dtype == np.float64 and out.flags.c_contiguous and out.size >= n
    rc = lib.hsort_inputs_generate(out.ctypes.data, n, DISTS[dist], seed & (2**64 - 1), threads)
    if rc != 0:
        raise ValueError(f"unknown distribution {dist!r}")
    return out[:n] if out.size != n else out


def special_alphabet() -> np.ndarray:
    """The 15 special float64 bit patterns (±NaN, ±inf, ±DBL_MAX, ±1, ±denorm-min, ±0, ...)."""
    lib = _load()
    k = lib.hsort_inputs_num_special()
    a = np.empty(k, dtype=np.uint64)
    lib.hsort_inputs_special(a.ctypes.data)
    return a

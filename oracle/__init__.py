"""Python face of the CPU oracle (oracle/oracle.cpp).

TEST INFRASTRUCTURE ONLY: imported by tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / ``--impl reference`` leg — never by the product package
``paper_conf_ipps_gowanlockk18a_b200``.  It shares no code with the CUDA path.

Every function follows the passage cited in oracle.cpp; pins live in tests/test_oracle_*.py.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.cpp")
_SO = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

_U64 = ctypes.c_uint64
_P = ctypes.c_void_p


_PAR_SRC = os.path.join(_HERE, "par_baseline.cpp")
_PAR_SO = os.path.join(_HERE, "libparbaseline.so")
_par = None


def build_par(force: bool = False) -> str:
    """Compile the parallel-CPU baseline (GNU parallel-mode sort, -fopenmp) into its own library."""
    if force or not os.path.exists(_PAR_SO) or os.path.getmtime(_PAR_SO) < os.path.getmtime(_PAR_SRC):
        subprocess.check_call(["g++", "-O2", "-std=c++20", "-fopenmp", "-shared", "-fPIC", _PAR_SRC,
                               "-o", _PAR_SO + ".tmp"])
        os.replace(_PAR_SO + ".tmp", _PAR_SO)
    return _PAR_SO


def par_sort_f64(A, threads: int = 0) -> np.ndarray:
    """The parallel-CPU baseline: __gnu_parallel::sort under totalOrder on `threads` cores."""
    global _par
    with _lock:
        if _par is None:
            build_par()
            lib = ctypes.CDLL(_PAR_SO)
            lib.par_sort_f64.argtypes = [_P, _P, _U64, ctypes.c_int]
            lib.par_sort_f64.restype = None
            lib.par_max_threads.argtypes = []
            lib.par_max_threads.restype = ctypes.c_int
            lib.par_multiway_merge_u64.argtypes = [_P, _P, ctypes.c_int, _P, ctypes.c_int]
            lib.par_multiway_merge_u64.restype = None
            _par = lib
    A = np.ascontiguousarray(A, dtype=np.float64)
    B = np.empty_like(A)
    _par.par_sort_f64(A.ctypes.data, B.ctypes.data, A.size, int(threads))
    return B


def par_multiway_merge_u64(keys, off, threads: int = 0) -> np.ndarray:
    """CPU-merge reference: __gnu_parallel::multiway_merge of the sorted runs keys[off[j]:off[j+1]]."""
    par_sort_f64(np.zeros(0))  # loads the library
    keys = np.ascontiguousarray(keys, dtype=np.uint64)
    off = np.ascontiguousarray(off, dtype=np.uint64)
    out = np.empty(int(off[-1] - off[0]), dtype=np.uint64)
    _par.par_multiway_merge_u64(keys.ctypes.data, off.ctypes.data, off.size - 1, out.ctypes.data,
                                int(threads))
    return out


def build(force: bool = False) -> str:
    """Compile oracle.cpp into liboracle.so (serial, -O2, C++20)."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        subprocess.check_call(
            ["g++", "-O2", "-std=c++20", "-shared", "-fPIC", _SRC, "-o", _SO + ".tmp"])
        os.replace(_SO + ".tmp", _SO)
    return _SO


def _load():
    global _lib
    with _lock:
        if _lib is None:
            build()
            lib = ctypes.CDLL(_SO)
            sig = {
                "oracle_total_order_cmp": ([ctypes.c_double, ctypes.c_double], ctypes.c_int),
                "oracle_sort_f64": ([_P, _P, _U64], None),
                "oracle_sort_u64": ([_P, _P, _U64], None),
                "oracle_key": ([_U64], _U64),
                "oracle_key_inv": ([_U64], _U64),
                "oracle_keys_from_f64": ([_P, _P, _U64], None),
                "oracle_f64_from_keys": ([_P, _P, _U64], None),
                "oracle_digit_histograms": ([_P, _U64, _P], None),
                "oracle_counting_sort_pass": ([_P, _P, _U64, ctypes.c_int], None),
                "oracle_merge_runs": ([_P, _P, ctypes.c_int, _P], None),
                "oracle_corank": ([_P, _P, ctypes.c_int, _U64, _P], None),
                "oracle_pipemerge_count": ([_U64, ctypes.c_int], _U64),
                "oracle_is_sorted_f64": ([_P, _U64], ctypes.c_int),
                "oracle_multiset_hash": ([_P, _U64, _P], None),
                "oracle_sort_pairs_f64": ([_P, _P, _P, _P, _U64], None),
                "oracle_sort_f32": ([_P, _P, _U64, ctypes.c_int], None),
                "oracle_sort_desc_f64": ([_P, _P, _U64], None),
                "oracle_sort_pairs_u64": ([_P, _P, _P, _P, _U64], None),
            }
            for name, (args, res) in sig.items():
                f = getattr(lib, name)
                f.argtypes = args
                f.restype = res
            _lib = lib
    return _lib


def _c(a: np.ndarray, dtype) -> np.ndarray:
    return np.ascontiguousarray(a, dtype=dtype)


def total_order_cmp(a: float, b: float) -> int:
    return _load().oracle_total_order_cmp(a, b)


def sort_f64(A: np.ndarray) -> np.ndarray:
    """B = A sorted ascending under IEEE 754 totalOrder."""
    A = _c(A, np.float64)
    B = np.empty_like(A)
    _load().oracle_sort_f64(A.ctypes.data, B.ctypes.data, A.size)
    return B


def sort_u64(K: np.ndarray) -> np.ndarray:
    K = _c(K, np.uint64)
    B = np.empty_like(K)
    _load().oracle_sort_u64(K.ctypes.data, B.ctypes.data, K.size)
    return B


def key(u: int) -> int:
    return _load().oracle_key(u)


def key_inv(k: int) -> int:
    return _load().oracle_key_inv(k)


def keys_from_f64(A: np.ndarray) -> np.ndarray:
    A = _c(A, np.float64)
    K = np.empty(A.size, dtype=np.uint64)
    _load().oracle_keys_from_f64(A.ctypes.data, K.ctypes.data, A.size)
    return K


def f64_from_keys(K: np.ndarray) -> np.ndarray:
    K = _c(K, np.uint64)
    B = np.empty(K.size, dtype=np.float64)
    _load().oracle_f64_from_keys(K.ctypes.data, B.ctypes.data, K.size)
    return B


def digit_histograms(K: np.ndarray) -> np.ndarray:
    K = _c(K, np.uint64)
    h = np.zeros((8, 256), dtype=np.uint64)
    _load().oracle_digit_histograms(K.ctypes.data, K.size, h.ctypes.data)
    return h


def counting_sort_pass(K: np.ndarray, digit: int) -> np.ndarray:
    K = _c(K, np.uint64)
    out = np.empty_like(K)
    _load().oracle_counting_sort_pass(K.ctypes.data, out.ctypes.data, K.size, digit)
    return out


def _pack_runs(runs):
    runs = [_c(r, np.uint64) for r in runs]
    off = np.zeros(len(runs) + 1, dtype=np.uint64)
    for j, r in enumerate(runs):
        off[j + 1] = off[j] + r.size
    keys = np.concatenate(runs) if runs else np.zeros(0, dtype=np.uint64)
    return _c(keys, np.uint64), off


def sort_f32(A, descending: bool = False) -> np.ndarray:
    """float32 keys sorted by binary32 totalOrder (or its reverse) (oracle.cpp)."""
    A = np.ascontiguousarray(A, dtype=np.float32)
    B = np.empty_like(A)
    _load().oracle_sort_f32(A.ctypes.data, B.ctypes.data, A.size, int(descending))
    return B


def sort_desc_f64(A) -> np.ndarray:
    A = np.ascontiguousarray(A, dtype=np.float64)
    B = np.empty_like(A)
    _load().oracle_sort_desc_f64(A.ctypes.data, B.ctypes.data, A.size)
    return B


def sort_pairs_f64(A, V):
    """(B, VB): the pairs stably sorted by A under IEEE totalOrder (oracle.cpp)."""
    A = np.ascontiguousarray(A, dtype=np.float64)
    V = np.ascontiguousarray(V, dtype=np.uint64)
    assert A.size == V.size
    B = np.empty_like(A)
    VB = np.empty_like(V)
    _load().oracle_sort_pairs_f64(A.ctypes.data, V.ctypes.data, B.ctypes.data, VB.ctypes.data, A.size)
    return B, VB


def sort_pairs_u64(A, V):
    A = np.ascontiguousarray(A, dtype=np.uint64)
    V = np.ascontiguousarray(V, dtype=np.uint64)
    assert A.size == V.size
    B = np.empty_like(A)
    VB = np.empty_like(V)
    _load().oracle_sort_pairs_u64(A.ctypes.data, V.ctypes.data, B.ctypes.data, VB.ctypes.data, A.size)
    return B, VB


def merge_runs(runs) -> np.ndarray:
    keys, off = _pack_runs(runs)
    out = np.empty(keys.size, dtype=np.uint64)
    _load().oracle_merge_runs(keys.ctypes.data, off.ctypes.data, len(runs), out.ctypes.data)
    return out


def corank(runs, o: int) -> np.ndarray:
    keys, off = _pack_runs(runs)
    ranks = np.zeros(len(runs), dtype=np.uint64)
    _load().oracle_corank(keys.ctypes.data, off.ctypes.data, len(runs), o, ranks.ctypes.data)
    return ranks


def pipemerge_count(n_b: int, n_gpu: int) -> int:
    return _load().oracle_pipemerge_count(n_b, n_gpu)


def is_sorted_f64(B: np.ndarray) -> bool:
    B = _c(B, np.float64)
    return bool(_load().oracle_is_sorted_f64(B.ctypes.data, B.size))


def multiset_hash(A: np.ndarray) -> tuple[int, int]:
    A = _c(A, np.float64)
    out = np.zeros(2, dtype=np.uint64)
    _load().oracle_multiset_hash(A.ctypes.data, A.size, out.ctypes.data)
    return int(out[0]), int(out[1])

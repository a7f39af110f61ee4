"""paper_conf_ipps_gowanlockk18a_b200 — B200-native heterogeneous float64 sort.

Thin Python binding (argument marshalling only) over the C ABI in ``include/hsort.h``
(``libhsort.so``, built in-tree from ``csrc/``).  Every step of the sort runs in the library:
the sm_100a kernels (radix.cu, merge.cu) and the native host runtime (api.cpp, pool.cpp,
host_merge.cpp).  There is no Python or CPU fallback: if the extension is missing this module
raises on import of any entry point.

Method: Gowanlock & Karsin, "Sorting Large Datasets with Heterogeneous CPU/GPU Architectures"
(PAPER.md; §III).  Names follow the paper: A (input), B (output), W (working memory),
n, n_b (batches), b_s (batch size), n_s (streams/slots), p_s (pinned buffer), n_GPU.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading
from typing import Any

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libhsort.so")

_U64 = ctypes.c_uint64
_P = ctypes.c_void_p
_I = ctypes.c_int
_lock = threading.Lock()
_lib = None

STATUS = {
    0: "HSORT_OK", -1: "HSORT_ERR_INVALID", -2: "HSORT_ERR_NOT_INITIALIZED",
    -3: "HSORT_ERR_HOST_OOM", -4: "HSORT_ERR_DEVICE_OOM", -5: "HSORT_ERR_CUDA",
    -6: "HSORT_ERR_NCCL", -7: "HSORT_ERR_BUSY", -8: "HSORT_ERR_INTERNAL",
}
MODES = {0: "BLINE", 1: "RESIDENT", 2: "STREAM"}


class HsortError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"{STATUS.get(code, code)}: {msg}")
        self.code = code


class hsort_stats(ctypes.Structure):
    _fields_ = [
        ("n", _U64), ("b_s", _U64), ("n_b", _U64),
        ("n_gpus", ctypes.c_int32), ("n_s", ctypes.c_int32), ("mode", ctypes.c_int32),
        ("passes_run", ctypes.c_int32), ("passes_skipped", ctypes.c_int32),
        ("direct_in", ctypes.c_int32), ("direct_out", ctypes.c_int32), ("merge_k", ctypes.c_int32),
        ("merge_gpu_fraction", ctypes.c_double),
        ("t_total", ctypes.c_double), ("t_sort_phase", ctypes.c_double),
        ("t_merge_phase", ctypes.c_double), ("t_gpu_sort", ctypes.c_double),
        ("t_h2d", ctypes.c_double), ("t_d2h", ctypes.c_double), ("t_stage", ctypes.c_double),
        ("t_merge_cpu", ctypes.c_double), ("t_merge_gpu", ctypes.c_double),
        ("t_init", ctypes.c_double),
        ("bytes_h2d", _U64), ("bytes_d2h", _U64), ("t_host_alloc", ctypes.c_double),
        ("pipe_merges", _U64), ("t_pipemerge", ctypes.c_double), ("t_pipemerge_wait", ctypes.c_double),
        ("msd_buckets", ctypes.c_int32), ("reserved0", ctypes.c_int32), ("t_setup", ctypes.c_double),
    ]


class hsort_plan_t(ctypes.Structure):
    _fields_ = [
        ("n", _U64), ("b_s", _U64), ("n_b", _U64),
        ("n_gpus", ctypes.c_int32), ("n_s", ctypes.c_int32), ("mode", ctypes.c_int32),
        ("last_batch", _U64), ("device_bytes_per_gpu", _U64), ("host_bytes", _U64),
        ("batches_per_stream", ctypes.c_double), ("schedule", ctypes.c_int32),
    ]


# symbol -> (argtypes, restype); the full ABI of include/hsort.h
SIGNATURES = {
    "hsort_init": ([], _I),
    "hsort_finalize": ([], _I),
    "hsort_sort": ([_P, _P, _U64, _U64, _I], _I),
    "hsort_sort_u64": ([_P, _P, _U64, _U64, _I], _I),
    "hsort_sort_lane": ([_I, _P, _P, _U64, _U64], _I),
    "hsort_sort_typed": ([_P, _P, _U64, _I, _I], _I),
    "hsort_sort_device_typed": ([_P, _P, _U64, _I, _I, _P], _I),
    "hsort_sort_pairs": ([_P, _P, _P, _P, _U64], _I),
    "hsort_sort_pairs_u64": ([_P, _P, _P, _P, _U64], _I),
    "hsort_sort_pairs_ex": ([_P, _P, _P, _P, _U64, _U64, _I, _I], _I),
    "hsort_sort_device_pairs": ([_P, _P, _P, _P, _U64, _I, _P], _I),
    "hsort_set_option": ([ctypes.c_char_p, ctypes.c_int64], _I),
    "hsort_get_option": ([ctypes.c_char_p, ctypes.POINTER(ctypes.c_int64)], _I),
    "hsort_get_stats": ([ctypes.POINTER(hsort_stats)], _I),
    "hsort_last_error": ([], ctypes.c_char_p),
    "hsort_version": ([], ctypes.c_char_p),
    "hsort_plan": ([_U64, _U64, _I, _U64, ctypes.POINTER(hsort_plan_t)], _I),
    "hsort_sort_device": ([_P, _P, _U64, _P], _I),
    "hsort_sort_device_keys": ([_P, _P, _U64, _I, _I, _P], _I),
    "hsort_device_histograms": ([_P, _U64, _I, _P, _P], _I),
    "hsort_device_radix_pass": ([_P, _P, _U64, _I, _P], _I),
    "hsort_device_corank": ([_P, _P, _I, _U64, _U64, _P, _P], _I),
    "hsort_device_merge": ([_P, _P, _I, _P, _I, _P], _I),
    "hsort_par_memcpy": ([_P, _P, _U64, _I], _I),
    "hsort_host_merge": ([_P, _P, _I, _P, _I, _I], _I),
    "hsort_host_corank": ([_P, _P, _I, _U64, _P], _I),
    "hsort_pipemerge_count": ([_U64, _I], _U64),
    "hsort_device_count": ([], _I),
    "hsort_get_kernel_times": ([ctypes.POINTER(ctypes.c_float), _I, ctypes.POINTER(_I)], _I),
    "hsort_device_upper_bounds": ([_P, _U64, _P, _U64, _P, _P], _I),
    "hsort_get_last_plan": ([ctypes.POINTER(_I), ctypes.POINTER(_I), ctypes.POINTER(_U64)], _I),
    "hsort_host_upper_bounds": ([_P, _U64, _P, _U64, _P], _I),
    "hsort_get_launch_count": ([], _U64),
    "hsort_sample_positions": ([_U64, _U64, _P], _I),
    "hsort_select_splitters": ([_P, _U64, _I, _P], _I),
}


def build(force: bool = False, jobs: int = 8) -> str:
    """Compile libhsort.so in-tree (nvcc -gencode arch=compute_100a,code=sm_100a)."""
    if force:
        subprocess.check_call(["make", "-C", _HERE, "clean"])
    subprocess.check_call(["make", "-C", _HERE, f"-j{jobs}"], stdout=subprocess.DEVNULL)
    return LIB_PATH


def lib() -> ctypes.CDLL:
    """Load libhsort.so; raises if it has not been built (no fallback path exists)."""
    global _lib
    with _lock:
        if _lib is None:
            if not os.path.exists(LIB_PATH):
                raise ImportError(
                    f"{LIB_PATH} not found: build it with __graft_entry__.build() or "
                    f"`make -C {_HERE}` (the CUDA extension is required; there is no fallback)")
            L = ctypes.CDLL(LIB_PATH)
            for name, (args, res) in SIGNATURES.items():
                f = getattr(L, name)
                f.argtypes = args
                f.restype = res
            _lib = L
    return _lib


def _check(rc: int) -> None:
    if rc != 0:
        msg = lib().hsort_last_error()
        raise HsortError(rc, msg.decode() if msg else "")


def _host_ptr(x: Any, dtype) -> tuple[int, int]:
    """(address, n elements) of a C-contiguous host buffer (numpy array or CPU torch tensor)."""
    if isinstance(x, np.ndarray):
        if x.dtype != dtype or not x.flags.c_contiguous:
            raise TypeError(f"expected C-contiguous {np.dtype(dtype)} array")
        return x.ctypes.data, x.size
    try:
        import torch
    except ImportError:  # pragma: no cover
        torch = None
    if torch is not None and isinstance(x, torch.Tensor):
        want = {np.float64: torch.float64, np.uint64: torch.uint64}[dtype]
        if x.device.type != "cpu" or x.dtype != want or not x.is_contiguous():
            raise TypeError(f"expected contiguous CPU tensor of {want}")
        return x.data_ptr(), x.numel()
    raise TypeError(f"unsupported buffer type {type(x)}")


def _dev_ptr(t) -> int:
    if hasattr(t, "data_ptr") and getattr(t, "is_cuda", False):
        return t.data_ptr()
    if isinstance(t, int):
        return t
    raise TypeError("expected a CUDA torch tensor or a raw device address")


def _stream_ptr(stream) -> int | None:
    if stream is None:
        try:
            import torch
            return torch.cuda.current_stream().cuda_stream
        except Exception:  # pragma: no cover
            return None
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


# ---- lifecycle -------------------------------------------------------------------------------
def hsort_init() -> None:
    _check(lib().hsort_init())


def hsort_finalize() -> None:
    _check(lib().hsort_finalize())


def hsort_device_count() -> int:
    return lib().hsort_device_count()


def hsort_version() -> str:
    return lib().hsort_version().decode()


def hsort_last_error() -> str:
    return lib().hsort_last_error().decode()


# ---- the sort --------------------------------------------------------------------------------
def hsort_sort(A, B=None, batch_elems: int = 0, n_gpus: int = 0):
    """B = A sorted under IEEE 754 totalOrder (host -> host).  B=None allocates; B may be A."""
    a, n = _host_ptr(A, np.float64)
    if B is None:
        B = np.empty(n, dtype=np.float64)
    b, nb = _host_ptr(B, np.float64)
    if nb != n:
        raise ValueError("A and B must have the same length")
    _check(lib().hsort_sort(a, b, n, batch_elems, n_gpus))
    return B


def hsort_sort_lane(lane: int, A, B=None, batch_elems: int = 0):
    """hsort_sort on GPU context `lane` alone; calls on different lanes may run concurrently
    (the ctypes call releases the GIL)."""
    a, n = _host_ptr(A, np.float64)
    if B is None:
        B = np.empty(n, dtype=np.float64)
    b, nb = _host_ptr(B, np.float64)
    if nb != n:
        raise ValueError("A and B must have the same length")
    _check(lib().hsort_sort_lane(lane, a, b, n, batch_elems))
    return B


def hsort_sort_u64(A, B=None, batch_elems: int = 0, n_gpus: int = 0):
    a, n = _host_ptr(A, np.uint64)
    if B is None:
        B = np.empty(n, dtype=np.uint64)
    b, nb = _host_ptr(B, np.uint64)
    if nb != n:
        raise ValueError("A and B must have the same length")
    _check(lib().hsort_sort_u64(a, b, n, batch_elems, n_gpus))
    return B


KEY_F64, KEY_F32 = 0, 1


def hsort_sort_typed(A, B=None, descending: bool = False):
    """B = A sorted by IEEE totalOrder (descending: its reverse); A float64 or float32 numpy array
    (host -> host; float64 ascending = hsort_sort, else one GPU, one batch)."""
    if not isinstance(A, np.ndarray) or A.dtype not in (np.float64, np.float32) or not A.flags.c_contiguous:
        raise TypeError("expected a C-contiguous float64 or float32 numpy array")
    if B is None:
        B = np.empty_like(A)
    if not isinstance(B, np.ndarray) or B.dtype != A.dtype or B.size != A.size or not B.flags.c_contiguous:
        raise ValueError("B must be a C-contiguous array of A's dtype and length")
    kt = KEY_F64 if A.dtype == np.float64 else KEY_F32
    _check(lib().hsort_sort_typed(A.ctypes.data, B.ctypes.data, A.size, kt, int(descending)))
    return B


def hsort_sort_pairs(A, V, B=None, VB=None):
    """(B, VB) = the pairs (A[i], V[i]) stably sorted by A under IEEE totalOrder (host -> host,
    one GPU, n <= 2^30).  A float64, V uint64 payloads (e.g. np.arange(n): stable argsort)."""
    a, n = _host_ptr(A, np.float64)
    v, nv = _host_ptr(V, np.uint64)
    if B is None:
        B = np.empty(n, dtype=np.float64)
    if VB is None:
        VB = np.empty(n, dtype=np.uint64)
    b, nb = _host_ptr(B, np.float64)
    vb, nvb = _host_ptr(VB, np.uint64)
    if not (n == nv == nb == nvb):
        raise ValueError("A, V, B, VB must have the same length")
    _check(lib().hsort_sort_pairs(a, v, b, vb, n))
    return B, VB


def hsort_sort_pairs_u64(A, V, B=None, VB=None):
    a, n = _host_ptr(A, np.uint64)
    v, nv = _host_ptr(V, np.uint64)
    if B is None:
        B = np.empty(n, dtype=np.uint64)
    if VB is None:
        VB = np.empty(n, dtype=np.uint64)
    b, nb = _host_ptr(B, np.uint64)
    vb, nvb = _host_ptr(VB, np.uint64)
    if not (n == nv == nb == nvb):
        raise ValueError("A, V, B, VB must have the same length")
    _check(lib().hsort_sort_pairs_u64(a, v, b, vb, n))
    return B, VB


def hsort_sort_pairs_ex(A, V, B=None, VB=None, batch_elems: int = 0, n_gpus: int = 1):
    """Key/value sort with hsort_sort's batch size and GPU count (RESIDENT key/value plan: stable
    batch sorts in HBM + the key/value K4/K5 merge).  A float64 or uint64, V uint64 payloads."""
    f64 = A.dtype == np.float64 if isinstance(A, np.ndarray) else A.dtype.is_floating_point
    dt = np.float64 if f64 else np.uint64
    a, n = _host_ptr(A, dt)
    v, nv = _host_ptr(V, np.uint64)
    if B is None:
        B = np.empty(n, dtype=dt)
    if VB is None:
        VB = np.empty(n, dtype=np.uint64)
    b, nb = _host_ptr(B, dt)
    vb, nvb = _host_ptr(VB, np.uint64)
    if not (n == nv == nb == nvb):
        raise ValueError("A, V, B, VB must have the same length")
    _check(lib().hsort_sort_pairs_ex(a, v, b, vb, n, batch_elems, n_gpus, int(f64)))
    return B, VB


def hsort_set_option(key: str, value: int) -> None:
    _check(lib().hsort_set_option(key.encode(), int(value)))


def hsort_get_option(key: str) -> int:
    v = ctypes.c_int64()
    _check(lib().hsort_get_option(key.encode(), ctypes.byref(v)))
    return v.value


def hsort_get_stats() -> dict:
    s = hsort_stats()
    _check(lib().hsort_get_stats(ctypes.byref(s)))
    d = {f: getattr(s, f) for f, _ in hsort_stats._fields_}
    d["mode_name"] = MODES.get(d["mode"], "?")
    return d


def hsort_plan(n: int, batch_elems: int = 0, n_gpus: int = 1, device_bytes: int = 0) -> dict:
    p = hsort_plan_t()
    _check(lib().hsort_plan(n, batch_elems, n_gpus, device_bytes, ctypes.byref(p)))
    d = {f: getattr(p, f) for f, _ in hsort_plan_t._fields_}
    d["mode_name"] = MODES.get(d["mode"], "?")
    return d


# ---- device-resident entry points (torch CUDA tensors) -----------------------------------------
def hsort_sort_device(d_in, d_out, stream=None) -> None:
    """d_out = totalOrder-sorted d_in (float64 CUDA tensors, same length); stream-ordered."""
    n = d_in.numel()
    if d_out.numel() != n:
        raise ValueError("length mismatch")
    _check(lib().hsort_sort_device(_dev_ptr(d_in), _dev_ptr(d_out), n, _stream_ptr(stream)))


def hsort_sort_device_keys(d_in, d_out, in_f64: bool, out_f64: bool, stream=None) -> None:
    n = d_in.numel()
    _check(lib().hsort_sort_device_keys(_dev_ptr(d_in), _dev_ptr(d_out), n, int(in_f64),
                                        int(out_f64), _stream_ptr(stream)))


def hsort_sort_device_typed(d_in, d_out, descending: bool = False, stream=None) -> None:
    """d_out = d_in sorted by IEEE totalOrder (or its reverse); float64 or float32 CUDA tensors."""
    import torch
    kt = {torch.float64: KEY_F64, torch.float32: KEY_F32}[d_in.dtype]
    if d_out.dtype != d_in.dtype or d_out.numel() != d_in.numel():
        raise ValueError("d_out must match d_in in dtype and length")
    _check(lib().hsort_sort_device_typed(_dev_ptr(d_in), _dev_ptr(d_out), d_in.numel(), kt,
                                         int(descending), _stream_ptr(stream)))


def hsort_sort_device_pairs(d_keys_in, d_vals_in, d_keys_out, d_vals_out, keys_f64: bool = True,
                            stream=None) -> None:
    """(d_keys_out, d_vals_out) = pairs stably sorted by key; 8-byte CUDA tensors, stream-ordered."""
    n = d_keys_in.numel()
    if not (d_vals_in.numel() == d_keys_out.numel() == d_vals_out.numel() == n):
        raise ValueError("length mismatch")
    _check(lib().hsort_sort_device_pairs(_dev_ptr(d_keys_in), _dev_ptr(d_vals_in),
                                         _dev_ptr(d_keys_out), _dev_ptr(d_vals_out), n,
                                         int(keys_f64), _stream_ptr(stream)))


def hsort_device_histograms(d_keys, in_f64: bool, d_hist, stream=None) -> None:
    _check(lib().hsort_device_histograms(_dev_ptr(d_keys), d_keys.numel(), int(in_f64),
                                         _dev_ptr(d_hist), _stream_ptr(stream)))


def hsort_device_radix_pass(d_src, d_dst, digit: int, stream=None) -> None:
    _check(lib().hsort_device_radix_pass(_dev_ptr(d_src), _dev_ptr(d_dst), d_src.numel(), digit,
                                         _stream_ptr(stream)))


def _offsets(off) -> np.ndarray:
    return np.ascontiguousarray(np.asarray(off, dtype=np.uint64))


def hsort_device_corank(d_keys, off, step: int, n_bounds: int, d_ranks, stream=None) -> None:
    o = _offsets(off)
    _check(lib().hsort_device_corank(_dev_ptr(d_keys), o.ctypes.data, o.size - 1, step, n_bounds,
                                     _dev_ptr(d_ranks), _stream_ptr(stream)))


def hsort_device_merge(d_keys, off, d_out, out_f64: bool, stream=None) -> None:
    o = _offsets(off)
    _check(lib().hsort_device_merge(_dev_ptr(d_keys), o.ctypes.data, o.size - 1, _dev_ptr(d_out),
                                    int(out_f64), _stream_ptr(stream)))


# ---- host-native components -------------------------------------------------------------------
def hsort_par_memcpy(dst: np.ndarray, src: np.ndarray, threads: int = 0) -> None:
    if dst.nbytes < src.nbytes:
        raise ValueError("dst too small")
    _check(lib().hsort_par_memcpy(dst.ctypes.data, src.ctypes.data, src.nbytes, threads))


def hsort_host_merge(keys: np.ndarray, off, out_f64: bool = False, threads: int = 0) -> np.ndarray:
    keys = np.ascontiguousarray(keys, dtype=np.uint64)
    o = _offsets(off)
    total = int(o[-1] - o[0])
    out = np.empty(total, dtype=np.float64 if out_f64 else np.uint64)
    _check(lib().hsort_host_merge(keys.ctypes.data, o.ctypes.data, o.size - 1, out.ctypes.data,
                                  int(out_f64), threads))
    return out


def hsort_host_corank(keys: np.ndarray, off, o: int) -> np.ndarray:
    keys = np.ascontiguousarray(keys, dtype=np.uint64)
    of = _offsets(off)
    r = np.zeros(of.size - 1, dtype=np.uint64)
    _check(lib().hsort_host_corank(keys.ctypes.data, of.ctypes.data, of.size - 1, o, r.ctypes.data))
    return r


def hsort_get_last_plan() -> dict:
    """Plan of the last GPUSort on the current device: passes run, elision, outliers."""
    na, el, no = _I(), _I(), _U64()
    _check(lib().hsort_get_last_plan(ctypes.byref(na), ctypes.byref(el), ctypes.byref(no)))
    return {"num_active": na.value, "elided": bool(el.value), "n_outliers": no.value}


def hsort_get_kernel_times() -> dict:
    """Per-kernel durations (ms) of the last device sort (needs option kernel_timing=1)."""
    buf = (ctypes.c_float * 16)()
    na = _I()
    m = lib().hsort_get_kernel_times(buf, 16, ctypes.byref(na))
    if m < 0:
        _check(m)
    v = list(buf[:m])
    out = {"num_active": na.value}
    if m >= 11:
        out.update(hist=v[0], scan=v[1], passes=v[2:10], copy=v[10])
    return out


def hsort_device_upper_bounds(d_keys, d_values, d_out, stream=None) -> None:
    _check(lib().hsort_device_upper_bounds(_dev_ptr(d_keys), d_keys.numel(), _dev_ptr(d_values),
                                           d_values.numel(), _dev_ptr(d_out), _stream_ptr(stream)))


def hsort_host_upper_bounds(keys: np.ndarray, values: np.ndarray) -> np.ndarray:
    keys = np.ascontiguousarray(keys, dtype=np.uint64)
    values = np.ascontiguousarray(values, dtype=np.uint64)
    out = np.empty(values.size, dtype=np.uint64)
    _check(lib().hsort_host_upper_bounds(keys.ctypes.data, keys.size, values.ctypes.data,
                                         values.size, out.ctypes.data))
    return out


def hsort_get_launch_count() -> int:
    """Kernels the library has launched since load (differences count a region's launches)."""
    return lib().hsort_get_launch_count()


def hsort_sample_positions(n: int, s: int) -> np.ndarray:
    """Regular sample positions of a sorted run of n keys (A13 splitter sampling)."""
    pos = np.zeros(s, dtype=np.uint64)
    _check(lib().hsort_sample_positions(n, s, pos.ctypes.data if s else None))
    return pos


def hsort_select_splitters(samples: np.ndarray, P: int) -> np.ndarray:
    """P - 1 splitters at the P-quantiles of the merged sorted samples (A13)."""
    samples = np.ascontiguousarray(samples, dtype=np.uint64)
    spl = np.zeros(max(P - 1, 0), dtype=np.uint64)
    _check(lib().hsort_select_splitters(samples.ctypes.data if samples.size else None, samples.size,
                                        P, spl.ctypes.data if spl.size else None))
    return spl


def hsort_pipemerge_count(n_b: int, n_gpus: int) -> int:
    return lib().hsort_pipemerge_count(n_b, n_gpus)


__all__ = [n for n in SIGNATURES] + ["HsortError", "build", "lib", "LIB_PATH"]

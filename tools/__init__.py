"""Measurement tools (not the oracle, not the product).

workcount: algorithmic work counters of the run-walk sweep (tools/workcount.c), the numerator of
the k_tm_walk roofline in bench.py.  Pinned in tests/test_workcount.py.
peaks: measured on-chip throughput ceilings (tools/peaks.cu: scattered 32-byte L1 / L2 loads,
shared-memory reads), the denominators of the on-chip roofline in bench.py.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libworkcount.so")
_PEAKS_SO = os.path.join(_HERE, "libpeaks.so")
_lib = None
_peaks = None


def build(force: bool = False) -> str:
    src = os.path.join(_HERE, "workcount.c")
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O2", "-std=c99", "-fPIC", "-shared", src, "-o", _SO])
    build_peaks(force)
    return _SO


def build_peaks(force: bool = False) -> str:
    src = os.path.join(_HERE, "peaks.cu")
    if force or not os.path.exists(_PEAKS_SO) or os.path.getmtime(_PEAKS_SO) < os.path.getmtime(src):
        nvcc = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
        subprocess.check_call([nvcc, "-O3", "-std=c++17", "-gencode", "arch=compute_100a,code=sm_100a", "-lineinfo",
                               "-Xcompiler", "-fPIC", "-shared", "-cudart", "static", src, "-o", _PEAKS_SO])
    return _PEAKS_SO


def measure_peaks(device: int = 0) -> dict:
    """Run the on-chip microbenchmarks on `device` (needs a GPU; ~0.1 s)."""
    global _peaks
    if _peaks is None:
        build_peaks()
        _peaks = C.CDLL(_PEAKS_SO)
        _peaks.peaks_measure.restype = C.c_int
        _peaks.peaks_measure.argtypes = [C.c_int, C.c_void_p]
    out = np.zeros(9, np.float64)
    rc = _peaks.peaks_measure(int(device), out.ctypes.data)
    if rc != 0:
        raise RuntimeError(f"peaks_measure failed ({rc})")
    keys = ("l1_scatter32_bytes_per_s", "l1_scatter32_requests_per_s", "l1_scatter32_requests_per_clk_sm",
            "l2_scatter32_bytes_per_s", "l2_scatter32_requests_per_s", "smem_read_bytes_per_s",
            "smem_read_bytes_per_clk_sm", "sms", "kernel_clock_mhz")
    return dict(zip(keys, out.tolist()))


class _Forest(C.Structure):
    _fields_ = [("n_trees", C.c_int32), ("tree_offset", C.c_void_p), ("feature", C.c_void_p),
                ("left", C.c_void_p), ("right", C.c_void_p), ("value", C.c_void_p)]


class _Counts(C.Structure):
    _fields_ = [("decisions", C.c_int64), ("runs", C.c_int64), ("run_decisions", C.c_int64),
                ("run_blocks", C.c_int64), ("resume_blocks", C.c_int64)]


def _load():
    global _lib
    if _lib is None:
        build()
        lib = C.CDLL(_SO)
        lib.wc_count.restype = C.c_int
        lib.wc_count.argtypes = [C.c_void_p, C.c_void_p, C.c_int64, C.c_int32, C.c_void_p, C.c_int32, C.c_void_p]
        _lib = lib
    return _lib


def count(models, features, freqs):
    """Work counters summed over the forest members of `models` (workloads.ModelSpec list) for
    every (kernel, clock) of `features` x `freqs`."""
    lib = _load()
    c = np.ascontiguousarray
    features = c(features, dtype=np.float32)
    freqs = c(freqs, dtype=np.float32)
    n_k, F = features.shape
    out = _Counts()
    for m in models:
        if m is None or m.forest_weight == 0.0:
            continue
        keep = [c(m.tree_offset, dtype=np.int64), c(m.feature, dtype=np.int32), c(m.left, dtype=np.int32),
                c(m.right, dtype=np.int32), c(m.value, dtype=np.float32)]
        f = _Forest(len(keep[0]) - 1, *[a.ctypes.data for a in keep])
        if lib.wc_count(C.byref(f), features.ctypes.data, n_k, F, freqs.ctypes.data, len(freqs), C.byref(out)) != 0:
            raise ValueError("wc_count: invalid arguments")
    return {k: int(getattr(out, k)) for k, _ in _Counts._fields_}

"""Measurement tools (not the oracle, not the product).

workcount: algorithmic work counters of the run-walk sweep (tools/workcount.c), the numerator of
the k_tm_walk roofline in bench.py.  Pinned in tests/test_workcount.py.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libworkcount.so")
_lib = None


def build(force: bool = False) -> str:
    src = os.path.join(_HERE, "workcount.c")
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O2", "-std=c99", "-fPIC", "-shared", src, "-o", _SO])
    return _SO


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

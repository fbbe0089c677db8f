"""CPU oracle for SYnergy's predict+select path — TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / `--impl reference` legs
may import this package.  The product package (paper_conf_sc_fandccfc23_b200/) never imports
it and shares no code with it (oracle.c restates the data format on its own).

Functions (each follows oracle.c, which cites PAPER.md):
  build()                                     compile liboracle.so (gcc, -ffp-contract=off)
  model_eval(spec, x)                         raw fp64 model output for one input vector
  predict(w_or_args...)                       normalised / raw fp32 predictions
  select(S, E, default_idx, targets)          int32 choices (+ runner-up gaps)
  sweep(workload)                             predict + select

Parity status: pinned (see tests/test_oracle_*.py and DESIGN.md "Oracle pins").
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    src = os.path.join(_HERE, "oracle.c")
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < max(
            os.path.getmtime(src), os.path.getmtime(os.path.join(_HERE, "oracle.h"))):
        subprocess.check_call(["gcc", "-O2", "-std=c99", "-ffp-contract=off", "-fno-fast-math",
                               "-fPIC", "-shared", src, "-o", _SO, "-lm"])
    return _SO


class _Model(C.Structure):
    _fields_ = [("n_inputs", C.c_int32), ("linear_weight", C.c_double),
                ("lin_w", C.c_void_p), ("lin_b", C.c_double), ("forest_weight", C.c_double),
                ("n_trees", C.c_int32), ("tree_offset", C.c_void_p), ("feature", C.c_void_p),
                ("left", C.c_void_p), ("right", C.c_void_p), ("value", C.c_void_p),
                ("svr_weight", C.c_double), ("n_sv", C.c_int32), ("sv", C.c_void_p), ("dual_coef", C.c_void_p),
                ("svr_gamma", C.c_double), ("svr_intercept", C.c_double), ("in_mean", C.c_void_p),
                ("in_scale", C.c_void_p)]


def _load():
    global _lib
    if _lib is None:
        build()
        lib = C.CDLL(_SO)
        P = C.c_void_p
        lib.oracle_model_eval.restype = C.c_double
        lib.oracle_model_eval.argtypes = [P, P, P]
        lib.oracle_predict.restype = C.c_int
        lib.oracle_predict.argtypes = [P, P, P, C.c_int64, C.c_int32, P, C.c_int32, C.c_int32,
                                       P, P, P]
        lib.oracle_select.restype = C.c_int
        lib.oracle_select.argtypes = [P, P, C.c_int64, C.c_int32, C.c_int32, P, P, C.c_int32,
                                      P, P]
        lib.oracle_pareto.restype = C.c_int
        lib.oracle_pareto.argtypes = [P, P, C.c_int64, C.c_int32, P]
        lib.oracle_choice_error.restype = C.c_int
        lib.oracle_choice_error.argtypes = [P, P, C.c_int64, C.c_int32, C.c_int32, P, P, C.c_int32, P, P, P,
                                            P, P]
        lib.oracle_sweep4.restype = C.c_int
        lib.oracle_sweep4.argtypes = [P, P, C.c_int64, C.c_int32, P, C.c_int32, C.c_int32, P, P,
                                      C.c_int32, P, P]
        lib.oracle_sweep.restype = C.c_int
        lib.oracle_sweep.argtypes = [P, P, P, C.c_int64, C.c_int32, P, C.c_int32, C.c_int32,
                                     P, P, C.c_int32, P, P, P, P, P]
        _lib = lib
    return _lib


def _ptr(a):
    return None if a is None else a.ctypes.data


class _Keep:
    """Holds a ctypes model struct and the numpy arrays it points into."""

    def __init__(self, spec):
        c = np.ascontiguousarray
        self.arrays = dict(
            lin_w=None if spec.lin_w is None else c(spec.lin_w, dtype=np.float64),
            tree_offset=c(spec.tree_offset, dtype=np.int64), feature=c(spec.feature, dtype=np.int32),
            left=c(spec.left, dtype=np.int32), right=c(spec.right, dtype=np.int32),
            value=c(spec.value, dtype=np.float32))
        svr = getattr(spec, "svr_weight", 0.0)
        for k in ("sv", "dual_coef", "in_mean", "in_scale"):
            v = getattr(spec, k, None)
            self.arrays[k] = None if v is None else c(v, dtype=np.float32 if k == "sv" else np.float64)
        a = self.arrays
        n_trees = len(a["tree_offset"]) - 1 if spec.forest_weight != 0.0 else 0
        n_sv = 0 if (svr == 0.0 or a["sv"] is None) else int(a["sv"].shape[0])
        self.s = _Model(int(spec.n_inputs), float(spec.linear_weight), _ptr(a["lin_w"]),
                        float(spec.lin_b), float(spec.forest_weight), int(n_trees),
                        _ptr(a["tree_offset"]), _ptr(a["feature"]), _ptr(a["left"]),
                        _ptr(a["right"]), _ptr(a["value"]), float(svr), n_sv, _ptr(a["sv"]),
                        _ptr(a["dual_coef"]), float(getattr(spec, "svr_gamma", 0.0)),
                        float(getattr(spec, "svr_intercept", 0.0)), _ptr(a["in_mean"]), _ptr(a["in_scale"]))

    @property
    def ref(self):
        return C.byref(self.s)


class OracleError(RuntimeError):
    pass


def model_eval(spec, x, count_visits=False):
    lib = _load()
    k = _Keep(spec)
    x = np.ascontiguousarray(x, dtype=np.float32)
    v = np.zeros(1, np.int64)
    out = lib.oracle_model_eval(k.ref, _ptr(x), _ptr(v) if count_visits else None)
    return (out, int(v[0])) if count_visits else out


def predict(speedup, energy, features, freqs, default_idx, count_visits=False):
    lib = _load()
    ks, ke = _Keep(speedup), _Keep(energy)
    features = np.ascontiguousarray(features, dtype=np.float32)
    freqs = np.ascontiguousarray(freqs, dtype=np.float32)
    n_k, F = features.shape
    n_f = freqs.shape[0]
    S = np.empty((n_k, n_f), np.float32)
    E = np.empty((n_k, n_f), np.float32)
    v = np.zeros(1, np.int64)
    rc = lib.oracle_predict(ks.ref, ke.ref, _ptr(features), n_k, F, _ptr(freqs), n_f,
                            int(default_idx), _ptr(S), _ptr(E), _ptr(v))
    if rc != 0:
        raise OracleError("oracle_predict: invalid arguments")
    return (S, E, int(v[0])) if count_visits else (S, E)


def _targets(targets):
    kinds = np.ascontiguousarray([k for k, _ in targets], dtype=np.int32)
    xs = np.ascontiguousarray([x for _, x in targets], dtype=np.float32)
    return kinds, xs


def select(S, E, default_idx, targets, with_gap=False):
    lib = _load()
    S = np.ascontiguousarray(S, dtype=np.float32)
    E = np.ascontiguousarray(E, dtype=np.float32)
    if S.ndim == 1:
        S, E = S[None], E[None]
    n_k, n_f = S.shape
    kinds, xs = _targets(targets)
    ch = np.empty((n_k, len(kinds)), np.int32)
    gap = np.empty((n_k, len(kinds)), np.float64)
    rc = lib.oracle_select(_ptr(S), _ptr(E), n_k, n_f, int(default_idx), _ptr(kinds), _ptr(xs),
                           len(kinds), _ptr(ch), _ptr(gap))
    if rc != 0:
        raise OracleError("oracle_select: invalid arguments")
    return (ch, gap) if with_gap else ch


def sweep(speedup, energy, features, freqs, default_idx, targets, want_pred=False,
          with_gap=False, count_visits=False):
    lib = _load()
    ks, ke = _Keep(speedup), _Keep(energy)
    features = np.ascontiguousarray(features, dtype=np.float32)
    freqs = np.ascontiguousarray(freqs, dtype=np.float32)
    n_k, F = features.shape
    n_f = freqs.shape[0]
    kinds, xs = _targets(targets)
    ch = np.empty((n_k, len(kinds)), np.int32)
    S = np.empty((n_k, n_f), np.float32) if want_pred else None
    E = np.empty((n_k, n_f), np.float32) if want_pred else None
    gap = np.empty((n_k, len(kinds)), np.float64) if with_gap else None
    v = np.zeros(1, np.int64)
    rc = lib.oracle_sweep(ks.ref, ke.ref, _ptr(features), n_k, F, _ptr(freqs), n_f,
                          int(default_idx), _ptr(kinds), _ptr(xs), len(kinds), _ptr(ch), _ptr(S),
                          _ptr(E), _ptr(gap), _ptr(v))
    if rc != 0:
        raise OracleError("oracle_sweep: invalid arguments")
    out = {"choice": ch}
    if want_pred:
        out["S"], out["E"] = S, E
    if with_gap:
        out["gap"] = gap
    if count_visits:
        out["visits"] = int(v[0])
    return out


def sweep4(models, features, freqs, default_idx, targets, want_pred=False):
    """Four-model variant: models = [speedup, energy, edp|None, ed2p|None]."""
    lib = _load()
    keeps = [None if m is None else _Keep(m) for m in models]
    arr = (C.c_void_p * 4)(*[None if k is None else C.cast(C.pointer(k.s), C.c_void_p) for k in keeps])
    features = np.ascontiguousarray(features, dtype=np.float32)
    freqs = np.ascontiguousarray(freqs, dtype=np.float32)
    n_k, F = features.shape
    kinds, xs = _targets(targets)
    ch = np.empty((n_k, len(kinds)), np.int32)
    P = np.empty((4, n_k, freqs.shape[0]), np.float32) if want_pred else None
    rc = lib.oracle_sweep4(arr, _ptr(features), n_k, F, _ptr(freqs), freqs.shape[0], int(default_idx),
                           _ptr(kinds), _ptr(xs), len(kinds), _ptr(ch), _ptr(P))
    if rc != 0:
        raise OracleError("oracle_sweep4: invalid arguments")
    return {"choice": ch, "P": P} if want_pred else {"choice": ch}


def pareto(S, E):
    """uint8 front mask [n_k][n_f] of the (max S, min E) Pareto front per kernel."""
    lib = _load()
    S = np.ascontiguousarray(S, dtype=np.float32)
    E = np.ascontiguousarray(E, dtype=np.float32)
    if S.ndim == 1:
        S, E = S[None], E[None]
    front = np.empty(S.shape, np.uint8)
    if lib.oracle_pareto(_ptr(S), _ptr(E), S.shape[0], S.shape[1], _ptr(front)) != 0:
        raise OracleError("oracle_pareto: invalid arguments")
    return front


def choice_error(S_true, E_true, default_idx, targets, choice_pred):
    """(ape [n_k][n_t], mape [n_t], rmse [n_t], counted [n_t]) of predicted choices vs truth."""
    lib = _load()
    S_true = np.ascontiguousarray(S_true, dtype=np.float32)
    E_true = np.ascontiguousarray(E_true, dtype=np.float32)
    choice_pred = np.ascontiguousarray(choice_pred, dtype=np.int32)
    n_k, n_f = S_true.shape
    kinds, xs = _targets(targets)
    n_t = len(kinds)
    ape = np.empty((n_k, n_t), np.float64)
    mape = np.empty(n_t, np.float64)
    rmse = np.empty(n_t, np.float64)
    cnt = np.empty(n_t, np.int64)
    if lib.oracle_choice_error(_ptr(S_true), _ptr(E_true), n_k, n_f, int(default_idx), _ptr(kinds), _ptr(xs),
                               n_t, _ptr(choice_pred), _ptr(ape), _ptr(mape), _ptr(rmse), _ptr(cnt)) != 0:
        raise OracleError("oracle_choice_error: invalid arguments")
    return ape, mape, rmse, cnt


def sweep_workload(w, **kw):
    return sweep(w.speedup, w.energy, w.features, w.freqs, w.default_idx, w.targets, **kw)


def _sweep_range(args):
    """Worker for the all-core parity run: one contiguous kernel range, single-threaded."""
    cfg, row0, n = args
    from paper_conf_sc_fandccfc23_b200 import workloads as W
    w = W.make_config(cfg, row0=row0, n=n)
    return row0, sweep_workload(w)["choice"]

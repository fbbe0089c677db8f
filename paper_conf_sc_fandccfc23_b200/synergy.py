"""Thin Python binding of libsynergy.so (include/synergy.h) — argument marshalling only.

Every step of the path (model inference, normalisation, objectives, argmin) runs in the
sm_100a kernels behind the C ABI; PyTorch supplies device memory and the current stream.
There is no CPU fallback: if the in-tree libsynergy.so is missing or cannot load, every call
raises.  Names follow the C ABI: predict / select / sweep / sweep_host.
"""
from __future__ import annotations

import ctypes as C
import os
import re
from typing import Optional, Sequence, Tuple

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
_ROOT = os.path.dirname(_PKG)
LIB_PATH = os.path.join(_PKG, "libsynergy.so")
HEADER = os.path.join(_ROOT, "include", "synergy.h")

SYN_OK, SYN_ERR_INVALID_ARG, SYN_ERR_UNSUPPORTED, SYN_ERR_CUDA, SYN_ERR_OOM = range(5)
# synergy_last_launch variant codes
VARIANT_TREE_MAJOR, VARIANT_GENERAL = 4000, 5000
STATUS_NAMES = {0: "SYN_OK", 1: "SYN_ERR_INVALID_ARG", 2: "SYN_ERR_UNSUPPORTED", 3: "SYN_ERR_CUDA",
                4: "SYN_ERR_OOM"}


class SynergyError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS_NAMES.get(status, status)}: {msg}")
        self.status = status


class _Target(C.Structure):
    _fields_ = [("kind", C.c_int32), ("x", C.c_float)]


class _ModelDesc(C.Structure):
    _fields_ = [("n_inputs", C.c_int32), ("linear_weight", C.c_double), ("lin_w", C.c_void_p),
                ("lin_b", C.c_double), ("forest_weight", C.c_double), ("n_trees", C.c_int32),
                ("tree_offset", C.c_void_p), ("feature", C.c_void_p), ("left", C.c_void_p),
                ("right", C.c_void_p), ("value", C.c_void_p), ("svr_weight", C.c_double),
                ("n_sv", C.c_int32), ("sv", C.c_void_p), ("dual_coef", C.c_void_p), ("svr_gamma", C.c_double),
                ("svr_intercept", C.c_double), ("in_mean", C.c_void_p), ("in_scale", C.c_void_p)]


_lib = None


def exported_symbols_from_header(path: str = HEADER):
    """Function names declared in include/synergy.h (the ABI the library must export)."""
    src = open(path).read()
    return sorted(set(re.findall(r"^\s*(?:const\s+)?\w+\s*\*?\s*(synergy_\w+)\s*\(", src, re.M)))


def load(path: str = LIB_PATH) -> C.CDLL:
    """Load the in-tree library (raises OSError if it is missing: no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(path):
        raise OSError(f"libsynergy.so not built at {path} (run python -m paper_conf_sc_fandccfc23_b200.build)")
    lib = C.CDLL(path)
    P, I32, I64 = C.c_void_p, C.c_int32, C.c_int64
    sig = {
        "synergy_last_error": (C.c_char_p, []),
        "synergy_version": (I32, []),
        "synergy_model_create": (I32, [P, I32, P]),
        "synergy_model_destroy": (I32, [P]),
        "synergy_model_info": (I32, [P, P, P, P, P, P]),
        "synergy_clocks_create": (I32, [P, I32, I32, P]),
        "synergy_clocks_destroy": (I32, [P]),
        "synergy_clocks_info": (I32, [P, P]),
        "synergy_predict": (I32, [P, P, P, I64, I32, P, I32, P, P, P]),
        "synergy_select": (I32, [P, P, I64, I32, I32, P, I32, P, P]),
        "synergy_sweep": (I32, [P, P, P, I64, I32, P, I32, P, I32, P, P, P, P]),
        "synergy_sweep4": (I32, [P, P, I64, I32, P, I32, P, I32, P, P, P]),
        "synergy_plan": (I32, [P, I64, I32, P, P, P]),
        "synergy_pareto": (I32, [P, P, I64, I32, P, P]),
        "synergy_choice_error": (I32, [P, P, I64, I32, I32, P, I32, P, P, P, P]),
        "synergy_workspace_create": (I32, [I32, P]),
        "synergy_workspace_destroy": (I32, [P]),
        "synergy_sweep_host": (I32, [P, P, P, P, I64, I32, P, I32, P, I32, P, P]),
        "synergy_last_launch": (I32, [P, P, P, P, P]),
        "synergy_timing_enable": (I32, [I32]),
        "synergy_timing_read": (I32, [I32, P, P, P, P, P]),
        "synergy_prepare": (I32, [P, I32, I64, I32, P, P]),
        "synergy_config_set": (I32, [C.c_char_p, I64]),
        "synergy_config_get": (I32, [C.c_char_p, P]),
    }
    for name, (res, args) in sig.items():
        fn = getattr(lib, name)
        fn.restype = res
        fn.argtypes = args
    _lib = lib
    return lib


def _check(status: int):
    if status != SYN_OK:
        raise SynergyError(status, load().synergy_last_error().decode())


def _targets(targets: Sequence[Tuple[int, float]]):
    arr = (_Target * max(len(targets), 1))()
    for i, (k, x) in enumerate(targets):
        arr[i].kind = int(k)
        arr[i].x = float(x)
    return arr, len(targets)


def _stream(stream) -> Optional[int]:
    import torch
    if stream is None:
        stream = torch.cuda.current_stream()
    return stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream)


def _dev_ptr(t, dtype, shape=None, name="tensor"):
    import torch
    if t is None:
        return None
    if not isinstance(t, torch.Tensor) or not t.is_cuda:
        raise TypeError(f"{name} must be a CUDA torch.Tensor")
    if t.dtype != dtype or not t.is_contiguous():
        raise TypeError(f"{name} must be contiguous {dtype}")
    if shape is not None and tuple(t.shape) != tuple(shape):
        raise ValueError(f"{name} shape {tuple(t.shape)} != {tuple(shape)}")
    return t.data_ptr()


class Model:
    """Device-resident model handle (synergy_model_create) built from a workloads.ModelSpec."""

    def __init__(self, spec, device: int = 0):
        lib = load()
        c = np.ascontiguousarray
        self._keep = [
            None if spec.lin_w is None else c(spec.lin_w, dtype=np.float64),
            c(spec.tree_offset, dtype=np.int64), c(spec.feature, dtype=np.int32),
            c(spec.left, dtype=np.int32), c(spec.right, dtype=np.int32), c(spec.value, dtype=np.float32)]
        lw, off, fe, le, ri, va = self._keep
        n_trees = len(off) - 1 if spec.forest_weight != 0.0 else 0
        d = _ModelDesc(int(spec.n_inputs), float(spec.linear_weight), None if lw is None else lw.ctypes.data,
                       float(spec.lin_b), float(spec.forest_weight), int(n_trees), off.ctypes.data,
                       fe.ctypes.data, le.ctypes.data, ri.ctypes.data, va.ctypes.data)
        svr_w = float(getattr(spec, "svr_weight", 0.0))
        if svr_w != 0.0:
            sv = c(spec.sv, dtype=np.float32)
            du, mn, sc = (c(spec.dual_coef, dtype=np.float64), c(spec.in_mean, dtype=np.float64),
                          c(spec.in_scale, dtype=np.float64))
            self._keep += [sv, du, mn, sc]
            d.svr_weight = svr_w
            d.n_sv = int(sv.shape[0])
            d.sv, d.dual_coef, d.in_mean, d.in_scale = sv.ctypes.data, du.ctypes.data, mn.ctypes.data, sc.ctypes.data
            d.svr_gamma = float(spec.svr_gamma)
            d.svr_intercept = float(spec.svr_intercept)
        h = C.c_void_p()
        _check(lib.synergy_model_create(C.byref(d), int(device), C.byref(h)))
        self._h = h
        self.device = int(device)
        self._keep = None

    @property
    def handle(self):
        return self._h

    def info(self):
        lib = load()
        ni, nt, md = C.c_int32(), C.c_int32(), C.c_int32()
        nn, nb = C.c_int64(), C.c_int64()
        _check(lib.synergy_model_info(self._h, C.byref(ni), C.byref(nt), C.byref(nn), C.byref(md), C.byref(nb)))
        return {"n_inputs": ni.value, "n_trees": nt.value, "n_nodes": nn.value, "max_depth": md.value,
                "device_bytes": nb.value}

    def close(self):
        if getattr(self, "_h", None):
            load().synergy_model_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class Clocks:
    """Device-resident core-clock table (synergy_clocks_create)."""

    def __init__(self, freqs, device: int = 0):
        lib = load()
        f = np.ascontiguousarray(freqs, dtype=np.float32)
        h = C.c_void_p()
        _check(lib.synergy_clocks_create(f.ctypes.data, int(f.shape[0]), int(device), C.byref(h)))
        self._h = h
        self.n = int(f.shape[0])
        self.device = int(device)

    @property
    def handle(self):
        return self._h

    def close(self):
        if getattr(self, "_h", None):
            load().synergy_clocks_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def predict(speedup: Model, energy: Model, features, clocks: Clocks, default_idx: int,
            out_speedup=None, out_energy=None, stream=None):
    """synergy_predict: normalised (or raw when default_idx == -1) fp32 predictions."""
    import torch
    n_k, F = features.shape
    if out_speedup is None:
        out_speedup = torch.empty((n_k, clocks.n), dtype=torch.float32, device=features.device)
    if out_energy is None:
        out_energy = torch.empty((n_k, clocks.n), dtype=torch.float32, device=features.device)
    _check(load().synergy_predict(speedup.handle, energy.handle, _dev_ptr(features, torch.float32, name="features"),
                                  n_k, F, clocks.handle, int(default_idx),
                                  _dev_ptr(out_speedup, torch.float32, (n_k, clocks.n), "out_speedup"),
                                  _dev_ptr(out_energy, torch.float32, (n_k, clocks.n), "out_energy"),
                                  _stream(stream)))
    return out_speedup, out_energy


def select(S, E, default_idx: int, targets, out=None, stream=None):
    """synergy_select: int32 choices [n_k][n_targets] from normalised predictions."""
    import torch
    n_k, n_f = S.shape
    tg, n_t = _targets(targets)
    if out is None:
        out = torch.empty((n_k, n_t), dtype=torch.int32, device=S.device)
    _check(load().synergy_select(_dev_ptr(S, torch.float32, name="S"), _dev_ptr(E, torch.float32, (n_k, n_f), "E"),
                                 n_k, n_f, int(default_idx), tg, n_t,
                                 _dev_ptr(out, torch.int32, (n_k, n_t), "out"), _stream(stream)))
    return out


def sweep(speedup: Model, energy: Model, features, clocks: Clocks, default_idx: int, targets,
          out=None, out_speedup=None, out_energy=None, stream=None):
    """synergy_sweep: fused predict + select; predictions written only if buffers are given."""
    import torch
    n_k, F = features.shape
    tg, n_t = _targets(targets)
    if out is None:
        out = torch.empty((n_k, n_t), dtype=torch.int32, device=features.device)
    _check(load().synergy_sweep(speedup.handle, energy.handle, _dev_ptr(features, torch.float32, name="features"),
                                n_k, F, clocks.handle, int(default_idx), tg, n_t,
                                _dev_ptr(out, torch.int32, (n_k, n_t), "out"),
                                _dev_ptr(out_speedup, torch.float32, (n_k, clocks.n), "out_speedup"),
                                _dev_ptr(out_energy, torch.float32, (n_k, clocks.n), "out_energy"),
                                _stream(stream)))
    return out


def sweep4(models, features, clocks: Clocks, default_idx: int, targets, out=None, out_pred=None, stream=None):
    """synergy_sweep4: four-model variant, models = [speedup, energy, edp|None, ed2p|None];
    out_pred (optional) = float32 [4][n_k][n_f] normalised predictions."""
    import torch
    n_k, F = features.shape
    tg, n_t = _targets(targets)
    if out is None:
        out = torch.empty((n_k, n_t), dtype=torch.int32, device=features.device)
    handles = (C.c_void_p * 4)(*[None if m is None else m.handle.value for m in models])
    _check(load().synergy_sweep4(handles, _dev_ptr(features, torch.float32, name="features"), n_k, F,
                                 clocks.handle, int(default_idx), tg, n_t,
                                 _dev_ptr(out, torch.int32, (n_k, n_t), "out"),
                                 _dev_ptr(out_pred, torch.float32, (4, n_k, clocks.n), "out_pred"),
                                 _stream(stream)))
    return out


def plan(choice, clocks: Clocks, out=None, stream=None):
    """synergy_plan: chosen clocks in MHz per kernel per target (NaN where no choice)."""
    import torch
    n_k, n_t = choice.shape
    if out is None:
        out = torch.empty((n_k, n_t), dtype=torch.float32, device=choice.device)
    _check(load().synergy_plan(_dev_ptr(choice, torch.int32, name="choice"), n_k, n_t, clocks.handle,
                               _dev_ptr(out, torch.float32, (n_k, n_t), "out"), _stream(stream)))
    return out


def pareto(S, E, out=None, stream=None):
    """synergy_pareto: uint8 [n_k][n_f] mask of the (max S, min E) Pareto front per kernel."""
    import torch
    n_k, n_f = S.shape
    if out is None:
        out = torch.empty((n_k, n_f), dtype=torch.uint8, device=S.device)
    _check(load().synergy_pareto(_dev_ptr(S, torch.float32, name="S"), _dev_ptr(E, torch.float32, (n_k, n_f), "E"),
                                 n_k, n_f, _dev_ptr(out, torch.uint8, (n_k, n_f), "out"), _stream(stream)))
    return out


def choice_error(S_true, E_true, default_idx, targets, choice_pred, stream=None):
    """synergy_choice_error: (err [n_k][n_t][2] = (APE, pred - actual), summary [n_t][3] =
    (MAPE, RMSE, counted)) of predicted choices against the ground-truth table."""
    import torch
    n_k, n_f = S_true.shape
    tg, n_t = _targets(targets)
    err = torch.empty((n_k, n_t, 2), dtype=torch.float64, device=S_true.device)
    summ = torch.empty((n_t, 3), dtype=torch.float64, device=S_true.device)
    _check(load().synergy_choice_error(_dev_ptr(S_true, torch.float32, name="S_true"),
                                       _dev_ptr(E_true, torch.float32, (n_k, n_f), "E_true"), n_k, n_f,
                                       int(default_idx), tg, n_t,
                                       _dev_ptr(choice_pred, torch.int32, (n_k, n_t), "choice_pred"),
                                       err.data_ptr(), summ.data_ptr(), _stream(stream)))
    return err, summ


class Workspace:
    """synergy_sweep_host: host features in, host choices out (H2D + sweep + D2H on `stream`)."""

    def __init__(self, device: int = 0):
        h = C.c_void_p()
        _check(load().synergy_workspace_create(int(device), C.byref(h)))
        self._h = h

    def sweep_host(self, speedup: Model, energy: Model, h_features, clocks: Clocks, default_idx: int,
                   targets, h_out, stream=None):
        """h_features / h_out: host buffers (numpy or CPU torch tensors, ideally pinned).
        Returns after enqueueing; h_out is valid once `stream` is synchronised."""
        tg, n_t = _targets(targets)
        n_k, F = h_features.shape
        fp = h_features.data_ptr() if hasattr(h_features, "data_ptr") else h_features.ctypes.data
        op = h_out.data_ptr() if hasattr(h_out, "data_ptr") else h_out.ctypes.data
        _check(load().synergy_sweep_host(self._h, speedup.handle, energy.handle, fp, n_k, F, clocks.handle,
                                         int(default_idx), tg, n_t, op, _stream(stream)))
        return h_out

    def close(self):
        if getattr(self, "_h", None):
            load().synergy_workspace_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def prepare(models, n_kernels: int, n_features: int, clocks: Clocks, stream=None):
    """synergy_prepare: create the persistent scratch for calls of this shape on `stream` (so later
    calls only enqueue kernels, e.g. inside a CUDA-graph capture).  models = [speedup, energy] or
    [speedup, energy, edp|None, ed2p|None]."""
    handles = (C.c_void_p * len(models))(*[None if m is None else m.handle.value for m in models])
    _check(load().synergy_prepare(handles, len(models), int(n_kernels), int(n_features), clocks.handle,
                                  _stream(stream)))


def config_set(key: str, value: int):
    """synergy_config_set: a launch-configuration knob (results do not depend on it)."""
    _check(load().synergy_config_set(key.encode(), int(value)))


def config_get(key: str) -> int:
    v = C.c_int64()
    _check(load().synergy_config_get(key.encode(), C.byref(v)))
    return v.value


def last_launch():
    k, b, v = C.c_int32(), C.c_int32(), C.c_int32()
    e, g = C.c_int64(), C.c_int64()
    _check(load().synergy_last_launch(C.byref(k), C.byref(e), C.byref(g), C.byref(b), C.byref(v)))
    return {"kernels": k.value, "evals": e.value, "grid": g.value, "block": b.value, "variant": v.value}


def timing_enable(on: bool = True):
    """synergy_timing_enable: bracket every library kernel launch with CUDA events."""
    _check(load().synergy_timing_enable(1 if on else 0))


def timing_read(cap: int = 32):
    """synergy_timing_read: {kernel name: (total_ms, launches, busy_ms)} since the previous read
    (busy_ms: the union of the kernel's launch intervals)."""
    names = (C.c_char_p * cap)()
    ms = (C.c_double * cap)()
    busy = (C.c_double * cap)()
    cnt = (C.c_int64 * cap)()
    n = C.c_int32()
    _check(load().synergy_timing_read(cap, names, ms, busy, cnt, C.byref(n)))
    return {names[k].decode(): (ms[k], cnt[k], busy[k]) for k in range(min(n.value, cap))}

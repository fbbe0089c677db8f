"""CPU-side checks of the C-ABI library: it loads, exports every symbol include/synergy.h
declares, and rejects invalid arguments on the host before touching a device."""
import ctypes as C
import subprocess

import numpy as np
import pytest

from paper_conf_sc_fandccfc23_b200 import build as B
from paper_conf_sc_fandccfc23_b200 import synergy as syn


@pytest.fixture(scope="module")
def lib():
    B.build()
    return syn.load()


def test_header_declares_the_boundary():
    names = syn.exported_symbols_from_header()
    for required in ("synergy_predict", "synergy_select", "synergy_sweep", "synergy_model_create",
                     "synergy_clocks_create", "synergy_sweep_host", "synergy_last_error"):
        assert required in names


def test_library_exports_every_declared_symbol(lib):
    out = subprocess.run(["nm", "-D", "--defined-only", B.LIB], capture_output=True, text=True, check=True).stdout
    exported = {line.split()[-1] for line in out.splitlines() if line.strip()}
    for name in syn.exported_symbols_from_header():
        assert name in exported, name
        assert hasattr(lib, name)


def test_library_is_sm100a(lib):
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", B.LIB], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_version_and_error_string(lib):
    assert lib.synergy_version() == 3
    h = C.c_void_p()
    assert lib.synergy_model_create(None, 0, C.byref(h)) == syn.SYN_ERR_INVALID_ARG
    assert b"desc" in lib.synergy_last_error()


def test_host_validation_before_device(lib):
    h = C.c_void_p()
    bad = np.array([100.0, 100.0, 200.0], np.float32)            # not strictly ascending
    assert lib.synergy_clocks_create(bad.ctypes.data, 3, 0, C.byref(h)) == syn.SYN_ERR_INVALID_ARG
    nan = np.array([100.0, np.nan], np.float32)
    assert lib.synergy_clocks_create(nan.ctypes.data, 2, 0, C.byref(h)) == syn.SYN_ERR_INVALID_ARG
    tg, n_t = syn._targets([(4, 150.0)])
    assert lib.synergy_select(None, None, 1, 8, 0, tg, n_t, None, None) == syn.SYN_ERR_INVALID_ARG
    assert b"x=150" in lib.synergy_last_error()
    tg, n_t = syn._targets([(0, 0.0)])
    assert lib.synergy_select(None, None, 1, 0, 0, tg, n_t, None, None) == syn.SYN_ERR_INVALID_ARG
    assert lib.synergy_select(None, None, -1, 8, 0, tg, n_t, None, None) == syn.SYN_ERR_INVALID_ARG
    assert lib.synergy_select(None, None, 0, 8, 0, tg, n_t, None, None) == syn.SYN_OK   # empty batch no-op


def test_model_validation(lib):
    from paper_conf_sc_fandccfc23_b200 import workloads as W

    def create(spec):
        d = syn._ModelDesc(int(spec.n_inputs), float(spec.linear_weight), None, float(spec.lin_b),
                           float(spec.forest_weight), int(len(spec.tree_offset) - 1), spec.tree_offset.ctypes.data,
                           spec.feature.ctypes.data, spec.left.ctypes.data, spec.right.ctypes.data,
                           spec.value.ctypes.data)
        h = C.c_void_p()
        return lib.synergy_model_create(C.byref(d), 0, C.byref(h))

    base = dict(n_inputs=3, forest_weight=1.0, tree_offset=np.array([0, 3], np.int64),
                value=np.array([0.5, 1.0, 2.0], np.float32))
    cyc = W.ModelSpec(feature=np.array([0, 0, -1], np.int32), left=np.array([1, 0, -1], np.int32),
                      right=np.array([2, 2, -1], np.int32), **base)
    assert create(cyc) == syn.SYN_ERR_INVALID_ARG                          # node 2 reached twice
    oob = W.ModelSpec(feature=np.array([0, -1, -1], np.int32), left=np.array([1, -1, -1], np.int32),
                      right=np.array([5, -1, -1], np.int32), **base)
    assert create(oob) == syn.SYN_ERR_INVALID_ARG                          # child outside tree
    badf = W.ModelSpec(feature=np.array([3, -1, -1], np.int32), left=np.array([1, -1, -1], np.int32),
                       right=np.array([2, -1, -1], np.int32), **base)
    assert create(badf) == syn.SYN_ERR_INVALID_ARG                         # feature >= n_inputs
    none = W.ModelSpec(n_inputs=3)
    assert create(none) == syn.SYN_ERR_INVALID_ARG                         # no member
    for bad in (np.inf, -np.inf, np.nan):                                  # non-finite leaf value
        nf = W.ModelSpec(feature=np.array([0, -1, -1], np.int32), left=np.array([1, -1, -1], np.int32),
                         right=np.array([2, -1, -1], np.int32), n_inputs=3, forest_weight=1.0,
                         tree_offset=np.array([0, 3], np.int64), value=np.array([0.5, 1.0, bad], np.float32))
        assert create(nf) == syn.SYN_ERR_INVALID_ARG
        assert b"not finite" in lib.synergy_last_error()
    # a NaN threshold is allowed (x <= NaN is false: every input goes right)
    nan_thr = W.ModelSpec(feature=np.array([0, -1, -1], np.int32), left=np.array([1, -1, -1], np.int32),
                          right=np.array([2, -1, -1], np.int32), n_inputs=3, forest_weight=1.0,
                          tree_offset=np.array([0, 3], np.int64), value=np.array([np.nan, 1.0, 2.0], np.float32))
    assert create(nan_thr) in (syn.SYN_OK, syn.SYN_ERR_INVALID_ARG, syn.SYN_ERR_CUDA)
    if create(nan_thr) == syn.SYN_ERR_INVALID_ARG:                         # only "no device" may fail it
        assert b"device" in lib.synergy_last_error()


def test_target_kinds_and_tuning_keys(lib):
    """ES_ABS / PL_ABS (kinds 6, 7) are accepted, kind 8 is not; tuning keys round-trip and an
    unknown key is INVALID_ARG (all host-side, no device needed)."""
    for kind in (6, 7):
        tg, n_t = syn._targets([(kind, 25.0)])
        assert lib.synergy_select(None, None, 0, 8, 0, tg, n_t, None, None) == syn.SYN_OK
        tg, n_t = syn._targets([(kind, 101.0)])
        assert lib.synergy_select(None, None, 0, 8, 0, tg, n_t, None, None) == syn.SYN_ERR_INVALID_ARG
    tg, n_t = syn._targets([(8, 0.0)])
    assert lib.synergy_select(None, None, 0, 8, 0, tg, n_t, None, None) == syn.SYN_ERR_INVALID_ARG
    old = syn.config_get("tm_kb")
    syn.config_set("tm_kb", 64)
    assert syn.config_get("tm_kb") == 64
    syn.config_set("tm_kb", old)
    with pytest.raises(syn.SynergyError) as ei:
        syn.config_set("no_such_knob", 1)
    assert ei.value.status == syn.SYN_ERR_INVALID_ARG


def test_model_desc_layout_matches_header():
    """The binding's ctypes struct lists syn_model_desc's fields in header order."""
    import re
    src = open(syn.HEADER).read()
    body = src[src.index("typedef struct {\n    int32_t n_inputs;"):src.index("} syn_model_desc;")]
    names = re.findall(r"\b(\w+);", body)
    assert [f for f, _ in syn._ModelDesc._fields_] == names


@pytest.mark.parametrize("bad", ["scale0", "nsv0", "nan_dual", "neg_gamma", "null_sv", "nan_sv"])
def test_svr_model_validation(lib, bad):
    """SVR members are validated on the host (synergy.h: synergy_model_create)."""
    from paper_conf_sc_fandccfc23_b200 import workloads as W
    _, en, _, _ = W.make_models_svr("c1", n_sv=20)
    en.in_scale = en.in_scale.copy()
    en.dual_coef = en.dual_coef.copy()
    en.sv = en.sv.copy()
    if bad == "scale0":
        en.in_scale[2] = 0.0
    elif bad == "nsv0":
        en.sv = en.sv[:0]
    elif bad == "nan_dual":
        en.dual_coef[3] = np.nan
    elif bad == "neg_gamma":
        en.svr_gamma = -1.0
    elif bad == "nan_sv":
        en.sv[5, 1] = np.inf
    with pytest.raises(syn.SynergyError) as ei:
        if bad == "null_sv":
            d = syn._ModelDesc(en.n_inputs, 0.0, None, 0.0, 0.0, 0, None, None, None, None, None, 1.0, 4, None,
                               None, 0.5, 0.0, None, None)
            h = C.c_void_p()
            syn._check(lib.synergy_model_create(C.byref(d), 0, C.byref(h)))
        else:
            syn.Model(en)
    assert ei.value.status == syn.SYN_ERR_INVALID_ARG

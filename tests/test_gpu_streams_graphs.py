"""The fused path on several streams at once and inside a CUDA graph (DESIGN.md §6 slab pipeline:
library-owned difference-array buffers and side stream per (device, caller stream); the side
stream forks from and joins the caller's stream with events, so a captured call is a fork-join
graph).  Results are compared with the CPU oracle, bit for bit."""
import numpy as np
import pytest

import oracle
from paper_conf_sc_fandccfc23_b200 import workloads as W
from gpu_util import assert_bits_equal

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _build():
    from paper_conf_sc_fandccfc23_b200 import build
    build.build()
    oracle.build()


def _workload(seed):
    # several kernel slabs at tm_slab = 64: the pipeline runs (finish i || walk i + 1)
    return W.fuzz_workload(seed, 300, 64, F=5, n_trees=4, max_depth=8, p_leaf=0.1)


def _run(w, stream, S, E, out):
    import torch
    from paper_conf_sc_fandccfc23_b200 import synergy as syn
    sp, en, ck = syn.Model(w.speedup), syn.Model(w.energy), syn.Clocks(w.freqs)
    feats = torch.from_numpy(np.ascontiguousarray(w.features)).cuda()
    return (sp, en, ck, feats), lambda: syn.sweep(sp, en, feats, ck, w.default_idx, w.targets, out=out,
                                                  out_speedup=S, out_energy=E, stream=stream)


def _buffers(w):
    import torch
    S = torch.full((w.n_kernels, w.n_freqs), -1.0, dtype=torch.float32, device="cuda")
    E = torch.full_like(S, -1.0)
    out = torch.full((w.n_kernels, len(w.targets)), -9, dtype=torch.int32, device="cuda")
    return S, E, out


def _check(w, S, E, out):
    ref = oracle.sweep_workload(w, want_pred=True)
    assert_bits_equal(S.cpu().numpy(), ref["S"], "S")
    assert_bits_equal(E.cpu().numpy(), ref["E"], "E")
    assert np.array_equal(out.cpu().numpy(), ref["choice"])


@pytest.fixture
def slabs64():
    from paper_conf_sc_fandccfc23_b200 import synergy as syn
    syn.config_set("tm_slab", 64)
    syn.config_set("tm_kb", 32)
    yield
    syn.config_set("tm_slab", 0)
    syn.config_set("tm_kb", 0)


def test_two_streams_concurrently(slabs64):
    import torch
    ws = [_workload(5), _workload(6)]
    streams = [torch.cuda.Stream(), torch.cuda.Stream()]
    bufs = [_buffers(w) for w in ws]
    runs = [_run(w, s.cuda_stream, *b) for w, s, b in zip(ws, streams, bufs)]
    torch.cuda.synchronize()
    for _ in range(3):                                   # interleaved calls on both streams
        for (_, call), s in zip(runs, streams):
            with torch.cuda.stream(s):
                call()
    torch.cuda.synchronize()
    for w, b in zip(ws, bufs):
        _check(w, *b)


def test_captured_in_cuda_graph(slabs64):
    import torch
    w = _workload(7)
    S, E, out = _buffers(w)
    s = torch.cuda.Stream()
    keep, call = _run(w, s.cuda_stream, S, E, out)
    with torch.cuda.stream(s):
        call()                                           # warm-up: builds the cached buffers
    torch.cuda.synchronize()
    S.fill_(-1.0); E.fill_(-1.0); out.fill_(-9)
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        call()
    for _ in range(3):
        g.replay()
    torch.cuda.synchronize()
    _check(w, S, E, out)


def test_prepare_then_capture_on_a_fresh_stream(slabs64):
    """synergy_prepare creates the clock-cut copies, difference arrays and side stream, so the very
    first sweep on the stream can be captured."""
    import torch
    from paper_conf_sc_fandccfc23_b200 import synergy as syn
    w = _workload(8)
    S, E, out = _buffers(w)
    s = torch.cuda.Stream()
    keep, call = _run(w, s.cuda_stream, S, E, out)
    syn.prepare([keep[0], keep[1]], w.n_kernels, w.n_features, keep[2], stream=s.cuda_stream)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        call()
    g.replay()
    torch.cuda.synchronize()
    _check(w, S, E, out)


def test_unprepared_capture_is_refused():
    """Without prepare / warm-up, the persistent scratch cannot be created inside a capture: the
    call returns SYN_ERR_UNSUPPORTED (nothing is enqueued) instead of breaking the capture."""
    import torch
    from paper_conf_sc_fandccfc23_b200 import synergy as syn
    w = _workload(9)
    S, E, out = _buffers(w)
    s = torch.cuda.Stream()
    keep, call = _run(w, s.cuda_stream, S, E, out)
    g = torch.cuda.CUDAGraph()
    with pytest.raises(syn.SynergyError) as ei:
        with torch.cuda.graph(g, stream=s):
            call()
    assert ei.value.status == syn.SYN_ERR_UNSUPPORTED
    torch.cuda.synchronize()


def test_single_launch_path_prepare_then_capture():
    """A small batch takes the single-launch k_tm_small (no difference arrays): prepare makes the
    clock-cut copies, then the call is captured and replayed."""
    import torch
    from paper_conf_sc_fandccfc23_b200 import synergy as syn
    w = W.fuzz_workload(10, 40, 64, F=5, n_trees=4, max_depth=8, p_leaf=0.1)
    S, E, out = _buffers(w)
    s = torch.cuda.Stream()
    keep, call = _run(w, s.cuda_stream, S, E, out)
    syn.prepare([keep[0], keep[1]], w.n_kernels, w.n_features, keep[2], stream=s.cuda_stream)
    torch.cuda.synchronize()
    with torch.cuda.stream(s):
        call()
    torch.cuda.synchronize()
    assert syn.last_launch()["kernels"] == 1              # k_tm_small alone
    S.fill_(-1.0); E.fill_(-1.0); out.fill_(-9)
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        call()
    for _ in range(2):
        g.replay()
    torch.cuda.synchronize()
    _check(w, S, E, out)


@pytest.mark.gpu
def test_timing_busy_is_union_of_launch_intervals(slabs64):
    """synergy_timing_read's busy time is the union of a kernel's launch intervals: never above the
    summed launch durations, and below it only when launches overlap (the slab pipeline's walks on
    two streams); results are unchanged with timing on."""
    import torch
    from paper_conf_sc_fandccfc23_b200 import synergy as syn
    w = _workload(77)
    S, E, out = _buffers(w)
    _, fn = _run(w, None, S, E, out)
    fn()
    torch.cuda.synchronize()
    syn.timing_read()
    syn.timing_enable(True)
    try:
        for _ in range(3):
            fn()
        torch.cuda.synchronize()
    finally:
        syn.timing_enable(False)
    t = syn.timing_read()
    assert "k_tm_walk" in t and "k_tm_finish" in t
    for name, (total, launches, busy) in t.items():
        assert launches > 0 and total > 0.0
        assert 0.0 < busy <= total * (1 + 1e-6) + 1e-3, (name, total, busy)
    _check(w, S, E, out)

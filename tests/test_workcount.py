"""Pins for the run-walk work counters (tools/workcount.c, a measurement tool separate from the
oracle), the numerator of the k_tm_walk roofline.  Checked against an independent formulation: a depth-first
walk of each tree over the clock-index interval that splits at clock thresholds (each leaf reached
owns one run of consecutive clocks), written here from the tree definition."""
import numpy as np

from paper_conf_sc_fandccfc23_b200 import workloads as W


def interval_runs(spec, t, x_static, freqs):
    """(runs, sum of leaf depths, sum of max(1, ceil(depth/2)), resume-walk block fetches) for one
    (kernel, tree).  Resume fetches, counted per reachable node: every 2-level block (the root and
    every reachable internal node at even depth) is fetched once when first reached, plus once
    more for every clock split inside it (its node or the reachable child) whose reachable clock
    interval has clocks on both sides: the first clock of the right side resumes at that block."""
    base = spec.tree_offset[t]
    F = len(x_static)
    runs = dec = blk = res = 0
    stack = [(0, 0, len(freqs), 0)]
    while stack:
        n, lo, hi, d = stack.pop()
        f = spec.feature[base + n]
        if d % 2 == 0 and (f >= 0 or d == 0):
            res += 1                                           # block first reached
        if f < 0:
            runs += 1
            dec += d
            blk += max(1, (d + 1) // 2)
            continue
        thr = spec.value[base + n]
        L, R = spec.left[base + n], spec.right[base + n]
        if f < F:
            stack.append((L if x_static[f] <= thr else R, lo, hi, d + 1))
            continue
        s = int(np.searchsorted(freqs, thr, side="right"))     # #clocks <= thr
        if lo < s < hi:
            res += 1                                           # right side resumes at this block
        if s < hi and max(s, lo) < hi:
            stack.append((R, max(s, lo), hi, d + 1))
        if s > lo:
            stack.append((L, lo, min(s, hi), d + 1))
    return runs, dec, blk, res


def _check(w):
    import tools
    r = tools.count([w.speedup, w.energy], w.features, w.freqs)
    runs = dec = blk = res = 0
    for k in range(w.n_kernels):
        for m in (w.speedup, w.energy):
            if m.forest_weight == 0.0:
                continue
            for t in range(m.n_trees):
                a, b, c, e = interval_runs(m, t, w.features[k], w.freqs)
                runs += a
                dec += b
                blk += c
                res += e
    assert (r["runs"], r["run_decisions"], r["run_blocks"]) == (runs, dec, blk)
    assert r["resume_blocks"] == res


def test_workcount_c1():
    _check(W.make_config("c1"))


def test_decisions_are_t_times_d_on_complete_trees():
    """Direct traversal of complete depth-D trees takes exactly T*D decisions per evaluation."""
    import tools
    w = W.make_config("c1")
    r = tools.count([w.speedup, w.energy], w.features, w.freqs)
    assert r["decisions"] == w.n_kernels * w.n_freqs * 2 * 10 * 8


def test_workcount_fuzz_unbalanced_exact_thresholds():
    for seed in range(4):
        _check(W.fuzz_workload(50 + seed, 5, 33, F=4, n_trees=4, max_depth=7, exact_thresholds=True))

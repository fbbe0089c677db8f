"""Pins for the forest mean's summation (oracle.c: exact_sum; reading Q8).

The paper fixes no summation order for the Random Forest mean (PAPER L386 names the model only),
so the oracle takes the plain real-number definition: the exact sum of the fp32 leaf values,
rounded once to fp64, divided by T.  Pinned against Python's math.fsum (an independent library
implementation of the correctly rounded sum) on leaves spanning the whole fp32 range, where a
sequential fp64 sum would round.
"""
import math

import numpy as np

from paper_conf_sc_fandccfc23_b200 import workloads as W


def stump_forest(values):
    """T one-leaf trees with the given leaf values (each tree is a stump)."""
    T = len(values)
    return W.ModelSpec(n_inputs=2, forest_weight=1.0, tree_offset=np.arange(T + 1, dtype=np.int64),
                       feature=np.full(T, -1, np.int32), left=np.full(T, -1, np.int32),
                       right=np.full(T, -1, np.int32), value=np.asarray(values, np.float32))


def test_cancellation_case_sequential_sum_would_lose():
    """1e30 + 1 - 1e30: the sequential fp64 sum gives 0, the exact sum 1."""
    import oracle
    vals = np.array([1e30, 1.0, -1e30], np.float32)
    seq = 0.0
    for v in vals:
        seq += float(v)
    assert seq == 0.0
    assert oracle.model_eval(stump_forest(vals), np.zeros(2, np.float32)) == 1.0 / 3.0


def test_matches_math_fsum_on_wide_range_leaves():
    import oracle
    rng = np.random.default_rng(31)
    for trial in range(300):
        T = int(rng.integers(1, 700))
        mant = rng.uniform(-1, 1, size=T)
        exps = rng.integers(-60, 60, size=T) if trial % 2 else rng.integers(-3, 3, size=T)
        vals = (mant * np.exp2(exps)).astype(np.float32)
        expect = math.fsum(float(v) for v in vals) / T
        got = oracle.model_eval(stump_forest(vals), np.zeros(2, np.float32))
        assert got == expect, (trial, got, expect)


def test_order_invariance():
    import oracle
    rng = np.random.default_rng(5)
    vals = (rng.uniform(-1, 1, 257) * np.exp2(rng.integers(-40, 40, 257))).astype(np.float32)
    ref = oracle.model_eval(stump_forest(vals), np.zeros(2, np.float32))
    for _ in range(20):
        assert oracle.model_eval(stump_forest(rng.permutation(vals)), np.zeros(2, np.float32)) == ref


def test_equals_sequential_sum_when_exact():
    """On the bench forests (leaves in [0.25, 4), <= 1000 trees) every partial sum is exact, so the
    exact-sum mean is also the plain sequential fp64 mean."""
    import oracle
    w = W.make_config("c1")
    rng = np.random.default_rng(2)
    sp = w.speedup
    for _ in range(200):
        x = np.concatenate([w.features[rng.integers(0, w.n_kernels)], [w.freqs[rng.integers(0, w.n_freqs)]]]).astype(np.float32)
        seq = 0.0
        for t in range(sp.n_trees):
            base = sp.tree_offset[t]
            n = 0
            while sp.feature[base + n] >= 0:
                n = sp.left[base + n] if x[sp.feature[base + n]] <= sp.value[base + n] else sp.right[base + n]
            seq += float(sp.value[base + n])
        assert oracle.model_eval(sp, x) == seq / sp.n_trees

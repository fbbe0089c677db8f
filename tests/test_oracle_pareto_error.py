"""Pins for the oracle's Pareto front and frequency-choice error metrics.

* Pareto front ("the red line is the Pareto front", L247, L374): against an independent
  sort-based skyline formulation, and against the selection definitions (the speed/energy
  extremes and every ES/PL choice are Pareto-optimal on tie-free inputs, L418).
* Choice error (Table 2): zero for perfect predictions, the hand-worked golden
  example, and exact rational arithmetic.
"""
import json
import os
from fractions import Fraction

import numpy as np

from paper_conf_sc_fandccfc23_b200.workloads import ES, MAX_PERF, MIN_ED2P, MIN_EDP, MIN_ENERGY, PL

TARGETS = [(MAX_PERF, 0.0), (MIN_ENERGY, 0.0), (MIN_EDP, 0.0), (MIN_ED2P, 0.0), (ES, 25.0), (ES, 50.0),
           (PL, 25.0), (PL, 50.0)]


def skyline(S, E):
    """Sort by speedup descending: a valid point is on the front iff its energy is below every
    strictly faster point's and minimal among the equally fast ones."""
    n = len(S)
    valid = [np.isfinite(S[i]) and np.isfinite(E[i]) and S[i] > 0 and E[i] > 0 for i in range(n)]
    idx = sorted([i for i in range(n) if valid[i]], key=lambda i: (-S[i], E[i]))
    front = np.zeros(n, np.uint8)
    best_faster = np.inf
    g = 0
    while g < len(idx):
        h = g
        while h < len(idx) and S[idx[h]] == S[idx[g]]:
            h += 1
        emin = min(E[i] for i in idx[g:h])
        for i in idx[g:h]:
            if E[i] == emin and E[i] < best_faster:
                front[i] = 1
        best_faster = min(best_faster, emin)
        g = h
    return front


def test_pareto_matches_skyline_with_ties_and_invalid():
    import oracle
    rng = np.random.default_rng(17)
    for _ in range(400):
        n = int(rng.integers(1, 40))
        S = (rng.integers(1, 12, n) / 8).astype(np.float32)
        E = (rng.integers(1, 12, n) / 8).astype(np.float32)
        S[rng.uniform(size=n) < 0.05] = 0.0
        E[rng.uniform(size=n) < 0.05] = np.nan
        np.testing.assert_array_equal(oracle.pareto(S, E)[0], skyline(S, E))


def test_selected_tradeoffs_lie_on_the_front():
    import oracle
    rng = np.random.default_rng(4)
    for _ in range(200):
        n = int(rng.integers(2, 60))
        S = rng.uniform(0.3, 1.3, n).astype(np.float32)
        E = rng.uniform(0.4, 1.6, n).astype(np.float32)
        d = int(rng.integers(0, n))
        front = oracle.pareto(S, E)[0]
        ch = oracle.select(S, E, d, [(MAX_PERF, 0.0), (MIN_ENERGY, 0.0), (ES, 10.0), (ES, 50.0), (ES, 90.0),
                                     (PL, 10.0), (PL, 50.0), (PL, 90.0)])[0]
        assert all(front[c] == 1 for c in ch)


def test_choice_error_zero_for_perfect_predictions():
    import oracle
    rng = np.random.default_rng(2)
    S = rng.uniform(0.3, 1.3, (50, 37)).astype(np.float32)
    E = rng.uniform(0.4, 1.6, (50, 37)).astype(np.float32)
    S[:, 20] = E[:, 20] = 1.0
    ch = oracle.select(S, E, 20, TARGETS)
    ape, mape, rmse, cnt = oracle.choice_error(S, E, 20, TARGETS, ch)
    assert np.all(ape == 0.0) and np.all(mape == 0.0) and np.all(rmse == 0.0) and np.all(cnt == 50)


def test_choice_error_hand_example():
    """Golden worked example (tests/golden/worked_example.json): truth MIN_EDP = clock 2
    (EDP 0.8/0.9); a prediction of clock 3 gives EDP 1.0: APE = (1.0 - 0.8/0.9)/(0.8/0.9) = 0.125."""
    import oracle
    with open(os.path.join(os.path.dirname(__file__), "golden", "worked_example.json")) as f:
        g = json.load(f)
    S = np.array([g["S"]], np.float32)
    E = np.array([g["E"]], np.float32)
    ape, mape, rmse, cnt = oracle.choice_error(S, E, g["default_idx"], [(MIN_EDP, 0.0), (MAX_PERF, 0.0)],
                                               np.array([[3, 1]], np.int32))
    edp2 = Fraction(float(np.float32(0.8))) / Fraction(float(np.float32(0.9)))
    assert abs(ape[0, 0] - float((1 - edp2) / edp2)) < 1e-15
    # MAX_PERF truth = clock 4 (S 1.05), predicted clock 1 (S 0.75): APE = 0.3/1.05
    assert abs(ape[0, 1] - float((Fraction(float(np.float32(1.05))) - Fraction(float(np.float32(0.75)))) /
                                 Fraction(float(np.float32(1.05))))) < 1e-15
    assert cnt.tolist() == [1, 1]
    assert abs(rmse[1] - float(np.float32(1.05)) + float(np.float32(0.75))) < 1e-15


def test_choice_error_exact_rationals_and_missing():
    import oracle
    rng = np.random.default_rng(9)
    n_k, n_f, d = 30, 17, 5
    S = (rng.integers(2, 12, (n_k, n_f)) / 8).astype(np.float32)
    E = (rng.integers(2, 12, (n_k, n_f)) / 8).astype(np.float32)
    S[:, d] = 1.0
    E[:, d] = 1.0
    pred = rng.integers(-1, n_f, (n_k, len(TARGETS))).astype(np.int32)
    truth = oracle.select(S, E, d, TARGETS)
    ape, mape, rmse, cnt = oracle.choice_error(S, E, d, TARGETS, pred)
    for t, (kind, _) in enumerate(TARGETS):
        def obj(k, i):
            s, e = Fraction(float(S[k, i])), Fraction(float(E[k, i]))
            return {MAX_PERF: s, ES: s, MIN_ENERGY: e, PL: e, MIN_EDP: e / s, MIN_ED2P: e / s / s}[kind]
        apes = []
        for k in range(n_k):
            if pred[k, t] < 0:
                assert np.isnan(ape[k, t])
                continue
            a = abs(obj(k, pred[k, t]) - obj(k, truth[k, t])) / abs(obj(k, truth[k, t]))
            assert abs(ape[k, t] - float(a)) <= 1e-15 * max(1.0, float(a))
            apes.append(a)
        assert cnt[t] == len(apes)
        assert abs(mape[t] - float(sum(apes) / len(apes))) < 1e-14
        # RMSE over the counted kernels (L388-L392): sqrt(mean of (pred - actual)^2), exact rationals.
        # Some predictions are -1 (not counted), so normalising by n_k instead would fail here.
        ms = sum((obj(k, pred[k, t]) - obj(k, truth[k, t])) ** 2 for k in range(n_k) if pred[k, t] >= 0) / len(apes)
        assert len(apes) < n_k
        assert abs(Fraction(rmse[t]) ** 2 - ms) <= Fraction(1, 10 ** 14) * max(ms, Fraction(1, 10 ** 6))
        assert ms > 0

"""Pins for the oracle's selection step (oracle.c: select_kernel).

Each test checks the oracle against something other than itself (TASK ③): hand-worked
examples from the paper's definitions (tests/golden/), exact rational arithmetic, an
independent Pareto-front formulation, and properties the definitions imply.
Definitions: EDP = e*t, ED2P = e*t^2; ES_x (L259-L267); PL_x (L269-L271);
t = 1/S (speedup axes of Figs 2/5/7, L69).  Readings: DESIGN.md Q1-Q5, Q14, Q16.
"""
import json
import os
from fractions import Fraction

import numpy as np
import pytest

from paper_conf_sc_fandccfc23_b200.workloads import (ES, ES_ABS, MAX_PERF, MIN_ED2P, MIN_EDP, MIN_ENERGY,
                                                     PL, PL_ABS, TARGET_NAMES)

GOLD = os.path.join(os.path.dirname(__file__), "golden")
KIND = {v: k for k, v in TARGET_NAMES.items()}


def _load_golden(name):
    with open(os.path.join(GOLD, name)) as f:
        g = json.load(f)
    S = np.array([float(v) for v in g["S"]], np.float32)
    E = np.array([float(v) for v in g["E"]], np.float32)
    targets = [(KIND[k], float(x)) for k, x, _ in g["expected"]]
    expected = [c for _, _, c in g["expected"]]
    return S, E, g["default_idx"], targets, expected


@pytest.mark.parametrize("name", ["worked_example.json", "non_pareto_default.json", "absolute_targets.json"])
def test_golden_examples(oracle_lib, name):
    S, E, d, targets, expected = _load_golden(name)
    ch = oracle_lib.select(S, E, d, targets)
    assert ch[0].tolist() == expected


# ------------------------------------------------------------ exact rational brute force

def _valid(s, e):
    return np.isfinite(s) and np.isfinite(e) and s > 0 and e > 0


def _brute(S, E, d, targets):
    """Definition with exact rationals; min over feasible of (key, index) (lowest index wins)."""
    n = len(S)
    if not _valid(S[d], E[d]):
        return [-1] * len(targets)
    V = [i for i in range(n) if _valid(S[i], E[i])]
    s = {i: Fraction(float(S[i])) for i in V}
    e = {i: Fraction(float(E[i])) for i in V}
    i_min = min(V, key=lambda i: (e[i], i))
    out = []
    for kind, x in targets:
        fr = Fraction(float(np.float32(x))) / 100   # oracle: (double)x / 100.0, exact on our grid
        cand = []
        for i in V:
            t = 1 / s[i]                                      # time normalised to default
            if kind == MAX_PERF:
                cand.append((-s[i], i))
            elif kind == MIN_ENERGY:
                cand.append((e[i], i))
            elif kind == MIN_EDP:
                cand.append((e[i] * t, i))
            elif kind == MIN_ED2P:
                cand.append((e[i] * t * t, i))
            elif kind == ES:
                if e[i] <= e[d] - fr * (e[d] - e[i_min]):
                    cand.append((-s[i], i))
            elif kind == PL:
                if s[i] >= s[d] - fr * (s[d] - s[i_min]):
                    cand.append((e[i], i))
            elif kind == ES_ABS:                             # L11/L46, Q1
                if e[i] <= (1 - fr) * e[d]:
                    cand.append((-s[i], i))
            elif kind == PL_ABS:
                if s[i] >= (1 - fr) * s[d]:
                    cand.append((e[i], i))
        out.append(min(cand)[1] if cand else -1)
    return out


def _grid_case(rng, n):
    """Values on a k/8 grid (exact in fp32/fp64) so ties are exact; some invalid entries."""
    S = rng.integers(1, 17, size=n).astype(np.float32) / 8
    E = rng.integers(1, 17, size=n).astype(np.float32) / 8
    bad = rng.uniform(size=n) < 0.1
    kinds = rng.integers(0, 4, size=n)
    S[bad & (kinds == 0)] = 0.0
    E[bad & (kinds == 1)] = -0.5
    S[bad & (kinds == 2)] = np.inf
    E[bad & (kinds == 3)] = np.nan
    return S, E


ALL_TARGETS = [(MAX_PERF, 0.0), (MIN_ENERGY, 0.0), (MIN_EDP, 0.0), (MIN_ED2P, 0.0)] + \
    [(ES, x) for x in (0.0, 25.0, 50.0, 75.0, 100.0)] + [(PL, x) for x in (0.0, 25.0, 50.0, 75.0, 100.0)]


# absolute-saving targets with x whose x/100 and 1 - x/100 are exact dyadic fractions
ABS_TARGETS = [(ES_ABS, x) for x in (0.0, 12.5, 25.0, 50.0, 75.0, 100.0)] + \
    [(PL_ABS, x) for x in (0.0, 25.0, 50.0, 87.5, 100.0)] + [(ES, 37.5), (PL, 62.5)]


def test_rational_brute_force_with_ties(oracle_lib):
    rng = np.random.default_rng(1234)
    n_cases = 10_000
    for c in range(n_cases):
        n = int(rng.integers(1, 9))
        S, E = _grid_case(rng, n)
        d = int(rng.integers(0, n))
        for tg in (ALL_TARGETS, ABS_TARGETS):
            ch = oracle_lib.select(S, E, d, tg)[0].tolist()
            assert ch == _brute(S, E, d, tg), (c, S, E, d)


# ------------------------------------------------------------- Pareto-front formulation

def _pareto_select(S, E, d, targets):
    """Independent formulation (PAPER L247, L69 'the red line is the Pareto front'): build the
    (max S, min E) Pareto set by pairwise dominance, then ES_x = highest-S front point with
    E <= threshold, PL_x = lowest-E front point with S >= threshold, MAX_PERF / MIN_ENERGY =
    front extremes.  Valid on tie-free inputs only."""
    n = len(S)
    pts = [(float(S[i]), float(E[i])) for i in range(n)]
    front = [i for i in range(n)
             if not any((pts[j][0] >= pts[i][0] and pts[j][1] <= pts[i][1] and pts[j] != pts[i])
                        for j in range(n))]
    e_min = min(front, key=lambda i: pts[i][1])
    out = []
    for kind, x in targets:
        fr = Fraction(x) / 100
        if kind == MAX_PERF:
            out.append(max(front, key=lambda i: pts[i][0]))
        elif kind == MIN_ENERGY:
            out.append(e_min)
        elif kind == ES:
            thr = Fraction(pts[d][1]) - fr * (Fraction(pts[d][1]) - Fraction(pts[e_min][1]))
            ok = [i for i in front if Fraction(pts[i][1]) <= thr]
            out.append(max(ok, key=lambda i: pts[i][0]))
        elif kind == PL:
            thr = Fraction(pts[d][0]) - fr * (Fraction(pts[d][0]) - Fraction(pts[e_min][0]))
            ok = [i for i in front if Fraction(pts[i][0]) >= thr]
            out.append(min(ok, key=lambda i: pts[i][1]))
    return out


def test_pareto_cross_check(oracle_lib):
    rng = np.random.default_rng(99)
    targets = [(MAX_PERF, 0.0), (MIN_ENERGY, 0.0)] + [(ES, x) for x in (0, 10, 25, 33, 50, 75, 90, 100)] + \
        [(PL, x) for x in (0, 10, 25, 33, 50, 75, 90, 100)]
    targets = [(k, float(x)) for k, x in targets]
    checked = 0
    for _ in range(3000):
        n = int(rng.integers(1, 9))
        S = rng.uniform(0.3, 1.3, size=n).astype(np.float32)
        E = rng.uniform(0.5, 1.5, size=n).astype(np.float32)
        if len(set(S.tolist())) < n or len(set(E.tolist())) < n:
            continue
        d = int(rng.integers(0, n))
        ch = oracle_lib.select(S, E, d, targets[:9])[0].tolist() + \
            oracle_lib.select(S, E, d, targets[9:])[0].tolist()          # <= 16 targets per call
        assert ch == _pareto_select(S, E, d, targets)
        checked += 1
    assert checked > 2500


# ------------------------------------------------------------------ definition properties

def _oracle_preds(oracle_lib, cfg="c1"):
    from paper_conf_sc_fandccfc23_b200 import workloads as W
    w = W.make_config(cfg)
    S, E = oracle_lib.predict(w.speedup, w.energy, w.features, w.freqs, w.default_idx)
    return w, S, E


def test_es100_is_min_energy_and_pl100_equals_min_energy(oracle_lib):
    """'ES_100 is the frequency with the lowest [energy]' (reading Q2)."""
    w, S, E = _oracle_preds(oracle_lib)
    ch = oracle_lib.select(S, E, w.default_idx, [(ES, 100.0), (PL, 100.0), (MIN_ENERGY, 0.0)])
    for k in range(S.shape[0]):
        assert E[k, ch[k, 0]] == E[k].min()
        assert ch[k, 1] == ch[k, 2]


def test_x0_constraints_and_nesting(oracle_lib):
    """ES_0: max S subject to E <= E_def; PL_0: min E subject to S >= S_def.  Monotone in x:
    ES feasible sets shrink as x grows (thr in [E_min, E_def]); PL with S_minE <= S_def grows."""
    w, S, E = _oracle_preds(oracle_lib)
    d = w.default_idx
    xs = [0.0, 10.0, 25.0, 50.0, 75.0, 90.0, 100.0]
    es = oracle_lib.select(S, E, d, [(ES, x) for x in xs])
    pl = oracle_lib.select(S, E, d, [(PL, x) for x in xs])
    for k in range(S.shape[0]):
        assert E[k, es[k, 0]] <= E[k, d] and S[k, es[k, 0]] == S[k][E[k] <= E[k, d]].max()
        assert S[k, pl[k, 0]] >= S[k, d] and E[k, pl[k, 0]] == E[k][S[k] >= S[k, d]].min()
        for a in range(len(xs) - 1):
            assert S[k, es[k, a + 1]] <= S[k, es[k, a]]
            assert E[k, es[k, a + 1]] <= E[k, es[k, a]]
            imin = int(np.argmin(E[k]))
            if S[k, imin] <= S[k, d]:
                assert E[k, pl[k, a + 1]] <= E[k, pl[k, a]]
                assert S[k, pl[k, a + 1]] <= S[k, pl[k, a]]
            else:
                assert pl[k, a] == imin


def test_dominance_and_edp_definitions(oracle_lib):
    w, S, E = _oracle_preds(oracle_lib)
    ch = oracle_lib.select(S, E, w.default_idx, ALL_TARGETS)
    for k in range(S.shape[0]):
        assert np.all(S[k, ch[k, 0]] >= S[k, ch[k]])         # MAX_PERF dominates in speed
        assert np.all(E[k, ch[k, 1]] <= E[k, ch[k]])         # MIN_ENERGY dominates in energy
        # EDP = E*T and ED2P = E*T^2 with T = 1/S, exact rationals (L253)
        s = [Fraction(float(v)) for v in S[k]]
        e = [Fraction(float(v)) for v in E[k]]
        edp = [e[i] / s[i] for i in range(len(s))]
        ed2p = [e[i] / (s[i] * s[i]) for i in range(len(s))]
        for key, col in ((edp, 2), (ed2p, 3)):
            best = min(key)
            # the chosen clock's rational objective is within 1 ulp (fp64) of the true minimum
            assert float(key[ch[k, col]]) <= float(best) * (1 + 1e-15)


def test_normalised_default_is_one(oracle_lib):
    w, S, E = _oracle_preds(oracle_lib)
    assert np.all(S[:, w.default_idx] == 1.0) and np.all(E[:, w.default_idx] == 1.0)


def test_constant_predictions_all_tie_to_index0(oracle_lib):
    S = np.ones((3, 17), np.float32)
    E = np.ones((3, 17), np.float32)
    ch = oracle_lib.select(S, E, 5, ALL_TARGETS)
    assert np.all(ch == 0)


def test_invalid_default_gives_minus_one(oracle_lib):
    S = np.ones((1, 4), np.float32)
    E = np.ones((1, 4), np.float32)
    S[0, 2] = np.nan
    assert np.all(oracle_lib.select(S, E, 2, ALL_TARGETS) == -1)
    E[0, 2] = 0.0
    S[0, 2] = 1.0
    assert np.all(oracle_lib.select(S, E, 2, ALL_TARGETS) == -1)


def test_validation(oracle_lib):
    S = np.ones((1, 4), np.float32)
    with pytest.raises(oracle_lib.OracleError):
        oracle_lib.select(S, S, 4, ALL_TARGETS)            # default out of range
    with pytest.raises(oracle_lib.OracleError):
        oracle_lib.select(S, S, 0, [(ES, 101.0)])          # x outside [0, 100]
    with pytest.raises(oracle_lib.OracleError):
        oracle_lib.select(S, S, 0, [(8, 0.0)])             # unknown kind
    with pytest.raises(oracle_lib.OracleError):
        oracle_lib.select(S, S, 0, [(ES_ABS, -1.0)])       # x outside [0, 100]
    with pytest.raises(oracle_lib.OracleError):
        oracle_lib.select(S, S, 0, [(ES, float("nan"))])
    with pytest.raises(oracle_lib.OracleError):
        oracle_lib.select(S, S, 0, [(MAX_PERF, 0.0)] * 17)  # > 16 targets

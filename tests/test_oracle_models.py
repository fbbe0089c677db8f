"""Pins for the oracle's model-evaluation and normalisation steps (oracle.c: oracle_model_eval,
predict_kernel) against library routines and closed forms.

  * Random Forest regression (Table 2): scikit-learn RandomForestRegressor /
    DecisionTreeRegressor predictions, exported to the sklearn `tree_` layout the C-ABI uses
    (thresholds rounded toward -inf to fp32, leaves rounded to fp32 and written back into
    the sklearn trees so both sides evaluate the same fp32 numbers; Q9/Q10).
  * Linear / Lasso (L386): sklearn LinearRegression / Lasso.predict.
  * Default-clock normalisation (L69): S = E = 1 exactly at default; invariance to 2^k scaling.
"""
import numpy as np
import pytest
from sklearn.ensemble import RandomForestRegressor
from sklearn.linear_model import Lasso, LinearRegression
from sklearn.tree import DecisionTreeRegressor

from paper_conf_sc_fandccfc23_b200 import workloads as W


def _round_down_f32(t):
    t32 = t.astype(np.float32)
    up = t32.astype(np.float64) > t
    t32[up] = np.nextafter(t32[up], np.float32(-np.inf))
    return t32


def export_sklearn(estimators, n_inputs):
    """sklearn trees -> ModelSpec (same arrays as tree_.feature/children_*/threshold/value).
    Leaves are rounded to fp32 and written back into the sklearn trees."""
    feats, lefts, rights, vals, off = [], [], [], [], [0]
    for est in estimators:
        t = est.tree_
        leaf = t.children_left < 0
        v = np.where(leaf, t.value[:, 0, 0], t.threshold)
        v32 = np.where(leaf, t.value[:, 0, 0].astype(np.float32), _round_down_f32(t.threshold))
        t.value[:, 0, 0] = np.where(leaf, v32.astype(np.float64), t.value[:, 0, 0])
        feats.append(np.where(leaf, -1, t.feature).astype(np.int32))
        lefts.append(t.children_left.astype(np.int32))
        rights.append(t.children_right.astype(np.int32))
        vals.append(v32.astype(np.float32))
        off.append(off[-1] + t.node_count)
        del v
    return W.ModelSpec(n_inputs=n_inputs, forest_weight=1.0, tree_offset=np.array(off, np.int64),
                       feature=np.concatenate(feats), left=np.concatenate(lefts),
                       right=np.concatenate(rights), value=np.concatenate(vals))


def _dvfs_data(rng, n, F, freqs):
    X = np.empty((n, F + 1), np.float32)
    X[:, :F] = np.floor(np.exp2(rng.uniform(0, 10, size=(n, F))))
    X[:, F] = freqs[rng.integers(0, len(freqs), size=n)]
    beta = 1 / (1 + np.exp(-(np.log2(1 + X[:, 0]) - np.log2(1 + X[:, 1])) / 3))
    y = 1.0 / (beta * 1312.0 / X[:, F] + 1 - beta) + rng.normal(0, 0.01, size=n)
    return X, y


def test_random_forest_matches_sklearn_exactly(oracle_lib):
    rng = np.random.default_rng(7)
    F = 6
    freqs = W.clock_table(64)
    X, y = _dvfs_data(rng, 3000, F, freqs)
    rf = RandomForestRegressor(n_estimators=25, max_depth=9, random_state=0).fit(X, y)
    spec = export_sklearn(rf.estimators_, F + 1)
    ref = rf.predict(X[:500])            # mean of per-tree fp32-rounded leaves, fp64
    got = np.array([oracle_lib.model_eval(spec, x) for x in X[:500]])
    # fp32 leaves in a narrow range: the fp64 sum is exact, so order does not matter
    np.testing.assert_array_equal(got, ref)


def test_decision_tree_threshold_equality_goes_left(oracle_lib):
    """x == threshold routes left (sklearn: X[:, f] <= threshold; Q9)."""
    X = np.array([[0.0], [1.0], [2.0], [3.0]], np.float32)
    y = np.array([0.0, 0.0, 1.0, 1.0])
    dt = DecisionTreeRegressor(max_depth=1).fit(X, y)
    spec = export_sklearn([dt], 1)
    thr = spec.value[0]
    assert spec.feature[0] == 0
    below = oracle_lib.model_eval(spec, np.array([thr], np.float32))
    above = oracle_lib.model_eval(spec, np.array([np.nextafter(thr, np.float32(np.inf))], np.float32))
    assert below == dt.predict(np.array([[thr]], np.float32))[0] == 0.0
    assert above == 1.0
    # hand-built 3-node tree, node ids shuffled: root 0 -> leaves 2 (left) / 1 (right)
    hand = W.ModelSpec(n_inputs=2, forest_weight=1.0, tree_offset=np.array([0, 3]),
                       feature=np.array([1, -1, -1], np.int32), left=np.array([2, -1, -1], np.int32),
                       right=np.array([1, -1, -1], np.int32),
                       value=np.array([500.0, 2.5, 0.75], np.float32))
    assert oracle_lib.model_eval(hand, np.array([9.0, 500.0], np.float32)) == 0.75
    assert oracle_lib.model_eval(hand, np.array([9.0, 500.5], np.float32)) == 2.5


@pytest.mark.parametrize("cls", [LinearRegression, Lasso])
def test_linear_matches_sklearn(oracle_lib, cls):
    rng = np.random.default_rng(3)
    F = 12
    X, y = _dvfs_data(rng, 500, F, W.clock_table(128))
    m = cls().fit(X.astype(np.float64), y) if cls is LinearRegression else cls(alpha=1e-4, max_iter=10000).fit(X.astype(np.float64), y)
    spec = W.ModelSpec(n_inputs=F + 1, linear_weight=1.0, lin_w=m.coef_.astype(np.float64),
                       lin_b=float(m.intercept_))
    ref = m.predict(X[:200].astype(np.float64))
    got = np.array([oracle_lib.model_eval(spec, x) for x in X[:200]])
    np.testing.assert_allclose(got, ref, rtol=1e-12, atol=1e-12)
    zero = W.ModelSpec(n_inputs=F + 1, linear_weight=1.0, lin_w=np.zeros(F + 1), lin_b=0.625)
    assert oracle_lib.model_eval(zero, X[0]) == 0.625


def test_identical_trees_equal_one_tree_and_stump(oracle_lib):
    rng = np.random.default_rng(11)
    freqs = W.clock_table(33)
    one = W.random_forest_spec(rng, 4, freqs, 1, 6)
    T = 37
    n = one.n_nodes
    many = W.ModelSpec(n_inputs=5, forest_weight=1.0, tree_offset=np.arange(T + 1, dtype=np.int64) * n,
                       feature=np.tile(one.feature, T), left=np.tile(one.left, T),
                       right=np.tile(one.right, T), value=np.tile(one.value, T))
    for _ in range(50):
        x = np.concatenate([np.floor(np.exp2(rng.uniform(0, 10, 4))), [freqs[rng.integers(0, 33)]]]).astype(np.float32)
        assert oracle_lib.model_eval(many, x) == oracle_lib.model_eval(one, x)
    stump = W.ModelSpec(n_inputs=5, forest_weight=1.0, tree_offset=np.array([0, 1]),
                        feature=np.array([-1], np.int32), left=np.array([-1], np.int32),
                        right=np.array([-1], np.int32), value=np.array([1.375], np.float32))
    assert oracle_lib.model_eval(stump, np.zeros(5, np.float32)) == 1.375


def test_weighted_ensemble_closed_form(oracle_lib):
    """Ensemble reading Q7: m = w_lin*lin + w_forest*forest (linear first)."""
    stump = W.ModelSpec(n_inputs=2, forest_weight=0.5, tree_offset=np.array([0, 1]),
                        feature=np.array([-1], np.int32), left=np.array([-1], np.int32),
                        right=np.array([-1], np.int32), value=np.array([3.0], np.float32),
                        linear_weight=0.25, lin_w=np.array([1.0, 2.0]), lin_b=0.5)
    assert oracle_lib.model_eval(stump, np.array([1.0, 4.0], np.float32)) == 0.25 * 9.5 + 0.5 * 3.0


def test_visit_count_complete_trees(oracle_lib):
    w = W.make_config("c1")
    r = oracle_lib.sweep_workload(w, count_visits=True)
    assert r["visits"] == w.n_kernels * w.n_freqs * 2 * 10 * 8   # T*D per model per eval


def test_normalisation_exact_and_scale_invariant(oracle_lib):
    w = W.make_config("c1")
    S, E = oracle_lib.predict(w.speedup, w.energy, w.features, w.freqs, w.default_idx)
    assert np.all(S[:, w.default_idx] == 1.0) and np.all(E[:, w.default_idx] == 1.0)
    sp2 = w.speedup.contiguous()
    sp2.value = sp2.value.copy()
    leaf = sp2.feature < 0
    sp2.value[leaf] *= np.float32(8.0)                    # 2^3: exact in fp32 and fp64
    S2, E2 = oracle_lib.predict(sp2, w.energy, w.features, w.freqs, w.default_idx)
    np.testing.assert_array_equal(S2, S)
    np.testing.assert_array_equal(E2, E)
    Sr, _ = oracle_lib.predict(sp2, w.energy, w.features, w.freqs, -1)
    Sr1, _ = oracle_lib.predict(w.speedup, w.energy, w.features, w.freqs, -1)
    np.testing.assert_array_equal(Sr, Sr1 * 8)


def test_sklearn_forest_full_pipeline_normalised(oracle_lib):
    """Normalised predictions through oracle_predict equal (float)(sk(k,f)/sk(k,f_def))."""
    rng = np.random.default_rng(5)
    F = 4
    freqs = W.clock_table(40)
    d = W.default_index(freqs)
    X, y = _dvfs_data(rng, 2000, F, freqs)
    rf = RandomForestRegressor(n_estimators=10, max_depth=7, random_state=1).fit(X, y)
    spec = export_sklearn(rf.estimators_, F + 1)
    feats = X[:20, :F].copy()
    S, E = oracle_lib.predict(spec, spec, feats, freqs, d)
    P = np.empty((20, len(freqs)))
    for i, f in enumerate(freqs):
        Xi = np.concatenate([feats, np.full((20, 1), f, np.float32)], axis=1)
        P[:, i] = rf.predict(Xi)
    np.testing.assert_array_equal(S, (P / P[:, d:d + 1]).astype(np.float32))


def export_svr(pipe, n_inputs):
    """sklearn Pipeline(StandardScaler, SVR(kernel="rbf")) -> ModelSpec SVR member; the support
    vectors are rounded to fp32 (the model format) and written back into the sklearn SVR."""
    scaler, svr = pipe.named_steps["standardscaler"], pipe.named_steps["svr"]
    sv32 = svr.support_vectors_.astype(np.float32)
    svr.support_vectors_[:] = sv32.astype(np.float64)
    svr._sparse = False
    return W.ModelSpec(n_inputs=n_inputs, svr_weight=1.0, sv=sv32, dual_coef=svr.dual_coef_[0].copy(),
                       svr_gamma=float(svr._gamma), svr_intercept=float(svr.intercept_[0]),
                       in_mean=scaler.mean_.copy(), in_scale=scaler.scale_.copy())


def test_svr_rbf_matches_sklearn(oracle_lib):
    """SVR with RBF kernel (Table 2) on standardized inputs: scikit-learn predictions."""
    from sklearn.pipeline import make_pipeline
    from sklearn.preprocessing import StandardScaler
    from sklearn.svm import SVR
    rng = np.random.default_rng(12)
    F = 5
    X, y = _dvfs_data(rng, 600, F, W.clock_table(64))
    pipe = make_pipeline(StandardScaler(), SVR(kernel="rbf", gamma=0.3, C=3.0, epsilon=0.01)).fit(X.astype(np.float64), y)
    spec = export_svr(pipe, F + 1)
    assert spec.n_sv > 50
    Xt = X[:200]
    ref = pipe.predict(Xt.astype(np.float64))
    got = np.array([oracle_lib.model_eval(spec, x) for x in Xt])
    np.testing.assert_allclose(got, ref, rtol=1e-11, atol=1e-12)


def test_svr_closed_form_and_ensemble_order(oracle_lib):
    """Two support vectors in 2-D with hand-computed distances; svr joins the ensemble last (Q7)."""
    spec = W.ModelSpec(n_inputs=2, svr_weight=1.0, sv=np.array([[0.0, 0.0], [1.0, -1.0]], np.float32),
                       dual_coef=np.array([2.0, -0.5]), svr_gamma=0.25, svr_intercept=0.125,
                       in_mean=np.array([1.0, 10.0]), in_scale=np.array([2.0, 4.0]))
    x = np.array([3.0, 6.0], np.float32)        # z = (1, -1): d0^2 = 2, d1^2 = 0
    assert abs(oracle_lib.model_eval(spec, x) - (0.125 + 2.0 * np.exp(-0.5) - 0.5)) < 1e-15
    x = np.array([1.0, 10.0], np.float32)       # z = (0, 0): d0^2 = 0, d1^2 = 2
    assert abs(oracle_lib.model_eval(spec, x) - (0.125 + 2.0 - 0.5 * np.exp(-0.5))) < 1e-15
    both = W.ModelSpec(n_inputs=2, svr_weight=0.5, sv=spec.sv, dual_coef=spec.dual_coef, svr_gamma=0.25,
                       svr_intercept=0.125, in_mean=spec.in_mean, in_scale=spec.in_scale,
                       linear_weight=2.0, lin_w=np.array([1.0, 0.0]), lin_b=0.0)
    want = 2.0 * 1.0 + 0.5 * (0.125 + 2.0 - 0.5 * np.exp(-0.5))
    assert abs(oracle_lib.model_eval(both, x) - want) < 1e-15

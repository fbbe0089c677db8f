"""Pins for the four-model variant of the oracle (oracle.c: oracle_sweep4, SURVEY
NEXT f1): direct EDP / ED2P regressors replace the derived E/S, E/S^2 keys of MIN_EDP / MIN_ED2P."""
import numpy as np

from paper_conf_sc_fandccfc23_b200 import workloads as W


def lookup_tree(freqs, values, F):
    """One tree splitting only on the clock (input F) at midpoints, leaf i = values[i]: the model's
    output at clock i is exactly values[i] (a per-clock lookup table)."""
    feature, left, right, value = [], [], [], []

    def node(a, b):
        idx = len(feature)
        feature.append(-1); left.append(-1); right.append(-1); value.append(0.0)
        if b - a == 1:
            value[idx] = values[a]
            return idx
        mid = (a + b) // 2
        feature[idx] = F
        value[idx] = float(np.float32(0.5 * (float(freqs[mid - 1]) + float(freqs[mid]))))
        l = node(a, mid); r = node(mid, b)
        left[idx], right[idx] = l, r
        return idx

    node(0, len(freqs))
    return W.ModelSpec(n_inputs=F + 1, forest_weight=1.0, tree_offset=np.array([0, len(feature)], np.int64),
                       feature=np.array(feature, np.int32), left=np.array(left, np.int32),
                       right=np.array(right, np.int32), value=np.array(value, np.float32))


def test_without_direct_models_equals_two_model_oracle():
    import oracle
    w = W.make_config("c1")
    r4 = oracle.sweep4([w.speedup, w.energy, None, None], w.features, w.freqs, w.default_idx, w.targets)
    np.testing.assert_array_equal(r4["choice"], oracle.sweep_workload(w)["choice"])


def test_direct_models_decide_edp_and_ed2p_by_argmin():
    """With per-clock lookup-table EDP/ED2P models the MIN_EDP / MIN_ED2P choices are the first
    argmin of the tables (numpy), independent of S and E; other targets are unchanged."""
    import oracle
    rng = np.random.default_rng(8)
    w = W.make_config("c1")
    F, n_f, d = w.n_features, w.n_freqs, w.default_idx
    for trial in range(20):
        edp = rng.integers(1, 9, size=n_f).astype(np.float32) / 4        # ties on a grid
        ed2p = rng.integers(1, 9, size=n_f).astype(np.float32) / 4
        bad = rng.integers(0, n_f)
        if bad != d:
            edp[bad] = -1.0                                               # not a candidate
        models = [w.speedup, w.energy, lookup_tree(w.freqs, edp, F), lookup_tree(w.freqs, ed2p, F)]
        r = oracle.sweep4(models, w.features, w.freqs, d, w.targets)["choice"]
        base = oracle.sweep_workload(w)["choice"]
        e = edp.astype(np.float64).copy()
        e[e <= 0] = np.inf
        assert np.all(r[:, 2] == int(np.argmin(e)))
        assert np.all(r[:, 3] == int(np.argmin(ed2p)))
        np.testing.assert_array_equal(r[:, [0, 1, 4, 5]], base[:, [0, 1, 4, 5]])


def test_table2_best_models_config():
    import oracle
    models, freqs, d = W.make_models4("c1")
    feats = W.make_features("c1")
    r = oracle.sweep4(models, feats, freqs, d, W.targets_six(), want_pred=True)
    P = r["P"]
    assert np.all(P[:, :, d] == 1.0)                                      # every model normalised
    assert (r["choice"] >= 0).all()

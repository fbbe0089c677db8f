"""Seeded synthetic workloads shaped like the paper's.

This module is the ONLY code shared by the CUDA path and the CPU oracle: it draws
inputs (feature vectors, core-clock tables, "trained-shaped" regression models and
energy-target lists) and holds none of the method's arithmetic (no prediction,
normalisation, objective or selection).  Both sides receive the same arrays.

Paper passages the shapes follow (PAPER.md line numbers):
  * static feature vector k (10 instruction-class counts)  L291-L311 (§6.1, Table 1)
  * core-clock tables, V100 196 clocks 135..1530 MHz       L59-L65  (Fig. 1)
  * default clock 1312 MHz                                  L69      (§2.2)
  * model families Linear / RandomForest                    L386, Table 2 (L398-L412)
  * energy targets MAX_PERF, MIN_ENERGY, MIN_EDP, MIN_ED2P,
    ES_x, PL_x                                              L182, L253-L271, Table 2
  * CloverLeaf / MiniWeather at 64 GPUs (config c5)         L362, L416

Model description format (the C-ABI's `syn_model_desc`, include/synergy.h):
scikit-learn's `tree_` layout, structure-of-arrays over all nodes of all trees,
node ids tree-local (root = 0), children -1 at leaves, `value` = split threshold at
internal nodes and leaf value at leaves (fp32), `tree_offset[t]..tree_offset[t+1]`
the node range of tree t.  Input index F (== n_inputs-1) is the core clock in MHz.
"""
from __future__ import annotations

from dataclasses import dataclass, field
from typing import Optional

import numpy as np

# Energy-target kinds (include/synergy.h: syn_target_kind).  PAPER L182, L382, Table 2.
# ES_ABS / PL_ABS: the absolute-saving reading of L11/L46 (Q1).
MAX_PERF, MIN_ENERGY, MIN_EDP, MIN_ED2P, ES, PL, ES_ABS, PL_ABS = 0, 1, 2, 3, 4, 5, 6, 7
TARGET_NAMES = {MAX_PERF: "MAX_PERF", MIN_ENERGY: "MIN_ENERGY", MIN_EDP: "MIN_EDP",
                MIN_ED2P: "MIN_ED2P", ES: "ES", PL: "PL", ES_ABS: "ES_ABS", PL_ABS: "PL_ABS"}

N_STATIC = 12           # Table 1's ten counts + two synthetic count columns
SEED_BASE = 0x5EED0000
FEATURE_CHUNK = 1 << 16  # rows per independently seeded feature chunk (shard-regenerable)

# Table 1 column order: int_add int_mul int_div int_bw float_add float_mul float_div sf
# gl_access loc_access, then two extra synthetic count columns.
_OFTEN_ABSENT = (2, 6, 7, 9)   # int_div, float_div, sf, loc_access -> zero prob 0.25


def targets_six():
    """The six-objective list of configs c1, c2, c4, c5."""
    return [(MAX_PERF, 0.0), (MIN_ENERGY, 0.0), (MIN_EDP, 0.0), (MIN_ED2P, 0.0),
            (ES, 50.0), (PL, 50.0)]


def targets_es_pl():
    """Config c3: ES_x / PL_x for x in {25, 50, 75} (BASELINE.json configs[2])."""
    return [(ES, 25.0), (ES, 50.0), (ES, 75.0), (PL, 25.0), (PL, 50.0), (PL, 75.0)]


@dataclass
class ModelSpec:
    """Host-side model description; mirrors `syn_model_desc` field by field."""
    n_inputs: int
    linear_weight: float = 0.0
    lin_w: Optional[np.ndarray] = None     # float64 [n_inputs]
    lin_b: float = 0.0
    forest_weight: float = 0.0
    tree_offset: np.ndarray = field(default_factory=lambda: np.zeros(1, np.int64))
    feature: np.ndarray = field(default_factory=lambda: np.zeros(0, np.int32))
    left: np.ndarray = field(default_factory=lambda: np.zeros(0, np.int32))
    right: np.ndarray = field(default_factory=lambda: np.zeros(0, np.int32))
    value: np.ndarray = field(default_factory=lambda: np.zeros(0, np.float32))
    # SVR with RBF kernel (Table 2 "SVR"), scikit-learn convention on standardized
    # inputs: svr(x) = intercept + sum_j dual_coef[j] * exp(-gamma * ||(x - in_mean)/in_scale - sv[j]||^2)
    svr_weight: float = 0.0
    sv: Optional[np.ndarray] = None          # float32 [n_sv][n_inputs] (standardized space)
    dual_coef: Optional[np.ndarray] = None   # float64 [n_sv]
    svr_gamma: float = 0.0
    svr_intercept: float = 0.0
    in_mean: Optional[np.ndarray] = None     # float64 [n_inputs]
    in_scale: Optional[np.ndarray] = None    # float64 [n_inputs]

    @property
    def n_sv(self) -> int:
        return 0 if self.svr_weight == 0.0 or self.sv is None else int(self.sv.shape[0])

    @property
    def n_trees(self) -> int:
        return int(len(self.tree_offset) - 1) if self.forest_weight != 0.0 else 0

    @property
    def n_nodes(self) -> int:
        return int(self.tree_offset[-1]) if self.forest_weight != 0.0 else 0

    def contiguous(self) -> "ModelSpec":
        c = np.ascontiguousarray
        return ModelSpec(
            n_inputs=int(self.n_inputs), linear_weight=float(self.linear_weight),
            lin_w=None if self.lin_w is None else c(self.lin_w, dtype=np.float64),
            lin_b=float(self.lin_b), forest_weight=float(self.forest_weight),
            tree_offset=c(self.tree_offset, dtype=np.int64), feature=c(self.feature, dtype=np.int32),
            left=c(self.left, dtype=np.int32), right=c(self.right, dtype=np.int32),
            value=c(self.value, dtype=np.float32), svr_weight=float(self.svr_weight),
            sv=None if self.sv is None else c(self.sv, dtype=np.float32),
            dual_coef=None if self.dual_coef is None else c(self.dual_coef, dtype=np.float64),
            svr_gamma=float(self.svr_gamma), svr_intercept=float(self.svr_intercept),
            in_mean=None if self.in_mean is None else c(self.in_mean, dtype=np.float64),
            in_scale=None if self.in_scale is None else c(self.in_scale, dtype=np.float64))


@dataclass
class Workload:
    name: str
    features: np.ndarray        # float32 [n_kernels, F], row-major
    freqs: np.ndarray           # float32 [n_freqs], strictly ascending MHz
    default_idx: int
    speedup: ModelSpec
    energy: ModelSpec
    targets: list               # [(kind, x)]
    n_kernels_total: int = 0    # full config size when `features` is a shard/sample
    row0: int = 0               # first global row of `features`

    @property
    def n_kernels(self) -> int:
        return int(self.features.shape[0])

    @property
    def n_features(self) -> int:
        return int(self.features.shape[1])

    @property
    def n_freqs(self) -> int:
        return int(self.freqs.shape[0])

    def target_arrays(self):
        kinds = np.array([k for k, _ in self.targets], dtype=np.int32)
        xs = np.array([x for _, x in self.targets], dtype=np.float32)
        return kinds, xs


# --------------------------------------------------------------------------- clocks

def clock_table(n_freqs: int, f_lo: int = 135, f_hi: int = 1530) -> np.ndarray:
    """V100-shaped clock table (PAPER): f_i = f_lo + round_half_even(i*(f_hi-f_lo)/(n-1)).

    Integers, exact in fp32, strictly ascending for n <= f_hi-f_lo+1.
    """
    if n_freqs == 1:
        return np.array([f_lo], dtype=np.float32)
    i = np.arange(n_freqs, dtype=np.float64)
    f = f_lo + np.round(i * (f_hi - f_lo) / (n_freqs - 1))   # numpy rounds half to even
    return f.astype(np.float32)


def default_index(freqs: np.ndarray, f_default: float = 1312.0) -> int:
    """Index nearest to the V100 default clock 1312 MHz; lowest index on a tie."""
    d = np.abs(freqs.astype(np.float64) - f_default)
    return int(np.flatnonzero(d == d.min())[0])


# ------------------------------------------------------------------------- features

def _feature_chunk(seed_seq: np.random.SeedSequence, chunk: int, rows: int, F: int) -> np.ndarray:
    rng = np.random.Generator(np.random.PCG64(np.random.SeedSequence(
        seed_seq.entropy, spawn_key=tuple(seed_seq.spawn_key) + (chunk,))))
    v = np.floor(np.exp2(rng.uniform(0.0, 10.0, size=(rows, F))))
    pz = np.full(F, 0.05)
    for j in _OFTEN_ABSENT:
        if j < F:
            pz[j] = 0.25
    v[rng.uniform(size=(rows, F)) < pz] = 0.0
    return v.astype(np.float32)


def gen_features(seed_seq, n_rows: int, F: int, row0: int = 0, n: Optional[int] = None) -> np.ndarray:
    """Rows [row0, row0+n) of an unbounded seeded feature population (n defaults to n_rows-row0).

    Values floor(2^U(0,10)) (integer counts 1..1023, exact in fp32), zeros with prob 0.25
    for often-absent op classes else 0.05.  Chunked so any shard regenerates alone.
    """
    if n is None:
        n = n_rows - row0
    out = np.empty((n, F), dtype=np.float32)
    r = row0
    while r < row0 + n:
        c = r // FEATURE_CHUNK
        c0 = c * FEATURE_CHUNK
        rows = FEATURE_CHUNK          # chunk contents never depend on n_rows
        blk = _feature_chunk(seed_seq, c, rows, F)
        a = r - c0
        b = min(rows, row0 + n - c0)
        out[r - row0:r - row0 + (b - a)] = blk[a:b]
        r += b - a
    return out


# ---------------------------------------------------------------------------- trees

class _DVFS:
    """Analytic DVFS shape used only to give leaves plausible values (not the method).

    beta (compute-boundness) = sigmoid(a . z + a0) of log-scaled box-centre features;
    S(f) = 1 / (beta f_def / f + 1 - beta);  P(f) = 0.3 + 0.7 (f/f_max)^2.5;
    E(f) = P(f) / S(f) / P(f_def).  Convex energy with a mid-range minimum.
    """

    def __init__(self, rng, F, freqs, def_idx):
        self.a = rng.normal(0.0, 1.0, size=F)
        self.a0 = rng.normal(0.0, 0.5)
        self.f_def = float(freqs[def_idx])
        self.f_max = float(freqs[-1])

    def beta(self, centre):                 # centre [..., F]
        z = np.log2(1.0 + centre) / 10.0 - 0.5
        return 1.0 / (1.0 + np.exp(-(z @ self.a + self.a0) * 2.0))

    def speedup(self, beta, f):
        return 1.0 / (beta * self.f_def / f + 1.0 - beta)

    def power(self, f):
        return 0.3 + 0.7 * (f / self.f_max) ** 2.5

    def energy(self, beta, f):
        return self.power(f) / self.speedup(beta, f) / self.power(self.f_def)


def _complete_trees(rng, n_trees, depth, F, freqs, dvfs: _DVFS, which: str, p_freq=0.25,
                    noise=0.01):
    """Complete binary trees of depth `depth`, BFS-numbered (children 2n+1, 2n+2).

    Splits on the clock (input F) with prob p_freq at a midpoint between adjacent table
    clocks inside the node's clock box, else on a static feature at integer+0.5 inside the
    node's box (so generated inputs never sit exactly on a threshold).  Leaves evaluate the
    analytic DVFS shape at the box centre plus N(0, noise), clamped to [0.25, 4).
    """
    nf = len(freqs)
    fr = freqs.astype(np.float64)
    nn = (1 << (depth + 1)) - 1
    feature = np.full((n_trees, nn), -1, dtype=np.int32)
    value = np.zeros((n_trees, nn), dtype=np.float32)
    # boxes for the current level: static [lo, hi) in count units, clock index [ilo, ihi]
    lo = np.zeros((n_trees, 1, F))
    hi = np.full((n_trees, 1, F), 1024.0)
    ilo = np.zeros((n_trees, 1), dtype=np.int64)
    ihi = np.full((n_trees, 1), nf - 1, dtype=np.int64)
    for lev in range(depth):
        m = 1 << lev
        first = m - 1
        use_f = (rng.uniform(size=(n_trees, m)) < p_freq) & (ihi > ilo)
        # static split: feature uniform, threshold integer+0.5 strictly inside the box
        j = rng.integers(0, F, size=(n_trees, m))
        blo = np.take_along_axis(lo, j[..., None], 2)[..., 0]
        bhi = np.take_along_axis(hi, j[..., None], 2)[..., 0]
        cand_lo = np.floor(blo)          # thr = k + 0.5 with blo <= k, k + 1 <= bhi
        cand_hi = np.ceil(bhi) - 1.0
        ok = cand_hi >= cand_lo
        # log-uniform-ish integer inside [cand_lo, cand_hi]
        u = rng.uniform(size=(n_trees, m))
        l0 = np.log2(cand_lo + 1.0)
        l1 = np.log2(np.maximum(cand_hi, cand_lo) + 1.0)
        k = np.clip(np.floor(np.exp2(l0 + u * (l1 - l0)) - 1.0), cand_lo, np.maximum(cand_hi, cand_lo))
        thr_s = k + 0.5
        # degenerate static box and no clock room: fall back to an out-of-box static split
        use_f = use_f | (~ok & (ihi > ilo))
        # clock split: position s in (ilo, ihi], threshold midpoint of clocks s-1, s
        s = ilo + 1 + np.floor(rng.uniform(size=(n_trees, m)) * np.maximum(ihi - ilo, 1)).astype(np.int64)
        s = np.minimum(s, np.maximum(ihi, ilo + 1))
        s = np.clip(s, 1, max(nf - 1, 1))
        thr_f = 0.5 * (fr[s - 1] + fr[np.minimum(s, nf - 1)]) if nf > 1 else np.zeros_like(fr[s - 1])
        feat = np.where(use_f, F, j).astype(np.int32)
        thr = np.where(use_f, thr_f, np.where(ok, thr_s, 1e9))
        feature[:, first:first + m] = feat
        value[:, first:first + m] = thr.astype(np.float32)
        # children boxes
        lo2 = np.repeat(lo, 2, axis=1)
        hi2 = np.repeat(hi, 2, axis=1)
        ilo2 = np.repeat(ilo, 2, axis=1)
        ihi2 = np.repeat(ihi, 2, axis=1)
        L = np.arange(m) * 2
        tr = np.arange(n_trees)[:, None]
        st = ~use_f
        jj = j
        # static: left child hi = thr, right child lo = thr
        hi2[tr, L, jj] = np.where(st, np.minimum(hi2[tr, L, jj], thr), hi2[tr, L, jj])
        lo2[tr, L + 1, jj] = np.where(st, np.maximum(lo2[tr, L + 1, jj], thr), lo2[tr, L + 1, jj])
        # clock: left child ihi = s-1, right child ilo = s
        ihi2[:, L] = np.where(use_f, np.minimum(ihi2[:, L], s - 1), ihi2[:, L])
        ilo2[:, L + 1] = np.where(use_f, np.maximum(ilo2[:, L + 1], s), ilo2[:, L + 1])
        lo, hi, ilo, ihi = lo2, hi2, ilo2, ihi2
    # leaves
    m = 1 << depth
    first = m - 1
    centre = 0.5 * (lo + np.minimum(hi, 1024.0))
    beta = dvfs.beta(centre)
    fc = 0.5 * (fr[np.clip(ilo, 0, nf - 1)] + fr[np.clip(ihi, 0, nf - 1)])
    if which == "speedup":
        y = dvfs.speedup(beta, fc)
    elif which == "edp":                          # E * T, T = 1/S
        y = dvfs.energy(beta, fc) / dvfs.speedup(beta, fc)
    else:
        y = dvfs.energy(beta, fc)
    y = y + rng.normal(0.0, noise, size=y.shape)
    value[:, first:] = np.clip(y, 0.25, np.nextafter(np.float32(4.0), np.float32(0.0))).astype(np.float32)
    # children arrays
    n = np.arange(nn)
    left = np.where(n < first, 2 * n + 1, -1).astype(np.int32)
    right = np.where(n < first, 2 * n + 2, -1).astype(np.int32)
    return feature, value, np.broadcast_to(left, (n_trees, nn)), np.broadcast_to(right, (n_trees, nn))


def forest_model(seed_seq, n_trees, depth, F, freqs, def_idx, which, batch=32, p_freq=0.25) -> ModelSpec:
    rng = np.random.Generator(np.random.PCG64(seed_seq))
    dvfs = _DVFS(rng, F, freqs, def_idx)
    feats, vals, lefts, rights = [], [], [], []
    t = 0
    while t < n_trees:
        b = min(batch, n_trees - t)
        f, v, l, r = _complete_trees(rng, b, depth, F, freqs, dvfs, which, p_freq=p_freq)
        feats.append(f.reshape(-1)); vals.append(v.reshape(-1))
        lefts.append(np.ascontiguousarray(l).reshape(-1)); rights.append(np.ascontiguousarray(r).reshape(-1))
        t += b
    nn = (1 << (depth + 1)) - 1
    return ModelSpec(n_inputs=F + 1, forest_weight=1.0,
                     tree_offset=np.arange(n_trees + 1, dtype=np.int64) * nn,
                     feature=np.concatenate(feats), left=np.concatenate(lefts),
                     right=np.concatenate(rights), value=np.concatenate(vals))


def linear_speedup_model(seed_seq, F, freqs, def_idx) -> ModelSpec:
    """Linear speedup regressor (Table 2 "Best" for MAX_PERF/PL: Linear).  w_F > 0 on the clock,
    small static weights, b set so S(f_def) ~ 1 for a typical kernel and S > 0 on the table."""
    rng = np.random.Generator(np.random.PCG64(seed_seq))
    f_def = float(freqs[def_idx])
    w = np.zeros(F + 1)
    w[:F] = rng.normal(0.0, 2e-5, size=F)
    w[F] = rng.uniform(0.6, 0.9) / f_def
    b = 1.0 - w[F] * f_def - float(np.sum(w[:F]) * 100.0)
    return ModelSpec(n_inputs=F + 1, linear_weight=1.0, lin_w=w, lin_b=b)


def linear_ed2p_model(seed_seq, F, freqs, def_idx) -> ModelSpec:
    """Linear ED2P regressor (Table 2 "Best" for MIN_ED2P: Linear): ED2P = E*T^2 falls with the
    clock on compute-bound kernels; negative clock weight, b so ED2P(f_def) ~ 1 and > 0."""
    rng = np.random.Generator(np.random.PCG64(seed_seq))
    f_def, f_max = float(freqs[def_idx]), float(freqs[-1])
    w = np.zeros(F + 1)
    w[:F] = rng.normal(0.0, 1e-5, size=F)
    w[F] = -rng.uniform(0.3, 0.6) / f_max
    b = 1.0 - w[F] * f_def - float(np.sum(w[:F]) * 100.0)
    return ModelSpec(n_inputs=F + 1, linear_weight=1.0, lin_w=w, lin_b=b)


def svr_energy_model(seed_seq, F, freqs, def_idx, n_sv=512, gamma=0.5) -> ModelSpec:
    """SVR_RBF energy regressor (Table 2: SVR evaluated for MIN_ENERGY / EDP / ES), shaped like a
    trained model: standardized inputs (log-count features, clock), support vectors drawn from the
    input distribution, dual coefficients fitted by least squares to the analytic DVFS energy at
    the support vectors (so predictions follow the convex energy-vs-clock shape)."""
    rng = np.random.Generator(np.random.PCG64(seed_seq))
    dvfs = _DVFS(rng, F, freqs, def_idx)
    feats = np.floor(np.exp2(rng.uniform(0.0, 10.0, size=(n_sv, F))))
    clk = freqs[rng.integers(0, len(freqs), size=n_sv)].astype(np.float64)
    X = np.concatenate([feats, clk[:, None]], axis=1)
    mean = np.concatenate([np.full(F, 256.0), [float(np.mean(freqs))]])
    scale = np.concatenate([np.full(F, 300.0), [float(np.std(freqs))]])
    Z = ((X - mean) / scale).astype(np.float32)
    y = dvfs.energy(dvfs.beta(feats), clk)
    K = np.exp(-gamma * ((Z[:, None, :].astype(np.float64) - Z[None, :, :]) ** 2).sum(-1))
    b = float(np.mean(y))
    dual = np.linalg.solve(K + 1e-2 * np.eye(n_sv), y - b)
    return ModelSpec(n_inputs=F + 1, svr_weight=1.0, sv=Z, dual_coef=dual, svr_gamma=gamma,
                     svr_intercept=b, in_mean=mean, in_scale=scale)


# ------------------------------------------------------------------------ configs

CONFIGS = {
    # name: (n_kernels, n_freqs, speedup, energy, targets)   speedup/energy: ("rf", T, D) | ("lin",)
    "c1": (16, 64, ("rf", 10, 8), ("rf", 10, 8), "six"),
    "c2": (1_000, 196, ("rf", 100, 12), ("rf", 100, 12), "six"),
    "c3": (100_000, 196, ("rf", 500, 12), ("rf", 500, 12), "espl"),
    "c4": (10_000_000, 128, ("lin",), ("rf", 100, 12), "six"),
    "c5": (64 * 56, 196, ("rf", 100, 12), ("rf", 100, 12), "six"),
}
CONFIG_INDEX = {"c1": 1, "c2": 2, "c3": 3, "c4": 4, "c5": 5}
C5_BLOCK = 56   # CloverLeaf-shaped 48 + MiniWeather-shaped 8 kernels per rank


def _seeds(cfg: str):
    ss = np.random.SeedSequence(SEED_BASE + CONFIG_INDEX[cfg])
    feat_ss, sp_ss, en_ss = ss.spawn(3)
    return feat_ss, sp_ss, en_ss


def _model(spec, seed_seq, F, freqs, def_idx, which):
    if spec[0] == "lin":
        return linear_speedup_model(seed_seq, F, freqs, def_idx)
    _, T, D = spec
    return forest_model(seed_seq, T, D, F, freqs, def_idx, which)


def make_models(cfg: str):
    n_k, n_f, sp, en, tg = CONFIGS[cfg]
    _, sp_ss, en_ss = _seeds(cfg)
    freqs = clock_table(n_f)
    d = default_index(freqs)
    return (_model(sp, sp_ss, N_STATIC, freqs, d, "speedup"),
            _model(en, en_ss, N_STATIC, freqs, d, "energy"), freqs, d)


def make_models4(cfg: str = "c2"):
    """Four-model variant on config cfg's shapes, each target's
    model family from Table 2's "Best" column (L403-L412): speedup Linear (MAX_PERF, PL), energy
    RandomForest (MIN_ENERGY, ES), EDP RandomForest (MIN_EDP), ED2P Linear (MIN_ED2P)."""
    n_k, n_f, sp, en, tg = CONFIGS[cfg]
    ss = np.random.SeedSequence(SEED_BASE + 100 + CONFIG_INDEX[cfg])
    s_sp, s_en, s_edp, s_ed2p = ss.spawn(4)
    freqs = clock_table(n_f)
    d = default_index(freqs)
    T, D = (en[1], en[2]) if en[0] == "rf" else (100, 12)
    return ([linear_speedup_model(s_sp, N_STATIC, freqs, d),
             forest_model(s_en, T, D, N_STATIC, freqs, d, "energy"),
             forest_model(s_edp, T, D, N_STATIC, freqs, d, "edp"),
             linear_ed2p_model(s_ed2p, N_STATIC, freqs, d)], freqs, d)


def make_models_svr(cfg: str = "c2", n_sv: int = 512, ensemble: bool = False):
    """SVR variant (Table 2 "SVR") on config cfg's shapes: the
    config's speedup model and an SVR_RBF energy model (n_sv support vectors).  ensemble=True
    instead makes the energy model 0.5 * forest + 0.5 * SVR (the weighted-ensemble reading Q7)."""
    sp, en, freqs, d = make_models(cfg)
    ss = np.random.SeedSequence(SEED_BASE + 200 + CONFIG_INDEX[cfg])
    svr = svr_energy_model(ss, N_STATIC, freqs, d, n_sv=n_sv)
    if ensemble:
        svr = ModelSpec(n_inputs=en.n_inputs, forest_weight=0.5, tree_offset=en.tree_offset, feature=en.feature,
                        left=en.left, right=en.right, value=en.value, svr_weight=0.5, sv=svr.sv,
                        dual_coef=svr.dual_coef, svr_gamma=svr.svr_gamma, svr_intercept=svr.svr_intercept,
                        in_mean=svr.in_mean, in_scale=svr.in_scale)
    return sp, svr, freqs, d


def make_features(cfg: str, row0: int = 0, n: Optional[int] = None) -> np.ndarray:
    n_k = CONFIGS[cfg][0]
    feat_ss, _, _ = _seeds(cfg)
    if n is None:
        n = n_k - row0
    if cfg == "c5":   # 64 identical replicas of one 56-kernel application block (weak scaling)
        blk = gen_features(feat_ss, C5_BLOCK, N_STATIC)
        rows = (np.arange(row0, row0 + n) % C5_BLOCK)
        return np.ascontiguousarray(blk[rows])
    return gen_features(feat_ss, n_k, N_STATIC, row0=row0, n=n)


def make_config(cfg: str, row0: int = 0, n: Optional[int] = None, models=None) -> Workload:
    """Config `cfg` (BASELINE.json configs[0..4] = c1..c5), optionally rows [row0, row0+n) only."""
    n_k, n_f, sp, en, tg = CONFIGS[cfg]
    if models is None:
        models = make_models(cfg)
    spm, enm, freqs, d = models
    feats = make_features(cfg, row0, n)
    targets = targets_six() if tg == "six" else targets_es_pl()
    return Workload(cfg, feats, freqs, d, spm, enm, targets, n_kernels_total=n_k, row0=row0)


# ---------------------------------------------------------------------- fuzz cases

def random_tree_arrays(rng, F, freqs, max_depth, p_leaf=0.2, p_freq=0.3, shuffle=True,
                       exact_thresholds=False, value_range=(0.25, 4.0), p_special_thr=0.0):
    """One unbalanced tree (early-leaf prob p_leaf) in sklearn layout with node ids shuffled.

    With exact_thresholds, some thresholds are set equal to existing feature values / clocks so
    `x == thr` (routes left) is exercised; p_special_thr makes that fraction of the thresholds
    NaN (everything goes right), +-inf or +-0.0.
    """
    feature, left, right, value = [], [], [], []

    def new():
        feature.append(-1); left.append(-1); right.append(-1); value.append(0.0)
        return len(feature) - 1

    def grow(n, d):
        if d >= max_depth or (d > 0 and rng.uniform() < p_leaf):
            feature[n] = -1
            value[n] = float(rng.uniform(*value_range))
            return
        if rng.uniform() < p_freq:
            f = F
            if exact_thresholds and rng.uniform() < 0.5:
                thr = float(freqs[rng.integers(0, len(freqs))])
            else:
                thr = float(rng.uniform(float(freqs[0]) - 10, float(freqs[-1]) + 10))
        else:
            f = int(rng.integers(0, F))
            if exact_thresholds and rng.uniform() < 0.5:
                thr = float(np.floor(np.exp2(rng.uniform(0, 10))))
            else:
                thr = float(np.exp2(rng.uniform(-1, 10)))
        if p_special_thr > 0.0 and rng.uniform() < p_special_thr:
            thr = float([np.nan, np.inf, -np.inf, -0.0, 0.0][rng.integers(0, 5)])
        feature[n] = f
        value[n] = thr
        l = new(); r = new()
        left[n] = l; right[n] = r
        grow(l, d + 1); grow(r, d + 1)

    root = new()
    grow(root, 0)
    feature = np.array(feature, np.int32); left = np.array(left, np.int32)
    right = np.array(right, np.int32); value = np.array(value, np.float32)
    if shuffle and len(feature) > 1:
        perm = np.concatenate([[0], 1 + rng.permutation(len(feature) - 1)])   # keep root at 0
        inv = np.empty_like(perm); inv[perm] = np.arange(len(perm))
        # new id of old node o is inv[o]; build arrays indexed by new ids
        nf_ = np.empty_like(feature); nl = np.empty_like(left); nr = np.empty_like(right)
        nv = np.empty_like(value)
        nf_[inv] = feature; nv[inv] = value
        nl[inv] = np.where(left >= 0, inv[np.maximum(left, 0)], -1)
        nr[inv] = np.where(right >= 0, inv[np.maximum(right, 0)], -1)
        feature, left, right, value = nf_, nl, nr, nv
    return feature, left, right, value


def random_forest_spec(rng, F, freqs, n_trees, max_depth, **kw) -> ModelSpec:
    parts = [random_tree_arrays(rng, F, freqs, max_depth, **kw) for _ in range(n_trees)]
    off = np.zeros(n_trees + 1, np.int64)
    off[1:] = np.cumsum([len(p[0]) for p in parts])
    return ModelSpec(n_inputs=F + 1, forest_weight=1.0, tree_offset=off,
                     feature=np.concatenate([p[0] for p in parts]),
                     left=np.concatenate([p[1] for p in parts]),
                     right=np.concatenate([p[2] for p in parts]),
                     value=np.concatenate([p[3] for p in parts]))


def fuzz_workload(seed: int, n_kernels: int, n_freqs: int, F: int = 5, n_trees: int = 3,
                  max_depth: int = 4, targets=None, linear: str = "none", specials: float = 0.0,
                  **kw) -> Workload:
    """Small random case: unbalanced shuffled trees, optional linear member (none|only|both).

    specials > 0: that fraction of the feature entries is replaced by values no counter produces
    (NaN, +-inf, negative counts, -0.0, huge values), to exercise the split semantics x <= thr
    (NaN goes right, -0.0 == 0.0) on both sides (Q16)."""
    rng = np.random.default_rng(seed)
    if n_freqs <= 1395:
        freqs = clock_table(n_freqs)
    else:
        freqs = np.arange(n_freqs, dtype=np.float32) + 100.0
    d = default_index(freqs)
    feats = np.floor(np.exp2(rng.uniform(0, 10, size=(n_kernels, F)))).astype(np.float32)
    feats[rng.uniform(size=feats.shape) < 0.1] = 0.0
    if specials > 0.0:
        pick = rng.uniform(size=feats.shape) < specials
        vals = np.array([np.nan, np.inf, -np.inf, -0.0, -1.0, -517.25, 3.0e38, -3.0e38], np.float32)
        feats[pick] = vals[rng.integers(0, len(vals), size=int(pick.sum()))]

    def one():
        if linear == "only":
            m = ModelSpec(n_inputs=F + 1)
        else:
            m = random_forest_spec(rng, F, freqs, n_trees, max_depth, **kw)
        if linear in ("only", "both"):
            m.linear_weight = 1.0 if linear == "only" else 0.5
            m.lin_w = rng.normal(0, 1e-3, size=F + 1)
            m.lin_w[F] = abs(m.lin_w[F]) + 1e-3
            m.lin_b = 1.0
            if linear == "both":
                m.forest_weight = 0.5
        return m

    sp, en = one(), one()
    if targets is None:
        targets = targets_six() + [(ES, 0.0), (ES, 25.0), (ES, 75.0), (ES, 100.0),
                                   (PL, 0.0), (PL, 25.0), (PL, 75.0), (PL, 100.0),
                                   (ES_ABS, 40.0), (PL_ABS, 20.0)]
    return Workload(f"fuzz{seed}", feats, freqs, d, sp, en, targets, n_kernels_total=n_kernels)

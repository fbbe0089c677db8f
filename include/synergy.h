/* synergy.h — C ABI of the B200 (sm_100a) SYnergy predict+select library (libsynergy.so).
 *
 * The operation (PAPER.md = the SYnergy paper, SC'23; "L<n>" = line n):
 *   §6.2 Prediction phase, L316-L322: for a new workload's static feature vector k'
 *   (Table 1) and the device's core-clock vector f (L59-L65, L312) build the
 *   prediction dataset P = (k', f), predict the metrics with the trained single-target
 *   models (L320; families Linear / Lasso / RandomForest, L386 and Table 2), then "find the
 *   frequency configuration f-hat by using a search algorithm for different energy targets,
 *   e.g. MIN_EDP, ES_25 or PL_25" (L322).  Energy targets: EDP = e*t, ED2P = e*t^2 (L253),
 *   ES_x (L259-L267), PL_x (L269-L271), MAX_PERF / MIN_ENERGY (L382, Table 2), all relative
 *   to the default clock (L69).  The library evaluates every (kernel, clock) pair of a batch
 *   of kernels with a speedup model and an energy model, normalises both to the default
 *   clock, and returns one clock index per kernel per target.  The readings of points the
 *   paper leaves open are DESIGN.md Q1-Q23 (exhaustive lowest-index argmin, potential-saving
 *   ES/PL, x <= threshold goes left, exact leaf sums, ...).
 *
 * Conventions for every call:
 *   - All calls return syn_status; no C++ exception crosses the ABI.  On a non-OK status the
 *     reason is available from synergy_last_error() (thread-local, valid until the next call
 *     on the same thread).
 *   - Argument errors are detected on the host before anything is enqueued; on error NOTHING
 *     is enqueued and outputs are untouched.
 *   - Device-side calls are asynchronous on `stream` (a cudaStream_t; NULL = legacy default
 *     stream).  Results are valid after the caller synchronises that stream.  Launch failures
 *     return SYN_ERR_CUDA.
 *   - "d_" pointers are device pointers on the model's device, "h_" pointers host pointers.
 *     The caller owns every buffer it passes.  The library keeps its own scratch, all of it
 *     stream-ordered (allocated from a library-owned CUDA memory pool on the call's stream, never
 *     with a host synchronisation): per (model, clock table) a clock-cut copy of the forest built
 *     by k_cut_blocks on the stream of the first call that pairs them (calls on other streams wait
 *     for its event); per (device, stream) the int64 difference arrays of the sweep, kept zeroed
 *     between calls and grown on demand (SYN_ERR_OOM possible); for calls spanning several kernel
 *     slabs a second array, a side stream and events (the finish of slab i overlaps the walk of
 *     slab i + 1; the call joins the side stream before returning); and per call the general
 *     path's and the SVR member's scratch (freed stream-ordered before the call returns).
 *     synergy_prepare creates the persistent pieces for a shape; after it (or after one call of
 *     that shape on a stream) later such calls only enqueue work, so they may be captured into a
 *     CUDA graph.  A call that would have to create persistent scratch while its stream is being
 *     captured returns SYN_ERR_UNSUPPORTED instead.
 *   - Paths: the tree-major kernels (k_tm_walk + k_tm_finish) when every forest's leaves fit the
 *     int64 fixed-point range and the per-tree task table fits shared memory (about 25 000 trees
 *     per call, any F), or for small batches (at most one kernel per SM) the single-launch
 *     k_tm_small (direct walks and the finish in one CTA per kernel); otherwise the general exact
 *     kernels (k_gen_forest + k_gen_finish: direct traversal, 320-bit exact leaf sums), which
 *     accept every valid model.  All return the same bits.
 *   - Layouts are row-major and contiguous: features [n_kernels][n_features] fp32,
 *     predictions [n_kernels][n_freqs] fp32, choices [n_kernels][n_targets] int32.
 *   - Handles (models, clock tables, workspaces) are bound to the device they were created
 *     on and must be used with that device current.  Models and clock tables are immutable
 *     and may be shared across streams and host threads.
 */
#ifndef SYNERGY_H
#define SYNERGY_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define SYNERGY_VERSION 3
#define SYNERGY_MAX_FREQS 4096
#define SYNERGY_MAX_TARGETS 16
#define SYNERGY_MAX_INPUTS 255
#define SYNERGY_MAX_DEPTH 64

typedef enum {
    SYN_OK = 0,
    SYN_ERR_INVALID_ARG = 1,   /* bad pointer, size, index, target, model or clock table   */
    SYN_ERR_UNSUPPORTED = 2,   /* well-formed but beyond the library's limits              */
    SYN_ERR_CUDA = 3,          /* a CUDA runtime call or kernel launch failed              */
    SYN_ERR_OOM = 4            /* device or host allocation failed                         */
} syn_status;

/* Energy targets (Listing 3, Table 2). */
typedef enum {
    SYN_MAX_PERF = 0,    /* highest speedup                                         */
    SYN_MIN_ENERGY = 1,  /* lowest energy                                           */
    SYN_MIN_EDP = 2,     /* lowest E*T, T = 1/S                  (L253)             */
    SYN_MIN_ED2P = 3,    /* lowest E*T^2                         (L253)             */
    SYN_ES = 4,          /* highest speedup with E <= E_def - x%(E_def - E_min)  (L267) */
    SYN_PL = 5,          /* lowest energy with S >= S_def - x%(S_def - S(i_minE)) (L271) */
    SYN_ES_ABS = 6,      /* highest speedup with E <= (1 - x%) E_def; -1 if none  (L11, L46) */
    SYN_PL_ABS = 7       /* lowest energy with S >= (1 - x%) S_def; -1 if none   (L11, L46) */
} syn_target_kind;

typedef struct {
    int32_t kind;        /* syn_target_kind                                         */
    float x;             /* percentage in [0, 100] for SYN_ES / PL / ES_ABS / PL_ABS, else ignored */
} syn_target;

typedef void *syn_stream;   /* cudaStream_t */

/* Model description (host memory; copied by synergy_model_create).  The forest uses
 * scikit-learn's `tree_` layout: structure of arrays over the nodes of all trees, node ids
 * tree-local with root 0, children -1 at leaves, value = split threshold (internal node,
 * x[feature] <= value goes left) or leaf value.  Input index n_inputs-1 is the core clock
 * in MHz; inputs 0..n_inputs-2 are the static features.  Output (Q7/Q8):
 *   m(x) = 0;  m += linear_weight * (lin_b + sum_j lin_w[j] x[j])   if linear_weight != 0
 *              m += forest_weight * mean_t leaf_t(x)                if forest_weight != 0
 *              m += svr_weight * svr(x)                             if svr_weight != 0
 * in fp64: fp64 fma over j in order for the linear member; for the forest the exact sum of the
 * fp32 leaves rounded once to fp64 (order-free, Q8), then / n_trees; a weight of
 * exactly 1 skips its multiplication.
 * SVR with RBF kernel (Table 2 "SVR"; scikit-learn SVR on StandardScaler inputs):
 *   svr(x) = svr_intercept + sum_j dual_coef[j] * exp(-svr_gamma * ||z(x) - sv[j]||^2),
 *   z(x)_d = (x[d] - in_mean[d]) / in_scale[d],
 * fp64.  Over a clock sweep the squared distance splits into a static-feature part and a
 * clock part, so the device evaluates sum_j (dual_j e^{-gamma A_kj}) e^{-gamma B_ji}: a
 * [kernels x SVs] x [SVs x clocks] fp64 contraction (Q24).  It agrees with the plain
 * definition within 2^-40 * (|svr_intercept| + sum_j |dual_coef[j]|), NOT bit for bit.
 * Calls whose models have an SVR member take stream-ordered scratch per SVR model of about
 * (n_sv * (n_freqs + min(n_kernels, 2^25 / n_sv)) + splits * n_kernels * n_freqs) * 8 bytes
 * (splits <= 16) from a library-owned CUDA memory pool on the device (cudaMallocFromPoolAsync /
 * cudaFreeAsync on the call's stream; the pool keeps freed memory mapped, so after the first
 * call of a given size no device memory is mapped), the only allocation a hot call makes. */
typedef struct {
    int32_t n_inputs;            /* F + 1, 1 .. SYNERGY_MAX_INPUTS                        */
    double linear_weight;        /* 0 => no linear member                                 */
    const double *lin_w;         /* [n_inputs]                                            */
    double lin_b;
    double forest_weight;        /* 0 => no forest member                                 */
    int32_t n_trees;             /* >= 1 when forest_weight != 0                          */
    const int64_t *tree_offset;  /* [n_trees+1] node range of each tree                   */
    const int32_t *feature;      /* [n_nodes] split input, -1 = leaf                      */
    const int32_t *left;         /* [n_nodes] tree-local child ids (ignored at leaves)    */
    const int32_t *right;
    const float *value;          /* [n_nodes] threshold or leaf value                     */
    double svr_weight;           /* 0 => no SVR_RBF member (the fields below are ignored) */
    int32_t n_sv;                /* support vectors, 1 .. 2^24                            */
    const float *sv;             /* [n_sv][n_inputs] support vectors, standardized space  */
    const double *dual_coef;     /* [n_sv] dual coefficients (alpha_j - alpha_j^*)        */
    double svr_gamma;            /* RBF gamma, finite, >= 0                               */
    double svr_intercept;
    const double *in_mean;       /* [n_inputs] standardization, in_scale finite and != 0  */
    const double *in_scale;
} syn_model_desc;

typedef struct syn_model syn_model;      /* opaque, device-resident, immutable */
typedef struct syn_clocks syn_clocks;    /* opaque, device-resident, immutable */
typedef struct syn_workspace syn_workspace;

/* Thread-local message for the last non-OK status ("" if none). */
const char *synergy_last_error(void);
int32_t synergy_version(void);

/* Validate, re-lay (breadth-first, children adjacent) and upload a model to `device`.
 * INVALID_ARG: null arrays, n_inputs out of range, a child id outside its tree, a node
 * reached twice (not a tree), a split feature outside [0, n_inputs), a non-finite leaf value,
 * all member weights 0, an SVR member with NULL arrays, n_sv outside [1, 2^24], non-finite
 * values or a zero scale.  (Thresholds may be any fp32, NaN included: x <= NaN is false.)
 * UNSUPPORTED: depth > SYNERGY_MAX_DEPTH, a tree of more than 2^23 - 1 nodes or more than
 * 2^31 - 16 nodes in all.  OOM / CUDA otherwise.
 * Synchronous (returns after the upload). */
syn_status synergy_model_create(const syn_model_desc *desc, int32_t device, syn_model **out);
syn_status synergy_model_destroy(syn_model *model);
/* Any output pointer may be NULL.  max_depth = deepest root-to-leaf path (edges). */
syn_status synergy_model_info(const syn_model *model, int32_t *n_inputs, int32_t *n_trees,
                              int64_t *n_nodes, int32_t *max_depth, int64_t *device_bytes);

/* Core-clock table f: h_freqs[n_freqs] in MHz, finite and strictly
 * ascending (INVALID_ARG otherwise), 1 <= n_freqs <= SYNERGY_MAX_FREQS.  Synchronous. */
syn_status synergy_clocks_create(const float *h_freqs, int32_t n_freqs, int32_t device,
                                 syn_clocks **out);
syn_status synergy_clocks_destroy(syn_clocks *clocks);
syn_status synergy_clocks_info(const syn_clocks *clocks, int32_t *n_freqs);

/* Create the persistent scratch a call of this shape needs on `stream` (clock-cut copies, the
 * sweep's difference arrays and slab-pipeline stream), enqueueing only the k_cut_blocks builds, so
 * that later calls with these models, this clock table, at most n_kernels kernels and this stream
 * only enqueue kernels (e.g. inside a CUDA-graph capture).  models[0..1] speedup / energy,
 * models[2..3] (n_models == 4) the four-model variant's direct models or NULL.  Errors as
 * synergy_sweep4 (no feature or output buffers are needed). */
syn_status synergy_prepare(const syn_model *const *models, int32_t n_models, int64_t n_kernels,
                           int32_t n_features, const syn_clocks *clocks, syn_stream stream);

/* Predictions for every (kernel, clock) pair:
 *   d_speedup[k][i] = (float)(mS(k, f_i) / mS(k, f_def)),  d_energy likewise with mE,
 * or (float)m when default_idx == -1 (raw model outputs).  n_kernels == 0 is a no-op.
 * INVALID_ARG: null model / clocks / non-empty buffers, n_kernels < 0, n_features + 1 !=
 * n_inputs of either model, default_idx outside [-1, n_freqs), handle on another device. */
syn_status synergy_predict(const syn_model *speedup, const syn_model *energy,
                           const float *d_features, int64_t n_kernels, int32_t n_features,
                           const syn_clocks *clocks, int32_t default_idx,
                           float *d_speedup, float *d_energy, syn_stream stream);

/* Target selection on given normalised predictions:
 *   valid_i = S_i, E_i finite and > 0; if the default is invalid all choices are -1;
 *   baselines S_def, E_def, E_min (lowest index of the minimum), S_minE; per target the
 *   objective key / constraint of syn_target_kind evaluated in fp64; d_choice[k][t] = the
 *   lowest index i minimising the key among valid feasible candidates, -1 if none.
 * INVALID_ARG: null buffers, n_kernels < 0, n_freqs outside [1, SYNERGY_MAX_FREQS],
 * default_idx outside [0, n_freqs), n_targets outside [1, SYNERGY_MAX_TARGETS], unknown kind,
 * ES/PL x NaN or outside [0, 100]. */
syn_status synergy_select(const float *d_speedup, const float *d_energy, int64_t n_kernels,
                          int32_t n_freqs, int32_t default_idx, const syn_target *h_targets,
                          int32_t n_targets, int32_t *d_choice, syn_stream stream);

/* Fused predict + select in one kernel: predictions stay on chip unless d_speedup /
 * d_energy are non-NULL (then they are also written, as synergy_predict would).
 * default_idx must be in [0, n_freqs).  Other errors as predict + select. */
syn_status synergy_sweep(const syn_model *speedup, const syn_model *energy,
                         const float *d_features, int64_t n_kernels, int32_t n_features,
                         const syn_clocks *clocks, int32_t default_idx,
                         const syn_target *h_targets, int32_t n_targets, int32_t *d_choice,
                         float *d_speedup, float *d_energy, syn_stream stream);

/* Four-model variant (single-target models F_t, F_e, F_edp, F_ed2p; Table 2
 * "Best" pairs MIN_EDP with RandomForest, MIN_ED2P with Linear).  models[0] speedup, [1] energy,
 * [2] direct EDP model, [3] direct ED2P model; [2] and [3] may be NULL (that target's key is then
 * derived as E/S resp. E/S^2, as in synergy_sweep).  Each model is normalised by its own default-
 * clock prediction; MIN_EDP / MIN_ED2P minimise the direct model's normalised prediction (a clock
 * also needs that prediction finite and > 0).  d_pred (nullable): [4][n_kernels][n_freqs]
 * normalised predictions (rows of absent models untouched).  Errors as synergy_sweep. */
syn_status synergy_sweep4(const syn_model *const *models, const float *d_features, int64_t n_kernels,
                          int32_t n_features, const syn_clocks *clocks, int32_t default_idx,
                          const syn_target *h_targets, int32_t n_targets, int32_t *d_choice,
                          float *d_pred, syn_stream stream);

/* Frequency plan emission ("the predicted frequency configuration is made available
 * to the SYCL library at runtime"; L187 q.submit(MIN_EDP, ...)): d_mhz[k][t] = f[d_choice[k][t]]
 * in MHz, NaN where the choice is -1 (or out of range).  Applying clocks needs privileged NVML
 * access (L330, L342), so the library only emits the plan.  INVALID_ARG: null buffers,
 * n_kernels < 0, n_targets outside [1, SYNERGY_MAX_TARGETS]. */
syn_status synergy_plan(const int32_t *d_choice, int64_t n_kernels, int32_t n_targets,
                        const syn_clocks *clocks, float *d_mhz, syn_stream stream);

/* Pareto front per kernel ("the red line is the Pareto front", L247, L374):
 * d_front[k][i] = 1 iff clock i is a valid candidate (S, E finite and > 0) and no valid clock j
 * has S_j >= S_i and E_j <= E_i with one strict, else 0.  Inputs as synergy_select.
 * INVALID_ARG: null buffers, n_kernels < 0, n_freqs outside [1, SYNERGY_MAX_FREQS]. */
syn_status synergy_pareto(const float *d_speedup, const float *d_energy, int64_t n_kernels,
                          int32_t n_freqs, uint8_t *d_front, syn_stream stream);

/* Frequency-choice error (Table 2: APE / MAPE / RMSE "between the predicted and
 * actual optimal frequency"): per kernel and target, the target's objective on the ground-truth
 * table (d_speedup_true, d_energy_true) at the predicted clock d_choice_pred[k][t] vs at the
 * actual optimal clock (the target selected on the ground truth, as synergy_select).  Objective:
 * MAX_PERF, ES_x -> S; MIN_ENERGY, PL_x -> E; MIN_EDP -> E/S; MIN_ED2P -> (E/S)/S (fp64).
 * d_err[k][t] = {APE, predicted - actual} (NaN, NaN where either clock is -1);
 * d_summary[t] = {MAPE, RMSE, kernels counted} over the counted kernels (fp64, fixed-order
 * reduction).  Errors as synergy_select plus null d_choice_pred / d_err / d_summary. */
syn_status synergy_choice_error(const float *d_speedup_true, const float *d_energy_true,
                                int64_t n_kernels, int32_t n_freqs, int32_t default_idx,
                                const syn_target *h_targets, int32_t n_targets,
                                const int32_t *d_choice_pred, double *d_err, double *d_summary,
                                syn_stream stream);

/* End-to-end host-buffer path: copies h_features host->device into the workspace, runs
 * synergy_sweep, copies the choices device->host into h_choice, all enqueued on `stream`
 * (h_choice is valid after the stream is synchronised; pinned host buffers make the copies
 * asynchronous).  The workspace grows on demand (the only allocating call; OOM possible) and
 * must not be used by two streams at once. */
syn_status synergy_workspace_create(int32_t device, syn_workspace **out);
syn_status synergy_workspace_destroy(syn_workspace *ws);
syn_status synergy_sweep_host(syn_workspace *ws, const syn_model *speedup,
                              const syn_model *energy, const float *h_features,
                              int64_t n_kernels, int32_t n_features, const syn_clocks *clocks,
                              int32_t default_idx, const syn_target *h_targets,
                              int32_t n_targets, int32_t *h_choice, syn_stream stream);

/* Launch statistics of the last sweep/predict/select enqueued by this host thread (for tests and
 * benchmarks): kernels launched, evaluations, grid, block, variant (4000 = tree-major kernels,
 * 5000 = general exact kernels, 0 = standalone kernels).  NULLs ok. */
syn_status synergy_last_launch(int32_t *kernels_launched, int64_t *evals, int64_t *grid,
                               int32_t *block, int32_t *variant);

/* Per-kernel device timing for measurement (bench.py's roofline).  While enabled, every library
 * kernel launch is bracketed by two CUDA events recorded on its launch stream (two extra stream
 * operations per launch; off by default).  synergy_timing_read synchronises the recorded events,
 * sums the elapsed time per kernel name since the previous read, clears the record and returns
 * up to `cap` entries: names[k] (static strings, e.g. "k_tm_walk", "k_svr_tc"), total_ms[k] (sum of
 * the launch durations), busy_ms[k] (length of the union of the launch intervals, on the time axis
 * of the first recorded event: less than total_ms when launches of one kernel overlap on several
 * streams, as the slab pipeline's walks do; busy_ms may be NULL), launches[k]; *n_kernels = number
 * of distinct kernels recorded.  Process-wide, thread-safe. */
syn_status synergy_timing_enable(int32_t on);
syn_status synergy_timing_read(int32_t cap, const char **names, double *total_ms, double *busy_ms,
                               int64_t *launches, int32_t *n_kernels);

/* Tuning knobs (launch-configuration choices only; results are identical for every setting), for
 * tests and benchmarks.  Initialised once from the environment (SYNERGY_<KEY upper-case>), then
 * process-wide.  Keys: "algo" (0 automatic, 1 force the general exact kernels), "tm_kb" (k_tm_walk
 * kernels per feature block, 32..1024), "tm_nt" (k_tm_walk threads per CTA, 512 or 1024), "tm_ctas",
 * "tm_nsub", "tm_split" (per-tree clock-range split, -1 automatic, 0 off, 1 on), "split_piece"
 * (model create: target cost of one split piece in quarters of the mean tree cost, default 4),
 * "tm_dyn" (task pools, -1 automatic), "tm_pdl" (default 1), "tm_slab", "tm_lpt" (expected-cost tree order for
 * batches of about one task per lane: -1 automatic, 0 off, 1 on), "tm_pipe" (slab pipeline:
 * 0 in order on the caller's stream, 1 finishes on a side stream, 2 (default) also the walks
 * alternating between the caller's stream and a second walk stream),
 * "tm_kt", "gen_kt", "svr_splits", "svr_tc" (tcgen05 SVR contraction, default 1), "tm_small"
 * (single-launch k_tm_small for small batches: -1 automatic, 0 off, 1 on); 0 = automatic
 * unless noted.  INVALID_ARG: unknown key. */
syn_status synergy_config_set(const char *key, int64_t value);
syn_status synergy_config_get(const char *key, int64_t *value);

#ifdef __cplusplus
}
#endif
#endif /* SYNERGY_H */

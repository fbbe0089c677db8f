/* oracle.h — plain, slow, single-threaded CPU oracle for SYnergy's predict+select path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load liboracle.so.  The product path
 * (paper_conf_sc_fandccfc23_b200/) never includes, links or calls anything here, and
 * this file shares no header, helper or table with the CUDA library: it restates the
 * data-format spec (scikit-learn `tree_` arrays) on its own.
 *
 * Paper passages (PAPER.md line numbers):
 *   prediction dataset P = (k', f), models F_t/F_e, search for f-hat  L316-L322 (§6.2)
 *   EDP = e*t, ED2P = e*t^2                                          L253 (§5.1)
 *   ES_x (x% of the potential saving vs default; ES_100 = min energy) L259-L267 (§5.2)
 *   PL_x (x% of the potential performance loss, same interval)        L269-L271 (§5.3)
 *   absolute-saving reading "best performance with x% energy savings"  L11, L46 (§1)
 *   model families Linear / RandomForest                              L386, Table 2
 * Readings of silent/ambiguous points: DESIGN.md "Readings" (Q1..Q23 of SURVEY §8(c)).
 * Compile: gcc -O2 -std=c99 -ffp-contract=off (no fast-math).
 */
#ifndef SYNERGY_ORACLE_H
#define SYNERGY_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct {
    int32_t        n_inputs;       /* F + 1; input F is the core clock in MHz            */
    double         linear_weight;  /* 0 => no linear member                              */
    const double  *lin_w;          /* [n_inputs]                                         */
    double         lin_b;
    double         forest_weight;  /* 0 => no forest member                              */
    int32_t        n_trees;
    const int64_t *tree_offset;    /* [n_trees+1]                                        */
    const int32_t *feature;        /* [n_nodes] -1 = leaf                                */
    const int32_t *left;           /* tree-local child ids                               */
    const int32_t *right;
    const float   *value;          /* threshold (internal) / leaf value                  */
    double         svr_weight;     /* 0 => no SVR_RBF member                             */
    int32_t        n_sv;
    const float   *sv;             /* [n_sv][n_inputs], standardized space               */
    const double  *dual_coef;      /* [n_sv]                                             */
    double         svr_gamma, svr_intercept;
    const double  *in_mean, *in_scale;  /* [n_inputs]                                    */
} oracle_model;

/* Raw model output m(x) for one input vector x[0..n_inputs-1] (fp64).
 * Adds the number of internal-node decisions taken to *visits when visits != NULL
 * (T*D for complete depth-D trees: the roofline's algorithmic work unit). */
double oracle_model_eval(const oracle_model *m, const float *x, int64_t *visits);

/* S[k][i], E[k][i] (fp32) for kernels [0, n_k) and clocks [0, n_f).
 * default_idx >= 0: normalised by the model's own prediction at default_idx;
 * default_idx == -1: raw (float)m.  Returns 0, or -1 on invalid arguments. */
int oracle_predict(const oracle_model *speedup, const oracle_model *energy,
                   const float *features, int64_t n_k, int32_t n_features,
                   const float *freqs, int32_t n_f, int32_t default_idx,
                   float *S, float *E, int64_t *visits);

/* choice[k][t] for targets (kind[t], x[t]); kinds 0..7 = MAX_PERF, MIN_ENERGY, MIN_EDP,
 * MIN_ED2P, ES, PL (potential-saving reading, L267/L271), ES_ABS, PL_ABS (absolute reading
 * E <= (1-x%) E_def resp. S >= (1-x%) S_def, L11/L46; -1 when no clock qualifies).  gap (nullable) [n_k][n_t] receives the relative gap between the best
 * and the runner-up key among feasible candidates (+inf if fewer than two). */
int oracle_select(const float *S, const float *E, int64_t n_k, int32_t n_f,
                  int32_t default_idx, const int32_t *kind, const float *x, int32_t n_t,
                  int32_t *choice, double *gap);

/* predict (normalised) then select, one kernel at a time; S/E nullable. */
int oracle_sweep(const oracle_model *speedup, const oracle_model *energy,
                 const float *features, int64_t n_k, int32_t n_features,
                 const float *freqs, int32_t n_f, int32_t default_idx,
                 const int32_t *kind, const float *x, int32_t n_t,
                 int32_t *choice, float *S, float *E, double *gap, int64_t *visits);

/* Four-model variant: models[0] speedup, [1] energy, [2] EDP, [3] ED2P
 * ([2]/[3] nullable = derived).  MIN_EDP / MIN_ED2P use the direct model's normalised
 * prediction.  P (nullable) receives [4][n_k][n_f] normalised predictions. */
int oracle_sweep4(const oracle_model *const *models, const float *features, int64_t n_k,
                  int32_t n_features, const float *freqs, int32_t n_f, int32_t default_idx,
                  const int32_t *kind, const float *x, int32_t n_t, int32_t *choice, float *P);

/* Pareto front per kernel: front[k][i] = 1 iff clock i is valid and not
 * dominated in (max S, min E) by a valid clock. */
int oracle_pareto(const float *S, const float *E, int64_t n_k, int32_t n_f, uint8_t *front);

/* Frequency-choice error APE / MAPE / RMSE (Table 2) of predicted choices
 * against the targets selected on a ground-truth table (S_true, E_true); ape nullable. */
int oracle_choice_error(const float *S_true, const float *E_true, int64_t n_k, int32_t n_f,
                        int32_t default_idx, const int32_t *kind, const float *x, int32_t n_t,
                        const int32_t *choice_pred, double *ape, double *mape, double *rmse,
                        int64_t *counted);

#ifdef __cplusplus
}
#endif
#endif

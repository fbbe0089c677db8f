/* workcount.c — measurement tool: algorithmic work counters of the run-walk sweep.
 *
 * NOT the oracle and NOT the product.  bench.py uses these counts as the numerator of the
 * k_tm_walk roofline (DESIGN.md §6 "Rooflines"): how many 32-byte 2-level block fetches the
 * resume walks of a batch need, which is a property of the inputs (how many runs of consecutive
 * clocks reach the same leaf, and where consecutive clocks' paths part), not of the kernel.
 * It restates the model format (scikit-learn `tree_` arrays, include/synergy.h) on its own and
 * shares no code with oracle/ or the CUDA library.  Pinned against an independent interval
 * depth-first formulation in tests/test_workcount.py.
 *
 * Definitions, per (kernel k, tree t), clocks i = 0 .. n_f-1 in table order, x = (k's static
 * features, f_i), walk from the root with x[feature] <= threshold going left:
 *   run            a maximal set of consecutive clocks reaching the same leaf
 *   run_decisions  sum over runs of the leaf depth (internal decisions on the path)
 *   run_blocks     sum over runs of max(1, ceil(depth / 2))      (root-restart walks)
 *   resume_blocks  first run of the tree: max(1, ceil(depth / 2)); a later run starting at clock
 *                  i: ceil(depth / 2) - floor(d / 2), d = depth of the first node where the paths
 *                  of clocks i-1 and i differ (the walk resumes at the block holding that node)
 *   decisions      sum over every (clock, tree) of the leaf depth (direct traversal)
 * Compile: gcc -O2 -std=c99 -fPIC -shared.
 */
#include <stdint.h>
#include <stdlib.h>

typedef struct {
    int32_t n_trees;
    const int64_t *tree_offset;   /* [n_trees+1]                   */
    const int32_t *feature;       /* [n_nodes], -1 = leaf           */
    const int32_t *left, *right;  /* tree-local child ids           */
    const float *value;           /* threshold / leaf value         */
} wc_forest;

typedef struct {
    int64_t decisions, runs, run_decisions, run_blocks, resume_blocks;
} wc_counts;

static int64_t leaf_of(const wc_forest *m, int64_t base, const float *x, int32_t F, float f, int32_t *depth)
{
    int64_t n = 0;
    int32_t d = 0;
    for (;;) {
        const int32_t q = m->feature[base + n];
        if (q < 0) break;
        const float v = q == F ? f : x[q];
        n = (v <= m->value[base + n]) ? m->left[base + n] : m->right[base + n];
        ++d;
    }
    *depth = d;
    return n;
}

static int32_t part_depth(const wc_forest *m, int64_t base, const float *x, int32_t F, float fa, float fb)
{
    int64_t n = 0;
    int32_t d = 0;
    for (;;) {
        const int32_t q = m->feature[base + n];
        if (q < 0) return d;
        const float va = q == F ? fa : x[q], vb = q == F ? fb : x[q];
        const int la = va <= m->value[base + n], lb = vb <= m->value[base + n];
        if (la != lb) return d;
        n = la ? m->left[base + n] : m->right[base + n];
        ++d;
    }
}

/* Adds the counters of forest m over kernels [0, n_k) to *c.  Returns 0, -1 on bad arguments. */
int wc_count(const wc_forest *m, const float *features, int64_t n_k, int32_t F, const float *freqs,
             int32_t n_f, wc_counts *c)
{
    if (!m || !c || n_k < 0 || F < 0 || n_f < 1 || (n_k > 0 && !features) || !freqs) return -1;
    for (int64_t k = 0; k < n_k; ++k) {
        const float *x = features + k * F;
        for (int32_t t = 0; t < m->n_trees; ++t) {
            const int64_t base = m->tree_offset[t];
            int64_t prev = -1;
            for (int32_t i = 0; i < n_f; ++i) {
                int32_t dep = 0;
                const int64_t leaf = leaf_of(m, base, x, F, freqs[i], &dep);
                c->decisions += dep;
                if (i > 0 && leaf == prev) continue;
                const int32_t blocks = dep > 1 ? (dep + 1) / 2 : 1;
                c->runs += 1;
                c->run_decisions += dep;
                c->run_blocks += blocks;
                c->resume_blocks += i == 0 ? blocks : blocks - part_depth(m, base, x, F, freqs[i - 1], freqs[i]) / 2;
                prev = leaf;
            }
        }
    }
    return 0;
}

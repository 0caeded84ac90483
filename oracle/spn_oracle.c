/*
 * spn_oracle.c -- plain, slow, fp64 CPU oracle for SPN joint / marginal
 * log-likelihood.  TEST INFRASTRUCTURE ONLY: it may be called from tests/,
 * __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference leg,
 * never from the product path.  It shares no code, header or helper with the
 * CUDA library (paper_conf_cgo_sommera022_b200/csrc); the only common thing
 * is the flat graph input format, which each side marshals itself.
 *
 * What it computes is the plain recursive definition of an SPN's value
 * (§II-A: "the inference starts by querying the univariate
 * leaf distributions using the full (joint) or partial (marginal) evidence
 * ... the probabilities obtained from the leaf nodes are then propagated
 * upwards through the DAG, performing multiplication and weighted addition
 * at the corresponding nodes"), evaluated in log space:
 *
 *   val(gaussian)   = log N(x_f; mean, stddev)            (Table I)
 *   val(categorical)= log p_{floor(x_f)}, 0 <= x_f < K    (Table I; reading c3)
 *   val(histogram)  = log p_b for the bucket lb_b <= x_f < ub_b  (Table I; c2)
 *                     outside every bucket / category -> log 0 = -inf
 *   marginal query and x_f NaN -> 0 = log 1                (L37; reading c6)
 *   joint query and x_f NaN    -> NaN                      (reading c7)
 *   val(product)    = sum_i val(child_i)                   (Table I)
 *   val(sum)        = log sum_i w_i exp(val(child_i))      (Table I)
 *                     computed max-shifted; all terms -inf -> -inf (c8)
 *   out[s][r]       = val(root_r) for sample s             (multi-root, c10)
 *   argmax[s]       = lowest r with the largest non-NaN out[s][r]; -1 if none
 *
 * Recursive with a per-sample memo (DAG sharing), OpenMP over samples,
 * compiled -O2 without fast-math.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

enum { O_GAUSSIAN = 0, O_CATEGORICAL = 1, O_HISTOGRAM = 2, O_SUM = 3, O_PRODUCT = 4 };

typedef struct {
    const int32_t *kind, *feature, *n_children, *n_params;
    const int64_t *child_begin, *param_begin, *children;
    const double *weights, *params;
    const float *xs;      /* this sample's features */
    int marginal;
    double *memo;         /* [n_nodes] */
    int64_t *stamp;       /* [n_nodes] sample id that filled memo */
    int64_t sample;
} ctx_t;

static double leaf_value(const ctx_t *c, int64_t u) {
    double x = (double)c->xs[c->feature[u]];
    if (isnan(x)) return c->marginal ? 0.0 : NAN;
    const double *p = c->params + c->param_begin[u];
    int32_t np = c->n_params[u];
    switch (c->kind[u]) {
    case O_GAUSSIAN: {
        double mean = p[0], sd = p[1];
        double z = (x - mean) / sd;
        return -0.5 * z * z - log(sd) - 0.5 * log(2.0 * M_PI);
    }
    case O_CATEGORICAL: {
        if (!(x >= 0.0 && x < (double)np)) return -INFINITY;
        return log(p[(int64_t)floor(x)]);
    }
    case O_HISTOGRAM: {
        for (int32_t b = 0; b + 2 < np; b += 3)
            if (x >= p[b] && x < p[b + 1]) return log(p[b + 2]);
        return -INFINITY;
    }
    }
    return NAN;
}

static double node_value(ctx_t *c, int64_t u) {
    if (c->stamp[u] == c->sample) return c->memo[u];
    double v;
    int32_t k = c->kind[u];
    if (k == O_PRODUCT) {
        v = 0.0;
        const int64_t *ch = c->children + c->child_begin[u];
        for (int32_t i = 0; i < c->n_children[u]; ++i) v += node_value(c, ch[i]);
    } else if (k == O_SUM) {
        const int64_t *ch = c->children + c->child_begin[u];
        const double *w = c->weights + c->child_begin[u];
        int32_t n = c->n_children[u];
        /* pass 1: m = max_i (log w_i + val_i); children are memoised, so
           pass 2 re-reads them without re-evaluating. */
        double m = -INFINITY;
        int has_nan = 0;
        for (int32_t i = 0; i < n; ++i) {
            double t = log(w[i]) + node_value(c, ch[i]);
            if (isnan(t)) has_nan = 1;
            else if (t > m) m = t;
        }
        if (has_nan) v = NAN;
        else if (m == -INFINITY) v = -INFINITY;
        else {
            double s = 0.0;
            for (int32_t i = 0; i < n; ++i) s += exp(log(w[i]) + node_value(c, ch[i]) - m);
            v = m + log(s);
        }
    } else {
        v = leaf_value(c, u);
    }
    c->memo[u] = v;
    c->stamp[u] = c->sample;
    return v;
}

int oracle_num_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

/* Returns 0 on success, -1 on allocation failure. */
int oracle_eval(int64_t n_nodes, const int32_t *kind, const int32_t *feature,
                const int64_t *child_begin, const int32_t *n_children,
                const int64_t *param_begin, const int32_t *n_params,
                const int64_t *children, const double *weights,
                const double *params, int64_t n_roots, const int64_t *roots,
                int64_t n_samples, const float *x, int64_t ld, int marginal,
                double *out, int32_t *argmax, int n_threads) {
    int fail = 0;
#ifdef _OPENMP
    if (n_threads <= 0) n_threads = omp_get_max_threads();
#pragma omp parallel num_threads(n_threads)
#endif
    {
        ctx_t c;
        c.kind = kind; c.feature = feature; c.n_children = n_children;
        c.n_params = n_params; c.child_begin = child_begin;
        c.param_begin = param_begin; c.children = children;
        c.weights = weights; c.params = params; c.marginal = marginal;
        c.memo = (double *)malloc(sizeof(double) * (size_t)(n_nodes > 0 ? n_nodes : 1));
        c.stamp = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n_nodes > 0 ? n_nodes : 1));
        if (!c.memo || !c.stamp) {
            fail = 1;
        } else {
            for (int64_t i = 0; i < n_nodes; ++i) c.stamp[i] = -1;
#ifdef _OPENMP
#pragma omp for schedule(dynamic, 64)
#endif
            for (int64_t s = 0; s < n_samples; ++s) {
                c.sample = s;
                c.xs = x + s * ld;
                int32_t best = -1;
                double bv = 0.0;
                for (int64_t r = 0; r < n_roots; ++r) {
                    double v = node_value(&c, roots[r]);
                    out[s * n_roots + r] = v;
                    if (!isnan(v) && (best < 0 || v > bv)) { best = (int32_t)r; bv = v; }
                }
                if (argmax) argmax[s] = best;
            }
        }
        free(c.memo);
        free(c.stamp);
    }
    return fail ? -1 : 0;
}

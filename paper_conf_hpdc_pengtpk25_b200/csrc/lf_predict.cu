// lf_predict.cu -- LiteForm's lightweight predictors on the host (sections
// 5.1-5.2): from the Table 2/3 features
// decide whether CELL beats the fixed CSR format and how many column
// partitions P to use.  The paper's Random Forests need
// per-hardware training data; the forests here were trained on
// B200 timings of the mixed-skew suite by scripts/train_predictor.py, which
// generates lf_forest.h (profiles/r1_predictor.md has the evaluation).
// Inference is a few hundred node visits: no GPU work, no allocation.
#include <cmath>

#include "lf_forest.h"
#include "lf_internal.cuh"

namespace {

// the 12 forest inputs from the 8 features, same operations and order as
// scripts/train_predictor.py:derive (float64, then float32 like sklearn)
void derive(const double f[8], float x[lf_forest::kInputs]) {
    const double I = f[0], K = f[1], nnz = f[2], mean = f[3], mn = f[4], mx = f[5], sd = f[6], J = f[7];
    const double d[lf_forest::kInputs] = {I, K, nnz, mean, mn, mx, sd, J, K * J * 4.0, I * J * 4.0,
                                          mean > 0 ? sd / mean : 0.0, mean > 0 ? mx / mean : 0.0};
    for (int i = 0; i < lf_forest::kInputs; i++) x[i] = (float)d[i];
}

// sklearn RandomForestClassifier.predict: per-tree leaf probabilities summed
// in tree order, first class with the maximum sum
template <int NC>
int32_t forest_predict(const float *x, int n_trees, const int32_t *roots, const lf_forest::ForestNode *nodes,
                       const double (*proba)[NC], const int32_t *classes) {
    double acc[NC] = {};
    for (int t = 0; t < n_trees; t++) {
        int n = roots[t];
        while (nodes[n].feature >= 0) n = ((double)x[nodes[n].feature] <= nodes[n].threshold) ? nodes[n].left
                                                                                               : nodes[n].right;
        for (int c = 0; c < NC; c++) acc[c] += proba[nodes[n].leaf][c];
    }
    int best = 0;
    for (int c = 1; c < NC; c++)
        if (acc[c] > acc[best]) best = c;
    return classes[best];
}

}  // namespace

extern "C" lf_status lf_predict(const double features[8], int32_t max_parts, int32_t *use_cell, int32_t *n_parts) {
    if (!features || !use_cell || !n_parts) return LF_ERR_INVALID_ARG;
    if (max_parts < 0 || max_parts > LF_MAX_PARTS) return LF_ERR_INVALID_ARG;
    for (int i = 0; i < 8; i++)
        if (!std::isfinite(features[i]) || features[i] < 0) return LF_ERR_INVALID_ARG;
    using namespace lf_forest;
    float x[kInputs];
    derive(features, x);
    *use_cell = forest_predict<use_cell_n_classes>(x, use_cell_n_trees, use_cell_roots, use_cell_nodes,
                                                   use_cell_proba, use_cell_classes);
    int32_t P = forest_predict<parts_n_classes>(x, parts_n_trees, parts_roots, parts_nodes, parts_proba,
                                                parts_classes);
    const int cap = max_parts ? max_parts : LF_MAX_PARTS;
    while (P > cap) P >>= 1;
    *n_parts = P < 1 ? 1 : P;
    return LF_OK;
}

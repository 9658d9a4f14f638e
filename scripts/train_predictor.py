"""NEXT-1: train LiteForm's format / partition predictors (sections 5.1-5.2,
P:L665-749) on B200 timings and export them as C tables for liblf.so.

    python scripts/train_predictor.py profiles/r1_predictor_data.jsonl

Input: one record per (matrix of the mixed-skew suite, J) from
scripts/predictor_data.py: Table 2/3 features, the
time of the fixed-format CSR kernel (Alg. 1) and of CELL at P in {1,2,4,8}.
Labels:
    use_cell = CELL at its best P is >= 1.1x faster than CSR
    parts    = the P with the lowest CELL time
Model: scikit-learn RandomForestClassifier (the paper's model family,
P:L709-716), one for each label, on the features below.
Outputs:
    paper_conf_hpdc_pengtpk25_b200/csrc/lf_forest.h   the two forests as C arrays
    tests/golden/predictor_cases.txt   features -> sklearn's predictions, which
                                       the C predictor must reproduce exactly
    profiles/r1_predictor.md           leave-one-family-out evaluation
"""
import json
import os
import re
import sys

import numpy as np
from sklearn.ensemble import RandomForestClassifier

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PARTS = (1, 2, 4, 8)
FEATURES = ("n_rows", "n_cols", "nnz", "len_mean", "len_min", "len_max", "len_std", "J",
            "B_bytes", "C_bytes", "len_cv", "max_over_mean")
RF = dict(n_estimators=32, max_depth=8, min_samples_leaf=2, random_state=0)


def derive(f):
    """The 12 predictor inputs from the 8 Table 2/3 features, in float64 in
    the same operation order as lf_predict.cu's derive(), then float32 (the
    precision sklearn's trees compare in)."""
    I, K, nnz, mean, mn, mx, sd, J = (float(v) for v in f)
    d = [I, K, nnz, mean, mn, mx, sd, J, K * J * 4.0, I * J * 4.0,
         sd / mean if mean > 0 else 0.0, mx / mean if mean > 0 else 0.0]
    return np.array(d, dtype=np.float64).astype(np.float32)


def family(name):
    """matrix family = name without size / seed (leave-one-family-out CV)"""
    return re.sub(r"_\d+(_\d+)?$", "", name)


def load(path):
    recs = [json.loads(l) for l in open(path) if l.strip()]
    X = np.stack([derive(r["features"]) for r in recs])
    t_cell = np.array([[r["t_cell"][str(p)] for p in PARTS] for r in recs])
    t_csr = np.array([r["t_csr"] for r in recs])
    parts = np.array([PARTS[int(np.argmin(tc))] for tc in t_cell])
    use = (t_csr >= 1.1 * t_cell.min(axis=1)).astype(int)
    fam = np.array([family(r["name"]) for r in recs])
    return recs, X, t_cell, t_csr, use, parts, fam


def chosen_time(t_cell, t_csr, use, parts):
    return np.where(use == 1, t_cell[np.arange(len(parts)), [PARTS.index(p) for p in parts]], t_csr)


def export_forest(rf, name):
    """C arrays: per node feature (-1 = leaf), float64 threshold (compare
    (float)x <= thr, as sklearn does on float32 inputs), children, and per
    leaf the normalised class probabilities (value / value.sum(), float64,
    the per-tree predict_proba); trees are summed in order, argmax = first max."""
    feat, thr, left, right, leaf = [], [], [], [], []
    probs, roots = [], []
    for est in rf.estimators_:
        t = est.tree_
        base = len(feat)
        roots.append(base)
        for n in range(t.node_count):
            if t.children_left[n] == -1:
                v = t.value[n][0].astype(np.float64)
                s = v.sum()
                p = v / (s if s != 0.0 else 1.0)
                feat.append(-1)
                thr.append(0.0)
                left.append(-1)
                right.append(-1)
                leaf.append(len(probs))
                probs.append(p)
            else:
                feat.append(int(t.feature[n]))
                thr.append(float(t.threshold[n]))
                left.append(base + int(t.children_left[n]))
                right.append(base + int(t.children_right[n]))
                leaf.append(-1)
    nc = len(rf.classes_)
    out = [f"// {name}: {len(rf.estimators_)} trees, {len(feat)} nodes, classes {list(map(int, rf.classes_))}",
           f"static const int {name}_n_trees = {len(roots)};",
           f"static const int {name}_n_classes = {nc};",
           f"static const int32_t {name}_classes[{nc}] = {{{', '.join(str(int(c)) for c in rf.classes_)}}};",
           f"static const int32_t {name}_roots[{len(roots)}] = {{{', '.join(map(str, roots))}}};",
           f"static const ForestNode {name}_nodes[{len(feat)}] = {{"]
    for i in range(len(feat)):
        out.append(f"    {{{feat[i]}, {left[i]}, {right[i]}, {leaf[i]}, {thr[i]!r}}},")
    out.append("};")
    out.append(f"static const double {name}_proba[{len(probs)}][{nc}] = {{")
    for p in probs:
        out.append("    {" + ", ".join(repr(float(x)) for x in p) + "},")
    out.append("};")
    return "\n".join(out)


def main():
    path = sys.argv[1]
    recs, X, t_cell, t_csr, use, parts, fam = load(path)
    n = len(recs)
    best = np.minimum(t_cell.min(axis=1), t_csr)
    # leave-one-family-out evaluation
    fams = sorted(set(fam))
    pu, pp = np.zeros(n, int), np.zeros(n, int)
    for f in fams:
        tr, te = fam != f, fam == f
        m_u = RandomForestClassifier(**RF).fit(X[tr], use[tr])
        m_p = RandomForestClassifier(**RF).fit(X[tr], parts[tr])
        pu[te] = m_u.predict(X[te])
        pp[te] = m_p.predict(X[te])
    t_pred = chosen_time(t_cell, t_csr, pu, pp)
    t_oracle = chosen_time(t_cell, t_csr, use, parts)
    t_p1 = t_cell[:, 0]
    gm = lambda r: float(np.exp(np.mean(np.log(r))))  # noqa: E731
    # final models on everything
    m_u = RandomForestClassifier(**RF).fit(X, use)
    m_p = RandomForestClassifier(**RF).fit(X, parts)
    hdr = ["// lf_forest.h -- GENERATED by scripts/train_predictor.py from " + os.path.basename(path) + "; do not edit.",
           "// LiteForm's predictors (sections 5.1-5.2, P:L665-749) trained on B200 timings of the",
           "// mixed-skew suite: use_cell (CELL >= 1.1x faster than CSR) and parts (best P).",
           f"// inputs ({len(FEATURES)}): " + ", ".join(FEATURES),
           f"// sklearn RandomForestClassifier{RF}; {n} training records.",
           "#pragma once",
           "#include <cstdint>",
           "namespace lf_forest {",
           f"constexpr int kInputs = {len(FEATURES)};",
           "struct ForestNode { int32_t feature, left, right, leaf; double threshold; };",
           export_forest(m_u, "use_cell"), export_forest(m_p, "parts"), "}  // namespace lf_forest", ""]
    open(os.path.join(ROOT, "paper_conf_hpdc_pengtpk25_b200", "csrc", "lf_forest.h"), "w").write("\n".join(hdr))
    # cases: the training inputs plus perturbed ones, with sklearn's predictions
    rng = np.random.default_rng(0)
    raw = [list(map(float, r["features"])) for r in recs]
    for _ in range(200):
        f = list(raw[rng.integers(n)])
        k = rng.integers(8)
        f[k] = float(f[k] * rng.uniform(0.25, 4.0))
        raw.append(f)
    Xc = np.stack([derive(f) for f in raw])
    cu, cp = m_u.predict(Xc), m_p.predict(Xc)
    with open(os.path.join(ROOT, "tests", "golden", "predictor_cases.txt"), "w") as fh:
        fh.write("# features[8] (Table 2/3: n_rows n_cols nnz mean min max std J) -> sklearn use_cell parts\n")
        fh.write("# written by scripts/train_predictor.py with the forests in csrc/lf_forest.h\n")
        for f, a, b in zip(raw, cu, cp):
            fh.write(" ".join(repr(x) for x in f) + f" {int(a)} {int(b)}\n")
    # report
    L = ["# NEXT-1: format / partition predictor trained on B200 (round 1)", "",
         f"Data `{os.path.basename(path)}` ({n} records = matrices of the mixed-skew suite x J in "
         "{32..512}; `scripts/predictor_data.py`), models `scripts/train_predictor.py` "
         f"(RandomForestClassifier {RF}, inputs: {', '.join(FEATURES)}).", "",
         "Labels (P:L676-678, L743-749): use_cell = CELL at its best P >= 1.1x faster than the CSR kernel; "
         "parts = argmin over P in {1,2,4,8} of the CELL time.", "",
         "Leave-one-family-out cross-validation (the family being predicted is never in the training set):", "",
         "| quantity | value |", "|---|---|",
         f"| use_cell accuracy | {np.mean(pu == use):.3f} |",
         f"| parts accuracy | {np.mean(pp == parts):.3f} |",
         f"| label balance: use_cell=1 | {np.mean(use):.3f} |",
         f"| label balance: parts = 1/2/4/8 | {' / '.join(f'{np.mean(parts == p):.2f}' for p in PARTS)} |",
         f"| geomean time(predicted) / time(best of CSR, CELL P=1..8) | {gm(t_pred / best):.3f} |",
         f"| geomean time(labels) / time(best) | {gm(t_oracle / best):.3f} |",
         f"| geomean time(always CELL P=1, the round-1 stand-in) / time(best) | {gm(t_p1 / best):.3f} |",
         f"| geomean time(always CSR) / time(best) | {gm(t_csr / best):.3f} |",
         f"| worst time(predicted) / time(best) | {np.max(t_pred / best):.2f} |", "",
         "Per family (CV predictions):", "",
         "| family | records | use_cell acc | parts acc | geomean pred/best | geomean P=1/best |", "|---|---|---|---|---|---|"]
    for f in fams:
        m = fam == f
        L.append(f"| {f} | {m.sum()} | {np.mean(pu[m] == use[m]):.2f} | {np.mean(pp[m] == parts[m]):.2f} | "
                 f"{gm(t_pred[m] / best[m]):.3f} | {gm(t_p1[m] / best[m]):.3f} |")
    imp_u = sorted(zip(m_u.feature_importances_, FEATURES), reverse=True)[:5]
    imp_p = sorted(zip(m_p.feature_importances_, FEATURES), reverse=True)[:5]
    L += ["", "Feature importances (final models): use_cell " + ", ".join(f"{k} {v:.2f}" for v, k in imp_u) +
          "; parts " + ", ".join(f"{k} {v:.2f}" for v, k in imp_p) + ".", ""]
    open(os.path.join(ROOT, "profiles", "r1_predictor.md"), "w").write("\n".join(L))
    print("\n".join(L))


if __name__ == "__main__":
    main()

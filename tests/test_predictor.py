"""lf_predict (sections 5.1-5.2): the C forests in
csrc/lf_forest.h reproduce scikit-learn's predictions exactly on the cases
scripts/train_predictor.py wrote (training inputs + perturbed ones).  Host
only: no GPU.  The predictor's *accuracy* has no oracle (the paper ships no
weights): parity unpinned, evaluation in profiles/r1_predictor.md."""
import os

import numpy as np
import pytest

HERE = os.path.dirname(os.path.abspath(__file__))


@pytest.fixture(scope="module")
def lf():
    import paper_conf_hpdc_pengtpk25_b200 as lf
    return lf


def cases():
    out = []
    for line in open(os.path.join(HERE, "golden", "predictor_cases.txt")):
        if line.startswith("#") or not line.strip():
            continue
        v = line.split()
        out.append(([float(x) for x in v[:8]], int(v[8]), int(v[9])))
    return out


def test_c_forest_equals_sklearn(lf):
    cs = cases()
    assert len(cs) >= 400
    bad = [(f, u, p, lf.predict(f)) for f, u, p in cs if lf.predict(f) != (u, p)]
    assert not bad, bad[:5]
    # both labels actually occur (the forest is not constant)
    assert len({u for _, u, _ in cs}) == 2 and len({p for _, _, p in cs}) >= 2


def test_max_parts_clamps(lf):
    for f, _, p in cases():
        if p > 1:
            assert lf.predict(f, max_parts=1)[1] == 1
            assert lf.predict(f, max_parts=p)[1] == p
            break


def test_invalid_features(lf):
    with pytest.raises(lf.LfError):
        lf.predict([1, 2, 3, -1, 0, 0, 0, 32])
    with pytest.raises(lf.LfError):
        lf.predict([1, 2, 3, np.nan, 0, 0, 0, 32])
    with pytest.raises(lf.LfError):
        lf.predict([1] * 8, max_parts=1000)

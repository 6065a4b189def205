"""The on-line batching-policy selector (§5, P272-274).

* oracle/forest_ref.py pinned to a hand-evaluated two-tree forest (every rule of P274:
  comparison per node, leaf vectors summed over trees, larger sum wins) and to a library
  routine: sklearn's RandomForestClassifier.predict, which takes the argmax of the summed
  (averaged) leaf class-probability vectors, on forests trained here on random data.
* the C++ planner's VB_BATCH_AUTO choice (host-only plans) equals the oracle's on the
  committed B200 trees (csrc/forest_b200.json, a platform constant: reading C-25).
"""
import json
import os

import numpy as np
import pytest

import vbinputs
from oracle import forest_ref as fr
from paper_conf_ppopp_li0yjl19_b200 import _native as nv

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

# Tree A: mean K <= 100 ? leaf 0.9 : leaf 0.2.
# Tree B: B <= 64 ? (mean M <= 256 ? leaf 0.6 : leaf 0.0) : leaf 0.3.
HAND = {"trees": [
    {"feature": [2, -1, -1], "threshold": [100.0, -2, -2], "left": [1, -1, -1], "right": [2, -1, -1],
     "p_binary": [0.5, 0.9, 0.2]},
    {"feature": [3, 0, -1, -1, -1], "threshold": [64.0, 256.0, -2, -2, -2], "left": [1, 2, -1, -1, -1],
     "right": [4, 3, -1, -1, -1], "p_binary": [0.5, 0.5, 0.6, 0.0, 0.3]},
]}


@pytest.mark.parametrize("x, want", [
    ((100.0, 7.0, 50.0, 10.0), fr.BINARY),       # A 0.9 + B 0.6 = 1.5 > 0.5
    ((300.0, 7.0, 50.0, 10.0), fr.THRESHOLD),    # A 0.9 + B 0.0 = 0.9 < 1.1
    ((100.0, 7.0, 200.0, 100.0), fr.THRESHOLD),  # A 0.2 + B 0.3 = 0.5 < 1.5
    ((256.0, 7.0, 100.0, 64.0), fr.BINARY),      # equality goes left at both roots: 0.9 + 0.6
])
def test_hand_forest(x, want):
    assert fr.select(HAND, x) == want


def test_tie_goes_to_threshold():
    one = {"trees": [{"feature": [-1], "threshold": [-2.0], "left": [-1], "right": [-1], "p_binary": [0.5]}]}
    assert fr.select(one, (1.0, 1.0, 1.0, 1.0)) == fr.THRESHOLD


def test_features_are_float32_means():
    x = fr.features([1, 2, 4], [3, 3, 3], [16, 17, 17])
    assert x == [float(np.float32(7 / 3)), 3.0, float(np.float32(50 / 3)), 3.0]


def _export(forest):
    trees = []
    for est in forest.estimators_:
        t = est.tree_
        v = t.value[:, 0, :]
        p = v[:, 1] / v.sum(axis=1)
        trees.append({"feature": [int(f) if l != -1 else -1 for f, l in zip(t.feature, t.children_left)],
                      "threshold": [float(a) for a in t.threshold], "left": [int(a) for a in t.children_left],
                      "right": [int(a) for a in t.children_right], "p_binary": [float(a) for a in p]})
    return {"trees": trees}


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_oracle_matches_sklearn_predict(seed):
    from sklearn.ensemble import RandomForestClassifier
    rng = np.random.default_rng(seed)
    X = np.column_stack([rng.uniform(16, 1024, 300), rng.uniform(16, 1024, 300), rng.uniform(16, 2048, 300),
                         rng.integers(1, 4096, 300)]).astype(np.float32)
    y = ((X[:, 2] < 300) ^ (X[:, 3] > 1000) ^ (rng.random(300) < 0.2)).astype(int)
    f = RandomForestClassifier(n_estimators=7, max_depth=5, random_state=seed).fit(X, y)
    model = _export(f)
    Xt = np.column_stack([rng.uniform(16, 1024, 400), rng.uniform(16, 1024, 400), rng.uniform(16, 2048, 400),
                          rng.integers(1, 4096, 400)]).astype(np.float32)
    proba = f.predict_proba(Xt)
    for x, pr_ in zip(Xt, proba):
        if abs(pr_[0] - pr_[1]) < 1e-9:
            continue                                   # sklearn breaks exact ties by class order too
        assert fr.select(model, [float(v) for v in x]) == int(f.predict(x[None])[0])


def _model():
    with open(os.path.join(ROOT, "paper_conf_ppopp_li0yjl19_b200", "csrc", "forest_b200.json")) as fh:
        return json.load(fh)


@pytest.mark.parametrize("dtype,key", [("bf16", "tc"), ("f32", "f32")])
def test_planner_auto_matches_oracle(dtype, key):
    model = _model()[key]
    rng = np.random.default_rng(7)
    seen = set()
    for i in range(150):
        B = int(rng.integers(1, 600))
        hi = int(rng.choice([64, 256, 1024, 2048]))
        M, N, K = (rng.integers(1, hi + 1, B) for _ in range(3))
        ld = lambda c: vbinputs.padded_ld(c, dtype)  # noqa: E731
        plan = nv.plan_vbatched(M, N, K, ld(K), ld(N), ld(N), dtype, nv.VB_BATCH_AUTO, device=-1)
        want = fr.select(model, fr.features(M, N, K))
        assert plan.policy() == want, (i, B, hi)
        seen.add(want)
    # an informative test needs both outcomes unless the trained trees are a single class
    single = all(len(t["p_binary"]) == 1 for t in model["trees"])
    assert single or len(seen) == 2

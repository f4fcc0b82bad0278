"""The exported selector tree (paper_conf_cluster_linwds24_b200/selector_model.json) is a
valid tree whose evaluation reproduces its training labels' predictions (CPU)."""
import json
import os

import numpy as np

import paper_conf_cluster_linwds24_b200 as sf

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def eval_tree(t, x):
    node = 0
    while t["left"][node] >= 0:
        node = t["left"][node] if x[t["feature"][node]] <= t["threshold"][node] else t["right"][node]
    return t["value"][node]


def test_model_is_well_formed_and_matches_sklearn():
    m = json.load(open(sf.MODEL_PATH))
    t = m["tree"]
    n = len(t["feature"])
    assert all(len(t[k]) == n for k in ("threshold", "left", "right", "value"))
    assert all(-1 <= c < n for c in t["left"] + t["right"])
    assert all(0 <= v < m["classes"] for v in t["value"])
    data = os.path.join(ROOT, "profiles", m.get("trained_on", "selector_train_r01.jsonl"))
    if os.path.exists(data):
        from sklearn.tree import DecisionTreeClassifier
        X = np.array([json.loads(l)["features"] for l in open(data)])
        assert X.shape[1] == m["n_features"]
        T = np.array([[v if v is not None else np.inf for v in json.loads(l)["times"]] for l in open(data)])
        assert T.shape[1] == m["classes"]
        clf = DecisionTreeClassifier(max_depth=m["max_depth"], min_samples_leaf=2, random_state=0)
        clf.fit(X, np.argmin(T, 1))
        pred = clf.predict(X[:200])
        assert all(eval_tree(t, x) == p for x, p in zip(X[:200], pred))

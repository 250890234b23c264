"""Generator (gen/) properties: determinism and Table-1 shapes."""
import numpy as np
import pytest

from gen import CONFIGS, make_config, random_tiny


def test_deterministic():
    a, b = make_config("C2"), make_config("C2")
    assert np.array_equal(a.child_class, b.child_class)
    assert np.array_equal(a.u, b.u)


@pytest.mark.parametrize("name", ["C2", "C3", "C5"])
def test_shapes(name):
    spec = CONFIGS[name]
    eg = make_config(name)
    assert eg.num_nodes == spec["N"] and eg.num_classes == spec["M"]
    assert abs(eg.num_edges / eg.num_nodes - spec["d"]) < 0.15 * spec["d"]
    assert np.all(np.diff(eg.class_ptr) >= 1)
    assert eg.child_class.min() >= 0 and eg.child_class.max() < eg.num_classes
    # children are sets
    for i in range(0, eg.num_nodes, 97):
        kids = eg.children(i)
        assert len(set(kids)) == len(kids)
    assert eg.meta["scc_max"] <= spec["scc_max"]
    assert eg.meta["scc_classes"] > 0
    assert np.all(eg.u == np.round(eg.u)) and eg.u.min() >= 0 and eg.u.max() <= 100
    if spec["cost"] == "quadratic":
        qi, qj, w = eg.quad
        assert np.all(qi < qj) and np.all(w != 0) and np.all(np.abs(w) <= 10)
    if spec["cost"] == "mlp":
        assert eg.mlp["W1"].shape == (64, eg.num_nodes) and eg.mlp["W3"].shape == (1, 8)


def test_tiny_tree_has_one_parent_node():
    for s in range(20):
        eg = random_tiny(s, "tree", num_classes=6)
        cnt = np.zeros(eg.num_classes, int)
        for i in range(eg.num_nodes):
            for c in eg.children(i):
                cnt[c] += 1
        assert cnt[0] == 0 and np.all(cnt[1:] == 1)

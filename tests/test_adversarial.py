"""Set cover -> e-graph extraction (gen/adversarial.py):
the conversion is pinned by brute force (the optimum extraction is the
minimum-weight set cover, enumerated over subsets of sets), and the planted
instance reproduces the paper's point that the heuristic misses shared
subterms (P135)."""
import itertools

import numpy as np
import pytest

from gen.adversarial import maxsat_egraph, planted_cover, random_maxsat, random_set_cover
from oracle import brute
from oracle.greedy import greedy


def min_cover(eg):
    """minimum-weight set cover by enumerating subsets of the sets."""
    n, m = eg.meta["elements"], eg.meta["sets"]
    members = []
    for j in range(m):
        members.append({e for e in range(n)
                        if 1 + n + j in [int(c) for k in range(int(eg.class_ptr[1 + e]),
                                                             int(eg.class_ptr[2 + e]))
                                         for c in eg.children(k)]})
    w = eg.u[-m:]
    best = np.inf
    for r in range(1, m + 1):
        for sub in itertools.combinations(range(m), r):
            if set().union(*(members[j] for j in sub)) == set(range(n)):
                best = min(best, float(sum(w[j] for j in sub)))
    return best


@pytest.mark.parametrize("seed", range(6))
def test_optimum_extraction_is_min_cover(seed):
    eg = random_set_cover(7, 6, 0.35, seed)
    assert brute.exhaustive_optimum(eg) == min_cover(eg)
    g = greedy(eg)
    assert g["valid"] and g["dag_cost"] >= min_cover(eg)


def test_planted_heuristic_gap():
    eg = planted_cover(4, seed=1)
    assert min_cover(eg) == 8.0
    g = greedy(eg)
    assert g["dag_cost"] == 12.0 and g["root_cost"] == 12.0


def min_unsat_weight(eg):
    """weighted MaxSAT by enumerating all truth assignments."""
    n = eg.meta["vars"]
    best = np.inf
    for bits in itertools.product([False, True], repeat=n):
        unsat = sum(w for cl, w in zip(eg.meta["clause_list"], eg.meta["weights"])
                    if not any(bits[abs(l) - 1] == (l > 0) for l in cl))
        best = min(best, unsat)
    return best


@pytest.mark.parametrize("seed", range(6))
def test_maxsat_optimum_extraction(seed):
    """The optimum extraction of the converted e-graph is minus the maximum
    satisfied weight: min unsatisfied weight - total weight (enumerated over
    all 2^n assignments and, independently, over all extractions)."""
    eg = random_maxsat(6, 14, 3, seed)
    assert brute.exhaustive_optimum(eg) == min_unsat_weight(eg) - eg.meta["total_weight"]


def test_maxsat_handmade():
    """(x1 or x2) w3, (not x1) w2, (not x2 or x1) w1: x1 = F, x2 = T
    satisfies the first two (5); x1 = T satisfies the first and third (4):
    optimum -5, unsatisfied weight 1."""
    eg = maxsat_egraph([[1, 2], [-1], [-2, 1]], [3.0, 2.0, 1.0], 2)
    eg.meta["clause_list"] = [[1, 2], [-1], [-2, 1]]
    eg.meta["weights"] = [3.0, 2.0, 1.0]
    assert brute.exhaustive_optimum(eg) == -5.0
    assert min_unsat_weight(eg) == 1.0
    # every extraction is an assignment: 2^2 of them, all valid (acyclic)
    assert sum(1 for _ in brute.assignments(eg)) == 4

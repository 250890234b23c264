"""Adversarial e-graphs (Sec. 5.3):
minimum set cover converted to e-graph extraction.  Inputs only (no method
arithmetic).

Conversion (the common-subexpression construction the paper describes: the
converted graphs are "rich in common sub-expressions" and carry "less
graphical information"):

* the root e-class m_0 holds one e-node (cost 0) whose children are the
  element e-classes;
* element e-class e_i holds one e-node per set S_j containing e_i (cost 0),
  whose only child is the set e-class of S_j;
* set e-class s_j holds one leaf e-node of cost w_j (the set's weight).

Every extraction picks, for each element, one covering set; a set class used
by several elements is selected once (the cost of a term counts shared
subterms once), so f_b(s) = the weight of the chosen
cover, and the optimum extraction is a minimum-weight set cover.  The greedy
worklist sees every element's cost as the full weight of its
cheapest set and cannot trade a set's weight against its reuse (P135).

The instances here are random (a seeded universe of n elements and m sets,
each element in at least one set); :func:`planted_cover` plants a cover that
beats the greedy heuristic's choice.

MaxSAT (the paper's second adversarial family, Table 4 P400-401; the paper
defers its conversion to refs [42, 55]) -- :func:`maxsat_egraph`:

* the root e-class holds one e-node (cost 0) whose children are the variable
  e-classes;
* variable e-class x_i holds two e-nodes, "x_i true" and "x_i false" (cost
  0); the first's children are the clause e-classes of the clauses with the
  literal x_i, the second's those with the literal not-x_i;
* clause e-class c holds one leaf e-node of cost -w_c (a reward).

An extraction is exactly a truth assignment (one e-node per variable class,
so x and not-x are never both chosen), the clause classes it reaches are the
clauses it satisfies, each counted once (P100, P170), so f_b(s) = -(weight of
the satisfied clauses) and the optimum extraction is a maximum-weight
assignment: optimum = min unsatisfied weight - total weight.  The costs are
negative (rewards), which the linear relaxation accepts as they are; the
greedy worklist heuristic (P133) needs non-negative costs and is not applied.
"""
from __future__ import annotations

import numpy as np

from .egraph import EGraphInput


def set_cover_egraph(sets, weights, n_elems, name="setcover"):
    """E-graph of the weighted set cover instance ``sets`` (list of element
    lists) with ``weights``.  Class order: root, elements 0..n-1, sets."""
    m = len(sets)
    cover = [[] for _ in range(n_elems)]
    for j, s in enumerate(sets):
        for e in sorted(set(s)):
            cover[e].append(j)
    assert all(cover), "every element must lie in some set"
    sizes = [1] + [len(c) for c in cover] + [1] * m
    class_ptr = np.concatenate([[0], np.cumsum(sizes)]).astype(np.int32)
    kids = [list(range(1, 1 + n_elems))]
    for e in range(n_elems):
        kids += [[1 + n_elems + j] for j in cover[e]]
    kids += [[] for _ in range(m)]
    child_ptr = np.concatenate([[0], np.cumsum([len(k) for k in kids])]).astype(np.int64)
    child_class = np.array([c for k in kids for c in k], dtype=np.int32)
    u = np.zeros(len(kids))
    u[-m:] = np.asarray(weights, dtype=np.float64)
    return EGraphInput(name, class_ptr, child_ptr, child_class, u, 0,
                       meta={"kind": "setcover", "elements": n_elems, "sets": m})


def random_set_cover(n_elems, n_sets, density, seed, wmax=5):
    """Seeded random instance: element e is in set j with probability
    ``density`` (at least one set each); integer weights U{1..wmax}."""
    rng = np.random.default_rng(seed)
    inc = rng.random((n_sets, n_elems)) < density
    for e in range(n_elems):
        if not inc[:, e].any():
            inc[rng.integers(n_sets), e] = True
    sets = [list(np.nonzero(inc[j])[0]) for j in range(n_sets)]
    w = rng.integers(1, wmax + 1, n_sets).astype(np.float64)
    return set_cover_egraph(sets, w, n_elems, name=f"setcover{seed}")


def planted_cover(k=4, seed=0):
    """k disjoint 'block' sets of weight 2 cover all 2k elements (optimum 2k);
    2k singleton sets of weight 1.5 each cover one element.  The heuristic
    prices every element at its cheapest set (1.5 < 2) and extracts the
    singletons (3k); the optimum shares the blocks (2k)."""
    rng = np.random.default_rng(seed)
    n = 2 * k
    perm = rng.permutation(n)
    blocks = [sorted(perm[2 * b: 2 * b + 2].tolist()) for b in range(k)]
    singles = [[e] for e in range(n)]
    sets = blocks + singles
    w = [2.0] * k + [1.5] * n
    order = rng.permutation(len(sets))
    return set_cover_egraph([sets[i] for i in order], [w[i] for i in order], n,
                            name=f"planted{k}")


def maxsat_egraph(clauses, weights, n_vars, name="maxsat"):
    """E-graph of the weighted MaxSAT instance ``clauses`` (lists of non-zero
    ints, DIMACS style: +i / -i for x_i / not-x_i, 1-based) with ``weights``.
    Class order: root, variables 1..n, clauses."""
    m = len(clauses)
    pos = [[] for _ in range(n_vars)]
    neg = [[] for _ in range(n_vars)]
    for c, cl in enumerate(clauses):
        for lit in set(cl):
            assert lit != 0 and abs(lit) <= n_vars
            (pos if lit > 0 else neg)[abs(lit) - 1].append(1 + n_vars + c)
    sizes = [1] + [2] * n_vars + [1] * m
    class_ptr = np.concatenate([[0], np.cumsum(sizes)]).astype(np.int32)
    kids = [list(range(1, 1 + n_vars))]
    for i in range(n_vars):
        kids += [sorted(pos[i]), sorted(neg[i])]
    kids += [[] for _ in range(m)]
    child_ptr = np.concatenate([[0], np.cumsum([len(k) for k in kids])]).astype(np.int64)
    child_class = np.array([c for k in kids for c in k], dtype=np.int32)
    u = np.zeros(len(kids))
    u[-m:] = -np.asarray(weights, dtype=np.float64)
    return EGraphInput(name, class_ptr, child_ptr, child_class, u, 0,
                       meta={"kind": "maxsat", "vars": n_vars, "clauses": m,
                             "total_weight": float(np.sum(weights))})


def random_maxsat(n_vars, n_clauses, k, seed, wmax=5):
    """Seeded random weighted k-SAT instance (distinct variables per clause,
    random signs, integer weights U{1..wmax}) as an e-graph."""
    rng = np.random.default_rng(seed)
    clauses = []
    for _ in range(n_clauses):
        vs = rng.choice(n_vars, size=min(k, n_vars), replace=False) + 1
        clauses.append([int(v) if rng.random() < 0.5 else -int(v) for v in vs])
    w = rng.integers(1, wmax + 1, n_clauses).astype(np.float64)
    eg = maxsat_egraph(clauses, w, n_vars, name=f"maxsat{seed}")
    eg.meta["clause_list"] = clauses
    eg.meta["weights"] = w.tolist()
    return eg

"""Brute-force enumerator / certifier for tiny e-graphs -- TEST INFRASTRUCTURE.

Independent of smoothe_oracle.cpp (pure Python, different algorithms): it is
one of the things the oracle is pinned to.

The induced distribution (P3): every e-class independently draws one of its
e-nodes with probability cp; the selected term is the set of classes reached
from the root through the drawn e-nodes (constraints (a),
(b)).  P(n_i chosen) is the total probability of draws in which ec(i) is
reached and i is its drawn node -- the quantity p_i of Eq. 2.
"""
from __future__ import annotations

import itertools
from collections import deque

import numpy as np


def _class_nodes(eg):
    return [list(range(int(eg.class_ptr[j]), int(eg.class_ptr[j + 1])))
            for j in range(eg.num_classes)]


def _children(eg):
    return [sorted(set(int(c) for c in eg.child_class[eg.child_ptr[i]:eg.child_ptr[i + 1]]))
            for i in range(eg.num_nodes)]


def reach(eg, choice, kids=None):
    """Classes reached from the root when class j uses e-node choice[j] (BFS)."""
    kids = kids or _children(eg)
    seen = {eg.root}
    dq = deque([eg.root])
    while dq:
        j = dq.popleft()
        for c in kids[choice[j]]:
            if c not in seen:
                seen.add(c)
                dq.append(c)
    return seen


def acyclic(eg, choice, reached, kids=None):
    """Constraint (c) by Kahn's algorithm on the reached subgraph."""
    kids = kids or _children(eg)
    indeg = {j: 0 for j in reached}
    for j in reached:
        for c in kids[choice[j]]:
            indeg[c] += 1
    dq = deque(j for j in reached if indeg[j] == 0)
    n = 0
    while dq:
        j = dq.popleft()
        n += 1
        for c in kids[choice[j]]:
            indeg[c] -= 1
            if indeg[c] == 0:
                dq.append(c)
    return n == len(reached)


def assignments(eg):
    return itertools.product(*_class_nodes(eg))


def marginals(eg, cp):
    """Exact P(n_i chosen) under the induced distribution, by enumeration."""
    kids = _children(eg)
    p = np.zeros(eg.num_nodes)
    preach = np.zeros(eg.num_classes)
    for ch in assignments(eg):
        w = float(np.prod([cp[k] for k in ch]))
        if w == 0.0:
            continue
        for j in reach(eg, ch, kids):
            p[ch[j]] += w
            preach[j] += w
    return p, preach


def parents(eg):
    kids = _children(eg)
    pa = [[] for _ in range(eg.num_classes)]
    for i in range(eg.num_nodes):
        for c in kids[i]:
            pa[c].append(i)
    return pa


def certified(eg, cp, assumption, tol=1e-12):
    """True iff, for every non-root class with >= 2 parent e-nodes, the paper's
    aggregator applied to the TRUE parent marginals gives the TRUE class
    probability: ind (Eq. 6b) holds iff parent events are independent enough,
    cor (Eq. 7) iff they are nested."""
    p, preach = marginals(eg, cp)
    pa = parents(eg)
    for j in range(eg.num_classes):
        if j == eg.root or len(pa[j]) < 2:
            continue
        ind = 1.0 - np.prod([1.0 - p[k] for k in pa[j]])
        cor = max(p[k] for k in pa[j])
        val = {"independent": ind, "correlated": cor, "hybrid": 0.5 * ind + 0.5 * cor}[assumption]
        if abs(val - preach[j]) > tol:
            return False
    return True


def discrete_cost(eg, choice, reached):
    """f_b(s) = u^T s, shared terms counted once."""
    return float(sum(eg.u[choice[j]] for j in reached))


def exhaustive_optimum(eg):
    """min f_b(s) over all valid extractions (constraints (a)-(c))."""
    kids = _children(eg)
    best = np.inf
    for ch in assignments(eg):
        r = reach(eg, ch, kids)
        if acyclic(eg, ch, r, kids):
            best = min(best, discrete_cost(eg, ch, r))
    return best

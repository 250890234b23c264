"""Greedy worklist extraction (the paper's "heuristic method") -- TEST
INFRASTRUCTURE ONLY (see oracle/__init__.py).

PAPER.md:133 (Section 2, "Heuristic Methods"), followed step by step:

* every e-class cost starts at infinity;
* the aggregated cost of e-node n_i is u_i plus the costs of its child
  e-classes ch_i;
* the working queue starts with every leaf e-node (no child e-classes);
* when n_i is dequeued its aggregated cost is computed; if it beats the cost of
  its e-class ec(i), the e-class takes that cost and selects n_i, and the parent
  e-nodes pa_ec(i) are queued;
* repeat until the queue is empty; the extraction is then read top-down from
  the root through the selected e-nodes.

Reading G1 (ties): "beats" compares (cost, height, e-node
id) lexicographically, height = 1 + the largest height of the child e-classes
(0 for a leaf).  Costs decide as in the paper; among equal costs the shorter
derivation wins, so the selection can never close a cycle (height strictly
decreases along every selected edge, also through zero-cost e-nodes), and the
lowest id breaks the remaining ties, which makes the result independent of
the queue order.

The extraction's cost is f_b(s) of P100: the sum of u over the selected
e-nodes of the e-classes reached from the root, each e-class once (reading
S19) -- the cost the heuristic's tree estimate overstates when subexpressions
are shared (P135, Fig. 2b: 27 against the optimum 19).
"""
from __future__ import annotations

from collections import deque

import numpy as np

INF = float("inf")


def greedy(eg, order: str = "fifo", seed: int = 0):
    """Return dict(choice [M] (-1: class not extracted), class_cost [M],
    height [M], root_cost, dag_cost, valid).  ``order`` = "fifo" (the paper's
    queue), "lifo" or "random" (a seeded shuffle of each pop): the result must
    not depend on it (reading G1)."""
    M, N = eg.num_classes, eg.num_nodes
    ec = eg.ec()
    kids = [sorted(set(int(c) for c in eg.children(i))) for i in range(N)]
    pa = [[] for _ in range(M)]  # parent e-nodes of each class
    for i in range(N):
        for c in kids[i]:
            pa[c].append(i)
    cost = [INF] * M
    height = [0] * M
    sel = [-1] * M

    def key_of(j):
        return (cost[j], height[j], sel[j] if sel[j] >= 0 else N)

    rng = np.random.default_rng(seed)
    queue = deque(i for i in range(N) if not kids[i])
    queued = [False] * N
    for i in queue:
        queued[i] = True
    while queue:
        if order == "fifo":
            i = queue.popleft()
        elif order == "lifo":
            i = queue.pop()
        else:
            queue.rotate(-int(rng.integers(len(queue))))
            i = queue.popleft()
        queued[i] = False
        agg = float(eg.u[i]) + sum(cost[c] for c in kids[i])
        h = 1 + max((height[c] for c in kids[i]), default=-1)
        j = int(ec[i])
        if agg < INF and (agg, h, i) < key_of(j):
            cost[j], height[j], sel[j] = agg, h, i
            for k in pa[j]:
                if not queued[k]:
                    queued[k] = True
                    queue.append(k)
    # top-down: the e-classes the root's selection reaches
    root = int(eg.root)
    choice = np.full(M, -1, dtype=np.int64)
    valid = sel[root] >= 0
    dag = 0.0
    if valid:
        seen = {root}
        stack = [root]
        while stack:
            j = stack.pop()
            choice[j] = sel[j]
            for c in kids[sel[j]]:
                if c not in seen:
                    seen.add(c)
                    stack.append(c)
        dag = float(sum(float(eg.u[choice[j]]) for j in seen))
    return {"choice": choice, "class_cost": np.array(cost), "height": np.array(height),
            "root_cost": cost[root], "dag_cost": dag if valid else INF, "valid": bool(valid)}

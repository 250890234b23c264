"""Seeded e-graph generators (inputs only; none of the method's arithmetic).

An e-graph is given the way the paper states the problem (PAPER.md:91-101,
Sec. 2 "Notations and Problem Formulation"):

* e-classes m_0..m_{M-1}, the root e-class has index 0;
* e-nodes n_0..n_{N-1}; e-class j owns the contiguous node range
  ``class_ptr[j] .. class_ptr[j+1]-1`` (this is ec(i));
* ch_i, the set of child e-classes of e-node i, as CSR
  ``child_ptr[N+1]`` / ``child_class[E]``;
* u, the linear per-e-node cost.

Three sources:

* :func:`fig1c_fixture` -- the e-graph of Figures 1c/2/3 (PAPER.md:75-87,
  160-172, 225-239) as reconstructed in SURVEY.md Appendix A.
* :func:`random_tiny` -- tiny tree / DAG / cyclic graphs (config C1) that a
  brute-force enumerator can certify.
* :func:`synth_egraph` -- Table-1-shaped synthetic graphs:
  levelled classes, heavy-tailed class sizes, an "anchor" e-node per class
  whose children lie strictly deeper (so an acyclic extraction always exists,
  DESIGN.md reading S30), locality-windowed children, back edges that create
  bounded strongly connected components, and sibling e-nodes sharing child
  sets (commutativity-like).
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np


@dataclass
class EGraphInput:
    name: str
    class_ptr: np.ndarray            # int32 [M+1]
    child_ptr: np.ndarray            # int64 [N+1]
    child_class: np.ndarray          # int32 [E]
    u: np.ndarray                    # float64 [N], linear cost
    root: int = 0
    quad: tuple | None = None        # (i int32[P], j int32[P], w float64[P]), i<j
    mlp: dict | None = None          # W1 [H1][N], b1 [H1], W2 [H2][H1], b2, W3 [1][H2], b3 (float32)
    meta: dict = field(default_factory=dict)

    @property
    def num_classes(self) -> int:
        return len(self.class_ptr) - 1

    @property
    def num_nodes(self) -> int:
        return len(self.child_ptr) - 1

    @property
    def num_edges(self) -> int:
        return int(self.child_ptr[-1])

    def ec(self) -> np.ndarray:
        """ec(i): class of e-node i."""
        sizes = np.diff(self.class_ptr)
        return np.repeat(np.arange(self.num_classes, dtype=np.int32), sizes)

    def children(self, i: int) -> list[int]:
        return [int(c) for c in self.child_class[self.child_ptr[i]:self.child_ptr[i + 1]]]

    def cost_kind(self) -> str:
        if self.mlp is not None:
            return "mlp"
        if self.quad is not None:
            return "quadratic"
        return "linear"


def _csr(owner: np.ndarray, child: np.ndarray, n: int):
    """Sort (owner, child) pairs, drop duplicates (set semantics)."""
    if owner.size:
        key = owner.astype(np.int64) * (1 << 32) + child.astype(np.int64)
        key = np.unique(key)
        owner = (key >> 32).astype(np.int64)
        child = (key & 0xFFFFFFFF).astype(np.int32)
    ptr = np.zeros(n + 1, dtype=np.int64)
    np.add.at(ptr, owner + 1, 1)
    return np.cumsum(ptr), child.astype(np.int32)


# ---------------------------------------------------------------------------
# Figure 1c fixture
# ---------------------------------------------------------------------------

def fig1c_fixture() -> EGraphInput:
    """sec^2(a) + tan(a) after sec->1/cos and sec^2->1+tan^2 (Fig. 1c).

    Classes: m0 root {n0:+}, m1 sec^2 {n1:x^2, n2:+},
    m2 tan^2 {n3:x^2}, m3 sec {n4:sec, n5:1/x}, m4 "1" {n6}, m5 tan {n7},
    m6 cos {n8}, m7 alpha {n9}.  Costs are the circled numbers of Fig. 2
    (PAPER.md:162-170): solutions cost 32, 27 and 19.
    """
    class_ptr = np.array([0, 1, 3, 4, 6, 7, 8, 9, 10], dtype=np.int32)
    kids = [[1, 5], [3], [2, 4], [5], [7], [6], [], [7], [7], []]
    u = np.array([2, 5, 2, 5, 10, 5, 0, 10, 10, 0], dtype=np.float64)
    child_ptr = np.zeros(11, dtype=np.int64)
    child_ptr[1:] = np.cumsum([len(k) for k in kids])
    child_class = np.array([c for k in kids for c in k], dtype=np.int32)
    return EGraphInput("fig1c", class_ptr, child_ptr, child_class, u, 0,
                       meta={"levels": 4})


# ---------------------------------------------------------------------------
# Random tiny graphs (config C1)
# ---------------------------------------------------------------------------

def random_tiny(seed: int, kind: str = "dag", num_classes: int = 8,
                max_class_size: int = 4, max_children: int = 3,
                cost_max: int = 10) -> EGraphInput:
    """Tiny graph of one of three families.

    * ``tree``: every non-root class has exactly one parent e-node, and that
      parent sits in a lower-numbered class.
    * ``dag``: children only in higher-numbered classes; every class j>0 has
      at least one parent.
    * ``cyclic``: as ``dag`` plus back/self edges on non-first e-nodes; the
      first e-node of each class keeps forward-only children, so an acyclic
      extraction exists (reading S30).
    """
    rng = np.random.default_rng(seed)
    M = num_classes
    sizes = rng.integers(1, max_class_size + 1, M)
    class_ptr = np.zeros(M + 1, dtype=np.int32)
    class_ptr[1:] = np.cumsum(sizes)
    N = int(class_ptr[-1])
    ec = np.repeat(np.arange(M), sizes)
    kids: list[set] = [set() for _ in range(N)]
    if kind == "tree":
        for j in range(1, M):
            parent = int(rng.integers(0, class_ptr[j]))
            kids[parent].add(j)
    else:
        for i in range(N):
            c = ec[i]
            if c + 1 < M:
                for _ in range(int(rng.integers(0, max_children + 1))):
                    kids[i].add(int(rng.integers(c + 1, M)))
        for j in range(1, M):
            if not any(j in kids[i] for i in range(N)):
                kids[int(rng.integers(0, class_ptr[j]))].add(j)
        if kind == "cyclic":
            for i in range(N):
                c = ec[i]
                if i != class_ptr[c] and rng.random() < 0.5:
                    kids[i].add(int(rng.integers(0, c + 1)))
    u = rng.integers(0, cost_max + 1, N).astype(np.float64)
    child_ptr = np.zeros(N + 1, dtype=np.int64)
    child_ptr[1:] = np.cumsum([len(k) for k in kids])
    child_class = np.array([c for k in kids for c in sorted(k)], dtype=np.int32)
    return EGraphInput(f"tiny-{kind}-{seed}", class_ptr, child_ptr, child_class, u, 0,
                       meta={"kind": kind})


# ---------------------------------------------------------------------------
# Table-1-shaped synthetic graphs (configs C2-C5)
# ---------------------------------------------------------------------------

def synth_egraph(name: str, N: int, M: int, d: float, D: int, *, seed: int,
                 w_levels: int = 3, w_pos: float = 0.01, p_back: float = 0.0,
                 b_levels: int = 1, b_pos: float | None = None, scc_max: int = 64,
                 share_frac: float = 0.1, size_alpha: float = 2.5, root_size: int = 2,
                 max_children: int = 16, cost_model: str = "linear",
                 quad_window: int = 64, mlp_hidden: tuple = (64, 8),
                 mlp_scale: float = 1.0) -> EGraphInput:
    """Levelled synthetic e-graph with N e-nodes, M e-classes, about d child
    classes per e-node and D levels below the root."""
    rng = np.random.default_rng(seed)
    b_pos = w_pos if b_pos is None else b_pos

    # --- levels: root alone at level 0, the rest spread evenly over 1..D
    M1 = M - 1
    lvl_sizes = np.full(D + 1, 0, dtype=np.int64)
    lvl_sizes[0] = 1
    lvl_sizes[1:] = M1 // D
    lvl_sizes[1:1 + M1 % D] += 1
    lvl_start = np.zeros(D + 2, dtype=np.int64)
    lvl_start[1:] = np.cumsum(lvl_sizes)
    level = np.repeat(np.arange(D + 1), lvl_sizes)
    pos = (np.arange(M) - lvl_start[level] + 0.5) / lvl_sizes[level]

    # --- class sizes: 1 + heavy-tailed share of the N - M extra e-nodes
    wts = rng.pareto(size_alpha, M) + 1.0
    wts[0] = 0.0
    extra = rng.multinomial(N - M - (root_size - 1), wts / wts.sum())
    extra[0] = root_size - 1
    sizes = 1 + extra
    class_ptr = np.zeros(M + 1, dtype=np.int64)
    class_ptr[1:] = np.cumsum(sizes)
    assert class_ptr[-1] == N
    ec = np.repeat(np.arange(M), sizes)
    anchor = class_ptr[:-1]
    is_anchor = np.zeros(N, dtype=bool)
    is_anchor[anchor] = True
    nlev = level[ec]
    npos = pos[ec]

    def pick(lvl, x):
        sz = lvl_sizes[lvl]
        k = np.minimum((np.clip(x, 0.0, 0.999999) * sz).astype(np.int64), sz - 1)
        return lvl_start[lvl] + k

    # --- shared child sets: node copies the previous node of its class
    shared = (rng.random(N) < share_frac) & ~is_anchor
    src = np.maximum.accumulate(np.where(shared, 0, np.arange(N)))

    # --- child counts (deepest level: leaves)
    leaves = nlev == D
    mand = M - 1                                     # mandatory anchor edges
    free = max(1, int((~leaves & ~shared).sum()))
    lam = max(0.0, (d * N * (1.0 - share_frac) - mand) / free - 1.0)
    cnt = 1 + rng.poisson(lam, N)
    cnt = np.minimum(cnt, max_children)
    cnt[leaves | shared] = 0
    owner = np.repeat(np.arange(N), cnt)
    olev = nlev[owner]
    opos = npos[owner]
    S = owner.size
    back = (~is_anchor[owner]) & (rng.random(S) < p_back)
    tl = np.where(back,
                  np.maximum(1, olev - rng.integers(0, b_levels + 1, S)),
                  np.minimum(D, olev + rng.integers(1, w_levels + 1, S)))
    wp = np.where(back, b_pos, w_pos)
    child = pick(tl, opos + rng.uniform(-1.0, 1.0, S) * wp)

    # mandatory edge: anchor of the nearest class one level up -> j
    js = np.arange(1, M)
    pc = pick(level[js] - 1, pos[js])
    owner = np.concatenate([owner, anchor[pc]])
    child = np.concatenate([child, js])
    isback = level[child] <= level[ec[owner]]

    # --- bound SCC sizes by dropping back edges inside oversized components
    from scipy.sparse import csr_matrix
    from scipy.sparse.csgraph import connected_components
    for _ in range(64):
        A = csr_matrix((np.ones(owner.size, dtype=np.int8), (ec[owner], child)), shape=(M, M))
        _, lab = connected_components(A, directed=True, connection="strong")
        csz = np.bincount(lab)
        if csz.max() <= scc_max:
            break
        inbig = (csz[lab[ec[owner]]] > scc_max) & (lab[ec[owner]] == lab[child]) & isback
        drop = inbig & (rng.random(owner.size) < 0.35)
        keep = ~drop
        owner, child, isback = owner[keep], child[keep], isback[keep]

    # an upward edge that closes no cycle would only stretch the acyclic skeleton
    # beyond D levels: keep back edges inside strongly connected components only
    A = csr_matrix((np.ones(owner.size, dtype=np.int8), (ec[owner], child)), shape=(M, M))
    _, lab = connected_components(A, directed=True, connection="strong")
    keep = ~isback | (lab[ec[owner]] == lab[child])
    owner, child, isback = owner[keep], child[keep], isback[keep]

    ptr_ns, child_ns = _csr(owner, child, N)
    cnt_all = np.diff(ptr_ns)[src]
    child_ptr = np.zeros(N + 1, dtype=np.int64)
    child_ptr[1:] = np.cumsum(cnt_all)
    E = int(child_ptr[-1])
    offs = np.arange(E, dtype=np.int64) - np.repeat(child_ptr[:-1], cnt_all)
    child_class = child_ns[np.repeat(ptr_ns[src], cnt_all) + offs].astype(np.int32)

    # --- costs: U{1..100}, leaves U{0,1} (as in Fig. 2: constants cost 0)
    u = rng.integers(1, 101, N).astype(np.float64)
    nleaf = cnt_all == 0
    u[nleaf] = rng.integers(0, 2, int(nleaf.sum()))

    quad = None
    mlp = None
    if cost_model == "quadratic":
        i = rng.integers(0, N - 1, N)
        k = np.minimum(i + rng.integers(1, quad_window + 1, N), N - 1)
        key = np.unique(i.astype(np.int64) * N + k)
        qi = (key // N).astype(np.int32)
        qj = (key % N).astype(np.int32)
        keep = qi < qj
        qi, qj = qi[keep], qj[keep]
        w = rng.integers(1, 11, qi.size) * rng.choice([-1, 1], qi.size)
        quad = (qi, qj, w.astype(np.float64))
    elif cost_model == "mlp":
        H1, H2 = mlp_hidden
        lim1 = np.sqrt(6.0 / N)
        lim2 = np.sqrt(6.0 / H1)
        lim3 = np.sqrt(6.0 / H2)
        mlp = {
            "W1": rng.uniform(-lim1, lim1, (H1, N)).astype(np.float32),
            "b1": rng.uniform(-0.1, 0.1, H1).astype(np.float32),
            "W2": rng.uniform(-lim2, lim2, (H2, H1)).astype(np.float32),
            "b2": rng.uniform(-0.1, 0.1, H2).astype(np.float32),
            "W3": (mlp_scale * rng.uniform(-lim3, lim3, (1, H2))).astype(np.float32),
            "b3": np.zeros(1, dtype=np.float32),
        }

    # descriptive metadata (structure only)
    A = csr_matrix((np.ones(E, dtype=np.int8), (np.repeat(ec, cnt_all), child_class)), shape=(M, M))
    _, lab = connected_components(A, directed=True, connection="strong")
    csz = np.bincount(lab)
    selfloop = np.zeros(M, dtype=bool)
    sl = np.repeat(ec, cnt_all) == child_class
    selfloop[np.repeat(ec, cnt_all)[sl]] = True
    nontriv = (csz[lab] > 1) | selfloop
    meta = {
        "levels": D, "N": N, "M": M, "E": E, "d": E / N, "r": M / N,
        "scc_classes": int(nontriv.sum()), "scc_max": int(csz.max()),
        "num_scc_nontrivial": int(len(np.unique(lab[nontriv]))),
        "max_class_size": int(sizes.max()), "seed": seed,
    }
    return EGraphInput(name, class_ptr.astype(np.int32), child_ptr, child_class, u, 0,
                       quad=quad, mlp=mlp, meta=meta)

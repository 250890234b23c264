"""Learned MLP cost (Sec. 5.5).

"To train the MLP, we generate a synthetic dataset for each e-graph: the
training data consists of random discrete valid solutions, and the target
values are set as random negative numbers representing savings for these
solutions.  Regression is performed to optimize the MLP using this synthetic
dataset."  (P425)

* solutions: random logits theta ~ U(-a, a) per e-node, decoded by the
  library's own decode (smoothe_debug_step: argmax per class, reach from the
  root, acyclicity check, P279); the valid ones give binary vectors s in
  {0,1}^N (s_k = 1 iff class ec(k) is reached and chose k, P99);
* targets: y ~ U(-target_scale, 0), seeded (the paper's "random negative
  numbers representing savings");
* model: N -> H1 -> H2 -> 1 with ReLU (reading S22), fit by Adam on the mean
  squared error.  This is offline model preparation, not the hot path: it runs
  in PyTorch (on the GPU when available) and returns float32 weights in the
  layout smoothe_cost_model takes (row-major [out][in]).
"""
from __future__ import annotations

import numpy as np

from .smoothe import CostModel, Options, load_egraph_from, run_create


def sample_solutions(eg, num: int, seed: int = 0, scale: float = 3.0, batch: int = 128,
                     device: int = 0, max_batches: int = 64):
    """Up to ``num`` distinct-or-not valid extractions as s [num][N] float32."""
    g = load_egraph_from(eg, device=device)
    rng = np.random.default_rng(seed)
    cm = CostModel(np.asarray(eg.u, dtype=np.float64))
    run = run_create(g, cm, batch, Options(penalty_group=batch, lam=0.0))
    ec = eg.ec()
    out = []
    try:
        for _ in range(max_batches):
            th = rng.uniform(-scale, scale, (eg.num_nodes, batch)).astype(np.float32)
            d = run.debug_step(th)
            ok = np.nonzero(d["valid"])[0]
            for b in ok:
                reached = d["reached"][:, b].astype(bool)
                s = np.zeros(eg.num_nodes, np.float32)
                sel = np.nonzero(reached)[0]
                s[d["choice"][sel, b]] = 1.0
                assert np.all(ec[d["choice"][sel, b]] == sel)
                out.append(s)
                if len(out) == num:
                    return np.stack(out)
    finally:
        run.close()
        g.close()
    if not out:
        raise RuntimeError("no valid extraction sampled")
    return np.stack(out)


def train_mlp(S, seed: int = 0, hidden=(64, 8), target_scale: float = 10.0, epochs: int = 300,
              lr: float = 1e-2, device=None):
    """Fit N -> H1 -> H2 -> 1 to random negative targets on the solutions S.
    Returns (weights dict for CostModel.mlp, targets, (first, last) MSE)."""
    import torch

    dev = torch.device(device or ("cuda" if torch.cuda.is_available() else "cpu"))
    rng = np.random.default_rng(seed)
    y = -target_scale * rng.random(S.shape[0])
    gen = torch.Generator().manual_seed(seed)
    N = S.shape[1]
    H1, H2 = hidden
    model = torch.nn.Sequential(torch.nn.Linear(N, H1), torch.nn.ReLU(), torch.nn.Linear(H1, H2),
                                torch.nn.ReLU(), torch.nn.Linear(H2, 1))
    with torch.no_grad():
        for m in model:
            if isinstance(m, torch.nn.Linear):
                bound = 1.0 / np.sqrt(m.in_features)
                m.weight.copy_(torch.empty_like(m.weight).uniform_(-bound, bound, generator=gen))
                m.bias.copy_(torch.empty_like(m.bias).uniform_(-bound, bound, generator=gen))
    model = model.to(dev)
    X = torch.tensor(S, dtype=torch.float32, device=dev)
    Y = torch.tensor(y, dtype=torch.float32, device=dev)[:, None]
    opt = torch.optim.Adam(model.parameters(), lr=lr)
    first = last = None
    for _ in range(epochs):
        opt.zero_grad()
        loss = torch.mean((model(X) - Y) ** 2)
        loss.backward()
        opt.step()
        last = float(loss.detach())
        first = last if first is None else first
    l1, l2, l3 = model[0], model[2], model[4]
    w = {"W1": l1.weight, "b1": l1.bias, "W2": l2.weight, "b2": l2.bias, "W3": l3.weight,
         "b3": l3.bias}
    w = {k: v.detach().float().cpu().numpy().astype(np.float32) for k, v in w.items()}
    return w, y, (first, last)


def learned_cost_model(eg, num_solutions: int = 256, seed: int = 0, **kw) -> CostModel:
    """The paper's learned cost: linear u plus an MLP trained as P425 says."""
    S = sample_solutions(eg, num_solutions, seed=seed)
    w, _, _ = train_mlp(S, seed=seed, **kw)
    return CostModel(np.asarray(eg.u, dtype=np.float64), mlp=w)

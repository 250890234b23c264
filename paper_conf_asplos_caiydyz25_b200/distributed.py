"""Multi-GPU driver: seeds shard across ranks (one process per GPU), each rank
holds a full e-graph replica and optimises its own seeds with no data-path
collective (the paper's seed batching).
At the end the ranks agree on the best extraction:

  1. all-gather of the per-rank best (cost, step, global seed, time-to-best)
  2. lexicographic min over ranks (reading S20) -- identical on every rank
  3. broadcast of the winner's choice[M] from its owner rank

With NCCL the tensors live on the rank's GPU (NVLink/NVSwitch); with gloo on
the CPU (tests).  Because theta initialisation is keyed by the global seed
and penalty groups never straddle ranks, every seed's trajectory -- hence the
global best -- is bit-identical for every GPU count.
"""
from __future__ import annotations

import math

import numpy as np


def shard(global_seeds: int, world: int, rank: int):
    """(seed_begin, seeds_per_rank) of this rank; seeds split evenly."""
    if global_seeds % world:
        raise ValueError("global seed count must be divisible by the number of ranks")
    per = global_seeds // world
    return rank * per, per


def reduce_best(records):
    """records: list of (cost, step, seed, time_to_best, rank); lexicographic min
    of (cost, step, seed) over valid records (cost finite)."""
    valid = [r for r in records if math.isfinite(r[0])]
    if not valid:
        return None
    return min(valid, key=lambda r: (r[0], r[1], r[2]))


def global_best(run, dist=None, device=None):
    """Best extraction over all ranks.  Returns a dict with best_cost,
    best_step, best_seed, time_to_best_s, owner and choice (numpy int32 [M])."""
    choice, s = run.extract()
    cost = s["best_cost"] if s["valid"] else math.inf
    if dist is None or not dist.is_initialized() or dist.get_world_size() == 1:
        return {"best_cost": cost, "best_step": s["best_step"], "best_seed": s["best_seed"],
                "time_to_best_s": s["time_to_best_s"], "owner": 0, "choice": choice}
    import torch
    world, rank = dist.get_world_size(), dist.get_rank()
    mine = torch.tensor([cost, float(s["best_step"]), float(s["best_seed"]),
                         float(s["time_to_best_s"]), float(rank)], dtype=torch.float64,
                        device=device)
    bufs = [torch.empty_like(mine) for _ in range(world)]
    dist.all_gather(bufs, mine)
    recs = [tuple(b.cpu().tolist()) for b in bufs]
    win = reduce_best(recs)
    if win is None:
        return {"best_cost": math.inf, "best_step": -1, "best_seed": -1, "time_to_best_s": -1.0,
                "owner": -1, "choice": np.full_like(choice, -1)}
    owner = int(win[4])
    ch = torch.as_tensor(choice.astype(np.int32), device=device)
    dist.broadcast(ch, src=owner)
    return {"best_cost": win[0], "best_step": int(win[1]), "best_seed": int(win[2]),
            "time_to_best_s": win[3], "owner": owner, "choice": ch.cpu().numpy()}

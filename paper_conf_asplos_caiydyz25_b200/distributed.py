"""Multi-GPU driver: seeds shard across ranks (one process per GPU), each rank
holds a full e-graph replica and optimises its own seeds with no data-path
collective (the paper's seed batching).
During the run, termination is global (reading S21: patience counts steps
without improvement of the GLOBAL best): every CHECK_EVERY steps the ranks
all-gather their best (cost, step, seed) and stop together
(optimize_global).  At the end the ranks agree on the best extraction:

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
    if dist is None or not dist.is_initialized():
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


CHECK_EVERY = 8


def _gather_best(run, dist, device, extra=0.0):
    """all-gather of (cost, step, seed, extra, rank) per rank -> list of tuples."""
    s = run.summary()
    cost = s["best_cost"] if s["valid"] else math.inf
    rec = (cost, float(s["best_step"]), float(s["best_seed"]), float(extra))
    if dist is None or not dist.is_initialized():
        return [rec + (0.0,)]
    import torch
    mine = torch.tensor(rec + (float(dist.get_rank()),), dtype=torch.float64, device=device)
    bufs = [torch.empty_like(mine) for _ in range(dist.get_world_size())]
    dist.all_gather(bufs, mine)
    return [tuple(b.cpu().tolist()) for b in bufs]


def optimize_global(run, max_steps, patience=0, time_limit_s=0.0, dist=None, device=None,
                    check_every=CHECK_EVERY, clock=None):
    """Run up to max_steps steps on every rank with GLOBAL termination
    (reading S21): every check_every steps the ranks gather
    their best (cost, step, seed) and their elapsed time; all ranks stop
    together once the global best -- the lexicographic minimum, the same on
    every rank -- is `patience` or more steps old, or the slowest rank has
    used time_limit_s.  The run's own (rank-local) patience must be off.
    Because each seed's trajectory does not depend on the GPU count and the
    checks fall on the same steps, the stop step is the same for every GPU
    count.  Returns (steps_run, global best record or None, stopped_by)."""
    import time
    clock = clock or time.perf_counter
    t0 = clock()
    done, win, why = 0, None, "max_steps"
    while done < max_steps:
        n = min(check_every, max_steps - done)
        run.steps(n)
        done += n
        recs = _gather_best(run, dist, device, extra=clock() - t0)
        win = reduce_best([(r[0], r[1], r[2], r[3], r[4]) for r in recs])
        best_step = int(win[1]) if win is not None else -1
        if patience > 0 and done - (best_step + 1) >= patience:
            why = "patience"
            break
        if time_limit_s > 0 and max(r[3] for r in recs) >= time_limit_s:
            why = "time_limit"
            break
    return done, win, why

"""Multi-GPU driver logic on CPU: world_size-2 gloo process group.

The product path reduces each rank's best (cost, step, global seed) with an
all-gather, picks the lexicographic minimum (reading S20) and broadcasts the
owner's extraction.  Runs are replaced by stubs with fixed results here (the
GPU parts are covered by tests/test_gpu_parity.py::test_seed_sharding_bit_identical).
"""
import math
import os
import socket

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_asplos_caiydyz25_b200.distributed import global_best, reduce_best, shard


class StubRun:
    def __init__(self, cost, step, seed, choice):
        self.s = {"best_cost": cost, "best_step": step, "best_seed": seed, "valid": int(math.isfinite(cost)),
                  "time_to_best_s": 0.5 + step}
        self.c = np.asarray(choice, np.int32)

    def extract(self):
        return self.c.copy(), dict(self.s)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, cases, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    out = []
    for per_rank in cases:
        cost, step, seed, choice = per_rank[rank]
        r = global_best(StubRun(cost, step, seed, choice), dist)
        out.append((r["best_cost"], r["best_step"], r["best_seed"], r["owner"], r["choice"].tolist()))
    q.put((rank, out))
    dist.barrier()
    dist.destroy_process_group()


def test_shard():
    assert shard(1024, 8, 3) == (384, 128)
    with pytest.raises(ValueError):
        shard(100, 8, 0)


def test_reduce_best_lexicographic():
    inf = math.inf
    assert reduce_best([(5.0, 3, 10, 0, 0), (5.0, 2, 99, 0, 1)])[4] == 1      # earlier step wins
    assert reduce_best([(5.0, 2, 40, 0, 0), (5.0, 2, 7, 0, 1)])[4] == 1       # lower seed wins
    assert reduce_best([(4.0, 9, 40, 0, 0), (5.0, 0, 7, 0, 1)])[4] == 0       # cost first
    assert reduce_best([(inf, 0, 0, 0, 0), (inf, 0, 1, 0, 1)]) is None        # nothing valid


def test_global_best_gloo_world2():
    inf = math.inf
    cases = [
        # rank0 (cost, step, seed, choice), rank1 ...
        [(12.0, 4, 3, [0, 5, -1]), (11.0, 9, 70, [0, 6, 7])],     # rank 1 cheaper
        [(11.0, 4, 3, [0, 5, -1]), (11.0, 9, 70, [0, 6, 7])],     # tie on cost: earlier step (rank 0)
        [(inf, -1, -1, [-1, -1, -1]), (30.0, 2, 64, [0, 1, 2])],  # rank 0 found nothing valid
    ]
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, cases, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=120) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert res[0] == res[1]                       # every rank agrees
    (c0, s0, sd0, o0, ch0), (c1, s1, sd1, o1, ch1), (c2, s2, sd2, o2, ch2) = res[0]
    assert (c0, sd0, o0, ch0) == (11.0, 70, 1, [0, 6, 7])
    assert (c1, s1, o1, ch1) == (11.0, 4, 0, [0, 5, -1])
    assert (c2, o2, ch2) == (30.0, 1, [0, 1, 2])


def _bench_dry(gpus):
    import json
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    out = subprocess.run([sys.executable, os.path.join(root, "bench.py"), "--dry-run-cpu",
                          "--gpus", str(gpus), "--ttb-steps", "200", "--patience", "20"],
                         capture_output=True, text=True, timeout=300, cwd=root)
    assert out.returncode == 0, out.stderr[-2000:]
    return json.loads([l for l in out.stdout.splitlines() if l.startswith("{")][-1])


def test_bench_launcher_world2_global_patience():
    """`bench.py --gpus 2` without torchrun re-executes itself with 2 ranks
    (here on gloo, with bench's deterministic stand-in for the GPU run): the
    line reports n_gpus = 2, every rank agrees on the best and its
    extraction, and the ranks stop TOGETHER on the global patience (reading
    S21): rank 0's own seeds stop improving at step 21 (it alone would stop at
    step 48, as the 1-rank run does) but rank 1's keep improving until step
    45, so both run 72 steps."""
    one = _bench_dry(1)
    assert one["n_gpus"] == 1 and one["steps_run"] == 48 and one["stopped_by"] == "patience"
    two = _bench_dry(2)
    assert two["n_gpus"] == 2 and len(two["all_ranks"]) == 2
    keys = ("steps_run", "stopped_by", "best_cost", "best_step", "best_seed", "owner", "choice")
    r0, r1 = two["all_ranks"]
    assert all(r0[k] == r1[k] for k in keys)
    assert (r0["best_seed"], r0["best_step"], r0["owner"], r0["steps_run"]) == (15, 45, 1, 72)
    assert r0["choice"] == [15, 8]          # the owner's extraction, broadcast

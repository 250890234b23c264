"""The NCCL branch of the multi-GPU driver on the one GPU a test box has: a
world-1 NCCL process group runs the real collectives on device tensors --
the every-8-steps all-gather of the global termination (reading S21) and
the all-gather + broadcast of the best extraction -- around a real run, and
must agree with the run's own summary."""
import os
import socket

import numpy as np
import pytest

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_nccl_world1_global_patience_and_best():
    import torch
    import torch.distributed as dist
    import paper_conf_asplos_caiydyz25_b200 as sm
    from gen import make_config
    from paper_conf_asplos_caiydyz25_b200.distributed import global_best, optimize_global
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(_free_port())
    dev = torch.device("cuda", 0)
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=dev)
    try:
        eg = make_config("C2")
        g = sm.load_egraph_from(eg)
        run = sm.run_create(g, sm.CostModel.from_input(eg), 64,
                            sm.Options(penalty_group=8, rng_key=41))
        n, win, why = optimize_global(run, 400, patience=24, dist=dist, device=dev)
        s = run.summary()
        assert why == "patience" and n == s["steps_run"] and n < 400
        # the stop: the first multiple of 8 at least `patience` steps past the best
        assert n - (s["best_step"] + 1) >= 24 and n - 8 - (s["best_step"] + 1) < 24
        best = global_best(run, dist, device=dev)
        choice, s2 = run.extract()
        assert best["owner"] == 0 and best["best_cost"] == s2["best_cost"]
        assert best["best_step"] == s2["best_step"] and best["best_seed"] == s2["best_seed"]
        assert np.array_equal(best["choice"], choice)
        run.close()
        g.close()
    finally:
        dist.destroy_process_group()

"""Where the time goes over a long run (step time is data dependent: as cp
sharpens, the forward rows freeze at other sweeps).

    python scripts/long_run_profile.py [C4] [steps] [window]
Graph-replayed steps, with a profiled window of `window` direct-launch steps
(phase and sweep-kernel CUDA events) every steps/5 steps.  Prints one JSON
line per window.
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_asplos_caiydyz25_b200 as sm  # noqa: E402
from gen import CONFIGS, make_config  # noqa: E402
from gen.configs import rng_key  # noqa: E402


def main():
    name = sys.argv[1] if len(sys.argv) > 1 else "C4"
    steps = int(sys.argv[2]) if len(sys.argv) > 2 else 1000
    win = int(sys.argv[3]) if len(sys.argv) > 3 else 10
    B = int(sys.argv[4]) if len(sys.argv) > 4 else CONFIGS[name]["seeds_per_gpu"]
    spec = CONFIGS[name]
    eg = make_config(name)
    g = sm.load_egraph_from(eg, device=0)
    stream = torch.cuda.Stream()
    torch.cuda.set_stream(stream)
    opts = sm.Options(lam=float(np.mean(eg.u)), penalty_group=spec["group"], rng_key=rng_key(name),
                      cuda_stream=stream.cuda_stream)
    run = sm.run_create(g, sm.CostModel.from_input(eg), B, opts)
    done = 0
    every = max(win, steps // 5)
    while done < steps:
        n = min(every - win, steps - done)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        run.steps(n)
        e1.record(stream)
        torch.cuda.synchronize()
        graph_ms = e0.elapsed_time(e1) / max(1, n)
        done += n
        run.profile(True)
        run.steps(win)
        p = run.get_profile()
        run.profile(False)
        done += win
        s = run.summary()
        print(json.dumps({"config": name, "B": B, "after_step": done, "graph_ms_per_step": graph_ms,
                          "phases": {k: round(v / p["steps"], 3) for k, v in p["phase_ms"].items()},
                          "sweeps": {k: round(v / p["steps"], 3) for k, v in p["sweep_kernel_ms"].items()},
                          "frozen_sweeps_per_step": p["frozen_sweeps"] / p["steps"],
                          "best": s["best_cost"], "best_step": s["best_step"]}), flush=True)


if __name__ == "__main__":
    main()

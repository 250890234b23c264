"""Profiling driver: build a config's run and take a few steps (for ncu).

    python scripts/prof_step.py [C4] [steps]
Direct launches (no CUDA graph) so ncu sees every kernel by name.
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import paper_conf_asplos_caiydyz25_b200 as sm  # noqa: E402
from gen import CONFIGS, make_config  # noqa: E402
from gen.configs import rng_key  # noqa: E402


def main():
    name = sys.argv[1] if len(sys.argv) > 1 else "C4"
    steps = int(sys.argv[2]) if len(sys.argv) > 2 else 2
    spec = CONFIGS[name]
    eg = make_config(name)
    g = sm.load_egraph_from(eg, device=0)
    opts = sm.Options(lam=float(np.mean(eg.u)), penalty_group=spec["group"], rng_key=rng_key(name),
                      use_graphs=False)
    run = sm.run_create(g, sm.CostModel.from_input(eg), spec["seeds_per_gpu"], opts)
    run.steps(steps)
    run.synchronize()
    print(name, "K", run.K, run.extract()[1])


if __name__ == "__main__":
    main()

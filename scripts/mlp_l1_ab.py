"""A/B of the MLP layer-1 kernels: debug_step's f and grad_cp with the TMA
kernel (default) vs the register-staged one (SMOOTHE_MLP_TMA=0), same inputs.

    python scripts/mlp_l1_ab.py [C5] [seeds]
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
    name = sys.argv[1] if len(sys.argv) > 1 else "C5"
    B = int(sys.argv[2]) if len(sys.argv) > 2 else CONFIGS[name]["seeds_per_gpu"]
    spec = CONFIGS[name]
    eg = make_config(name)
    g = sm.load_egraph_from(eg, device=0)
    opts = sm.Options(lam=float(np.mean(eg.u)), penalty_group=spec["group"], rng_key=rng_key(name),
                      use_graphs=False)
    run = sm.run_create(g, sm.CostModel.from_input(eg), B, opts)
    th, m, v, _ = run.state()
    outs = []
    for env in ("1", "0"):
        os.environ["SMOOTHE_MLP_TMA"] = env
        outs.append(run.debug_step(theta=th, m=m, v=v))
    for k in ("f", "grad_cp", "loss"):
        a, b = (np.asarray(o[k], np.float64) for o in outs)
        d = np.abs(a - b) / np.maximum(np.abs(b), 1e-30)
        print(name, B, k, "max rel diff", float(d.max()), "n>1e-5", int((d > 1e-5).sum()), "of", d.size)


if __name__ == "__main__":
    main()

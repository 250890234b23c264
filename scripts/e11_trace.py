"""Relaxed vs sampled cost along the optimisation (Fig. 9;
SURVEY.md 2.5 E11): the library's per-step record (smoothe_run_get_trace) of
a run on the bench workloads.

    python scripts/e11_trace.py [steps] [C3 C4 ...]  -> gpurun_out/e11_<config>.json
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import paper_conf_asplos_caiydyz25_b200 as sm  # noqa: E402
from gen import CONFIGS, make_config  # noqa: E402
from gen.configs import rng_key  # noqa: E402


def main():
    steps = int(sys.argv[1]) if len(sys.argv) > 1 else 300
    names = sys.argv[2:] or ["C2", "C3", "C4", "C5"]
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    for name in names:
        spec = CONFIGS[name]
        eg = make_config(name)
        g = sm.load_egraph_from(eg, device=0)
        run = sm.run_create(g, sm.CostModel.from_input(eg), spec["seeds_per_gpu"],
                            sm.Options(lam=float(np.mean(eg.u)), penalty_group=spec["group"],
                                       rng_key=rng_key(name), lr=0.1))
        run.steps(steps)
        tr = run.trace()
        _, s = run.extract()
        rmin, smin = tr["relaxed_min"], tr["sampled_min"]
        fin = np.isfinite(smin)
        gap = np.abs(smin[fin] - rmin[fin]) / np.maximum(np.abs(smin[fin]), 1e-12)
        out = {"config": name, "steps": steps, "seeds": spec["seeds_per_gpu"],
               "best_cost": s["best_cost"], "best_step": s["best_step"],
               "relative_gap_min_sampled_vs_min_relaxed": {
                   "first": float(gap[0]) if gap.size else None,
                   "median": float(np.median(gap)) if gap.size else None,
                   "last": float(gap[-1]) if gap.size else None},
               "trace": {k: [float(x) for x in v] for k, v in tr.items()}}
        with open(os.path.join(ROOT, "gpurun_out", f"e11_{name}.json"), "w") as fh:
            json.dump(out, fh)
        print(name, "best", s["best_cost"], "at", s["best_step"], "gap", out["relative_gap_min_sampled_vs_min_relaxed"],
              flush=True)
        run.close()
        g.close()


if __name__ == "__main__":
    main()

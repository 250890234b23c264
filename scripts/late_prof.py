"""ncu window on a late step (the step time is data dependent): run N
graph-replayed steps unprofiled, then one direct-launch profiled step inside
cudaProfilerStart / Stop (use ncu --profile-from-start off).

    python scripts/late_prof.py [C4] [N]
"""
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
    n = int(sys.argv[2]) if len(sys.argv) > 2 else 300
    spec = CONFIGS[name]
    eg = make_config(name)
    g = sm.load_egraph_from(eg, device=0)
    stream = torch.cuda.Stream()
    torch.cuda.set_stream(stream)
    opts = sm.Options(lam=float(np.mean(eg.u)), penalty_group=spec["group"], rng_key=rng_key(name),
                      cuda_stream=stream.cuda_stream)
    run = sm.run_create(g, sm.CostModel.from_input(eg), spec["seeds_per_gpu"], opts)
    run.steps(n)
    torch.cuda.synchronize()
    run.profile(True)
    torch.cuda.profiler.start()
    run.steps(1)
    torch.cuda.synchronize()
    torch.cuda.profiler.stop()
    p = run.get_profile()
    print(name, "after", n, "sweeps", {k: round(v, 3) for k, v in p["sweep_kernel_ms"].items()})


if __name__ == "__main__":
    main()

"""Wall-time breakdown of the C-ABI end-to-end path (load, create, steps, extract)."""
import sys
import time

import numpy as np

sys.path.insert(0, ".")
import paper_conf_asplos_caiydyz25_b200 as sm  # noqa: E402
from gen import CONFIGS, make_config  # noqa: E402
from gen.configs import rng_key  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "C4"
steps = int(sys.argv[2]) if len(sys.argv) > 2 else 20
spec = CONFIGS[name]
eg = make_config(name)
import torch  # noqa: E402
torch.cuda.init()
for rep in range(2):
    t0 = time.perf_counter()
    g = sm.load_egraph_from(eg, device=0)
    t1 = time.perf_counter()
    opts = sm.Options(lam=float(np.mean(eg.u)), penalty_group=spec["group"], rng_key=rng_key(name))
    run = sm.run_create(g, sm.CostModel.from_input(eg), spec["seeds_per_gpu"], opts)
    run.synchronize()
    t2 = time.perf_counter()
    run.steps(1)
    run.synchronize()
    t3 = time.perf_counter()
    run.steps(steps - 1)
    run.synchronize()
    t4 = time.perf_counter()
    ch, s = run.extract()
    t5 = time.perf_counter()
    print(f"{name} rep{rep}: load {t1 - t0:.3f}s create {t2 - t1:.3f}s first step {t3 - t2:.3f}s "
          f"{steps - 1} steps {t4 - t3:.3f}s extract {t5 - t4:.3f}s total {t5 - t0:.3f}s")
    run.close()
    g.close()

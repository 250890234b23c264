"""k_wspmv's live-byte roofline on late steps (C4): N graph-replayed steps,
then W profiled (direct-launch) steps whose frozen-sweep kernel times and
device-counted live units give the achieved bandwidth, as bench.py computes
it for its first steps.

    python scripts/late_roofline.py [C4] [N] [W]
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
    n = int(sys.argv[2]) if len(sys.argv) > 2 else 300
    w = int(sys.argv[3]) if len(sys.argv) > 3 else 2
    spec = CONFIGS[name]
    eg = make_config(name)
    g = sm.load_egraph_from(eg, device=0)
    stream = torch.cuda.Stream()
    torch.cuda.set_stream(stream)
    B = spec["seeds_per_gpu"]
    run = sm.run_create(g, sm.CostModel.from_input(eg), B,
                        sm.Options(lam=float(np.mean(eg.u)), penalty_group=spec["group"],
                                   rng_key=rng_key(name), cuda_stream=stream.cuda_stream))
    run.steps(n)
    torch.cuda.synchronize()
    run.profile(True)
    run.steps(w)
    p = run.get_profile()
    run.profile(False)
    peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"]
    nw = max(1, p["frozen_sweeps"])
    le, lr, rw = p["frozen_live_edges"], p["frozen_live_rows"], p["frozen_rows_written"]
    live_bytes = 4.0 * min(128, B) * (le + 3.0 * lr + rw) / nw
    ms = p["sweep_kernel_ms"]["frozen"] / nw
    print(json.dumps({"config": name, "after_step": n, "profiled_steps": w,
                      "working_frozen_launches_per_step": nw / w, "avg_launch_ms": ms,
                      "live_bytes_per_launch": live_bytes,
                      "achieved_gbs": live_bytes / (ms * 1e-3) / 1e9,
                      "frac_of_measured_hbm": live_bytes / (ms * 1e-3) / 1e9 / peak,
                      "sweep_kernel_ms_per_step": {k: v / w for k, v in p["sweep_kernel_ms"].items()}}))


if __name__ == "__main__":
    main()

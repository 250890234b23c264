"""NEXT-1: the large-component penalty path (components above 64 classes) timed.

    python scripts/bench_large_scc.py [p_back ...]
C2-sized graphs with one large strongly connected component (scc_max
unbounded, back-edge probability p_back: 217 / 702 / 1112 classes at 0.06 /
0.1 / 0.15), 64 seeds in penalty groups of 8: graph-replayed step time,
and the per-phase CUDA-event breakdown (direct launches) with the penalty
phase alone.  One JSON line per graph.
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_asplos_caiydyz25_b200 as sm  # noqa: E402
from gen import make_config  # noqa: E402


def main():
    pbs = [float(x) for x in sys.argv[1:]] or [0.06, 0.1, 0.15]
    for pb in pbs:
        eg = make_config("C2", scc_max=10**9, p_back=pb)
        g = sm.load_egraph_from(eg, device=0)
        stream = torch.cuda.Stream()
        torch.cuda.set_stream(stream)
        run = sm.run_create(g, sm.CostModel.from_input(eg), 64,
                            sm.Options(penalty_group=8, rng_key=5, lam=float(np.mean(eg.u)),
                                       cuda_stream=stream.cuda_stream))
        run.steps(3)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        run.steps(10)
        e1.record(stream)
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / 10
        run.profile(True)
        run.steps(5)
        p = run.get_profile()
        run.profile(False)
        ph = {k: v / p["steps"] for k, v in p["phase_ms"].items()}
        n = g.info["scc_max"]
        flops = 8 * 21 * 2.0 * n ** 3   # groups x products (15 Horner + 1 + s ~ 5) x 2 n^3
        print(json.dumps({"p_back": pb, "scc_max": n, "num_scc": g.info["num_scc"],
                          "ms_per_step": ms, "phases_ms": ph,
                          "penalty_gemm_flops_per_step_est": flops,
                          "penalty_tflops_est": flops / (ph["penalty"] * 1e-3) / 1e12}), flush=True)
        run.close()
        g.close()


if __name__ == "__main__":
    main()

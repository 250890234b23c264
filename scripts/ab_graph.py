"""Graph-replay A/B of environment variants in one process (GPU box).

    python scripts/ab_graph.py C4 20 "SMOOTHE_FSKIP=1" "SMOOTHE_FSKIP=0" ...
Each variant creates a fresh run (the library reads its knobs at run
creation), takes 3 warm-up steps and times N graph-replayed steps with CUDA
events; variants alternate over 3 rounds and the median per variant prints.
"""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_asplos_caiydyz25_b200 as sm  # noqa: E402
from gen import CONFIGS, make_config  # noqa: E402
from gen.configs import rng_key  # noqa: E402


def main():
    name, n = sys.argv[1], int(sys.argv[2])
    variants = sys.argv[3:]
    spec = CONFIGS[name]
    eg = make_config(name)
    g = sm.load_egraph_from(eg, device=0)
    res = {v: [] for v in variants}
    stream = torch.cuda.Stream()  # a real stream: handle 0 (legacy default) means none
    for rnd in range(3):
        for v in variants:
            saved = {}
            for kv in v.split(","):
                k, val = kv.split("=")
                saved[k] = os.environ.get(k)
                os.environ[k] = val
            opts = sm.Options(lam=float(np.mean(eg.u)), penalty_group=spec["group"], rng_key=rng_key(name),
                              cuda_stream=stream.cuda_stream)
            run = sm.run_create(g, sm.CostModel.from_input(eg), spec["seeds_per_gpu"], opts)
            run.steps(3)
            run.synchronize()
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            run.steps(n)
            e1.record(stream)
            run.synchronize()
            torch.cuda.synchronize()
            ms = e0.elapsed_time(e1) / n
            res[v].append(ms)
            print(f"round {rnd} {v}: {ms:.3f} ms/step best={run.extract()[1]['best_cost']}", flush=True)
            run.close()
            for k, val in saved.items():
                if val is None:
                    os.environ.pop(k, None)
                else:
                    os.environ[k] = val
    for v in variants:
        print(f"{v:50s} median {np.median(res[v]):.3f} ms/step  all {['%.3f' % x for x in res[v]]}")


if __name__ == "__main__":
    main()

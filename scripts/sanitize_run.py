"""Workload for compute-sanitizer (memcheck / racecheck / initcheck /
synccheck): Fig. 1c and C2 through the C ABI -- graph replay and direct
launches, a debug step, the greedy heuristic -- plus a short C5 run (MLP
cost on tcgen05) and the frozen-sweep path forced on.

    compute-sanitizer --tool memcheck python scripts/sanitize_run.py [small|mlp|frozen]
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import paper_conf_asplos_caiydyz25_b200 as sm  # noqa: E402
from gen import fig1c_fixture, make_config  # noqa: E402


def run(eg, B, G, steps, graphs, **kw):
    g = sm.load_egraph_from(eg, device=0)
    r = sm.run_create(g, sm.CostModel.from_input(eg), B,
                      sm.Options(penalty_group=G, rng_key=9, use_graphs=graphs, **kw))
    r.steps(steps)
    th = r.theta()
    # the q stack / route dumps copy whole version stacks, whose slots hold
    # only the classes recomputed in each sweep (by design), to
    # the host before the versions are resolved: initcheck flags those host
    # copies, so its passes skip these two dumps (SAN_NODUMP=1)
    dump = eg.num_nodes < 10000 and not os.environ.get("SAN_NODUMP")
    r.debug_step(th, qstack=dump, route=dump)
    ch, s = r.extract()
    r.close()
    if eg.u.min() >= 0:
        g.greedy(eg.u)
    g.close()
    print(eg.name, B, "best", s["best_cost"], "graph_mode", s["graph_mode"], flush=True)


def main():
    what = sys.argv[1] if len(sys.argv) > 1 else "small"
    if what == "small":
        run(fig1c_fixture(), 4, 2, 5, True, prop_iters=4)
        run(make_config("C2"), 64, 8, 3, True)
        run(make_config("C2"), 64, 8, 2, False)
        run(make_config("C2"), 33, 3, 2, False, assumption="independent")
    elif what == "mlp":
        eg = make_config("C5")
        run(eg, 64, 8, 1, False)
    elif what == "frozen":
        os.environ["SMOOTHE_REV_W"] = "1"
        run(make_config("C2"), 64, 8, 2, False, prop_iters=60)
        run(make_config("C2"), 64, 8, 2, False, prop_iters=60, converge=True)


if __name__ == "__main__":
    main()

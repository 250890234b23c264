import sys, numpy as np
sys.path.insert(0, '/root/repo'); sys.path.insert(0, '/root/repo/tests')
import paper_conf_asplos_caiydyz25_b200 as sm, oracle as orc
from gen import make_config
from test_gpu_parity import DELTA
eg = make_config("C4"); B, G = 128, 16
g = sm.load_egraph_from(eg)
run = sm.run_create(g, sm.CostModel.from_input(eg), B, sm.Options(penalty_group=G, rng_key=21, use_graphs=True))
run.steps(4); th, m, v, n = run.state(); run.close(); g.close()
g = sm.load_egraph_from(eg)
run = sm.run_create(g, sm.CostModel.from_input(eg), B, sm.Options(lam=1.0, penalty_group=G, lr=0.1, rng_key=3))
d = run.debug_step(th, m, v, step_index=n, route=False)
e, s = 782571, 2
print("theta", th[e, s], "m", m[e, s], "v", v[e, s], "n", n)
for k in ("grad_theta", "grad_cp", "cp", "theta_out", "m_out", "v_out"):
    print("gpu", k, d[k][e, s])
og = orc.Graph(eg)
oo = orc.Options(assumption="hybrid", K=g.K_auto, lam=1.0, G=G, lr=0.1, route_delta=DELTA)
cols = slice(0, 16)
o = og.step(th[:, cols].astype(np.float64), oo, m=m[:, cols], v=v[:, cols], step_index=n, route=False, spread=True)
for k in ("grad_theta", "grad_cp", "cp", "theta_out", "m_out", "v_out", "grad_cp_spread"):
    print("orc", k, o[k][e, s])
u = orc.update(th[:, cols].astype(np.float64), d["grad_theta"][:, cols].astype(np.float64), oo, m=m[:, cols], v=v[:, cols], step_index=n)
print("orc update given gpu grad", u["theta_out"][e, s], u["m_out"][e, s], u["v_out"][e, s])
# the class of e
cp_ = np.asarray(eg.class_ptr) if hasattr(eg, 'class_ptr') else None

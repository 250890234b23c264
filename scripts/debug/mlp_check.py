"""Debug: MLP layer-1 accuracy on the GPU vs fp64 (f = f_mlp only, u = 0)."""
import os, sys
import numpy as np
ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
import paper_conf_asplos_caiydyz25_b200 as sm
import oracle
from gen import make_config

eg = make_config("C5")
eg.u = np.zeros_like(eg.u)
for B in (32, 64, 128):
    g = sm.load_egraph_from(eg, device=0)
    run = sm.run_create(g, sm.CostModel.from_input(eg), B, sm.Options(penalty_group=8, rng_key=3))
    theta = np.random.default_rng(1).uniform(-2, 2, (eg.num_nodes, B)).astype(np.float32)
    d = run.debug_step(theta, None, None, step_index=0, route=False)
    p = d["p"].astype(np.float64)
    W1 = eg.mlp["W1"].astype(np.float64); b1 = eg.mlp["b1"].astype(np.float64)
    W2 = eg.mlp["W2"].astype(np.float64); b2 = eg.mlp["b2"].astype(np.float64)
    W3 = eg.mlp["W3"].astype(np.float64); b3 = eg.mlp["b3"].astype(np.float64)
    z1 = W1 @ p + b1[:, None]
    z2 = W2 @ np.maximum(z1, 0) + b2[:, None]
    f = (W3 @ np.maximum(z2, 0) + b3[:, None])[0]
    err = np.abs(d["f"] - f)
    print(B, "f_mlp max abs err", err.max(), "rel", (err / np.maximum(np.abs(f), 1e-30)).max(),
          "min |z1|", np.abs(z1).min(), "typ |z1|", np.median(np.abs(z1)))
    run.close(); g.close()

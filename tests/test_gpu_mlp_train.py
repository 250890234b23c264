"""Learned MLP cost: random valid solutions from the library's
decode, random negative targets, regression; the trained model is then a
smoothe_cost_model whose decoded cost matches the MLP written out in fp64."""
import numpy as np
import pytest

from gen import make_config

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def sm():
    import torch
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    import paper_conf_asplos_caiydyz25_b200 as pkg
    pkg.lib()
    return pkg


def mlp64(w, s):
    z1 = np.maximum(w["W1"].astype(np.float64) @ s + w["b1"], 0.0)
    z2 = np.maximum(w["W2"].astype(np.float64) @ z1 + w["b2"], 0.0)
    return float((w["W3"].astype(np.float64) @ z2 + w["b3"])[0])


def test_learned_mlp_cost(sm):
    from paper_conf_asplos_caiydyz25_b200 import mlp_train
    eg = make_config("C2")
    S = mlp_train.sample_solutions(eg, 128, seed=1)
    assert S.shape == (128, eg.num_nodes)
    ec = eg.ec()
    for s in S[:8]:  # one e-node per selected class, the root selected
        sel = ec[s > 0]
        assert len(np.unique(sel)) == len(sel) and eg.root in sel
    w, y, (first, last) = mlp_train.train_mlp(S, seed=1, epochs=400)
    assert np.all(y <= 0) and last < 0.1 * first
    # decode the first solution through the library with the trained cost
    cm = sm.CostModel(eg.u, mlp=w)
    g = sm.load_egraph_from(eg)
    run = sm.run_create(g, cm, 32, sm.Options(penalty_group=8))
    th = np.random.default_rng(0).uniform(-1, 1, (eg.num_nodes, 32)).astype(np.float32)
    th[S[0] > 0, :] += 3.0
    d = run.debug_step(th)
    assert d["valid"][0] == 1
    ref = float(eg.u @ S[0]) + mlp64(w, S[0].astype(np.float64))
    assert abs(d["disc_cost"][0] - ref) <= 1e-4 * abs(ref) + 1e-3
    run.steps(20)
    _, s = run.extract()
    assert s["valid"] == 1
    run.close()
    g.close()

"""GPU path (libsmoothe.so through its C ABI) vs the fp64 oracle, element by
element on the same seeded inputs (SURVEY.md 8(c) parity protocol).  The
oracle takes every decision itself; no GPU array is ever an oracle input.

Bars (BASELINE.json north_star):
* bit-exact: theta initialisation, decoded choices, reached sets, validity,
  integer discrete costs (linear / quadratic with integer u, w);
* |gpu - ref| <= 1e-6 + 1e-4 |ref| for cp, q^K, p, f, h, loss, g_cp;
* g_theta = cp (g_cp - sum cp g_cp) cancels by construction, so its bound is
  1e-6 + 1e-4 * (magnitude of the terms combined): cp (|g_cp| + sum cp |g_cp|);
* theta', m', v' from the oracle's own step, with the g_theta bound carried
  through the optimiser (the oracle's update at g_ref -/+ bound), and the
  update alone given the GPU's gradient at 2e-5;
* max routing (reading S7'): the champion scan is an fp32 decision on the GPU
  and an fp64 one in the oracle.  Where a comparison of the oracle's scan is
  within DELTA (relative) of its threshold -- above the fp32-vs-fp64 error of
  p -- both outcomes are admissible: the oracle marks the decision and bounds,
  element by element, how far g_cp can move over every admissible routing
  (grad_cp_spread, an interval reverse pass; pinned in test_oracle_pins.py);
  the bar on g_cp / g_theta / theta' is widened by that bound and nowhere
  else.  Every other decision must route identically.  No seed is left out,
  and no GPU output is ever an oracle input.
For every comparison the fraction of elements inside the PLAIN bar
(1e-6 + 1e-4 |ref|) and the worst |gpu - ref| / (1e-6 + 1e-4 |ref|) are
logged to $SMOOTHE_PARITY_LOG (JSON lines) when set.
"""
import json
import os

import numpy as np
import pytest

from gen import CONFIGS, fig1c_fixture, make_config, random_tiny

pytestmark = pytest.mark.gpu

AGGS = ["independent", "correlated", "hybrid"]
RTOL, ATOL = 1e-4, 1e-6
# routing decisions closer than DELTA (relative) to the scan threshold may
# legitimately go either way in fp32 vs fp64 (reading S7')
DELTA = 1e-5


@pytest.fixture(scope="module")
def sm():
    import torch
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    import paper_conf_asplos_caiydyz25_b200 as pkg
    pkg.lib()
    return pkg


def log_stats(rec):
    path = os.environ.get("SMOOTHE_PARITY_LOG")
    if path:
        with open(path, "a") as fh:
            fh.write(json.dumps(rec) + "\n")


def plain_stats(got, ref):
    got = np.asarray(got, dtype=np.float64)
    ref = np.asarray(ref, dtype=np.float64)
    if ref.size == 0:
        return {"n": 0}
    r = np.abs(got - ref) / (ATOL + RTOL * np.abs(ref))
    return {"n": int(ref.size), "plain_pass": float(np.mean(r <= 1)), "worst_ratio": float(r.max())}


def close(name, got, ref, scale=None, rtol=RTOL, atol=ATOL, stats=None):
    got = np.asarray(got, dtype=np.float64)
    ref = np.asarray(ref, dtype=np.float64)
    if stats is not None:
        stats[name] = plain_stats(got, ref)
    scale = np.abs(ref) if scale is None else scale
    err = np.abs(got - ref) - (atol + rtol * scale)
    bad = np.argwhere(err > 0)
    assert bad.size == 0, (f"{name}: {len(bad)} of {ref.size} outside tolerance; first "
                           f"{bad[:3].tolist()} got {got[tuple(bad[0])]} ref {ref[tuple(bad[0])]}")


def class_sums(eg, x):
    """sum over the e-nodes of each class, broadcast back to the e-nodes."""
    ec = eg.ec()
    out = np.zeros((eg.num_classes,) + x.shape[1:])
    np.add.at(out, ec, x)
    return out[ec]


def route_mask(eg):
    """classes whose route is a decision: not the root, at least two parents."""
    npar = np.zeros(eg.num_classes, np.int64)
    for k in range(eg.num_nodes):
        for c in set(eg.child_class[eg.child_ptr[k]:eg.child_ptr[k + 1]].tolist()):
            npar[c] += 1
    m = npar >= 2
    m[eg.root] = False
    return m


def grad_scales(og, eg, th, oo, o, **kw):
    """|g_cp| scale; for the quadratic cost, whose negative pair weights make
    g_p = u + sum_k w p_k cancel, the same backward with |w| (the reverse mode
    is linear in g_p with non-negative coefficients)."""
    gco = o["grad_cp"]
    if eg.quad is not None:
        qi, qj, qw = eg.quad
        eg.quad = (qi, qj, np.abs(qw))
        oa = og.__class__(eg).step(th, oo, **kw)
        eg.quad = (qi, qj, qw)
        gco = np.maximum(np.abs(gco), np.abs(oa["grad_cp"]))
    return np.abs(gco)


def compare_step(sm, orc, eg, B, G, agg="hybrid", lam=1.0, theta=None, m=None, v=None,
                 step_index=0, K=-1, seed=0, cols=None, lr=0.1, label=None, routes=None):
    g = sm.load_egraph_from(eg, device=0)
    Kr = g.K_auto if K < 0 else K
    opts = sm.Options(assumption=agg, prop_iters=K, lam=lam, penalty_group=G, lr=lr, rng_key=3)
    run = sm.run_create(g, sm.CostModel.from_input(eg), B, opts)
    rng = np.random.default_rng(seed)
    if theta is None:
        theta = rng.uniform(-2, 2, (eg.num_nodes, B)).astype(np.float32)
    if routes is None:   # the route arrays are [K][M][B]: skip them on big graphs
        routes = Kr * eg.num_classes * B <= 4e7
    d = run.debug_step(theta, m, v, step_index=step_index, route=routes)
    cols = slice(None) if cols is None else cols
    th = theta[:, cols].astype(np.float64)
    og = orc.Graph(eg)
    assert og.K_auto == g.K_auto
    oo = orc.Options(assumption=agg, K=Kr, lam=lam, G=G, lr=lr, route_delta=DELTA)
    mo = None if m is None else m[:, cols]
    vo = None if v is None else v[:, cols]
    o = og.step(th, oo, m=mo, v=vo, step_index=step_index, route=routes, spread=True)
    sel = lambda a: a[:, cols]
    st = {}
    close("cp", sel(d["cp"]), o["cp"], stats=st)
    close("p", sel(d["p"]), o["p"], stats=st)
    close("f", d["f"][cols], o["f"], stats=st)
    nb = th.shape[1]
    close("h", d["h"][: nb // G], o["h"], stats=st)            # cols always start at seed 0
    # decode: bit-exact for every seed (no routing involved)
    assert np.array_equal(sel(d["choice"]), o["choice"])
    assert np.array_equal(sel(d["reached"]), o["reached"])
    assert np.array_equal(d["valid"][cols], o["valid"])
    ok = o["valid"] == 1
    if eg.mlp is None:
        assert np.array_equal(d["disc_cost"][cols][ok], o["disc_cost"][ok])
    else:
        close("disc_cost", d["disc_cost"][cols][ok], o["disc_cost"][ok])
    assert np.all(np.isinf(d["disc_cost"][cols][~ok]))
    # routing: identical wherever the oracle's scan is not within DELTA
    if routes and agg != "independent":
        rm = route_mask(eg)
        gr, orr = d["route"][:, :, cols][:, rm], o["route"][:, rm]
        firm = orr >= 0
        assert np.array_equal(gr[firm], orr[firm]), (
            f"{int((gr[firm] != orr[firm]).sum())} routes differ from the oracle's S7' scan")
        amb = orr <= -2
        st["route_near_threshold_decisions"] = int(amb.sum())
    sp = o["grad_cp_spread"]
    gsc = grad_scales(og, eg, th, oo, o, m=mo, v=vo, step_index=step_index)
    close("grad_cp", sel(d["grad_cp"]), o["grad_cp"], scale=gsc,
          atol=ATOL + sp, stats=st)
    cpo = o["cp"]
    gscale = cpo * (gsc + class_sums(eg, cpo * gsc))
    gspread = cpo * (sp + class_sums(eg, cpo * sp))
    close("grad_theta", sel(d["grad_theta"]), o["grad_theta"],
          scale=gscale, atol=ATOL + gspread, stats=st)
    # the optimiser: from the oracle's own step, the g_theta bound carried
    # through the update (the oracle's update at g -/+ bound) ...
    # The image of the interval [g - eb, g + eb] under the update is not
    # spanned by its end points: Adam's m'/sqrt(v') peaks inside at
    # g* = (1 - b1) b2 v / (b1 (1 - b2) m), and v' is smallest at g = 0
    # (DESIGN.md 5), so those points count too where they lie inside.
    eb = ATOL + RTOL * gscale + gspread
    g0 = o["grad_theta"]
    cands = [g0 - eb, g0 + eb]
    if mo is not None and vo is not None:
        b1, b2 = oo.beta1, oo.beta2
        m64, v64 = mo.astype(np.float64), vo.astype(np.float64)
        with np.errstate(divide="ignore", invalid="ignore"):
            gst = (1 - b1) * b2 * v64 / (b1 * (1 - b2) * m64)
        inside = np.isfinite(gst) & (np.abs(gst - g0) < eb)
        cands.append(np.where(inside, gst, g0))
    cands.append(np.where(np.abs(g0) < eb, 0.0, g0))
    ups = [orc.update(th, c, oo, m=mo, v=vo, step_index=step_index) for c in cands]
    for k in ("theta_out", "m_out", "v_out"):
        spread = np.max([np.abs(u_[k] - o[k]) for u_ in ups], axis=0)
        close(k, sel(d[k]), o[k], scale=np.abs(o[k]),
              atol=ATOL + spread, stats=st)
    # ... and the update alone given the GPU's gradient (no oracle step involved)
    # (scales: the magnitudes of the terms each output sums, as m' = b1 m +
    # (1 - b1) g cancels when m and g have opposite signs)
    gg = sel(d["grad_theta"]).astype(np.float64)
    u = orc.update(th, gg, oo, m=mo, v=vo, step_index=step_index)
    m0 = np.zeros_like(th) if mo is None else np.abs(mo.astype(np.float64))
    usc = {"m_out": oo.beta1 * m0 + (1 - oo.beta1) * np.abs(gg), "v_out": np.abs(u["v_out"]),
           "theta_out": np.abs(th) + np.abs(u["theta_out"] - th)}
    for k in ("theta_out", "m_out", "v_out"):
        close(k + "|gpu_grad", sel(d[k]), u[k], scale=usc[k], rtol=2e-5, atol=1e-6)
    st["near_threshold_decisions_per_seed"] = {"max": int(o["route_namb"].max()),
                                               "mean": float(o["route_namb"].mean())}
    st["grad_cp_widened_elements"] = float(np.mean(sp > 0))
    st["grad_cp_widened_past_bar"] = float(np.mean(sp > ATOL + RTOL * gsc))
    if cols == slice(None):
        close("loss", d["loss"], o["loss"], stats=st)
    log_stats({"test": label or eg.name, "B": nb, "K": Kr, "agg": agg,
               "min_route_margin": float(np.min(o["route_margin"])),
               **st})
    run.close()
    g.close()
    return d, o


def test_theta_init_bitexact(sm, orc):
    eg = make_config("C2")
    g = sm.load_egraph_from(eg)
    run = sm.run_create(g, sm.CostModel.from_input(eg), 96,
                        sm.Options(rng_key=0x5EED0002, seed_begin=5, penalty_group=8))
    th = run.theta()
    ref = orc.theta_init(0x5EED0002, 5, 96, eg.num_nodes)
    assert np.array_equal(th.astype(np.float64), ref)


@pytest.mark.parametrize("agg", AGGS)
def test_fig1c_step(sm, orc, agg):
    eg = fig1c_fixture()
    rng = np.random.default_rng(1)
    th = rng.uniform(-1, 1, (10, 4)).astype(np.float32)
    d, o = compare_step(sm, orc, eg, 4, 2, agg, theta=th)
    # the paper's closed form on the GPU path too
    c1, c4 = d["cp"][1], d["cp"][4]
    assert np.allclose(d["f"], 19 + 13 * c1 - 5 * c1 * c4, rtol=1e-6)


@pytest.mark.parametrize("agg", AGGS)
@pytest.mark.parametrize("kind", ["tree", "dag", "cyclic"])
def test_tiny_families(sm, orc, agg, kind):
    for s in range(6):
        eg = random_tiny(3000 + s, kind, num_classes=8)
        # B = 33: ragged (padded to 64 internally), 11 penalty groups of 3
        compare_step(sm, orc, eg, 33, 3, agg, lam=0.7, seed=s, K=3 + s % 4)


def converge_envelope(orc, og, eg, th, agg, K, lam, d, b, t_gpu, label):
    """Convergence mode (reading S1b) for seed b without GPU decisions in the
    oracle: the stopping sweep is an fp32 event (no q row of the seed changes
    bitwise).  From the oracle's own fixed-K q stack, t_lo = the first sweep
    whose largest relative row change is <= 2^-20 (16 fp32 ulps; a larger
    change cannot vanish in fp32), so fp32 may stop anywhere in [t_lo, K].
    The GPU's sweep count must lie there, and its p and g_cp must lie in the
    envelope of the oracle's own steps with K' = t_lo..K sweeps, widened by
    the parity bar and, for g_cp, the oracle's routing bound (compare_step)."""
    th = th[:, [b]].astype(np.float64)
    full = og.step(th, orc.Options(assumption=agg, K=K, lam=lam, G=1), qstack=True)
    q = full["qstack"][:, :, 0]
    dq = np.abs(q[1:] - q[:-1]) / np.maximum(np.abs(q[1:]), 1e-300)
    dq[:, (q[1:] == 0).all(axis=0)] = 0.0
    r = dq.max(axis=1)                       # r[t-1]: sweep t
    small = np.where(r <= 2.0 ** -20)[0]
    t_lo = int(small[0]) + 1 if small.size else K
    assert t_lo <= t_gpu <= K, (b, t_lo, t_gpu, K)
    outs = [og.step(th, orc.Options(assumption=agg, K=t, lam=lam, G=1, route_delta=DELTA), spread=True)
            for t in range(t_lo, K + 1)]
    gsc = np.abs(np.stack([o["grad_cp"] for o in outs])).max(axis=0)
    sp = np.stack([o["grad_cp_spread"] for o in outs]).max(axis=0)   # routing (reading S7')
    if eg.quad is not None:
        gsc = np.maximum(gsc, grad_scales(og, eg, th, orc.Options(assumption=agg, K=K, lam=lam, G=1), full))
    st = {}
    for key, scale in (("p", None), ("grad_cp", gsc)):
        ref = np.stack([o[key] for o in outs])
        lo, hi = ref.min(axis=0), ref.max(axis=0)
        got = d[key][:, [b]].astype(np.float64)
        sc = np.maximum(np.abs(lo), np.abs(hi)) if scale is None else scale
        tol = ATOL + RTOL * sc + (sp if key == "grad_cp" else 0.0)
        bad = np.argwhere((got < lo - tol) | (got > hi + tol))
        assert bad.size == 0, f"{label} seed {b} {key}: {len(bad)} outside the oracle envelope"
        st[key] = {"envelope_width_rel": float((np.abs(hi - lo) / (tol)).max())}
    log_stats({"test": label, "seed": int(b), "t_lo": t_lo, "t_gpu": int(t_gpu), "K": K, **st})


@pytest.mark.parametrize("agg", AGGS)
def test_tiny_frozen_and_converge(sm, orc, monkeypatch, agg):
    """Tiny cyclic graphs with K well past the freezing point: the frozen-sweep
    path forced on (ragged B = 33, groups of 3), and the convergence mode per
    seed (G = 1) against the oracle's envelope (converge_envelope)."""
    monkeypatch.setenv("SMOOTHE_REV_W", "1")
    for s in range(6):
        eg = random_tiny(3100 + s, "cyclic", num_classes=8)
        compare_step(sm, orc, eg, 33, 3, agg, lam=0.7, seed=s, K=12 + s, label=f"tiny_frozen_{agg}")
        g = sm.load_egraph_from(eg)
        run = sm.run_create(g, sm.CostModel.from_input(eg), 16,
                            sm.Options(assumption=agg, prop_iters=12 + s, lam=0.7,
                                       penalty_group=1, converge=True))
        th = np.random.default_rng(s).uniform(-2, 2, (eg.num_nodes, 16)).astype(np.float32)
        d = run.debug_step(th)
        og = orc.Graph(eg)
        for b in range(16):
            converge_envelope(orc, og, eg, th, agg, 12 + s, 0.7, d, b, int(d["sweeps"][b]),
                              f"tiny_converge_{agg}")
        run.close()
        g.close()


@pytest.mark.parametrize("B,agg,K", [(32, "hybrid", -1), (64, "independent", 12),
                                     (64, "correlated", 12), (256, "hybrid", 12)])
def test_long_lists_split_items(sm, orc, B, agg, K):
    """Classes of > 16 batches of 4 children and e-nodes of > 64 children: the
    reverse sweep splits them over several warps (HostGraph::rev_item) and
    combines the partial sums; every width V = 1, 2, 4 (two seed slices at
    256) and aggregator."""
    eg = random_tiny(3300, "dag", num_classes=200, max_class_size=40, max_children=150)
    assert np.diff(eg.child_ptr).max() > 64
    compare_step(sm, orc, eg, B, 8, agg, K=K)


def test_tiny_second_adam_step(sm, orc):
    eg = random_tiny(3100, "cyclic")
    rng = np.random.default_rng(2)
    B = 8
    m = rng.normal(0, 0.1, (eg.num_nodes, B)).astype(np.float32)
    v = rng.uniform(0, 0.05, (eg.num_nodes, B)).astype(np.float32)
    compare_step(sm, orc, eg, B, 4, m=m, v=v, step_index=6)


def test_one_hot_and_ties(sm, orc):
    """Degenerate inputs: one-hot logits (cp in {0,1}, q = 1 exactly, zero
    factors in the product), exact logit ties (lowest id wins)."""
    eg = random_tiny(3200, "cyclic", num_classes=8)
    rng = np.random.default_rng(3)
    B = 32
    th = np.zeros((eg.num_nodes, B), np.float32)
    ec = eg.ec()
    for j in range(eg.num_classes):
        idx = np.where(ec == j)[0]
        for b in range(B):
            if b % 3 == 0:
                th[rng.choice(idx), b] = 1e4      # one-hot
            elif b % 3 == 1:
                th[idx, b] = 0.25                 # all tied
            else:
                th[idx, b] = rng.uniform(-1, 1, idx.size)
    compare_step(sm, orc, eg, B, 4, theta=th, lam=0.5)


@pytest.mark.parametrize("B,G", [(64, 8), (100, 10), (200, 8)])
def test_c2_full(sm, orc, B, G):
    compare_step(sm, orc, make_config("C2"), B, G, seed=B)


@pytest.mark.parametrize("agg", ["independent", "correlated"])
def test_c2_aggregators(sm, orc, agg):
    compare_step(sm, orc, make_config("C2"), 64, 8, agg, seed=5)


@pytest.mark.parametrize("p_back,G,fp64", [(0.06, 8, "0"), (0.1, 8, "0"), (0.15, 16, "0"),
                                           (0.06, 1, "0"), (0.1, 8, "1")])
def test_large_scc(sm, orc, monkeypatch, p_back, G, fp64):
    """Components larger than 64 classes (217 / 702 / 1112 classes): the
    global-memory penalty path (tcgen05 3xTF32 GEMMs by default, the fp64
    CUDA-core GEMMs with SMOOTHE_BIG_FP64=1) and the block-wide decode
    closures.  The first half of the seeds favour the anchor e-nodes (children
    strictly deeper: a valid extraction), so both verdicts occur.  G = 1 is the
    exact per-seed penalty (no Eq. 11 averaging)."""
    monkeypatch.setenv("SMOOTHE_BIG_FP64", fp64)
    eg = make_config("C2", scc_max=10**9, p_back=p_back)
    assert eg.meta["scc_max"] > 64
    B = 64
    rng = np.random.default_rng(11)
    theta = rng.uniform(-2, 2, (eg.num_nodes, B)).astype(np.float32)
    # anchors just above every other logit (U(-2, 2)): the arg-max without
    # pushing cp towards 1, where 1 - p in fp32 loses the relative accuracy
    # the parity bar asks of the independence derivatives
    theta[eg.class_ptr[:-1], : B // 2] = 2.05
    d, o = compare_step(sm, orc, eg, B, G, theta=theta)
    assert o["valid"][: B // 2].all() and not o["valid"].all()
    assert np.all(o["h"] > 0)


@pytest.mark.parametrize("name,B,G,K,agg", [("C2", 64, 8, 80, "hybrid"),
                                             ("C2", 100, 10, 80, "hybrid"),
                                             ("C2", 200, 8, 70, "hybrid"),
                                             ("C2", 64, 8, 80, "independent"),
                                             ("C2", 64, 8, 80, "correlated"),
                                             ("C3", 32, 8, 60, "hybrid")])
def test_frozen_sweeps_parity(sm, orc, monkeypatch, name, B, G, K, agg):
    """The frozen reverse sweeps (W = class-level coefficients of the K-state,
    deferred g_cp pass) forced on with K beyond the
    freezing point: the step still matches the fp64 oracle."""
    monkeypatch.setenv("SMOOTHE_REV_W", "1")
    compare_step(sm, orc, make_config(name), B, G, agg, K=K, seed=B + K)


@pytest.mark.parametrize("name,B,K,agg,wpath", [("C2", 64, 80, "hybrid", "1"),
                                                ("C2", 32, 80, "independent", "1"),
                                                ("C5", 64, 57, "hybrid", "1"),
                                                ("C2", 64, 80, "hybrid", "0"),
                                                ("C2", 100, 40, "correlated", "0"),
                                                ("C3", 32, 60, "hybrid", "0")])
def test_converge_mode_parity(sm, orc, monkeypatch, name, B, K, agg, wpath):
    """Reading S1b ("repeat until convergence", P215): each seed's step stops
    at its first sweep that changes none of its q rows (an fp32 event), and
    the reverse mode runs the sweeps performed.  Checked per sampled seed
    against the oracle's own envelope (converge_envelope).  wpath: the
    converged seeds' pass-through runs in the frozen-sweep kernels ("1") or
    in the reverse kernel ("0")."""
    monkeypatch.setenv("SMOOTHE_REV_W", wpath)
    eg = make_config(name)
    g = sm.load_egraph_from(eg)
    opts = sm.Options(assumption=agg, prop_iters=K, lam=1.0, penalty_group=1, rng_key=3,
                      converge=True)
    run = sm.run_create(g, sm.CostModel.from_input(eg), B, opts)
    theta = np.random.default_rng(K + B).uniform(-2, 2, (eg.num_nodes, B)).astype(np.float32)
    d = run.debug_step(theta)
    sw = d["sweeps"]
    assert np.all((sw >= 1) & (sw <= K)), sw
    if name == "C2":
        assert np.median(sw) < K, sw  # most seeds converged
    og = orc.Graph(eg)
    for b in list(range(0, B, max(1, B // (8 if name == "C2" else 3)))):
        close(f"cp[{b}]", d["cp"][:, [b]], og.step(theta[:, [b]].astype(np.float64),
                                                    orc.Options(assumption=agg, K=1, G=1))["cp"])
        converge_envelope(orc, og, eg, theta, agg, K, 1.0, d, b, int(sw[b]),
                          f"converge_{name}_{agg}_w{wpath}")
    run.close()
    g.close()


def test_c3_quadratic_full(sm, orc):
    spec = CONFIGS["C3"]
    compare_step(sm, orc, make_config("C3"), spec["seeds_per_gpu"], spec["group"], seed=3)


def test_c5_mlp_full(sm, orc):
    spec = CONFIGS["C5"]
    compare_step(sm, orc, make_config("C5"), spec["seeds_per_gpu"], spec["group"], seed=4)


@pytest.mark.parametrize("B", [32, 64, 128, 256])
def test_mlp_layer1_tensor_cores(sm, B):
    """The tcgen05 layer-1 contraction (hi/lo TF32 split) at every seed-chunk
    width: with u = 0 the step's f is f_mlp alone, checked against the MLP in
    fp64 applied to the GPU's own p (1e-4 relative; measured ~4e-6).  C5's
    e-node count leaves the last split-K CTA without e-nodes, which must
    contribute zeros."""
    eg = make_config("C5")
    eg.u = np.zeros_like(eg.u)
    g = sm.load_egraph_from(eg, device=0)
    run = sm.run_create(g, sm.CostModel.from_input(eg), B, sm.Options(penalty_group=8, rng_key=3))
    theta = np.random.default_rng(B).uniform(-2, 2, (eg.num_nodes, B)).astype(np.float32)
    d = run.debug_step(theta, None, None, step_index=0)
    p = d["p"].astype(np.float64)
    w = {k: v.astype(np.float64) for k, v in eg.mlp.items()}
    z1 = w["W1"] @ p + w["b1"][:, None]
    z2 = w["W2"] @ np.maximum(z1, 0) + w["b2"][:, None]
    f = (w["W3"] @ np.maximum(z2, 0) + w["b3"][:, None])[0]
    close("f_mlp", d["f"], f, scale=np.abs(f) + (np.abs(w["W3"]) @ np.abs(np.maximum(z2, 0)))[0])
    run.close()
    g.close()


@pytest.mark.parametrize("N,B", [(300_000, 32), (300_000, 64), (300_000, 128), (7_777, 64),
                                 (1_000, 256)])
def test_mlp_l1_tma_bit_identical(sm, monkeypatch, N, B):
    """The TMA layer-1 kernel (default) against the register-staged one
    (SMOOTHE_MLP_TMA=0): the same products (the MMA truncates the raw W1 / p
    tiles to tf32 exactly as the register kernel's explicit split does) summed
    in the same order, so f and the gradient of a debug step are bit for bit
    equal -- at C5's size and on a ragged e-node count (7 777: last
    32-e-node tile partial).  On 1 000 e-nodes (most split-K CTAs without a
    tile) the two kernels split K into 32- and 64-e-node ranges, so the
    partial sums differ in order: equal to fp32 rounding there."""
    eg = make_config("C5") if N == 300_000 else make_config("C5", N=N, M=max(N // 18, 8))
    g = sm.load_egraph_from(eg, device=0)
    run = sm.run_create(g, sm.CostModel.from_input(eg), B, sm.Options(penalty_group=8, rng_key=5))
    run.steps(2)
    th, m, v, n = run.state()
    outs = []
    for env in ("1", "0"):
        monkeypatch.setenv("SMOOTHE_MLP_TMA", env)
        outs.append(run.debug_step(th, m, v, step_index=n))
    for k in ("f", "grad_cp", "loss", "theta_out"):
        a, b = np.asarray(outs[0][k], np.float64), np.asarray(outs[1][k], np.float64)
        if N == 1_000:
            assert np.allclose(a, b, rtol=1e-5, atol=1e-6 * np.abs(b).max()), k
        else:
            assert np.array_equal(a, b), k
    run.close()
    g.close()


def test_c4_full_size_first_group(sm, orc):
    """C4 at the bench launch configuration (128 seeds, G = 16): the oracle
    recomputes the first penalty group (16 seeds) exactly."""
    spec = CONFIGS["C4"]
    B, G = spec["seeds_per_gpu"], spec["group"]
    compare_step(sm, orc, make_config("C4"), B, G, seed=6, cols=slice(0, G))


@pytest.mark.parametrize("name,B,G", [("C3", 256, 8), ("C5", 512, 8)])
def test_single_gpu_batches(sm, orc, name, B, G):
    """The 8(d) P = 1 seed batches that fit the oracle's time: C3 with all
    256 seeds, C5 with 512 seeds on the GPU (the oracle recomputes the first
    64, eight penalty groups)."""
    cols = None if B <= 256 else slice(0, 64)
    compare_step(sm, orc, make_config(name), B, G, seed=B + 1, cols=cols, label=f"{name}_B{B}")


@pytest.mark.parametrize("name,B,G,steps,cols", [("C2", 64, 8, 7, None), ("C4", 32, 16, 3, slice(0, 16)),
                                                 ("C4", 128, 16, 4, slice(0, 16))])
def test_debug_step_after_graph_replay(sm, orc, name, B, G, steps, cols):
    """Parity from state produced by the timed path: steps replayed from the
    captured CUDA graph (graph_mode 1; on C4 the forward and reverse sweeps
    gated by conditional / switch nodes, persistent k_wspmv and plain sweep;
    128 seeds is the bench's launch configuration), then a debug step from
    that theta / m / v (Adam step steps + 1) against the oracle."""
    eg = make_config(name)
    g = sm.load_egraph_from(eg)
    run = sm.run_create(g, sm.CostModel.from_input(eg), B,
                        sm.Options(penalty_group=G, rng_key=21, use_graphs=True))
    run.steps(steps)
    th, m, v, n = run.state()
    assert n == steps
    assert run.extract()[1]["graph_mode"] == 1
    run.close()
    g.close()
    compare_step(sm, orc, eg, B, G, theta=th, m=m, v=v, step_index=n, cols=cols,
                 label=f"{name}_after_graph_replay")


@pytest.mark.parametrize("B", [32, 128])
def test_c4_graph_replay_and_direct_launches_identical(sm, B):
    """The benchmarked C4 path (CUDA-graph replay with the sweeps gated by
    conditional / switch nodes) against direct launches (every kernel of
    every sweep launched): theta after 3 steps and the best extraction bit
    for bit."""
    eg = make_config("C4")
    outs = []
    for use_graphs in (True, False):
        g = sm.load_egraph_from(eg)
        run = sm.run_create(g, sm.CostModel.from_input(eg), B,
                            sm.Options(penalty_group=16, rng_key=0x5EED0004, use_graphs=use_graphs))
        run.steps(3)
        ch, s = run.extract()
        assert s["graph_mode"] == (1 if use_graphs else 0)
        outs.append((run.theta(), ch, s))
        run.close()
        g.close()
    assert np.array_equal(outs[0][0], outs[1][0])
    assert np.array_equal(outs[0][1], outs[1][1])
    for k in ("best_cost", "best_step", "best_seed", "last_loss"):
        assert outs[0][2][k] == outs[1][2][k], k


@pytest.mark.parametrize("name,B,G,conv,env", [
    ("C4", 128, 16, False, {"SMOOTHE_WSPMV_PERSIST": "0"}),
    ("C4", 128, 16, False, {"SMOOTHE_WFUSE": "0"}),
    ("C4", 128, 16, False, {"SMOOTHE_RSWITCH": "0"}),
    ("C4", 128, 16, True, {"SMOOTHE_RSWITCH": "0"}),
    ("C4", 128, 16, False, {"SMOOTHE_RBLOCK": "1", "SMOOTHE_FBLOCK": "0", "SMOOTHE_PLAIN_IF": "1",
                            "SMOOTHE_WSPMV_PERSIST": "0", "SMOOTHE_WFUSE": "0", "SMOOTHE_RSWITCH": "0"}),
    ("C5", 64, 8, False, {"SMOOTHE_WFUSE": "0"})])
def test_schedule_variants_identical(sm, monkeypatch, name, B, G, conv, env):
    """The benchmarked C4 schedule at 128 seeds (graph replay; forward sweeps
    gated in blocks of 16 and reverse sweeps in blocks of 8 by conditional
    nodes -- a reverse block above the last forward sweep that changed a row
    runs k_wspmv alone --; persistent k_wspmv whose last chunk of a long class combines the
    partial rows; persistent plain reverse) against the plainer schedules it
    replaced (per-item k_wspmv blocks, k_wcombine launches, one conditional
    per reverse sweep, the plain sweep under its own conditional, ungated
    forward), and C5's fused combine against k_wcombine: theta after 3 steps
    and the best extraction bit for bit (the schedule never changes which sums
    are formed or their order)."""
    eg = make_config(name)
    outs = []
    for e in ({}, env):
        for k in env:
            monkeypatch.delenv(k, raising=False)
        for k, v in e.items():
            monkeypatch.setenv(k, v)
        g = sm.load_egraph_from(eg)
        run = sm.run_create(g, sm.CostModel.from_input(eg), B,
                            sm.Options(penalty_group=G, rng_key=0x5EED0128, converge=conv))
        run.steps(3)
        ch, s = run.extract()
        assert s["graph_mode"] == 1
        outs.append((run.theta(), ch, s))
        run.close()
        g.close()
    assert np.array_equal(outs[0][0], outs[1][0])
    assert np.array_equal(outs[0][1], outs[1][1])
    for k in ("best_cost", "best_step", "best_seed", "last_loss"):
        assert outs[0][2][k] == outs[1][2][k], k


@pytest.mark.parametrize("agg,conv", [("hybrid", False), ("independent", False), ("correlated", False),
                                      ("hybrid", True)])
def test_gated_schedule_small_graph(sm, orc, monkeypatch, agg, conv):
    """The large-graph schedule of the captured step (forward / reverse
    sweeps gated in blocks by conditional and switch nodes, persistent
    k_wspmv and plain reverse, dead-gradient skipping, frozen sweeps) forced
    on C2 with K = 150 (SMOOTHE_BIG_SCHED=1): bit for bit the ungated graph
    and direct launches after 5 steps, then a debug step from that state
    against the oracle."""
    eg = make_config("C2")
    for k, v in (("SMOOTHE_GLIVE", "1"), ("SMOOTHE_REV_W", "1"), ("SMOOTHE_WSPMV_PERSIST", "1"),
                 ("SMOOTHE_RBLOCK", "4"), ("SMOOTHE_FBLOCK", "4")):
        monkeypatch.setenv(k, v)
    outs = []
    for big, graphs in (("1", True), ("0", True), ("1", False)):
        monkeypatch.setenv("SMOOTHE_BIG_SCHED", big)
        g = sm.load_egraph_from(eg)
        run = sm.run_create(g, sm.CostModel.from_input(eg), 64,
                            sm.Options(penalty_group=8, rng_key=0x5EED0150, prop_iters=150,
                                       assumption=agg, converge=conv, use_graphs=graphs))
        run.steps(5)
        ch, s = run.extract()
        assert s["graph_mode"] == (1 if graphs else 0)
        outs.append((run.theta(), ch, s, run.state()))
        run.close()
        g.close()
    for o in outs[1:]:
        assert np.array_equal(outs[0][0], o[0])
        assert np.array_equal(outs[0][1], o[1])
        for k in ("best_cost", "best_step", "best_seed", "last_loss"):
            assert outs[0][2][k] == o[2][k], k
    if not conv:
        th, m, v, n = outs[0][3]
        compare_step(sm, orc, eg, 64, 8, agg=agg, theta=th, m=m, v=v, step_index=n, K=150,
                     label=f"C2_gated_{agg}")


def test_graphs_and_direct_launches_identical(sm):
    eg = make_config("C2")
    outs = []
    for use_graphs in (True, False):
        g = sm.load_egraph_from(eg)
        run = sm.run_create(g, sm.CostModel.from_input(eg), 64,
                            sm.Options(penalty_group=8, rng_key=11, use_graphs=use_graphs))
        run.steps(12)
        outs.append((run.theta(), run.extract()))
        run.close()
    assert np.array_equal(outs[0][0], outs[1][0])
    assert np.array_equal(outs[0][1][0], outs[1][1][0])
    assert outs[0][1][1]["best_cost"] == outs[1][1][1]["best_cost"]


@pytest.mark.parametrize("name,B,G", [("C2", 64, 8), ("C3", 32, 8), ("C5", 64, 8)])
def test_decode_overlap_identical(sm, monkeypatch, name, B, G):
    """Penalty and decode on the second stream give the
    same bits as the sequential step: theta, the best extraction and its
    step / seed (quadratic and MLP configs use the decode stream's own
    scratch buffers)."""
    eg = make_config(name)
    outs = []
    for ov in ("1", "0"):
        monkeypatch.setenv("SMOOTHE_DECODE_OVERLAP", ov)
        g = sm.load_egraph_from(eg)
        run = sm.run_create(g, sm.CostModel.from_input(eg), B,
                            sm.Options(penalty_group=G, rng_key=13))
        run.steps(8)
        outs.append((run.theta(), run.extract()))
        run.close()
    assert np.array_equal(outs[0][0], outs[1][0])
    assert np.array_equal(outs[0][1][0], outs[1][1][0])
    for k in ("best_cost", "best_step", "best_seed", "last_loss"):
        assert outs[0][1][1][k] == outs[1][1][1][k], k


@pytest.mark.parametrize("name,B,G,agg,steps", [
    ("C2", 64, 8, "hybrid", 6), ("C2", 32, 8, "independent", 6), ("C3", 32, 8, "correlated", 6),
    ("C5", 256, 8, "hybrid", 6), ("C4", 32, 16, "hybrid", 3)])
def test_change_propagation_bit_identical(sm, monkeypatch, name, B, G, agg, steps):
    """Skipping classes none of whose parent classes changed in the previous
    sweep (change propagation) gives the same bits as
    recomputing every class in every sweep (SMOOTHE_SWEEP_ALL=1): theta after
    several Adam steps, the best extraction, and the q stack (rebuilt from the
    version lists) and routes of a debug step.  C4 runs the persistent
    forward kernel (more classes than resident row groups)."""
    eg = make_config(name)
    small = name != "C4"   # the C4 q stack would be tens of GB on the host
    outs = []
    for env in ("0", "1"):
        monkeypatch.setenv("SMOOTHE_SWEEP_ALL", env)
        g = sm.load_egraph_from(eg)
        run = sm.run_create(g, sm.CostModel.from_input(eg), B,
                            sm.Options(penalty_group=G, rng_key=3, assumption=agg))
        run.steps(steps)
        th = run.theta()
        dump = run.debug_step(th, qstack=small, route=small)
        outs.append((run.theta(), run.extract(), dump))
        run.close()
    (t0, e0, d0), (t1, e1, d1) = outs
    assert np.array_equal(t0, t1)
    assert np.array_equal(e0[0], e1[0]) and e0[1]["best_cost"] == e1[1]["best_cost"]
    for key in ("qstack", "route", "qK", "grad_cp", "theta_out", "choice", "disc_cost"):
        if key in d0:
            assert np.array_equal(d0[key], d1[key]), key


@pytest.mark.parametrize("wmode,K,conv", [("0", -1, False), ("1", 80, False), ("1", 80, True)])
def test_seed_sharding_bit_identical(sm, monkeypatch, wmode, K, conv):
    """8(e): a run of 64 seeds equals two runs of 32 seeds (seed_begin 0, 32)
    seed by seed, and the lexicographic best of the shards is the full best.
    With the frozen-sweep path (SMOOTHE_REV_W=1, K = 80: most sweeps frozen)
    the per-seed decisions keep this exact."""
    monkeypatch.setenv("SMOOTHE_REV_W", wmode)
    eg = make_config("C2")
    g = sm.load_egraph_from(eg)
    cost = sm.CostModel.from_input(eg)
    full = sm.run_create(g, cost, 64, sm.Options(penalty_group=8, rng_key=5, prop_iters=K,
                                                 converge=conv))
    full.steps(15)
    tf = full.theta()
    cf, sf = full.extract()
    halves = []
    for sb in (0, 32):
        r = sm.run_create(g, cost, 32, sm.Options(penalty_group=8, rng_key=5, seed_begin=sb,
                                                  prop_iters=K, converge=conv))
        r.steps(15)
        halves.append((r.theta(), r.extract()))
    assert np.array_equal(np.concatenate([halves[0][0], halves[1][0]], axis=1), tf)
    bests = sorted((h[1][1]["best_cost"], h[1][1]["best_step"], h[1][1]["best_seed"], i)
                   for i, h in enumerate(halves))
    c, st, seed, i = bests[0]
    assert (c, st, seed) == (sf["best_cost"], sf["best_step"], sf["best_seed"])
    assert np.array_equal(halves[i][1][0], cf)


def test_best_of_seeds_fig1c(sm):
    eg = fig1c_fixture()
    g = sm.load_egraph_from(eg)
    run = sm.optimize(g, sm.CostModel.from_input(eg), 16, 100,
                      sm.Options(prop_iters=4, lam=1.0, penalty_group=4, rng_key=0x5EED0001))
    choice, s = run.extract()
    assert s["valid"] == 1 and s["best_cost"] == 19.0
    assert choice[1] == 2 and choice[3] == -1
    assert s["steps_run"] == 100 and s["time_to_best_s"] > 0


def test_extracted_solution_is_valid(sm, orc):
    from oracle import brute
    eg = make_config("C2")
    g = sm.load_egraph_from(eg)
    run = sm.optimize(g, sm.CostModel.from_input(eg), 64, 30,
                      sm.Options(penalty_group=8, rng_key=9))
    choice, s = run.extract()
    assert s["valid"] == 1
    # the extraction: every selected class's chosen node lies in it, its child
    # classes are selected, no cycle, and the cost is the sum of u
    sel = np.where(choice >= 0)[0]
    ch = {int(j): int(choice[j]) for j in sel}
    r = brute.reach(eg, [ch.get(j, int(eg.class_ptr[j])) for j in range(eg.num_classes)])
    assert r == set(ch)
    assert brute.acyclic(eg, [ch.get(j, int(eg.class_ptr[j])) for j in range(eg.num_classes)], r)
    assert sum(eg.u[ch[j]] for j in ch) == s["best_cost"]


def test_patience_stops_early(sm):
    eg = fig1c_fixture()
    g = sm.load_egraph_from(eg)
    run = sm.run_create(g, sm.CostModel.from_input(eg), 4,
                        sm.Options(prop_iters=4, penalty_group=4, patience=16))
    run.steps(1000)
    _, s = run.extract()
    assert s["steps_run"] < 1000


@pytest.mark.parametrize("name,B,G,agg,steps", [("C2", 128, 8, "hybrid", 6), ("C2", 256, 8, "independent", 4),
                                                ("C3", 128, 8, "correlated", 3), ("C4", 128, 16, "hybrid", 3)])
def test_reverse_tma_bit_identical(sm, monkeypatch, name, B, G, agg, steps):
    """The TMA-staged reverse sweep (opt-in SMOOTHE_REV_TMA=1: gather4 into a
    shared-memory ring, 128-seed slices) against the register kernel: the
    same arithmetic in the same order, so theta after several steps, the
    best extraction and a debug step's gradient are bit for bit equal."""
    eg = make_config(name)
    outs = []
    for env in ("1", "0"):
        monkeypatch.setenv("SMOOTHE_REV_TMA", env)
        g = sm.load_egraph_from(eg)
        run = sm.run_create(g, sm.CostModel.from_input(eg), B,
                            sm.Options(penalty_group=G, rng_key=17, assumption=agg))
        run.steps(steps)
        th = run.theta()
        d = run.debug_step(th)
        outs.append((run.theta(), run.extract(), d["grad_cp"]))
        run.close()
        g.close()
    assert np.array_equal(outs[0][0], outs[1][0])
    assert np.array_equal(outs[0][2], outs[1][2])
    assert np.array_equal(outs[0][1][0], outs[1][1][0])
    assert outs[0][1][1]["best_cost"] == outs[1][1][1]["best_cost"]


@pytest.mark.parametrize("name,B,G,agg,steps,conv", [
    ("C2", 64, 8, "hybrid", 6, 0), ("C3", 32, 8, "correlated", 4, 0), ("C5", 64, 8, "hybrid", 4, 0),
    ("C4", 32, 16, "hybrid", 3, 0), ("C4", 128, 16, "independent", 2, 0), ("C5", 64, 8, "hybrid", 3, 1)])
def test_dead_gradient_skip_identical(sm, monkeypatch, name, B, G, agg, steps, conv):
    """Reverse sweeps whose input g_q^t is all zero (live flag unset) are
    skipped (default) against running every sweep (SMOOTHE_GLIVE=0): the
    sweeps are linear in g_q with no source term, so theta after several
    steps, a debug step's gradient and the best extraction are equal
    (skipping can only leave a -0 where +0 would be added: compared as
    values, so -0 == +0)."""
    eg = make_config(name)
    outs = []
    for env in ("1", "0"):
        monkeypatch.setenv("SMOOTHE_GLIVE", env)
        g = sm.load_egraph_from(eg)
        run = sm.run_create(g, sm.CostModel.from_input(eg), B,
                            sm.Options(penalty_group=G, rng_key=19, assumption=agg, converge=bool(conv)))
        run.steps(steps)
        th, m, v, n = run.state()
        d = run.debug_step(th, m, v, step_index=n)
        outs.append((run.theta(), run.extract(), d["grad_cp"], d["grad_theta"]))
        run.close()
        g.close()
    assert np.array_equal(outs[0][0], outs[1][0])
    assert np.array_equal(outs[0][2], outs[1][2])
    assert np.array_equal(outs[0][3], outs[1][3])
    assert np.array_equal(outs[0][1][0], outs[1][1][0])
    assert outs[0][1][1]["best_cost"] == outs[1][1][1]["best_cost"]


def test_step_trace_relaxed_vs_sampled(sm):
    """The per-step record (smoothe_run_get_trace, E11 / PAPER.md:459-461):
    row k holds min / mean over seeds of the relaxed f(p_b) and the min of the
    sampled f_b(s) of step k; checked against a debug step taken as step k
    (its own f and decoded costs), and the run's best is the minimum of the
    sampled column at the recorded step."""
    eg = make_config("C2")
    g = sm.load_egraph_from(eg)
    run = sm.run_create(g, sm.CostModel.from_input(eg), 64, sm.Options(penalty_group=8, rng_key=23))
    run.steps(9)
    th, m, v, n = run.state()
    d = run.debug_step(th, m, v, step_index=n)   # step 9
    tr = run.trace()
    assert len(tr["relaxed_min"]) == 10
    assert tr["relaxed_min"][9] == d["f"].min()
    assert tr["relaxed_mean"][9] == pytest.approx(d["f"].mean(), rel=1e-12)
    ok = d["valid"] == 1
    assert tr["valid"][9] == ok.sum()
    assert tr["sampled_min"][9] == d["disc_cost"][ok].min()
    _, s = run.extract()
    smin = tr["sampled_min"]
    assert s["best_cost"] == smin.min() and s["best_step"] == int(np.argmin(smin))
    assert np.all(tr["relaxed_min"] <= tr["relaxed_mean"])
    run.close()
    g.close()


@pytest.mark.parametrize("name,B,G,steps", [("C2", 64, 8, 6), ("C3", 128, 8, 3), ("C5", 64, 8, 3)])
def test_version_pool_growth_bit_identical(sm, monkeypatch, name, B, G, steps):
    """Pooled version stacks: a run whose pools start far too
    small (SMOOTHE_POOL_FRAC=0.01) aborts the overflowing steps (no update, no
    keep-best), grows the pools and repeats them; theta, the best extraction
    and a debug step's q stack and routes (rebuilt from the pools) are bit
    for bit those of a run with pools for every sweep (SMOOTHE_POOL_FRAC=1)."""
    eg = make_config(name)
    outs = []
    for frac in ("0.01", "1"):
        monkeypatch.setenv("SMOOTHE_POOL_FRAC", frac)
        g = sm.load_egraph_from(eg)
        run = sm.run_create(g, sm.CostModel.from_input(eg), B,
                            sm.Options(penalty_group=G, rng_key=31))
        run.steps(steps)
        th, m, v, n = run.state()
        assert n == steps
        small = eg.num_nodes < 10000
        d = run.debug_step(th, m, v, step_index=n, qstack=small, route=small)
        ch, s = run.extract()
        outs.append((th, ch, s, d))
        run.close()
        g.close()
    (t0, c0, s0, d0), (t1, c1, s1, d1) = outs
    assert s0["pool_grows"] > 0 and s1["pool_grows"] == 0
    assert s0["pool_rows"] < s1["pool_rows"] or s1["pool_rows"] == s0["pool_rows"]
    assert np.array_equal(t0, t1) and np.array_equal(c0, c1)
    for k in ("best_cost", "best_step", "best_seed", "steps_run"):
        assert s0[k] == s1[k], k
    for k in ("qstack", "route", "grad_cp", "theta_out", "qK"):
        if k in d0:
            assert np.array_equal(d0[k], d1[k]), k

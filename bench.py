"""Benchmark of the SmoothE seed-parallel step on B200 (driver contract).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C4] [--impl ours|reference]

One JSON line on rank 0.  A "step" is one pass of the whole hot path
(softmax, K forward sweeps, cost, NOTEARS, K reverse
sweeps, softmax-backward + Adam, decode + validity, keep-best) over the
per-GPU seed batch.  metric = seed x e-node steps/s (BASELINE.json), value =
whole-job units/s with inputs resident in HBM; e2e = the same metric through
the C-ABI calls with HOST buffers (load + optimize + extract inside the timed
region).  Multi-GPU: seeds shard across ranks (weak scaling, no data-path
collective); the global best is min-reduced over NCCL at the end.

--impl reference runs the fp64 CPU oracle (oracle/) as it stands on the box's
host cores on a bounded sample of the same workload (tier: no reference code).
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import tempfile
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "seed x e-node steps/s (fwd+bwd) and time-to-best-cost at 1/2/4/8 B200"
UNIT = "seed*e-node*steps/s"


def log(*a):
    print(*a, file=sys.stderr, flush=True)


def workload(name):
    from gen import CONFIGS, make_config
    from gen.configs import rng_key
    spec = CONFIGS[name]
    t0 = time.time()
    eg = make_config(name)
    log(f"[bench] generated {name}: N={eg.num_nodes} M={eg.num_classes} E={eg.num_edges} "
        f"in {time.time() - t0:.1f}s")
    return spec, eg, rng_key(name)


def byte_model(N, M, K, Bl):
    """SURVEY.md 8(d) streaming model, bytes per unit (seed x e-node)."""
    r = M / N
    return {"fixed": 52 + 12 * r, "forward_sweep": 4 + 8 * r, "reverse_sweep": 12 + 12 * r,
            "step": 52 + 12 * r + K * (16 + 20 * r)}


def class_graph(eg):
    """distinct (class, child class) edges as CSR over the parent class"""
    M, N = eg.num_classes, eg.num_nodes
    src = eg.ec()[np.repeat(np.arange(N), np.diff(eg.child_ptr))]
    key = np.unique(src.astype(np.int64) * M + np.asarray(eg.child_class))
    src, dst = key // M, key % M
    return src, dst, np.searchsorted(src, np.arange(M + 1))


def hmax_classes(eg):
    """longest walk from each class (inf if it reaches a cycle): g_q^t_j is
    exactly 0 for t < K - hmax_j (the reverse window)"""
    M = eg.num_classes
    src, dst, ptr = class_graph(eg)
    outdeg = np.diff(ptr).astype(np.int64)
    order = np.argsort(dst, kind="stable")
    pptr = np.searchsorted(dst[order], np.arange(M + 1))
    h = np.full(M, -1, np.int64)
    frontier = np.where(outdeg == 0)[0]
    h[frontier] = 0
    while frontier.size:
        preds = np.concatenate([src[order[pptr[c]:pptr[c + 1]]] for c in frontier])
        np.subtract.at(outdeg, preds, 1)
        new = np.unique(preds[(outdeg[preds] == 0) & (h[preds] < 0)])
        for j in new:
            h[j] = h[dst[ptr[j]:ptr[j + 1]]].max() + 1
        frontier = new
    out = h.astype(float)
    out[h < 0] = np.inf
    return out


def active_fractions(eg, K):
    """Mean fraction of e-nodes / classes the reverse sweeps touch (activity
    windows: reverse sweep t skips class j unless dmin_j <= t - 1, its BFS depth
    from the root, and t > K - hmax_j)."""
    M, N = eg.num_classes, eg.num_nodes
    src, dst, ptr = class_graph(eg)
    dmin = np.full(M, np.iinfo(np.int64).max)
    dmin[eg.root] = 0
    frontier, d = np.array([eg.root]), 0
    while frontier.size:
        d += 1
        nxt = np.unique(np.concatenate([dst[ptr[j]:ptr[j + 1]] for j in frontier]))
        nxt = nxt[dmin[nxt] > d]
        dmin[nxt] = d
        frontier = nxt
    hm = hmax_classes(eg)
    sizes = np.diff(eg.class_ptr)
    nodes = classes = 0.0
    for t in range(1, K + 1):
        act = (dmin <= t - 1) & (t + hm > K)
        nodes += sizes[act].sum() / N
        classes += act.sum() / M
    return nodes / K, classes / K


class ClockSampler:
    """nvidia-smi clocks + throttle reasons during the timed region."""

    def __init__(self, index):
        self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
        q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
             "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
        try:
            self.p = subprocess.Popen(["nvidia-smi", f"--id={index}", f"--query-gpu={q}",
                                       "--format=csv,noheader,nounits", "-lms", "100"],
                                      stdout=self.f, stderr=subprocess.DEVNULL)
        except Exception:
            self.p = None

    def stop(self):
        if self.p is None:
            return None
        self.p.terminate()
        try:
            self.p.wait(timeout=5)
        except Exception:
            self.p.kill()
        self.f.flush()
        self.f.seek(0)
        rows = [l.strip().split(", ") for l in self.f.read().splitlines() if l.strip()]
        os.unlink(self.f.name)
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for r in rows:
            try:
                sm.append(float(r[1]))
                mx = float(r[2])
                for n, v in zip(names, r[5:9]):
                    if v.strip().lower() in ("active", "1"):
                        reasons.add(n)
            except Exception:
                continue
        if not sm:
            return None
        return {"sm_mhz": float(np.median(sm)), "sm_max_mhz": mx, "reasons": sorted(reasons),
                "samples": len(sm)}


def measured_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as fh:
            p = json.load(fh)
        return p.get("hbm_gbs", 6563.2), "measured"
    except Exception:
        return 6650.0, "fallback"


def ncu_traffic(config, kernel):
    """dram bytes per launch from a committed `ncu --set full` capture, if any."""
    try:
        with open(os.path.join(ROOT, "profiles", "traffic.json")) as fh:
            t = json.load(fh)
        return t.get(config, {}).get(kernel)
    except Exception:
        return None


# ---------------------------------------------------------------------------
# CPU legs: the fp64 oracle as it stands (bench's cpu_baseline / --impl reference)
# ---------------------------------------------------------------------------
def oracle_sample(eg, spec, key, steps, seeds):
    import oracle
    og = oracle.Graph(eg)
    G = min(spec["group"], seeds)
    while seeds % G:
        G -= 1
    opts = oracle.Options(K=-1, lam=float(np.mean(eg.u)), G=G, lr=0.1)
    th = oracle.theta_init(key, 0, seeds, eg.num_nodes)
    m = v = None
    t0 = time.perf_counter()
    for s in range(steps):
        o = og.step(th, opts, m=m, v=v, step_index=s)
        th, m, v = o["theta_out"], o["m_out"], o["v_out"]
    dt = time.perf_counter() - t0
    units = seeds * eg.num_nodes * steps
    cores = min(oracle.num_threads(), seeds)
    return {"value": units / dt, "unit": UNIT, "cores": cores, "kind": "oracle",
            "sample": f"{steps} step(s) x {seeds} seeds of {eg.name} (N={eg.num_nodes}, "
                      f"K={og.K_auto}), fp64 C++ -O3 OpenMP over seeds; {dt:.1f}s"}


def cpu_sample_size(name):
    # about 10-30 s of CPU work on the box (SURVEY.md 8(d) oracle timing)
    return {"C1": (50, 1), "C2": (10, 16), "C3": (2, 16), "C4": (1, 16), "C5": (1, 16)}[name]


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    spec, eg, key = workload(args.config)
    steps, seeds = cpu_sample_size(args.config)
    per_step = []
    cb = None
    for _ in range(args.warmup and 1):
        oracle_sample(eg, spec, key, 1, min(seeds, 4))
    for _ in range(max(1, args.steps)):
        cb = oracle_sample(eg, spec, key, steps, seeds)
        per_step.append(cb["value"])
    value = float(np.median(per_step))
    cb["value"] = value
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": f"{args.config} ({eg.name}) oracle sample",
                       "seeds_per_gpu": spec["seeds_per_gpu"]},
            "cpu_baseline": cb,
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


# ---------------------------------------------------------------------------
# GPU arm
# ---------------------------------------------------------------------------
def run_ours(args):
    import torch
    import torch.distributed as dist
    import paper_conf_asplos_caiydyz25_b200 as sm

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    spec, eg, key = workload(args.config)
    Bl, G = spec["seeds_per_gpu"], spec["group"]
    lam = float(np.mean(eg.u))      # reading S11: lambda = mean(u)
    cost = sm.CostModel.from_input(eg)
    # a real (non-legacy) stream: the library orders its private stream after
    # this one and this one after its work, so events here bracket the steps
    stream = torch.cuda.Stream()
    torch.cuda.set_stream(stream)
    opts = sm.Options(assumption="hybrid", prop_iters=-1, lam=lam, penalty_group=G, lr=0.1,
                      rng_key=key, seed_begin=rank * Bl, cuda_stream=stream.cuda_stream,
                      use_graphs=True, converge=args.converge)
    t0 = time.time()
    g = sm.load_egraph_from(eg, device=local)
    run = sm.run_create(g, cost, Bl, opts)
    torch.cuda.synchronize()
    log(f"[bench] rank {rank}: load+create {time.time() - t0:.1f}s, K={run.K}, "
        f"info={g.info}")
    N, M, K = eg.num_nodes, eg.num_classes, run.K

    run.steps(args.warmup)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    # timed region: K steps replayed from the step's CUDA graph
    clocks = ClockSampler(local)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    run.steps(args.steps)
    e1.record(stream)
    torch.cuda.synchronize()
    ck = clocks.stop()
    ms = e0.elapsed_time(e1)
    # second timed region, K more steps launched directly with CUDA events at
    # every phase boundary and around every sweep kernel (the roofline's
    # per-launch kernel time and the phase breakdown)
    run.profile(True)
    torch.cuda.synchronize()
    p0, p1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    p0.record(stream)
    run.steps(args.steps)
    p1.record(stream)
    torch.cuda.synchronize()
    prof_ms = p0.elapsed_time(p1)
    prof = run.get_profile()
    run.profile(False)
    if world > 1:
        t = torch.tensor([ms], device="cuda", dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    units_rank = Bl * N * args.steps
    value = units_rank * world / (ms * 1e-3)

    # time-to-best-cost: the same run continues (CUDA-graph replay) to a fixed
    # step budget; time is measured by the library from run creation (theta
    # initialisation included, load excluded) to the end of the step that first
    # produced the final global best
    done = args.warmup + 2 * args.steps
    if args.ttb_steps > done:
        run.steps(args.ttb_steps - done)
        run.synchronize()
    from paper_conf_asplos_caiydyz25_b200.distributed import global_best
    best = global_best(run, dist if world > 1 else None, device=torch.device("cuda", local))
    ttb = {"steps": max(done, args.ttb_steps), "time_to_best_s": best["time_to_best_s"],
           "best_cost": best["best_cost"], "best_step": best["best_step"],
           "best_seed": best["best_seed"],
           "note": "wall time on the GPU from run creation to the end of the best step"}
    # quality context: the paper's greedy worklist heuristic on
    # the same graph and u (smoothe_greedy, on the GPU; its own objective is
    # the linear cost, so for MLP / quadratic configs it ignores those terms)
    if rank == 0:
        tg = time.time()
        _, _, gr = g.greedy(eg.u)
        ttb["greedy"] = {"dag_cost": gr["dag_cost"], "wall_ms": (time.time() - tg) * 1e3,
                         "valid": gr["valid"], "linear_cost_only": eg.mlp is not None
                         or eg.quad is not None}

    # roofline for the dominant phase
    bm = byte_model(N, M, K, Bl)
    ph = prof["phase_ms"]
    # the dominant sweep kernel, timed alone (CUDA events around each launch on
    # the library's stream, inside the timed region)
    kms, kn = prof["sweep_kernel_ms"], prof["sweep_kernel_launches"]
    dom = max(("forward", "reverse", "frozen"), key=lambda k: kms.get(k, 0.0))
    units_launch = Bl * N
    peak, peak_src = measured_peaks()
    if dom == "frozen":
        # k_wspmv (frozen reverse sweeps): per working
        # launch it streams one W row per class edge and gathers one g_q row
        # per class edge (counted once per class row in the streaming model,
        # like the reverse sweep's gathers), reads g_q^t_i, updates S_i and
        # writes g_q^{t-1}_i: Bl (4 C + 16 M) bytes, C = distinct class edges.
        # Launches in sweeps with no frozen seed exit at once; the time of all
        # launches is charged to the working ones.
        C_edges = len(class_graph(eg)[0])
        nwork = max(1, prof.get("frozen_sweeps", 0))
        per_launch_ms = kms[dom] / nwork
        alg = Bl * (4.0 * C_edges + 16.0 * M)
        fn = fc = 1.0
        alg_unit = alg / units_launch
        kname = "k_wspmv"
    else:
        per_launch_ms = kms[dom] / max(1, kn[dom])
        # algorithmic bytes of the rows a launch touches (activity windows), on
        # average over the K launches: per e-node and per class terms of the
        # model (the forward kernel recomputes only classes whose parents
        # changed in the previous sweep, a data-dependent set)
        fn, fc = active_fractions(eg, K) if dom == "reverse" else (1.0, 1.0)
        per_node, per_class = (4.0, 8.0) if dom == "forward" else (12.0, 12.0)
        alg = Bl * (per_node * N * fn + per_class * M * fc)
        alg_unit = bm["forward_sweep" if dom == "forward" else "reverse_sweep"]
        kname = f"k_sweep_{dom}"
    achieved = alg / (per_launch_ms * 1e-3) / 1e9
    traffic = ncu_traffic(args.config, dom)
    # fwd+bwd share of the profiled step, applied to the graph-timed step
    fwdbwd_ms = (ms / args.steps) * sum(ph[k] for k in ("softmax", "forward", "cost", "penalty",
                                                        "reverse", "update")) / max(1e-9, sum(ph.values()))
    roof = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
            "frac": achieved / peak, "traffic": traffic, "kernel": kname,
            "alg_bytes_per_unit": alg_unit,
            "units_per_launch": units_launch, "avg_launch_ms": per_launch_ms,
            "kernel_share_of_step": kms[dom] / max(1e-9, sum(ph.values())),
            "alg_bytes_per_launch": alg, "active_node_frac": fn, "active_class_frac": fc,
            "peak_source": f"{peak_src} hbm_gbs (MEASURED_PEAKS.json)"}
    if dom == "frozen":
        roof["working_launches_per_step"] = nwork / max(1, prof["steps"])

    run.close()

    # the same workload in convergence mode (reading S1b, an option, not the
    # headline: the north star fixes the number of iterations): each seed's
    # sweeps stop at convergence; same graph, seeds and timing rules
    conv = None
    if not args.converge and not args.no_converge_leg:
        copts = sm.Options(assumption="hybrid", prop_iters=-1, lam=lam, penalty_group=G, lr=0.1,
                           rng_key=key, seed_begin=rank * Bl, cuda_stream=stream.cuda_stream,
                           use_graphs=True, converge=True)
        crun = sm.run_create(g, cost, Bl, copts)
        crun.steps(args.warmup)
        torch.cuda.synchronize()
        c0, c1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        c0.record(stream)
        crun.steps(args.steps)
        c1.record(stream)
        torch.cuda.synchronize()
        cms = c0.elapsed_time(c1)
        crun.close()
        conv = {"ms_per_step": cms / args.steps, "value": units_rank * world / (cms * 1e-3),
                "note": "smoothe_options.converge = 1 (reading S1b): each seed's sweeps stop at "
                        "its first change-free sweep; this rank's device time"}
    g.close()
    torch.cuda.synchronize()

    # e2e: the C-ABI calls with host buffers: load (H2D) + optimize (init + steps) + extract (D2H)
    e2e = None
    if not args.no_e2e:
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        t0 = time.perf_counter()
        g2 = sm.load_egraph_from(eg, device=local)
        r2 = sm.optimize(g2, cost, Bl, args.steps, opts)
        choice2, s2 = r2.extract()
        dt = time.perf_counter() - t0
        r2.close()
        g2.close()
        if world > 1:
            t = torch.tensor([dt], device="cuda", dtype=torch.float64)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            dt = float(t.item())
        h2d = (eg.class_ptr.nbytes + eg.child_ptr.nbytes + eg.child_class.nbytes + eg.u.nbytes
               + (sum(a.nbytes for a in eg.quad) if eg.quad is not None else 0)
               + (sum(a.nbytes for a in eg.mlp.values()) if eg.mlp is not None else 0))
        d2h = choice2.nbytes + 64
        e2e = {"value": units_rank * world / dt, "unit": UNIT,
               "h2d_bytes_per_step": h2d / args.steps, "d2h_bytes_per_step": d2h / args.steps,
               "seconds": dt, "includes": "load_egraph (host analysis + H2D), theta init, "
                                         f"{args.steps} steps, extract (D2H)"}

    cb = None
    if rank == 0 and world == 1 and not args.no_cpu:
        steps_c, seeds_c = cpu_sample_size(args.config)
        cb = oracle_sample(eg, spec, key, steps_c, seeds_c)

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms / args.steps, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": {"workload": f"{args.config}: {eg.name} synthetic e-graph "
                                   f"N={N} M={M} E={eg.num_edges} K={K} cost={eg.cost_kind()}",
                       "seeds_per_gpu": Bl, "global_seeds": Bl * world, "penalty_group": G,
                       "assumption": "hybrid", "optimizer": "adam lr=0.1",
                       "lambda": lam, "parallelism": f"seed-sharded dp{world}",
                       "sweeps": ("each seed until convergence, at most K (reading S1b)"
                                  if args.converge else "K (reading S1)"),
                       "l2": "inputs larger than L2 (cp %.0f MB, q-stack %.1f GB)" %
                             (N * Bl * 4 / 1e6, (K + 1) * M * Bl * 4 / 1e9)},
            "fwd_bwd_units_per_s": units_rank * world / (fwdbwd_ms * 1e-3),
            "phases_ms_per_step": {k: v / max(1, prof["steps"]) for k, v in ph.items()},
            "profiled_ms_per_step": prof_ms / args.steps,
            "sweep_kernel_ms_per_step": {k: v / max(1, prof["steps"])
                                         for k, v in prof["sweep_kernel_ms"].items()},
            "gpu_launches": prof["launches"],
            "time_to_best": ttb,
            "converge_mode": conv,
            "roofline": roof, "e2e": e2e, "cpu_baseline": cb, "clocks": ck,
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="C4")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--converge", action="store_true",
                    help="reading S1b: each seed's sweeps stop at convergence (not the default K)")
    ap.add_argument("--no-converge-leg", action="store_true",
                    help="skip the extra convergence-mode measurement")
    ap.add_argument("--ttb-steps", type=int, default=80,
                    help="step budget of the time-to-best-cost measurement (same run)")
    args = ap.parse_args()
    if args.warmup < 3:
        log("[bench] warmup raised to 3 (timing rules)")
        args.warmup = 3
    if args.impl == "reference":
        return run_reference(args)
    return run_ours(args)


if __name__ == "__main__":
    sys.exit(main())

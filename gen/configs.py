"""The five BASELINE.json configs as concrete seeded inputs.

| | family (Table 1 shape) | N | M | d | D | cost | seeds |
|---|---|---|---|---|---|---|---|
| C1 | Fig. 1c fixture + random tiny          | 10 | 8 | 1.0 | 4 | linear | 1 |
| C2 | flexc-like, cyclic                     | 5 000 | 1 233 | 1.8 | 24 | linear | 64 |
| C3 | tensat-like                            | 100 000 | 60 208 | 2.3 | 40 | quadratic | 256 |
| C4 | rover-like, deep, cyclic               | 1 000 000 | 168 160 | 5.5 | 96 | linear | 1024 |
| C5 | diospyros-like                         | 300 000 | 13 133 | 2.5 | 32 | linear+MLP | 512 |

``seeds`` is the whole-job seed batch B (at 8 GPUs for C3-C5); a run on P
GPUs holds B/P seeds per GPU (``seeds_per_gpu``), i.e. weak scaling from the
per-GPU batch the 8-GPU config implies.
gen_seed = 1000 + config#, rng_key = 0x5EED0000 + config# (SURVEY.md 8(d)).
"""
from __future__ import annotations

from .egraph import fig1c_fixture, synth_egraph

CONFIGS = {
    "C1": dict(kind="fixture", seeds=1, seeds_per_gpu=1, group=1),
    "C2": dict(kind="synth", N=5000, M=1233, d=1.8, d_boost=1.15, D=24, p_back=0.015,
               b_levels=3, scc_max=32, w_pos=0.03, cost="linear", seeds=64, seeds_per_gpu=64,
               group=8),
    "C3": dict(kind="synth", N=100_000, M=60_208, d=2.3, d_boost=1.1, D=40, p_back=0.01,
               b_levels=1, scc_max=32, w_pos=0.004, cost="quadratic", seeds=256,
               seeds_per_gpu=32, group=8),
    "C4": dict(kind="synth", N=1_000_000, M=168_160, d=5.5, d_boost=1.09, D=96, p_back=0.0015,
               b_levels=2, scc_max=64, w_pos=0.004, cost="linear", seeds=1024,
               seeds_per_gpu=128, group=16),
    "C5": dict(kind="synth", N=300_000, M=13_133, d=2.5, d_boost=1.05, D=32, p_back=0.002,
               b_levels=1, scc_max=32, w_pos=0.01, cost="mlp", seeds=512, seeds_per_gpu=64,
               group=8),
}


def config_number(name: str) -> int:
    return int(name[1:])


def rng_key(name: str) -> int:
    return 0x5EED0000 + config_number(name)


def make_config(name: str, **overrides):
    """Return the EGraphInput of a config (deterministic)."""
    spec = dict(CONFIGS[name])
    spec.update(overrides)
    if spec["kind"] == "fixture":
        return fig1c_fixture()
    return synth_egraph(name, spec["N"], spec["M"], spec["d"] * spec["d_boost"], spec["D"],
                        seed=1000 + config_number(name), p_back=spec["p_back"],
                        b_levels=spec["b_levels"], scc_max=spec["scc_max"],
                        w_pos=spec["w_pos"], cost_model=spec["cost"])

"""Seeded synthetic inputs shared by the oracle side (tests, bench cpu_baseline)
and the CUDA side (tests, bench, smoke).

This package holds NO arithmetic of the SmoothE method (no softmax, no
propagation, no cost evaluation, no penalty): it only draws e-graphs, costs and
cost-model weights from seeded generators, with the shapes of the paper's
Table 1.  See DESIGN.md "Input recipe".
"""
from .egraph import EGraphInput, fig1c_fixture, random_tiny, synth_egraph  # noqa: F401
from .configs import CONFIGS, make_config  # noqa: F401

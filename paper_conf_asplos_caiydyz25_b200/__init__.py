"""B200 (sm_100a) implementation of SmoothE's seed-parallel gradient step.

The product is libsmoothe.so (C ABI: include/smoothe.h); this package is its
thin Python binding plus the multi-GPU driver (torch.distributed).
"""
from .smoothe import (CostModel, EGraph, Options, Run, SmootheError, extract, lib,  # noqa: F401
                      load_egraph, load_egraph_from, optimize, release_cached_memory, run_create,
                      torch_stream, version)

"""ctypes wrapper of the fp64 SmoothE oracle -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package.  The
product package ``paper_conf_asplos_caiydyz25_b200`` never imports it, and the
oracle shares no code with the CUDA path (see smoothe_oracle.cpp header).

Pinned by tests/test_oracle_*.py against PAPER.md's worked example, closed
forms, invariants and brute-force enumeration (oracle/brute.py).  Functions
without such a pin are marked "parity unpinned" in DESIGN.md (whole-trajectory
parity only).
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "smoothe_oracle.cpp")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None

ASSUMPTIONS = {"independent": 0, "correlated": 1, "hybrid": 2}


def build(force: bool = False) -> str:
    """Compile the oracle (gcc/g++ -O3 -march=native -fopenmp, no hand SIMD)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["g++", "-std=c++17", "-O3", "-march=native", "-ffp-contract=off", "-fopenmp", "-fPIC",
                               "-shared", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


class _Cost(C.Structure):
    _fields_ = [("kind", C.c_int32), ("u", C.c_void_p), ("quad_nnz", C.c_int64),
                ("quad_i", C.c_void_p), ("quad_j", C.c_void_p), ("quad_w", C.c_void_p),
                ("H1", C.c_int32), ("H2", C.c_int32),
                ("W1", C.c_void_p), ("b1", C.c_void_p), ("W2", C.c_void_p),
                ("b2", C.c_void_p), ("W3", C.c_void_p), ("b3", C.c_void_p)]


class _Opts(C.Structure):
    _fields_ = [("assumption", C.c_int32), ("K", C.c_int32), ("lam", C.c_double),
                ("G", C.c_int32), ("lr", C.c_double), ("beta1", C.c_double),
                ("beta2", C.c_double), ("eps", C.c_double), ("optimizer", C.c_int32),
                ("route_delta", C.c_double), ("route_alt", C.c_int32)]


class _Dump(C.Structure):
    _fields_ = [(n, C.c_void_p) for n in
                ("cp", "qstack", "p", "f", "h", "loss", "grad_cp", "grad_theta", "theta_out",
                 "m_out", "v_out", "choice", "valid", "disc_cost", "reached", "route",
                 "route_margin", "route_margin_all", "route_namb", "grad_cp_spread")]


def lib():
    global _lib
    if _lib is None:
        _lib = C.CDLL(build())
        _lib.oracle_graph_new.restype = C.c_void_p
        _lib.oracle_graph_new.argtypes = [C.c_int32, C.c_int32, C.c_void_p, C.c_void_p,
                                          C.c_void_p, C.c_int32]
        _lib.oracle_graph_free.argtypes = [C.c_void_p]
        _lib.oracle_graph_info.argtypes = [C.c_void_p, C.c_void_p]
        _lib.oracle_graph_scc.argtypes = [C.c_void_p, C.c_void_p]
        _lib.oracle_philox4x32_10.argtypes = [C.c_void_p, C.c_void_p, C.c_void_p]
        _lib.oracle_theta_init.argtypes = [C.c_uint64, C.c_int64, C.c_int32, C.c_int32, C.c_void_p]
        _lib.oracle_expm.argtypes = [C.c_int32, C.c_void_p, C.c_void_p]
        _lib.oracle_step.restype = C.c_int
        _lib.oracle_step.argtypes = [C.c_void_p, C.POINTER(_Cost), C.POINTER(_Opts), C.c_int32,
                                     C.c_void_p, C.c_void_p, C.c_void_p, C.c_int32,
                                     C.POINTER(_Dump)]
        _lib.oracle_decode.argtypes = [C.c_void_p, C.POINTER(_Cost), C.c_int32, C.c_void_p,
                                       C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p]
        _lib.oracle_optimize.restype = C.c_int
        _lib.oracle_optimize.argtypes = [C.c_void_p, C.POINTER(_Cost), C.POINTER(_Opts), C.c_int32,
                                         C.c_uint64, C.c_int64, C.c_int32, C.c_int32,
                                         C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p]
        _lib.oracle_num_threads.restype = C.c_int
        _lib.oracle_update.argtypes = [C.c_int64, C.POINTER(_Opts), C.c_int32, C.c_void_p,
                                       C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p,
                                       C.c_void_p, C.c_void_p]
    return _lib


def _p(a):
    return None if a is None else a.ctypes.data


def num_threads() -> int:
    return lib().oracle_num_threads()


def philox4x32_10(ctr, key):
    c = np.ascontiguousarray(ctr, dtype=np.uint32)
    k = np.ascontiguousarray(key, dtype=np.uint32)
    out = np.zeros(4, dtype=np.uint32)
    lib().oracle_philox4x32_10(_p(c), _p(k), _p(out))
    return out


def theta_init(rng_key: int, seed_begin: int, B: int, N: int) -> np.ndarray:
    out = np.zeros((N, B), dtype=np.float64)
    lib().oracle_theta_init(rng_key, seed_begin, B, N, _p(out))
    return out


def expm(A: np.ndarray) -> np.ndarray:
    A = np.ascontiguousarray(A, dtype=np.float64)
    E = np.zeros_like(A)
    lib().oracle_expm(A.shape[0], _p(A), _p(E))
    return E


class Options:
    def __init__(self, assumption="hybrid", K=-1, lam=1.0, G=1, lr=0.1, beta1=0.9,
                 beta2=0.999, eps=1e-8, optimizer="adam", route_delta=1e-5, route_alt=0):
        """route_delta: relative margin below which a max-routing comparison
        may go either way (reading S7', smoothe_oracle.cpp backward());
        route_alt (pins of the spread bound only): 1 / 2 route decisions with
        several admissible routes to the highest / lowest admissible parent."""
        self.assumption, self.K, self.lam, self.G = assumption, K, lam, G
        self.lr, self.beta1, self.beta2, self.eps = lr, beta1, beta2, eps
        self.optimizer = optimizer
        self.route_delta, self.route_alt = route_delta, route_alt

    def c(self) -> _Opts:
        return _Opts(ASSUMPTIONS[self.assumption], self.K, self.lam, self.G, self.lr, self.beta1,
                     self.beta2, self.eps, 0 if self.optimizer == "adam" else 1,
                     self.route_delta, self.route_alt)


def update(theta, grad, opts: Options, m=None, v=None, step_index=0):
    """The oracle's optimiser step alone (same code as inside step())."""
    th = np.ascontiguousarray(theta, dtype=np.float64)
    g = np.ascontiguousarray(grad, dtype=np.float64)
    m = None if m is None else np.ascontiguousarray(m, dtype=np.float64)
    v = None if v is None else np.ascontiguousarray(v, dtype=np.float64)
    out = [np.zeros_like(th) for _ in range(3)]
    lib().oracle_update(th.size, C.byref(opts.c()), step_index, _p(th), _p(m), _p(v), _p(g),
                        _p(out[0]), _p(out[1]), _p(out[2]))
    return {"theta_out": out[0], "m_out": out[1], "v_out": out[2]}


class Graph:
    """Oracle view of an EGraphInput (gen.EGraphInput)."""

    def __init__(self, eg):
        self.eg = eg
        self._arrs = [np.ascontiguousarray(eg.class_ptr, dtype=np.int32),
                      np.ascontiguousarray(eg.child_ptr, dtype=np.int64),
                      np.ascontiguousarray(eg.child_class, dtype=np.int32)]
        self.h = lib().oracle_graph_new(eg.num_classes, eg.num_nodes, _p(self._arrs[0]),
                                        _p(self._arrs[1]), _p(self._arrs[2]), eg.root)
        if not self.h:
            raise ValueError("oracle rejected the e-graph")
        self.M, self.N = eg.num_classes, eg.num_nodes
        info = np.zeros(5, dtype=np.int64)
        lib().oracle_graph_info(self.h, _p(info))
        self.E, self.K_auto, self.num_scc, self.scc_classes, self.scc_max = (int(x) for x in info)
        self._cost_keep = None
        self.cost = self._make_cost(eg)

    def __del__(self):
        try:
            if self.h:
                lib().oracle_graph_free(self.h)
        except Exception:
            pass

    def _make_cost(self, eg) -> _Cost:
        u = np.ascontiguousarray(eg.u, dtype=np.float64)
        keep = [u]
        c = _Cost()
        c.kind = 0
        c.u = _p(u)
        if eg.quad is not None:
            qi, qj, qw = (np.ascontiguousarray(eg.quad[0], dtype=np.int32),
                          np.ascontiguousarray(eg.quad[1], dtype=np.int32),
                          np.ascontiguousarray(eg.quad[2], dtype=np.float64))
            keep += [qi, qj, qw]
            c.kind, c.quad_nnz, c.quad_i, c.quad_j, c.quad_w = 1, qi.size, _p(qi), _p(qj), _p(qw)
        if eg.mlp is not None:
            ws = {k: np.ascontiguousarray(v, dtype=np.float32) for k, v in eg.mlp.items()}
            keep += list(ws.values())
            c.kind = 2
            c.H1, c.H2 = ws["W1"].shape[0], ws["W2"].shape[0]
            c.W1, c.b1, c.W2, c.b2, c.W3, c.b3 = (_p(ws[k]) for k in ("W1", "b1", "W2", "b2", "W3", "b3"))
        self._cost_keep = keep
        return c

    def scc(self) -> np.ndarray:
        out = np.zeros(self.M, dtype=np.int32)
        lib().oracle_graph_scc(self.h, _p(out))
        return out

    def step(self, theta, opts: Options, m=None, v=None, step_index=0, qstack=False, route=False,
             spread=False):
        """One step for B seeds; theta [N][B] (any float dtype; upcast exactly).

        Every decision is the oracle's own (fp64).  Always returned:
        route_margin / route_margin_all [B], the smallest relative margin of a
        max-routing decision (reading S7', smoothe_oracle.cpp backward()) that
        the gradient uses / of any decision, and route_namb [B], the number
        of decisions (sweep, class) the gradient uses that have several
        admissible routes (comparisons within opts.route_delta may go either
        way).  route=True adds the oracle's routes [K][M][B] int32 (-1: root
        or no parents; -2 - k: fp64 outcome k, other routes admissible).
        spread=True adds grad_cp_spread [N][B]: an elementwise bound on how
        far g_cp can move over all admissible routings (0 where none
        reaches)."""
        theta = np.ascontiguousarray(theta, dtype=np.float64)
        N, B = theta.shape
        assert N == self.N
        m = None if m is None else np.ascontiguousarray(m, dtype=np.float64)
        v = None if v is None else np.ascontiguousarray(v, dtype=np.float64)
        K = self.K_auto if opts.K < 0 else opts.K
        out = {
            "cp": np.zeros((N, B)), "p": np.zeros((N, B)), "f": np.zeros(B),
            "h": np.zeros(B // opts.G), "loss": np.zeros(1), "grad_cp": np.zeros((N, B)),
            "grad_theta": np.zeros((N, B)), "theta_out": np.zeros((N, B)),
            "m_out": np.zeros((N, B)), "v_out": np.zeros((N, B)),
            "choice": np.zeros((self.M, B), dtype=np.int32), "valid": np.zeros(B, dtype=np.uint8),
            "disc_cost": np.zeros(B), "reached": np.zeros((self.M, B), dtype=np.uint8),
        }
        if qstack:
            out["qstack"] = np.zeros((K + 1, self.M, B))
        out["route_margin"] = np.zeros(B)
        out["route_margin_all"] = np.zeros(B)
        out["route_namb"] = np.zeros(B, dtype=np.int32)
        if spread:
            out["grad_cp_spread"] = np.zeros((N, B))
        if route:
            out["route"] = np.zeros((K, self.M, B), dtype=np.int32)
        d = _Dump(**{k: _p(a) for k, a in out.items()})
        rc = lib().oracle_step(self.h, C.byref(self.cost), C.byref(opts.c()), B, _p(theta), _p(m),
                               _p(v), step_index, C.byref(d))
        if rc != 0:
            raise ValueError("oracle_step failed (G must divide B)")
        out["loss"] = float(out["loss"][0])
        out["K"] = K
        return out

    def decode(self, theta):
        theta = np.ascontiguousarray(theta, dtype=np.float64)
        N, B = theta.shape
        choice = np.zeros((self.M, B), dtype=np.int32)
        reached = np.zeros((self.M, B), dtype=np.uint8)
        valid = np.zeros(B, dtype=np.uint8)
        cost = np.zeros(B)
        lib().oracle_decode(self.h, C.byref(self.cost), B, _p(theta), _p(choice), _p(reached),
                            _p(valid), _p(cost))
        return {"choice": choice, "reached": reached, "valid": valid, "disc_cost": cost}

    def optimize(self, opts: Options, B: int, rng_key: int, seed_begin: int = 0, steps: int = 100,
                 patience: int = 0):
        best_cost = np.zeros(1)
        best_step = np.zeros(1, dtype=np.int32)
        best_seed = np.zeros(1, dtype=np.int64)
        best_choice = np.zeros(self.M, dtype=np.int32)
        n = lib().oracle_optimize(self.h, C.byref(self.cost), C.byref(opts.c()), B, rng_key,
                                  seed_begin, steps, patience, _p(best_cost), _p(best_step),
                                  _p(best_seed), _p(best_choice))
        return {"steps_run": n, "best_cost": float(best_cost[0]), "best_step": int(best_step[0]),
                "best_seed": int(best_seed[0]), "best_choice": best_choice}

"""Thin ctypes binding of libsmoothe.so (include/smoothe.h) -- argument
marshalling only; every step of the SmoothE path runs in the library's CUDA
kernels.  There is no CPU fallback: if the shared library is missing or the
GPU is unusable, these calls raise.

Names follow the C ABI: load_egraph, run_create, run_steps, optimize,
extract, debug_step (see include/smoothe.h for semantics and citations).
"""
from __future__ import annotations

import ctypes as C
import os
from dataclasses import dataclass, field

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("SMOOTHE_LIB") or os.path.join(_HERE, "libsmoothe.so")

OK, E_INVALID_ARG, E_BAD_GRAPH, E_OOM, E_CUDA, E_NO_VALID, E_STATE = range(7)
STATUS_NAMES = ["OK", "E_INVALID_ARG", "E_BAD_GRAPH", "E_OOM", "E_CUDA", "E_NO_VALID", "E_STATE"]
ASSUMPTIONS = {"independent": 0, "correlated": 1, "hybrid": 2}
COST_KINDS = {"linear": 0, "quadratic": 1, "mlp": 2}
PHASES = ["softmax", "forward", "cost", "penalty", "reverse", "update", "decode", "best"]


class SmootheError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{STATUS_NAMES[status] if 0 <= status < 7 else status}: {msg}")
        self.status = status


class _Info(C.Structure):
    _fields_ = [("num_classes", C.c_int32), ("num_nodes", C.c_int32), ("num_edges", C.c_int64),
                ("root", C.c_int32), ("K_auto", C.c_int32), ("num_scc", C.c_int32),
                ("scc_classes", C.c_int32), ("scc_max", C.c_int32), ("max_class_size", C.c_int32),
                ("max_in_degree", C.c_int32), ("device", C.c_int32), ("device_bytes", C.c_int64)]


class _Cost(C.Structure):
    _fields_ = [("kind", C.c_int), ("u", C.c_void_p), ("quad_nnz", C.c_int64),
                ("quad_i", C.c_void_p), ("quad_j", C.c_void_p), ("quad_w", C.c_void_p),
                ("mlp_hidden1", C.c_int32), ("mlp_hidden2", C.c_int32),
                ("W1", C.c_void_p), ("b1", C.c_void_p), ("W2", C.c_void_p), ("b2", C.c_void_p),
                ("W3", C.c_void_p), ("b3", C.c_void_p)]


class _Opts(C.Structure):
    _fields_ = [("assumption", C.c_int), ("prop_iters", C.c_int32), ("lam", C.c_double),
                ("penalty_group", C.c_int32), ("lr", C.c_double), ("beta1", C.c_double),
                ("beta2", C.c_double), ("eps", C.c_double), ("optimizer", C.c_int32),
                ("patience", C.c_int32), ("time_limit_s", C.c_double), ("rng_key", C.c_uint64),
                ("seed_begin", C.c_int64), ("cuda_stream", C.c_void_p), ("use_graphs", C.c_int32),
                ("converge", C.c_int32)]


class _Summary(C.Structure):
    _fields_ = [("best_cost", C.c_double), ("best_seed", C.c_int64), ("best_step", C.c_int32),
                ("valid", C.c_int32), ("steps_run", C.c_int32), ("K", C.c_int32),
                ("time_to_best_s", C.c_double), ("step_time_s", C.c_double),
                ("last_loss", C.c_double), ("pool_rows", C.c_int64), ("pool_peak_rows", C.c_int64),
                ("pool_grows", C.c_int32), ("graph_mode", C.c_int32)]


class _Dump(C.Structure):
    _fields_ = [(n, C.c_void_p) for n in
                ("cp", "qK", "p", "grad_cp", "grad_theta", "theta_out", "m_out", "v_out", "f", "h",
                 "loss", "choice", "reached", "valid", "disc_cost", "qstack", "route", "sweeps")]


class _Greedy(C.Structure):
    _fields_ = [("dag_cost", C.c_double), ("root_cost", C.c_double), ("valid", C.c_int32),
                ("selected_classes", C.c_int32)]


class _Profile(C.Structure):
    _fields_ = [("phase_ms", C.c_double * 8), ("phase_launches", C.c_int64 * 8),
                ("steps", C.c_int64), ("launches", C.c_int64), ("num_seeds_padded", C.c_int32),
                ("sweep_kernel_ms", C.c_double * 3), ("sweep_kernel_launches", C.c_int64 * 3),
                ("frozen_sweeps", C.c_int64), ("frozen_live_edges", C.c_int64),
                ("frozen_live_rows", C.c_int64), ("frozen_rows_written", C.c_int64)]


_lib = None

# every function the header declares, with its ctypes signature
_SIGS = {
    "smoothe_load_egraph": (C.c_int, [C.c_int32, C.c_int32, C.c_void_p, C.c_void_p, C.c_void_p,
                                      C.c_int32, C.c_int, C.POINTER(C.c_void_p)]),
    "smoothe_egraph_get_info": (C.c_int, [C.c_void_p, C.POINTER(_Info)]),
    "smoothe_egraph_get_scc": (C.c_int, [C.c_void_p, C.c_void_p]),
    "smoothe_options_default": (C.c_int, [C.POINTER(_Opts)]),
    "smoothe_run_create": (C.c_int, [C.c_void_p, C.POINTER(_Cost), C.c_int32, C.POINTER(_Opts),
                                     C.POINTER(C.c_void_p)]),
    "smoothe_run_steps": (C.c_int, [C.c_void_p, C.c_int32]),
    "smoothe_run_synchronize": (C.c_int, [C.c_void_p]),
    "smoothe_optimize": (C.c_int, [C.c_void_p, C.POINTER(_Cost), C.c_int32, C.c_int32,
                                   C.POINTER(_Opts), C.POINTER(C.c_void_p)]),
    "smoothe_extract": (C.c_int, [C.c_void_p, C.c_void_p, C.POINTER(_Summary)]),
    "smoothe_debug_step": (C.c_int, [C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p, C.c_int32,
                                     C.POINTER(_Dump)]),
    "smoothe_get_theta": (C.c_int, [C.c_void_p, C.c_void_p]),
    "smoothe_get_state": (C.c_int, [C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p]),
    "smoothe_run_get_trace": (C.c_int, [C.c_void_p, C.c_void_p, C.c_int32, C.c_void_p]),
    "smoothe_greedy": (C.c_int, [C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p,
                                 C.POINTER(_Greedy)]),
    "smoothe_run_warm_start": (C.c_int, [C.c_void_p, C.c_void_p, C.c_float]),
    "smoothe_run_profile": (C.c_int, [C.c_void_p, C.c_int32]),
    "smoothe_run_get_profile": (C.c_int, [C.c_void_p, C.POINTER(_Profile)]),
    "smoothe_last_error": (C.c_char_p, []),
    "smoothe_version": (C.c_char_p, []),
    "smoothe_free_run": (None, [C.c_void_p]),
    "smoothe_release_cached_memory": (None, [C.c_int]),
    "smoothe_free_egraph": (None, [C.c_void_p]),
}


def lib():
    """Load libsmoothe.so; raises if it has not been built (no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} not built: run __graft_entry__.build() "
                              "(make -C paper_conf_asplos_caiydyz25_b200)")
        L = C.CDLL(LIB_PATH)
        for name, (res, args) in _SIGS.items():
            fn = getattr(L, name)
            fn.restype = res
            fn.argtypes = args
        _lib = L
    return _lib


def _check(status):
    if status != OK:
        raise SmootheError(status, lib().smoothe_last_error().decode())


def _p(a):
    return None if a is None else a.ctypes.data


def _c(a, dtype):
    return None if a is None else np.ascontiguousarray(a, dtype=dtype)


class EGraph:
    """smoothe_load_egraph: CSR e-graph -> library handle."""

    def __init__(self, class_ptr, child_ptr, child_class, root=0, device=0):
        self._h = None
        cp_ = _c(class_ptr, np.int32)
        chp = _c(child_ptr, np.int64)
        chc = _c(child_class, np.int32)
        if chc.size == 0:
            chc = np.zeros(1, np.int32)
        h = C.c_void_p()
        _check(lib().smoothe_load_egraph(len(cp_) - 1, len(chp) - 1, _p(cp_), _p(chp), _p(chc),
                                         int(root), int(device), C.byref(h)))
        self._h = h
        info = _Info()
        _check(lib().smoothe_egraph_get_info(h, C.byref(info)))
        self.info = {n: getattr(info, n) for n, _ in _Info._fields_}
        self.M, self.N = info.num_classes, info.num_nodes
        self.K_auto = info.K_auto

    def greedy(self, u):
        """smoothe_greedy: the paper's worklist heuristic on the
        device.  Returns (choice [M] int32, -1 outside the extraction,
        class_cost [M], result dict)."""
        ud = _c(u, np.float64)
        assert ud.shape == (self.N,)
        choice = np.zeros(self.M, np.int32)
        cost = np.zeros(self.M)
        r = _Greedy()
        _check(lib().smoothe_greedy(self._h, _p(ud), _p(choice), _p(cost), C.byref(r)))
        return choice, cost, {n: getattr(r, n) for n, _ in _Greedy._fields_}

    def scc(self):
        out = np.zeros(self.M, np.int32)
        _check(lib().smoothe_egraph_get_scc(self._h, _p(out)))
        return out

    def close(self):
        if self._h:
            lib().smoothe_free_egraph(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def load_egraph(class_ptr, child_ptr, child_class, root=0, device=0) -> EGraph:
    return EGraph(class_ptr, child_ptr, child_class, root, device)


def load_egraph_from(eg, device=0) -> EGraph:
    """Convenience: any object with class_ptr / child_ptr / child_class / root."""
    return EGraph(eg.class_ptr, eg.child_ptr, eg.child_class, eg.root, device)


@dataclass
class CostModel:
    """smoothe_cost_model (reading S24)."""
    u: np.ndarray
    quad: tuple | None = None
    mlp: dict | None = None
    _keep: list = field(default_factory=list, repr=False)

    @property
    def kind(self):
        return "mlp" if self.mlp is not None else "quadratic" if self.quad is not None else "linear"

    @classmethod
    def from_input(cls, eg):
        return cls(eg.u, eg.quad, eg.mlp)

    def c(self) -> _Cost:
        c = _Cost()
        u = _c(self.u, np.float64)
        self._keep = [u]
        c.kind = COST_KINDS[self.kind]
        c.u = _p(u)
        if self.quad is not None:
            qi, qj, qw = _c(self.quad[0], np.int32), _c(self.quad[1], np.int32), _c(self.quad[2], np.float64)
            self._keep += [qi, qj, qw]
            c.quad_nnz, c.quad_i, c.quad_j, c.quad_w = qi.size, _p(qi), _p(qj), _p(qw)
        if self.mlp is not None:
            ws = {k: _c(v, np.float32) for k, v in self.mlp.items()}
            self._keep += list(ws.values())
            c.mlp_hidden1, c.mlp_hidden2 = ws["W1"].shape[0], ws["W2"].shape[0]
            c.W1, c.b1, c.W2, c.b2, c.W3, c.b3 = (_p(ws[k]) for k in ("W1", "b1", "W2", "b2", "W3", "b3"))
        return c


@dataclass
class Options:
    """smoothe_options; defaults = smoothe_options_default()."""
    assumption: str = "hybrid"
    prop_iters: int = -1
    lam: float = 1.0
    penalty_group: int = 1
    lr: float = 0.1
    beta1: float = 0.9
    beta2: float = 0.999
    eps: float = 1e-8
    optimizer: str = "adam"
    patience: int = 0
    time_limit_s: float = 0.0
    rng_key: int = 0
    seed_begin: int = 0
    cuda_stream: int | None = None
    use_graphs: bool = True
    converge: bool = False

    def c(self) -> _Opts:
        return _Opts(ASSUMPTIONS[self.assumption], self.prop_iters, self.lam, self.penalty_group,
                     self.lr, self.beta1, self.beta2, self.eps, 0 if self.optimizer == "adam" else 1,
                     self.patience, self.time_limit_s, self.rng_key, self.seed_begin,
                     self.cuda_stream, 1 if self.use_graphs else 0, 1 if self.converge else 0)


def torch_stream():
    """The current torch CUDA stream handle (int) or None."""
    try:
        import torch
        if torch.cuda.is_available():
            return torch.cuda.current_stream().cuda_stream
    except Exception:
        pass
    return None


class Run:
    """A batch of B seeds being optimised (smoothe_run)."""

    def __init__(self, egraph: EGraph, cost: CostModel, num_seeds: int, options: Options, _h=None):
        self.egraph, self.cost, self.B, self.options = egraph, cost, int(num_seeds), options
        self._h = _h
        if _h is None:
            h = C.c_void_p()
            c = cost.c()
            o = options.c()
            _check(lib().smoothe_run_create(egraph._h, C.byref(c), self.B, C.byref(o), C.byref(h)))
            self._h = h
        self.K = options.prop_iters if options.prop_iters >= 0 else egraph.K_auto

    def steps(self, n: int):
        _check(lib().smoothe_run_steps(self._h, int(n)))

    def synchronize(self):
        _check(lib().smoothe_run_synchronize(self._h))

    def summary(self):
        """smoothe_extract without the extraction: the summary dict alone."""
        s = _Summary()
        st = lib().smoothe_extract(self._h, None, C.byref(s))
        if st not in (OK, E_NO_VALID):
            _check(st)
        return {n: getattr(s, n) for n, _ in _Summary._fields_}

    def extract(self):
        """(choice [M] int32 with -1 for unselected classes, summary dict)."""
        choice = np.zeros(self.egraph.M, np.int32)
        s = _Summary()
        st = lib().smoothe_extract(self._h, _p(choice), C.byref(s))
        if st not in (OK, E_NO_VALID):
            _check(st)
        return choice, {n: getattr(s, n) for n, _ in _Summary._fields_}

    def warm_start(self, choice, bias: float):
        """smoothe_run_warm_start: theta_k += bias at the chosen e-nodes."""
        ch = _c(choice, np.int32)
        assert ch.shape == (self.egraph.M,)
        _check(lib().smoothe_run_warm_start(self._h, _p(ch), float(bias)))

    def theta(self):
        out = np.zeros((self.egraph.N, self.B), np.float32)
        _check(lib().smoothe_get_theta(self._h, _p(out)))
        return out

    def trace(self, max_steps: int = 4096):
        """smoothe_run_get_trace: per-step relaxed vs sampled cost, dict of
        arrays (relaxed_min, relaxed_mean, sampled_min, valid)."""
        out = np.zeros((max_steps, 4), np.float64)
        n = C.c_int32(0)
        _check(lib().smoothe_run_get_trace(self._h, _p(out), int(max_steps), C.byref(n)))
        t = out[: n.value]
        return {"relaxed_min": t[:, 0], "relaxed_mean": t[:, 1], "sampled_min": t[:, 2],
                "valid": t[:, 3].astype(np.int64)}

    def state(self):
        """smoothe_get_state: (theta, m, v) [N][B] float32 and the steps run."""
        th, m, v = (np.zeros((self.egraph.N, self.B), np.float32) for _ in range(3))
        n = C.c_int32(0)
        _check(lib().smoothe_get_state(self._h, _p(th), _p(m), _p(v), C.byref(n)))
        return th, m, v, n.value

    def debug_step(self, theta=None, m=None, v=None, step_index=0, qstack=False, route=False):
        N, M, B = self.egraph.N, self.egraph.M, self.B
        G = self.options.penalty_group
        out = {k: np.zeros((N, B), np.float32) for k in
               ("cp", "p", "grad_cp", "grad_theta", "theta_out", "m_out", "v_out")}
        out.update(qK=np.zeros((M, B), np.float32), f=np.zeros(B), h=np.zeros(B // G),
                   loss=np.zeros(1), choice=np.zeros((M, B), np.int32),
                   reached=np.zeros((M, B), np.uint8), valid=np.zeros(B, np.uint8),
                   disc_cost=np.zeros(B), sweeps=np.zeros(B, np.int32))
        if qstack:
            out["qstack"] = np.zeros((self.K + 1, M, B), np.float32)
        if route:
            out["route"] = np.zeros((self.K, M, B), np.int32)
        d = _Dump(**{k: _p(a) for k, a in out.items()})
        th, mm, vv = _c(theta, np.float32), _c(m, np.float32), _c(v, np.float32)
        _check(lib().smoothe_debug_step(self._h, _p(th), _p(mm), _p(vv), int(step_index), C.byref(d)))
        out["loss"] = float(out["loss"][0])
        return out

    def profile(self, enable=True):
        _check(lib().smoothe_run_profile(self._h, 1 if enable else 0))

    def get_profile(self):
        p = _Profile()
        _check(lib().smoothe_run_get_profile(self._h, C.byref(p)))
        return {"phase_ms": dict(zip(PHASES, list(p.phase_ms))),
                "phase_launches": dict(zip(PHASES, list(p.phase_launches))),
                "steps": p.steps, "launches": p.launches, "num_seeds_padded": p.num_seeds_padded,
                "sweep_kernel_ms": {"forward": p.sweep_kernel_ms[0], "reverse": p.sweep_kernel_ms[1],
                                    "frozen": p.sweep_kernel_ms[2]},
                "sweep_kernel_launches": {"forward": p.sweep_kernel_launches[0],
                                          "reverse": p.sweep_kernel_launches[1],
                                          "frozen": p.sweep_kernel_launches[2]},
                "frozen_sweeps": p.frozen_sweeps, "frozen_live_edges": p.frozen_live_edges,
                "frozen_live_rows": p.frozen_live_rows,
                "frozen_rows_written": p.frozen_rows_written}

    def close(self):
        if self._h:
            lib().smoothe_free_run(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def run_create(egraph, cost, num_seeds, options=None) -> Run:
    return Run(egraph, cost, num_seeds, options or Options())


def optimize(egraph, cost, num_seeds, steps, options=None) -> Run:
    """smoothe_optimize: create a run, take `steps` steps, wait."""
    options = options or Options()
    h = C.c_void_p()
    c = cost.c()
    o = options.c()
    _check(lib().smoothe_optimize(egraph._h, C.byref(c), int(num_seeds), int(steps), C.byref(o),
                                  C.byref(h)))
    return Run(egraph, cost, num_seeds, options, _h=h)


def extract(run: Run):
    return run.extract()


def release_cached_memory(device: int = -1):
    """smoothe_release_cached_memory: return the recycled run blocks to the driver."""
    lib().smoothe_release_cached_memory(int(device))


def version() -> str:
    return lib().smoothe_version().decode()

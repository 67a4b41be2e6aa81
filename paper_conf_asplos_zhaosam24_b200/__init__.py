"""Python binding of libfelix (include/felix.h): argument marshalling only.

Every step of the hot path runs in libfelix's CUDA kernels (tcgen05 GEMMs, NVRTC-generated DAG
kernels, rounding / scoring / top-k kernels).  PyTorch supplies device memory and streams.  There
is no CPU fallback: importing this package without the built extension raises, and every device
call needs an sm_100a GPU.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass
from typing import Optional, Sequence

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libfelix.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(f"libfelix.so not built at {LIB_PATH}; run __graft_entry__.build() "
                      f"(python paper_conf_asplos_zhaosam24_b200/_build.py)")
_lib = ctypes.CDLL(LIB_PATH)

FELIX_STATUS = {0: "OK", 1: "INVALID_ARG", 2: "INVALID_DAG", 3: "SHAPE", 4: "UNSUPPORTED", 5: "CUDA",
                6: "NVRTC", 7: "OOM"}

EXPORTED = ["felix_last_error", "felix_abi_version", "felix_space_create", "felix_space_destroy",
            "felix_space_info", "felix_codegen", "felix_costmodel_load", "felix_costmodel_destroy",
            "felix_search", "felix_round_topk", "felix_eval", "felix_round", "felix_score",
            "felix_init_sample", "felix_profile_enable", "felix_profile_read", "felix_profile_reset",
            "felix_debug_trace", "felix_history_topk", "felix_space_set_statements", "felix_search_group",
            "felix_eval_ex", "felix_tune", "felix_merge_topk"]


class FelixError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"felix {FELIX_STATUS.get(status, status)}: {msg}")
        self.status = status


class _Var(ctypes.Structure):
    _fields_ = [("kind", ctypes.c_int32), ("_pad", ctypes.c_int32), ("lo", ctypes.c_int64), ("hi", ctypes.c_int64)]


class _Split(ctypes.Structure):
    _fields_ = [("extent", ctypes.c_int64), ("n", ctypes.c_int32), ("_pad", ctypes.c_int32),
                ("vars", ctypes.POINTER(ctypes.c_int32))]


class _SearchParams(ctypes.Structure):
    _fields_ = [("n_seeds", ctypes.c_int64), ("n_steps", ctypes.c_int32), ("lr", ctypes.c_float),
                ("beta1", ctypes.c_float), ("beta2", ctypes.c_float), ("eps", ctypes.c_float),
                ("lam", ctypes.c_float), ("rng_seed", ctypes.c_uint64), ("init_from_y", ctypes.c_int32),
                ("history", ctypes.c_int32), ("index_base", ctypes.c_int64)]


class _EvalOut(ctypes.Structure):
    _fields_ = [("phi", ctypes.c_void_p), ("g", ctypes.c_void_p), ("cost", ctypes.c_void_p), ("loss", ctypes.c_void_p),
                ("grad", ctypes.c_void_p), ("F", ctypes.c_void_p), ("search_path", ctypes.c_int32),
                ("_pad", ctypes.c_int32)]


class _SpaceInfo(ctypes.Structure):
    _fields_ = [("n_vars", ctypes.c_int32), ("n_nodes", ctypes.c_int32), ("n_features", ctypes.c_int32),
                ("n_constraints_user", ctypes.c_int32), ("n_roots_total", ctypes.c_int32),
                ("n_components", ctypes.c_int32), ("n_tuples_total", ctypes.c_int64), ("nvrtc_ms", ctypes.c_double),
                ("regs_fwd", ctypes.c_int32), ("regs_rev", ctypes.c_int32), ("dag_flops_fwd", ctypes.c_int64),
                ("dag_flops_rev", ctypes.c_int64)]


_P = ctypes.c_void_p
_lib.felix_last_error.restype = ctypes.c_char_p
_lib.felix_abi_version.restype = ctypes.c_int32
for _name in EXPORTED:
    if _name not in ("felix_last_error", "felix_abi_version", "felix_space_destroy", "felix_costmodel_destroy"):
        getattr(_lib, _name).restype = ctypes.c_int
_lib.felix_space_destroy.restype = None
_lib.felix_costmodel_destroy.restype = None


def _check_tensor(t, shape, dtype_name: str, device_index: int, what: str) -> None:
    """Argument validation before a pointer crosses the ABI: a CUDA tensor on the handle's device,
    of the given dtype, contiguous, of exactly `shape`."""
    import torch
    dt = getattr(torch, dtype_name)
    if not (isinstance(t, torch.Tensor) and t.is_cuda and t.dtype == dt and t.is_contiguous()
            and tuple(t.shape) == tuple(shape) and t.device.index == device_index):
        got = (tuple(t.shape), t.dtype, str(t.device)) if isinstance(t, torch.Tensor) else type(t)
        raise FelixError(1, f"{what} must be a contiguous {dtype_name} CUDA tensor {tuple(shape)} on cuda:{device_index}, got {got}")


def _check(status: int) -> None:
    if status != 0:
        raise FelixError(status, _lib.felix_last_error().decode(errors="replace"))


def _ptr(t) -> int:
    return 0 if t is None else int(t.data_ptr())


def _stream(stream) -> int:
    import torch
    if stream is None:
        stream = torch.cuda.current_stream()
    return int(stream.cuda_stream)


def _space_args(space):
    """Marshal a felix_inputs.Space-like object (vars, splits, nodes, feature_roots, constraint_roots)."""
    vars_ = (_Var * len(space.vars))()
    for j, v in enumerate(space.vars):
        vars_[j].kind, vars_[j].lo, vars_[j].hi = int(v.kind), int(v.lo), int(v.hi)
    keep = []
    splits = (_Split * max(1, len(space.splits)))()
    for s, sp in enumerate(space.splits):
        arr = (ctypes.c_int32 * len(sp.vars))(*[int(j) for j in sp.vars])
        keep.append(arr)
        splits[s].extent, splits[s].n = int(sp.extent), len(sp.vars)
        splits[s].vars = ctypes.cast(arr, ctypes.POINTER(ctypes.c_int32))
    nodes = np.ascontiguousarray(space.nodes)
    assert nodes.dtype.itemsize == 24
    fr = np.ascontiguousarray(space.feature_roots, dtype=np.int32)
    cr = np.ascontiguousarray(space.constraint_roots, dtype=np.int32)
    keep += [nodes, fr, cr]
    args = [vars_, len(space.vars), splits, len(space.splits), nodes.ctypes.data_as(_P), len(nodes),
            fr.ctypes.data_as(_P), len(fr), cr.ctypes.data_as(_P) if len(cr) else None, len(cr)]
    return args, keep


def search_group(spaces: Sequence["Space"], cm: "CostModel", ys, n_steps: int, *, lr=0.05, beta1=0.9, beta2=0.999,
                 eps=1e-8, lam=1.0, rng_seeds: Sequence[int] = None, index_bases: Sequence[int] = None,
                 init_from_y: bool = True, final_losses=None, stream=None):
    """felix_search_group: the spaces' searches in lock-step with one MLP pass per Adam step over the
    candidates of all of them (shared cost model).  ys[i]: device fp32 [n_vars_i, n_i], updated in place."""
    G = len(spaces)
    if G == 0:
        return ys
    if len(ys) != G:
        raise FelixError(1, "len(ys) != len(spaces)")
    for sp, y in zip(spaces, ys):
        sp._check_y(y)
    if final_losses is not None:
        if len(final_losses) != G:
            raise FelixError(1, "len(final_losses) != len(spaces)")
        for sp, y, l in zip(spaces, ys, final_losses):
            if l is not None:
                _check_tensor(l, (y.shape[1],), "float32", sp.device, "final_losses[i]")
    seeds = list(rng_seeds) if rng_seeds is not None else [0] * G
    bases = list(index_bases) if index_bases is not None else [0] * G
    params = (_SearchParams * G)()
    for i, y in enumerate(ys):
        params[i] = _SearchParams(int(y.shape[1]), int(n_steps), lr, beta1, beta2, eps, lam, int(seeds[i]) & (2**64 - 1),
                                  1 if init_from_y else 0, 0, int(bases[i]))
    hs = (_P * G)(*[sp._h.value for sp in spaces])
    yp = (_P * G)(*[_ptr(y) for y in ys])
    lp = (_P * G)(*[_ptr(l) for l in final_losses]) if final_losses is not None else None
    _check(_lib.felix_search_group(hs, G, cm._h, params, yp, lp, _P(_stream(stream))))
    return ys


_TUNE_KEYS = ("mlp", "cone_width", "replicas", "sc_warps", "chunks", "split_cone", "tile_cta_group", "chain_cta_group", "dphi_ksplit",
              "codegen_cone_width", "codegen_replicas", "trace", "round_bnb", "graph_steps", "pdl", "score_dmma", "dphi_tma")
_TUNE_DEFAULT = {k: (0 if k in ("trace", "round_bnb") else -1) for k in _TUNE_KEYS}


def merge_topk(key, score, sched, k: int):
    """felix_merge_topk: deterministic merge of gathered top-k records (host arrays; rows with key < 0
    are empty).  Returns (key int64 [m], score float64 [m], sched int32 [m, n_vars]), m <= k."""
    import numpy as np
    key = np.ascontiguousarray(key, dtype=np.int64)
    score = np.ascontiguousarray(score, dtype=np.float64)
    sched = np.ascontiguousarray(sched, dtype=np.int32)
    if sched.ndim != 2 or key.shape != (sched.shape[0],) or score.shape != key.shape:
        raise FelixError(1, "merge_topk: key [R], score [R], sched [R, n_vars] expected")
    n_vars = max(int(sched.shape[1]), 1)
    ko = np.zeros(k, np.int64)
    so = np.zeros(k, np.float64)
    xo = np.zeros((k, n_vars), np.int32)
    m = ctypes.c_int32(0)
    _check(_lib.felix_merge_topk(key.ctypes.data_as(_P), score.ctypes.data_as(_P), sched.ctypes.data_as(_P),
                                 ctypes.c_int64(key.shape[0]), ctypes.c_int32(n_vars), ctypes.c_int32(k),
                                 ko.ctypes.data_as(_P), so.ctypes.data_as(_P), xo.ctypes.data_as(_P), ctypes.byref(m)))
    return ko[:m.value], so[:m.value], xo[:m.value]


def tune(**knobs) -> None:
    """felix_tune: process-wide execution knobs (experiments / tests), e.g. tune(mlp=1, cone_width=8).
    MLP modes may be given by name: mlp="tile" | "chain" | "layers" | "auto"."""
    for k, v in knobs.items():
        if k == "mlp" and isinstance(v, str):
            v = {"auto": -1, "tile": 0, "chain": 1, "layers": 2}[v]
        _check(_lib.felix_tune(k.encode(), ctypes.c_int32(int(v))))


class tuned:
    """Context manager: set knobs for a block, restore the defaults afterwards."""

    def __init__(self, **knobs):
        self.knobs = knobs

    def __enter__(self):
        tune(**self.knobs)
        return self

    def __exit__(self, *exc):
        tune(**{k: _TUNE_DEFAULT[k] for k in self.knobs})
        return False


def abi_version() -> int:
    return int(_lib.felix_abi_version())


def codegen(space, compile: bool = False) -> str:
    """Generated CUDA source of a space's expression kernels (device-free; compile=True also runs
    NVRTC for sm_100a)."""
    args, keep = _space_args(space)
    ns = int(getattr(space, "n_statements", 1))
    n = ctypes.c_int64(0)
    _check(_lib.felix_codegen(*args, ns, 0, None, ctypes.c_int64(0), ctypes.byref(n)))
    buf = ctypes.create_string_buffer(n.value + 1)
    _check(_lib.felix_codegen(*args, ns, int(compile), buf, ctypes.c_int64(n.value + 1), ctypes.byref(n)))
    return buf.value.decode()


@dataclass
class SpaceInfo:
    n_vars: int
    n_nodes: int
    n_features: int
    n_constraints_user: int
    n_roots_total: int
    n_components: int
    n_tuples_total: int
    nvrtc_ms: float
    regs_fwd: int
    regs_rev: int
    dag_flops_fwd: int
    dag_flops_rev: int


class CostModel:
    """felix_costmodel_load: MLP dims [d0, ..., 1], W[l] fp32 [d_{l+1}, d_l], b[l] fp32 [d_{l+1}]."""

    def __init__(self, dims: Sequence[int], W: Sequence[np.ndarray], b: Sequence[np.ndarray], device: int = 0):
        L = len(dims) - 1
        Ws = [np.ascontiguousarray(w, dtype=np.float32) for w in W]
        bs = [np.ascontiguousarray(x, dtype=np.float32) for x in b]
        d = (ctypes.c_int32 * (L + 1))(*[int(x) for x in dims])
        wp = (_P * L)(*[w.ctypes.data for w in Ws])
        bp = (_P * L)(*[x.ctypes.data for x in bs])
        h = _P()
        _check(_lib.felix_costmodel_load(int(device), L, d, wp, bp, ctypes.byref(h)))
        self._h = h
        self.dims = tuple(int(x) for x in dims)
        self.device = device

    @classmethod
    def from_weights(cls, mlp, device: int = 0) -> "CostModel":
        return cls(mlp.dims, mlp.W, mlp.b, device)

    def __del__(self):
        h = getattr(self, "_h", None)
        if h and _lib is not None:
            _lib.felix_costmodel_destroy(h)
            self._h = None

    def mlp_flops_per_candidate_step(self) -> int:
        """Forward + input-gradient backward: 4 * sum d_l d_{l+1}."""
        return 4 * sum(self.dims[l] * self.dims[l + 1] for l in range(len(self.dims) - 1))


class Space:
    """felix_space_create + the search / rounding / scoring calls on it."""

    def __init__(self, space, device: int = 0):
        args, keep = _space_args(space)
        h = _P()
        _check(_lib.felix_space_create(int(device), *args, ctypes.byref(h)))
        self._h = h
        self.n_statements = int(getattr(space, "n_statements", 1))
        if self.n_statements != 1:
            _check(_lib.felix_space_set_statements(self._h, self.n_statements))
        self.device = device
        self.n_vars = len(space.vars)
        self.name = getattr(space, "name", "space")
        inf = _SpaceInfo()
        _check(_lib.felix_space_info(self._h, ctypes.byref(inf)))
        self.info = SpaceInfo(*[getattr(inf, f) for f, _ in _SpaceInfo._fields_])

    def __del__(self):
        h = getattr(self, "_h", None)
        if h and _lib is not None:
            _lib.felix_space_destroy(h)
            self._h = None

    # ---------------------------------------------------------------- primary calls
    def search(self, cm: CostModel, y, n_steps: int, *, lr=0.05, beta1=0.9, beta2=0.999, eps=1e-8, lam=1.0,
               rng_seed: int = 0, init_from_y: bool = True, index_base: int = 0, final_loss=None, history=False,
               stream=None):
        """felix_search on device y (torch fp32 [n_vars, n], updated in place).  history=True also records
        varValuesHistory (Alg. 1 l.13/17) for history_topk."""
        self._check_y(y)
        if final_loss is not None:
            _check_tensor(final_loss, (y.shape[1],), "float32", self.device, "final_loss")
        p = _SearchParams(int(y.shape[1]), int(n_steps), lr, beta1, beta2, eps, lam, int(rng_seed) & (2**64 - 1),
                          1 if init_from_y else 0, 1 if history else 0, int(index_base))
        _check(_lib.felix_search(self._h, cm._h, ctypes.byref(p), _P(_ptr(y)), _P(_ptr(final_loss)),
                                 _P(_stream(stream))))
        return y

    def round_topk(self, cm: CostModel, y, k: int, index_base: int = 0, stream=None):
        """felix_round_topk -> (idx int64 [m], score float64 [m], sched int32 [m, n_vars]) on the host."""
        self._check_y(y)
        idx = np.zeros(k, dtype=np.int64)
        sc = np.zeros(k, dtype=np.float64)
        sched = np.zeros((k, self.n_vars), dtype=np.int32)
        cnt = ctypes.c_int32(0)
        _check(_lib.felix_round_topk(self._h, cm._h, _P(_ptr(y)), ctypes.c_int64(y.shape[1]),
                                     ctypes.c_int64(index_base), int(k), idx.ctypes.data_as(_P),
                                     sc.ctypes.data_as(_P), sched.ctypes.data_as(_P), ctypes.byref(cnt),
                                     _P(_stream(stream))))
        m = cnt.value
        return idx[:m], sc[:m], sched[:m]

    def history_topk(self, cm: CostModel, k: int, stream=None):
        """felix_history_topk over the last search(history=True) -> (idx int64 [m], step int32 [m],
        score float64 [m], sched int32 [m, n_vars], n_unique) on the host."""
        idx = np.zeros(k, dtype=np.int64)
        step = np.zeros(k, dtype=np.int32)
        sc = np.zeros(k, dtype=np.float64)
        sched = np.zeros((k, self.n_vars), dtype=np.int32)
        cnt = ctypes.c_int32(0)
        nu = ctypes.c_int64(0)
        _check(_lib.felix_history_topk(self._h, cm._h, int(k), idx.ctypes.data_as(_P), step.ctypes.data_as(_P),
                                       sc.ctypes.data_as(_P), sched.ctypes.data_as(_P), ctypes.byref(cnt),
                                       ctypes.byref(nu), _P(_stream(stream))))
        m = cnt.value
        return idx[:m], step[:m], sc[:m], sched[:m], int(nu.value)

    # ---------------------------------------------------------------- test hooks
    def eval(self, cm: CostModel, y, lam: float = 1.0, stream=None, features: bool = False):
        """felix_eval(_ex): phi, g, cost, loss, grad at y; features=True adds the raw smoothed features
        F (float64 [n_features, n])."""
        import torch
        self._check_y(y)
        n = y.shape[1]
        dev = y.device
        out = dict(
            phi=torch.empty((self.info.n_features, n), dtype=torch.float32, device=dev),
            g=torch.empty((self.info.n_roots_total, n), dtype=torch.float32, device=dev),
            cost=torch.empty(n, dtype=torch.float32, device=dev),
            loss=torch.empty(n, dtype=torch.float32, device=dev),
            grad=torch.empty((self.n_vars, n), dtype=torch.float32, device=dev),
        )
        if features:
            out["F"] = torch.empty((self.info.n_features, n), dtype=torch.float64, device=dev)
        eo = _EvalOut(*[_ptr(out.get(k)) for k in ("phi", "g", "cost", "loss", "grad", "F")], 0, 0)
        _check(_lib.felix_eval_ex(self._h, cm._h, _P(_ptr(y)), ctypes.c_int64(n), ctypes.c_float(lam),
                                  ctypes.byref(eo), _P(_stream(stream))))
        return out

    def eval_search_path(self, cm: CostModel, y, lam: float = 1.0, stream=None):
        """felix_eval_ex(search_path=1): loss and dL/dy through the kernels of one felix_search Adam step
        (split-cone partial adjoints summed as the search's Adam prologue sums them)."""
        import torch
        self._check_y(y)
        n = y.shape[1]
        out = dict(loss=torch.empty(n, dtype=torch.float32, device=y.device),
                   grad=torch.empty((self.n_vars, n), dtype=torch.float32, device=y.device))
        eo = _EvalOut(0, 0, 0, _ptr(out["loss"]), _ptr(out["grad"]), 0, 1, 0)
        _check(_lib.felix_eval_ex(self._h, cm._h, _P(_ptr(y)), ctypes.c_int64(n), ctypes.c_float(lam),
                                  ctypes.byref(eo), _P(_stream(stream))))
        return out

    def round(self, y, stream=None):
        import torch
        self._check_y(y)
        n = y.shape[1]
        sched = torch.empty((n, self.n_vars), dtype=torch.int32, device=y.device)
        valid = torch.empty(n, dtype=torch.uint8, device=y.device)
        _check(_lib.felix_round(self._h, _P(_ptr(y)), ctypes.c_int64(n), _P(_ptr(sched)), _P(_ptr(valid)),
                                _P(_stream(stream))))
        return sched, valid

    def score(self, cm: CostModel, sched, stream=None):
        import torch
        n = sched.shape[0] if hasattr(sched, "shape") else 0
        _check_tensor(sched, (n, self.n_vars), "int32", self.device, "sched")
        out = torch.empty(n, dtype=torch.float64, device=sched.device)
        _check(_lib.felix_score(self._h, cm._h, _P(_ptr(sched)), ctypes.c_int64(n), _P(_ptr(out)),
                                _P(_stream(stream))))
        return out

    def init_sample(self, n: int, rng_seed: int, index_base: int = 0, device=None, stream=None):
        import torch
        y = torch.empty((self.n_vars, n), dtype=torch.float32, device=device or f"cuda:{self.device}")
        _check(_lib.felix_init_sample(self._h, ctypes.c_int64(n), ctypes.c_uint64(int(rng_seed) & (2**64 - 1)),
                                      ctypes.c_int64(index_base), _P(_ptr(y)), _P(_stream(stream))))
        return y

    def profile(self, enable: bool) -> None:
        _check(_lib.felix_profile_enable(self._h, 1 if enable else 0))

    def profile_read(self):
        ms = (ctypes.c_double * 4)()
        ln = (ctypes.c_int64 * 4)()
        _check(_lib.felix_profile_read(self._h, ms, ln))
        names = ("dag_fwd", "mlp_gemm", "dag_rev_adam", "init")
        return {nm: (ms[i], ln[i]) for i, nm in enumerate(names)}

    def profile_reset(self) -> None:
        _check(_lib.felix_profile_reset(self._h))

    def debug_trace(self, warps: bool = False):
        """uint64 [2][8192][8] globaltimer stamps (kernels generated after tune(trace=1)); warps=True also
        returns the forward kernel's per-warp cone-end stamps [8192][16]."""
        out = np.zeros(2 * 8192 * 8 + (8192 * 16 if warps else 0), dtype=np.uint64)
        _check(_lib.felix_debug_trace(self._h, out.ctypes.data_as(_P), ctypes.c_int64(out.size)))
        tr = out[:2 * 8192 * 8].reshape(2, 8192, 8)
        return (tr, out[2 * 8192 * 8:].reshape(8192, 16)) if warps else tr

    def _check_y(self, y) -> None:
        import torch
        if not (isinstance(y, torch.Tensor) and y.is_cuda and y.dtype == torch.float32 and y.dim() == 2
                and y.shape[0] == self.n_vars and y.is_contiguous() and y.device.index == self.device):
            raise FelixError(1, f"y must be a contiguous CUDA float32 tensor [{self.n_vars}, n] on cuda:{self.device}")

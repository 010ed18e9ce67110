"""ORACLE for the DGR solver iteration — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its ``cpu_baseline`` leg and
``--impl reference``) may import this package.  The product package
``paper_conf_dac_0159layhrr24_b200`` never imports it, and the two share no code.

``dgr_oracle.c`` is a plain fp64, single-threaded C implementation written from
/root/reference/PAPER.md (see the header of that file for the equation-by-equation
citations).  This module is argument marshalling only (ctypes + numpy).

Parity-pinned functions (tests/test_oracle_*.py): Philox (known-answer vectors),
Gumbel-softmax (sum to one, textbook softmax, shift invariance), demand (one-hot ==
integer rasterisation, conservation, brute-force expectation), loss (closed form,
brute force), reverse (central finite differences, torch autograd), Adam
(torch.optim.Adam), induction (a3 = 0 closed form, sort rules, top_p edge cases).
"Parity unpinned": the 100-iteration trajectory itself (the paper prints no values;
only quality properties are checked) — see DESIGN.md §3.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "dgr_oracle.c")
_SRC_FOREST = os.path.join(_HERE, "forest_oracle.c")   # row f1: DAG-forest construction
_LIB = os.path.join(_HERE, "liboracle.so")
_LIB32 = os.path.join(_HERE, "liboracle32.so")   # conditioning probe only (same source, real = float)
_libs = {}


def build(verbose: bool = False) -> str:
    for out, extra in ((_LIB, []), (_LIB32, ["-DODGR_REAL=float"])):
        cmd = ["gcc", "-O2", "-std=c11", "-shared", "-fPIC", *extra, "-o", out, _SRC, _SRC_FOREST, "-lm"]
        if verbose:
            print(" ".join(cmd))
        subprocess.check_call(cmd)
    return _LIB


class Weights(ctypes.Structure):
    """a1, a2, a3, beta (Q3), L (Q4), f kind/slope (Q2)."""
    _fields_ = [("a_wl", ctypes.c_double), ("a_via", ctypes.c_double), ("a_of", ctypes.c_double),
                ("beta", ctypes.c_double), ("n_layers", ctypes.c_double), ("f_kind", ctypes.c_int32),
                ("f_slope", ctypes.c_double)]


def weights(a_wl=0.5, a_via=4.0, a_of=500.0, beta=0.25, n_layers=5.0, f_kind=0, f_slope=1.0) -> Weights:
    return Weights(a_wl, a_via, a_of, beta, n_layers, f_kind, f_slope)


_dp = np.ctypeslib.ndpointer(dtype=np.float64, flags="C_CONTIGUOUS")
_i32 = np.ctypeslib.ndpointer(dtype=np.int32, flags="C_CONTIGUOUS")
_i64 = np.ctypeslib.ndpointer(dtype=np.int64, flags="C_CONTIGUOUS")
_f32 = np.ctypeslib.ndpointer(dtype=np.float32, flags="C_CONTIGUOUS")
_u32 = np.ctypeslib.ndpointer(dtype=np.uint32, flags="C_CONTIGUOUS")


def _load(fp32: bool = False):
    path = _LIB32 if fp32 else _LIB
    if path not in _libs:
        if not os.path.exists(path) or os.path.getmtime(path) < max(os.path.getmtime(_SRC), os.path.getmtime(_SRC_FOREST)):
            build()
        L = ctypes.CDLL(path)
        vp, c = ctypes.c_void_p, ctypes
        L.odgr_philox4x32_10.argtypes = [_u32, _u32, _u32]
        L.odgr_uniform.argtypes = [c.c_uint64, c.c_uint64, c.c_uint64, c.c_uint32]
        L.odgr_uniform.restype = c.c_double
        L.odgr_gumbel.argtypes = [c.c_uint64, c.c_uint64, c.c_uint64, c.c_uint32]
        L.odgr_gumbel.restype = c.c_double
        L.odgr_new.restype = vp
        L.odgr_new.argtypes = [c.c_int32, c.c_int32] + [c.c_int64] * 6 + [_i64] * 5 + [_i32, _i32] + \
            [_f32] * 4 + [c.c_uint64]
        L.odgr_free.argtypes = [vp]
        L.odgr_iteration.argtypes = [vp]
        L.odgr_iteration.restype = c.c_int64
        L.odgr_set_iteration.argtypes = [vp, c.c_int64]
        L.odgr_set_shard.argtypes = [vp, c.c_int64, c.c_int64]
        W = c.POINTER(Weights)
        L.odgr_forward_partial.argtypes = [vp, c.c_double, W, c.c_int, _dp, _dp,
                                           c.POINTER(c.c_double), c.POINTER(c.c_double)]
        L.odgr_forward_finish.argtypes = [vp, _dp, _dp, c.c_double, c.c_double, W, _dp]
        L.odgr_forward_finish.restype = c.c_double
        L.odgr_forward.argtypes = [vp, c.c_double, W, c.c_int, _dp]
        L.odgr_forward.restype = c.c_double
        L.odgr_backward.argtypes = [vp, c.c_double, W, _dp, _dp]
        L.odgr_backward_c.argtypes = [vp, c.c_double, W, _dp, _dp, _dp]
        L.odgr_adam.argtypes = [vp, c.c_double, _dp, _dp]
        L.odgr_next_iteration.argtypes = [vp]
        L.odgr_step.argtypes = [vp, c.c_int, c.c_double, c.c_double, W, _dp]
        L.odgr_get_logits.argtypes = [vp, _dp, _dp]
        L.odgr_set_logits.argtypes = [vp, _dp, _dp]
        L.odgr_get_adam.argtypes = [vp, _dp, _dp, _dp, _dp]
        L.odgr_get_probs.argtypes = [vp, _dp, _dp]
        L.odgr_get_demand.argtypes = [vp, _dp, _dp]
        L.odgr_induce.argtypes = [vp, c.c_double, c.c_double, c.c_double, _i32, _i32, _i64, _i32, _i32, _i32,
                                  _dp, _dp, _dp, _dp]
        L.odgr_real_bytes.restype = c.c_int32
        L.odgr_build_forest.restype = vp
        L.odgr_build_forest.argtypes = [c.c_int32, c.c_int32, c.c_int64, _i64, _i32, c.c_int32, c.c_int32, c.c_int32,
                                        c.c_uint64]
        L.odgr_forest_sizes.argtypes = [vp, _i64]
        L.odgr_forest_copy.argtypes = [vp] + [_i64] * 5 + [_i32] * 3 + [_f32] * 2
        L.odgr_forest_free.argtypes = [vp]
        _libs[path] = L
    return _libs[path]


def philox4x32_10(ctr, key) -> np.ndarray:
    out = np.zeros(4, dtype=np.uint32)
    _load().odgr_philox4x32_10(np.asarray(ctr, dtype=np.uint32), np.asarray(key, dtype=np.uint32), out)
    return out


def uniform(seed: int, idx: int, k: int, stream: int) -> float:
    return _load().odgr_uniform(seed, idx, k, stream)


def gumbel(seed: int, idx: int, k: int, stream: int) -> float:
    return _load().odgr_gumbel(seed, idx, k, stream)


@dataclass
class InduceResult:
    tree_choice: np.ndarray
    route: np.ndarray
    nucleus_off: np.ndarray
    nucleus: np.ndarray
    D_h: np.ndarray
    D_v: np.ndarray
    metrics: np.ndarray
    margin_tree: np.ndarray
    margin_route: np.ndarray
    margin_nucleus: np.ndarray


class Oracle:
    """fp64 CPU oracle over a ``forestgen.Forest``.

    ``fp32=True`` loads the same source compiled with ``real = float``: NOT a reference, only the
    conditioning probe that marks outputs fp32 arithmetic cannot pin to the tolerance."""

    def __init__(self, f, fp32: bool = False):
        self._L = L = _load(fp32)
        self.fp32 = fp32
        self.f = f
        self.X, self.Y = f.X, f.Y
        self._h = L.odgr_new(
            f.X, f.Y, f.n_nets, f.n_trees, f.n_subnets, f.n_paths, f.n_segs, f.n_tps,
            np.ascontiguousarray(f.net_tree_off, np.int64), np.ascontiguousarray(f.tree_sub_off, np.int64),
            np.ascontiguousarray(f.sub_path_off, np.int64), np.ascontiguousarray(f.path_seg_off, np.int64),
            np.ascontiguousarray(f.path_tp_off, np.int64), np.ascontiguousarray(f.seg, np.int32).reshape(-1),
            np.ascontiguousarray(f.tp_xy, np.int32).reshape(-1),
            np.ascontiguousarray(f.cap_h, np.float32).reshape(-1),
            np.ascontiguousarray(f.cap_v, np.float32).reshape(-1),
            np.ascontiguousarray(f.w_tree0, np.float32), np.ascontiguousarray(f.w_path0, np.float32),
            int(f.seed))
        self.last_t = 1.0

    def __del__(self):
        if getattr(self, "_h", None):
            self._L.odgr_free(self._h)
            self._h = None

    # --- state -------------------------------------------------------------------
    @property
    def iteration(self) -> int:
        return self._L.odgr_iteration(self._h)

    @iteration.setter
    def iteration(self, k: int):
        self._L.odgr_set_iteration(self._h, k)

    def set_shard(self, lo: int, hi: int):
        self._L.odgr_set_shard(self._h, lo, hi)

    def logits(self):
        wt = np.zeros(self.f.n_trees); wp = np.zeros(self.f.n_paths)
        self._L.odgr_get_logits(self._h, wt, wp)
        return wt, wp

    def set_logits(self, wt, wp):
        self._L.odgr_set_logits(self._h, np.ascontiguousarray(wt, np.float64), np.ascontiguousarray(wp, np.float64))

    def adam_state(self):
        a = [np.zeros(self.f.n_trees), np.zeros(self.f.n_trees), np.zeros(self.f.n_paths), np.zeros(self.f.n_paths)]
        self._L.odgr_get_adam(self._h, *a)
        return a

    def probs(self):
        q = np.zeros(self.f.n_trees); p = np.zeros(self.f.n_paths)
        self._L.odgr_get_probs(self._h, q, p)
        return q, p

    def demand(self):
        dh = np.zeros((self.Y, self.X)); dv = np.zeros((self.Y, self.X))
        self._L.odgr_get_demand(self._h, dh, dv)
        return dh, dv

    # --- the iteration -------------------------------------------------------------
    def forward(self, t: float, w: Weights, noise: bool = True) -> np.ndarray:
        out = np.zeros(4)
        self._L.odgr_forward(self._h, t, ctypes.byref(w), int(noise), out)
        self.last_t = t
        return out

    def forward_partial(self, t: float, w: Weights, noise: bool = True):
        dh = np.zeros((self.Y, self.X)); dv = np.zeros((self.Y, self.X))
        ewl = ctypes.c_double(); etp = ctypes.c_double()
        self._L.odgr_forward_partial(self._h, t, ctypes.byref(w), int(noise), dh, dv, ctypes.byref(ewl),
                                     ctypes.byref(etp))
        return dh, dv, ewl.value, etp.value

    def forward_finish(self, dh, dv, ewl, etp, w: Weights) -> np.ndarray:
        out = np.zeros(4)
        self._L.odgr_forward_finish(self._h, np.ascontiguousarray(dh, np.float64), np.ascontiguousarray(dv, np.float64),
                                    ewl, etp, ctypes.byref(w), out)
        return out

    def backward(self, t: float, w: Weights, costs: bool = False):
        """dw, du of the last forward (and, with costs=True, every candidate's c_i = d cost / d pi_i)."""
        dw = np.zeros(self.f.n_paths); du = np.zeros(self.f.n_trees)
        if costs:
            c = np.zeros(self.f.n_paths)
            self._L.odgr_backward_c(self._h, t, ctypes.byref(w), dw, du, c)
            return dw, du, c
        self._L.odgr_backward(self._h, t, ctypes.byref(w), dw, du)
        return dw, du

    def adam(self, lr: float, dw, du):
        self._L.odgr_adam(self._h, lr, np.ascontiguousarray(dw, np.float64), np.ascontiguousarray(du, np.float64))

    def next_iteration(self):
        self._L.odgr_next_iteration(self._h)

    def step(self, iters: int, t: float, lr: float, w: Weights) -> np.ndarray:
        out = np.zeros(4)
        self._L.odgr_step(self._h, iters, t, lr, ctypes.byref(w), out)
        self.last_t = t
        return out

    def induce(self, top_p: float, beta: float = 0.25, t_final: float | None = None) -> InduceResult:
        f = self.f
        t = self.last_t if t_final is None else t_final
        r = InduceResult(
            tree_choice=np.zeros(f.n_nets, np.int32), route=np.zeros(f.n_subnets, np.int32),
            nucleus_off=np.zeros(f.n_subnets + 1, np.int64), nucleus=np.zeros(max(1, f.n_paths), np.int32),
            D_h=np.zeros((f.Y, f.X), np.int32), D_v=np.zeros((f.Y, f.X), np.int32), metrics=np.zeros(5),
            margin_tree=np.zeros(f.n_nets), margin_route=np.zeros(f.n_subnets),
            margin_nucleus=np.zeros(f.n_subnets))
        self._L.odgr_induce(self._h, t, top_p, beta, r.tree_choice, r.route, r.nucleus_off, r.nucleus, r.D_h, r.D_v,
                            r.metrics, r.margin_tree, r.margin_route, r.margin_nucleus)
        r.nucleus = r.nucleus[: r.nucleus_off[-1]].copy()
        return r


def build_forest(X: int, Y: int, net_pin_off, pin_xy, n_tree_cand: int = 2, z_cap: int = 15, seed: int = 1,
                 c_cap: int = 0) -> dict:
    """Row f1 oracle (forest_oracle.c): the routing DAG forest of the given nets' pins (§4.2,
    P:524-539; readings Q8, Q14, Q14b, Q17).  Returns the CSR arrays of include/dgr.h's forest."""
    L = _load()
    npo = np.ascontiguousarray(net_pin_off, dtype=np.int64)
    pxy = np.ascontiguousarray(np.asarray(pin_xy, dtype=np.int32).reshape(-1))
    h = L.odgr_build_forest(int(X), int(Y), len(npo) - 1, npo, pxy, int(n_tree_cand), int(z_cap), int(c_cap), int(seed))
    try:
        sz = np.zeros(5, np.int64)
        L.odgr_forest_sizes(h, sz)
        nt, ns, np_, ng, ntp = (int(v) for v in sz)
        out = dict(net_tree_off=np.zeros(len(npo), np.int64), tree_sub_off=np.zeros(nt + 1, np.int64),
                   sub_path_off=np.zeros(ns + 1, np.int64), path_seg_off=np.zeros(np_ + 1, np.int64),
                   path_tp_off=np.zeros(np_ + 1, np.int64), sub_xy=np.zeros((max(ns, 1), 4), np.int32),
                   seg=np.zeros((max(ng, 1), 4), np.int32), tp_xy=np.zeros((max(ntp, 1), 2), np.int32),
                   w_tree0=np.zeros(max(nt, 1), np.float32), w_path0=np.zeros(max(np_, 1), np.float32))
        L.odgr_forest_copy(h, out["net_tree_off"], out["tree_sub_off"], out["sub_path_off"], out["path_seg_off"],
                           out["path_tp_off"], out["sub_xy"], out["seg"], out["tp_xy"], out["w_tree0"], out["w_path0"])
        out["sub_xy"], out["seg"], out["tp_xy"] = out["sub_xy"][:ns], out["seg"][:ng], out["tp_xy"][:ntp]
        out["w_tree0"], out["w_path0"] = out["w_tree0"][:nt], out["w_path0"][:np_]
        return out
    finally:
        L.odgr_forest_free(h)

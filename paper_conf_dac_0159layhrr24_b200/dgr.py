"""Python binding of libdgr (include/dgr.h) — argument marshalling only.

PyTorch supplies the device workspace (a uint8 CUDA tensor), the stream and, for multi-GPU,
the process group used to broadcast the NCCL unique id.  Every step of the solver iteration
(Gumbel-softmax, demand scatter, scan/loss/gradient map, reverse pass, Adam, induction) runs
in libdgr's sm_100a kernels.  There is no CPU fallback: a missing extension or a missing GPU
raises.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
_LIB = os.environ.get("DGR_LIB") or os.path.join(_PKG, "libdgr.so")   # DGR_LIB: A/B builds of libdgr
_lib = None


class DgrError(RuntimeError):
    pass


_P64 = ctypes.POINTER(ctypes.c_int64)
_P32 = ctypes.POINTER(ctypes.c_int32)
_PF = ctypes.POINTER(ctypes.c_float)


class _Desc(ctypes.Structure):
    _fields_ = [("X", ctypes.c_int32), ("Y", ctypes.c_int32),
                ("n_nets", ctypes.c_int64), ("n_trees", ctypes.c_int64), ("n_subnets", ctypes.c_int64),
                ("n_paths", ctypes.c_int64), ("n_segs", ctypes.c_int64), ("n_tps", ctypes.c_int64),
                ("net_tree_off", _P64), ("tree_sub_off", _P64), ("sub_path_off", _P64),
                ("path_seg_off", _P64), ("path_tp_off", _P64),
                ("seg", _P32), ("tp_xy", _P32), ("sub_xy", _P32),
                ("cap_h", _PF), ("cap_v", _PF), ("w_tree0", _PF), ("w_path0", _PF),
                ("seed", ctypes.c_uint64)]


class _PinsDesc(ctypes.Structure):
    _fields_ = [("X", ctypes.c_int32), ("Y", ctypes.c_int32), ("n_nets", ctypes.c_int64),
                ("net_pin_off", ctypes.c_void_p), ("pin_xy", ctypes.c_void_p), ("n_tree_cand", ctypes.c_int32),
                ("z_cap", ctypes.c_int32), ("seed", ctypes.c_uint64), ("c_cap", ctypes.c_int32)]


ALLREDUCE_FN = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32,
                                ctypes.c_void_p)


class _Dist(ctypes.Structure):
    _fields_ = [("rank", ctypes.c_int32), ("world", ctypes.c_int32), ("nccl_unique_id", ctypes.c_void_p),
                ("allreduce", ALLREDUCE_FN), ("allreduce_user", ctypes.c_void_p)]


F_KINDS = {"sigmoid": 0, "relu": 1, "leaky_relu": 2, "exp": 3, "celu": 4}
_DEFAULT_SLOPE = {0: 1.0, 1: 1.0, 2: 0.01, 3: 1.0, 4: 1.0}


class Weights(ctypes.Structure):
    """dgr_weights: a1, a2, a3, beta_v (Q3), L (Q4), overflow function f (0 sigmoid, 1 ReLU,
    2 LeakyReLU, 3 exp, 4 CELU; Fig. 6) and its slope / alpha (Q2)."""
    _fields_ = [("a_wl", ctypes.c_float), ("a_via", ctypes.c_float), ("a_of", ctypes.c_float),
                ("beta_via", ctypes.c_float), ("n_layers", ctypes.c_float), ("f_kind", ctypes.c_int32),
                ("f_slope", ctypes.c_float)]

    def __init__(self, a_wl=0.5, a_via=4.0, a_of=500.0, beta_via=0.25, n_layers=5.0, f_kind=0, f_slope=None):
        if isinstance(f_kind, str):
            f_kind = F_KINDS[f_kind]
        if f_slope is None:
            f_slope = _DEFAULT_SLOPE[int(f_kind)]
        super().__init__(a_wl, a_via, a_of, beta_via, n_layers, f_kind, f_slope)


class Loss(ctypes.Structure):
    _fields_ = [("total", ctypes.c_double), ("wl", ctypes.c_double), ("via", ctypes.c_double),
                ("overflow", ctypes.c_double)]

    def as_array(self) -> np.ndarray:
        return np.array([self.total, self.wl, self.via, self.overflow])


def lib_path() -> str:
    return _LIB


def load_library():
    """Load libdgr.so from the package directory (fails loudly when it was not built)."""
    global _lib
    if _lib is not None:
        return _lib
    import torch  # noqa: F401  (load torch's CUDA runtime / NCCL first so libdgr shares them)
    if not os.path.exists(_LIB):
        raise DgrError(f"{_LIB} is missing: build it with `python -m paper_conf_dac_0159layhrr24_b200.build` "
                       "(no CPU fallback exists)")
    L = ctypes.CDLL(_LIB)
    c, vp = ctypes, ctypes.c_void_p
    L.dgr_last_error.restype = c.c_char_p
    L.dgr_nccl_unique_id.argtypes = [vp]
    L.dgr_partition.argtypes = [c.POINTER(_Desc), c.c_int32, _P64]
    L.dgr_workspace_size.argtypes = [c.POINTER(_Desc), c.POINTER(_Dist)]
    L.dgr_workspace_size.restype = c.c_int64
    L.dgr_forest_load.argtypes = [c.POINTER(_Desc), c.POINTER(_Dist), vp, c.c_int64, vp, c.POINTER(vp)]
    L.dgr_forest_plan.argtypes = [c.POINTER(_Desc), c.POINTER(_Dist), vp, c.POINTER(vp)]
    L.dgr_handle_workspace_size.argtypes = [vp]
    L.dgr_handle_workspace_size.restype = c.c_int64
    L.dgr_bind_workspace.argtypes = [vp, c.POINTER(_Desc), c.POINTER(_Dist), vp, c.c_int64]
    L.dgr_step.argtypes = [vp, c.c_int32, c.c_float, c.c_float, c.POINTER(Weights), c.POINTER(Loss)]
    L.dgr_step_async.argtypes = [vp, c.c_int32, c.c_float, c.c_float, c.POINTER(Weights), c.POINTER(c.c_double)]
    L.dgr_sync.argtypes = [vp]
    L.dgr_get_demand.argtypes = [vp, _PF, _PF]
    L.dgr_get_logits.argtypes = [vp, _PF, _PF]
    L.dgr_induce.argtypes = [vp, c.c_float, _P32, _P32, _P64, _P32, _P32, _P32, c.POINTER(c.c_double)]
    L.dgr_get_info.argtypes = [vp, _P64]
    L.dgr_plan_info.argtypes = [c.POINTER(_Desc), c.POINTER(_Dist), _P64]
    L.dgr_free.argtypes = [vp]
    L.dgr_profile.argtypes = [vp, c.c_int32]
    L.dgr_profile_read.argtypes = [vp, c.POINTER(c.c_double), _P64]
    L.dgr_build_forest.argtypes = [c.POINTER(_PinsDesc), vp, c.POINTER(vp)]
    L.dgr_built_forest_sizes.argtypes = [vp, _P64]
    L.dgr_built_forest_download.argtypes = [vp] + [vp] * 10
    L.dgr_built_forest_free.argtypes = [vp]
    for fn in ("dgr_build_forest", "dgr_built_forest_sizes", "dgr_built_forest_download", "dgr_built_forest_free"):
        getattr(L, fn).restype = c.c_int
    for fn in ("dgr_nccl_unique_id", "dgr_partition", "dgr_forest_load", "dgr_forest_plan", "dgr_bind_workspace",
               "dgr_step", "dgr_step_async", "dgr_sync", "dgr_get_demand",
               "dgr_get_logits", "dgr_induce", "dgr_get_info", "dgr_free", "dgr_profile", "dgr_profile_read", "dgr_plan_info"):
        getattr(L, fn).restype = c.c_int
    _lib = L
    return L


def _check(rc: int):
    if rc != 0:
        raise DgrError(f"libdgr error {rc}: {load_library().dgr_last_error().decode()}")


def _ptr(a: np.ndarray, ct):
    return a.ctypes.data_as(ctypes.POINTER(ct))


class _DescHolder:
    """A dgr_forest_desc over contiguous copies of the forest's arrays (kept alive here)."""

    def __init__(self, f):
        self.arrays = dict(
            net_tree_off=np.ascontiguousarray(f.net_tree_off, np.int64),
            tree_sub_off=np.ascontiguousarray(f.tree_sub_off, np.int64),
            sub_path_off=np.ascontiguousarray(f.sub_path_off, np.int64),
            path_seg_off=np.ascontiguousarray(f.path_seg_off, np.int64),
            path_tp_off=np.ascontiguousarray(f.path_tp_off, np.int64),
            seg=np.ascontiguousarray(f.seg, np.int32).reshape(-1),
            tp_xy=np.ascontiguousarray(f.tp_xy, np.int32).reshape(-1),
            sub_xy=np.ascontiguousarray(f.sub_xy, np.int32).reshape(-1),
            cap_h=np.ascontiguousarray(f.cap_h, np.float32).reshape(-1),
            cap_v=np.ascontiguousarray(f.cap_v, np.float32).reshape(-1),
            w_tree0=np.ascontiguousarray(f.w_tree0, np.float32),
            w_path0=np.ascontiguousarray(f.w_path0, np.float32),
        )
        a = self.arrays
        self.desc = _Desc(
            int(f.X), int(f.Y), len(a["net_tree_off"]) - 1, len(a["tree_sub_off"]) - 1, len(a["sub_path_off"]) - 1,
            len(a["path_seg_off"]) - 1, len(a["seg"]) // 4, len(a["tp_xy"]) // 2,
            _ptr(a["net_tree_off"], ctypes.c_int64), _ptr(a["tree_sub_off"], ctypes.c_int64),
            _ptr(a["sub_path_off"], ctypes.c_int64), _ptr(a["path_seg_off"], ctypes.c_int64),
            _ptr(a["path_tp_off"], ctypes.c_int64), _ptr(a["seg"], ctypes.c_int32), _ptr(a["tp_xy"], ctypes.c_int32),
            _ptr(a["sub_xy"], ctypes.c_int32), _ptr(a["cap_h"], ctypes.c_float), _ptr(a["cap_v"], ctypes.c_float),
            _ptr(a["w_tree0"], ctypes.c_float), _ptr(a["w_path0"], ctypes.c_float), int(f.seed))
        self.X, self.Y = int(f.X), int(f.Y)
        self.n_nets, self.n_trees = self.desc.n_nets, self.desc.n_trees
        self.n_subnets, self.n_paths = self.desc.n_subnets, self.desc.n_paths

    def host_bytes(self) -> int:
        return int(sum(a.nbytes for a in self.arrays.values()))


def partition(forest, world: int) -> np.ndarray:
    """dgr_partition: contiguous, work-balanced net ranges for `world` ranks (host only)."""
    L = load_library()
    d = _DescHolder(forest)
    out = np.zeros(world + 1, np.int64)
    _check(L.dgr_partition(ctypes.byref(d.desc), world, _ptr(out, ctypes.c_int64)))
    return out


def plan_info(forest, rank: int = 0, world: int = 1) -> dict:
    """dgr_plan_info: the rank's tile / bundle plan, computed on the host (no GPU)."""
    L = load_library()
    d = _DescHolder(forest)
    out = np.zeros(8, np.int64)
    dist = _Dist(rank, world, None) if world > 1 else None
    if world > 1:
        # the plan does not need the NCCL id; pass a dummy so validation accepts world > 1
        buf = ctypes.create_string_buffer(128)
        dist.nccl_unique_id = ctypes.cast(buf, ctypes.c_void_p)
    _check(L.dgr_plan_info(ctypes.byref(d.desc), ctypes.byref(dist) if dist is not None else None,
                           _ptr(out, ctypes.c_int64)))
    keys = ("n_tiles", "n_global_tiles", "n_bundles", "n_slots", "workspace_bytes", "n_paths", "global_paths",
            "max_window")
    return {k: int(v) for k, v in zip(keys, out)}


def nccl_unique_id() -> bytes:
    L = load_library()
    buf = ctypes.create_string_buffer(128)
    _check(L.dgr_nccl_unique_id(buf))
    return buf.raw


@dataclass
class InduceResult:
    tree_choice: np.ndarray
    route: np.ndarray
    nucleus_off: np.ndarray
    nucleus: np.ndarray
    D_h: np.ndarray
    D_v: np.ndarray
    metrics: np.ndarray


class _DevBuf:
    """A library device buffer as a CUDA array (no copy)."""

    def __init__(self, ptr: int, n: int, dtype: int):
        self.__cuda_array_interface__ = {"shape": (int(n),), "typestr": ("<i8", "<i4", "<f8", "<f4")[dtype],
                                         "data": (int(ptr), False), "version": 3}


def torch_allreduce(group=None):
    """A dgr_dist.allreduce callback over a torch.distributed process group (e.g. gloo: the ranks'
    exchange without NCCL, so that several ranks can share one GPU).  Plumbing only: the buffer goes
    to the host, torch.distributed sums it, and it comes back."""
    import torch
    import torch.distributed as tdist

    def fn(buf, n, dtype, stream):
        try:
            st = torch.cuda.ExternalStream(stream) if stream else torch.cuda.current_stream()
            st.synchronize()
            dev = torch.as_tensor(_DevBuf(buf, n, dtype), device="cuda")
            host = dev.cpu()
            tdist.all_reduce(host, group=group)
            dev.copy_(host)
            torch.cuda.synchronize()
            return 0
        except Exception:   # the failing dgr_* call reports DGR_ENCCL
            return 1
    return fn


class Solver:
    """One rank's DGR solver over a forest (any object with forestgen.Forest's fields)."""

    def __init__(self, forest, rank: int = 0, world: int = 1, nccl_id: bytes | None = None, device=None,
                 stream=None, allreduce=None):
        """allreduce: optional Python callable (buf_ptr, count, dtype, stream_ptr) -> int replacing NCCL
        (dgr_dist.allreduce): sums `count` int64 / int32 / fp64 / fp32 (dtype 0 / 1 / 2 / 3) elements at
        device address buf_ptr over the ranks in place, after the work on stream_ptr (e.g.
        torch_allreduce() over a torch.distributed process group)."""
        import torch
        if not torch.cuda.is_available():
            raise DgrError("libdgr needs a CUDA device (no CPU fallback)")
        L = load_library()
        self._torch = torch
        self.device = torch.device(device) if device is not None else torch.device("cuda", torch.cuda.current_device())
        self.stream = stream if stream is not None else torch.cuda.current_stream(self.device)
        self._d = _DescHolder(forest)
        self.X, self.Y = self._d.X, self._d.Y
        self.n_nets, self.n_trees = self._d.n_nets, self._d.n_trees
        self.n_subnets, self.n_paths = self._d.n_subnets, self._d.n_paths
        self._idbuf = None
        dist = None
        self._ar = None
        # world == 1 with an NCCL id or a callback: the band exchange runs anyway (one-rank
        # communicator / the callback), the sharded path exercised on one GPU
        if allreduce is not None:
            self._ar = ALLREDUCE_FN(lambda _u, buf, n, dt, st: int(allreduce(buf, n, dt, st)))
            dist = _Dist(rank, world, None, self._ar, None)
        elif world > 1 or nccl_id is not None:
            if nccl_id is None or len(nccl_id) != 128:
                raise DgrError("world > 1 needs the 128-byte NCCL unique id from rank 0")
            self._idbuf = ctypes.create_string_buffer(nccl_id, 128)
            dist = _Dist(rank, world, ctypes.cast(self._idbuf, ctypes.c_void_p))
        self._dist = dist
        distp = ctypes.byref(dist) if dist is not None else None
        # plan once on the host, then bind a torch-allocated workspace (dgr_forest_plan + dgr_bind_workspace)
        self._h = ctypes.c_void_p()
        _check(L.dgr_forest_plan(ctypes.byref(self._d.desc), distp, ctypes.c_void_p(self.stream.cuda_stream),
                                 ctypes.byref(self._h)))
        nbytes = L.dgr_handle_workspace_size(self._h)
        if nbytes <= 0:
            raise DgrError("dgr_handle_workspace_size: " + L.dgr_last_error().decode())
        with torch.cuda.device(self.device):
            self.workspace = torch.empty(int(nbytes), dtype=torch.uint8, device=self.device)
        _check(L.dgr_bind_workspace(self._h, ctypes.byref(self._d.desc), distp,
                                    ctypes.c_void_p(self.workspace.data_ptr()), int(nbytes)))
        self.workspace_bytes = int(nbytes)

    # ----------------------------------------------------------------------------------
    def step(self, iters: int, temperature: float, lr: float = 0.3, weights: Weights | None = None,
             want_loss: bool = True) -> np.ndarray | None:
        w = weights if weights is not None else Weights()
        loss = Loss()
        _check(load_library().dgr_step(self._h, int(iters), float(temperature), float(lr), ctypes.byref(w),
                                       ctypes.byref(loss) if want_loss else None))
        return loss.as_array() if want_loss else None

    def step_async(self, iters: int, temperature: float, lr: float, weights: Weights | None,
                   loss_out: np.ndarray):
        """dgr_step_async: enqueue the iterations and a copy of their last loss into loss_out (4 float64,
        host memory, ideally pinned); valid after sync()."""
        assert loss_out.dtype == np.float64 and loss_out.size >= 4 and loss_out.flags.c_contiguous
        w = weights if weights is not None else Weights()
        _check(load_library().dgr_step_async(self._h, int(iters), float(temperature), float(lr), ctypes.byref(w),
                                             loss_out.ctypes.data_as(ctypes.POINTER(ctypes.c_double))))

    def sync(self):
        _check(load_library().dgr_sync(self._h))

    def demand(self):
        dh = np.zeros((self.Y, self.X), np.float32); dv = np.zeros((self.Y, self.X), np.float32)
        _check(load_library().dgr_get_demand(self._h, _ptr(dh, ctypes.c_float), _ptr(dv, ctypes.c_float)))
        return dh, dv

    def logits(self):
        wt = np.zeros(self.n_trees, np.float32); wp = np.zeros(self.n_paths, np.float32)
        _check(load_library().dgr_get_logits(self._h, _ptr(wt, ctypes.c_float), _ptr(wp, ctypes.c_float)))
        return wt, wp

    def induce(self, top_p: float = 0.9) -> InduceResult:
        r = InduceResult(
            tree_choice=np.zeros(self.n_nets, np.int32), route=np.zeros(self.n_subnets, np.int32),
            nucleus_off=np.zeros(self.n_subnets + 1, np.int64), nucleus=np.zeros(max(1, self.n_paths), np.int32),
            D_h=np.zeros((self.Y, self.X), np.int32), D_v=np.zeros((self.Y, self.X), np.int32),
            metrics=np.zeros(5, np.float64))
        _check(load_library().dgr_induce(
            self._h, float(top_p), _ptr(r.tree_choice, ctypes.c_int32), _ptr(r.route, ctypes.c_int32),
            _ptr(r.nucleus_off, ctypes.c_int64), _ptr(r.nucleus, ctypes.c_int32), _ptr(r.D_h, ctypes.c_int32),
            _ptr(r.D_v, ctypes.c_int32), r.metrics.ctypes.data_as(ctypes.POINTER(ctypes.c_double))))
        r.nucleus = r.nucleus[: r.nucleus_off[-1]].copy()
        return r

    def info(self) -> dict:
        a = np.zeros(12, np.int64)
        _check(load_library().dgr_get_info(self._h, _ptr(a, ctypes.c_int64)))
        return dict(k=int(a[0]), net_lo=int(a[1]), net_hi=int(a[2]), n_bundles=int(a[3]), n_slots=int(a[4]),
                    workspace_bytes=int(a[5]), world=int(a[6]), rank=int(a[7]), n_tiles=int(a[8]),
                    n_global_tiles=int(a[9]), n_pipe_tiles=int(a[10]), n_general_paths=int(a[11]))

    STAGES = ("KF", "allreduce", "KG", "KBF", "KB", "KL")   # KL: the loss kernel, once per call

    def profile(self, enable: bool = True):
        """Start (and clear) / stop per-stage CUDA-event timing of dgr_step."""
        _check(load_library().dgr_profile(self._h, int(bool(enable))))

    def profile_read(self) -> tuple[dict, dict]:
        """{stage: summed ms}, {stage: launches} since profile(True)."""
        ms = (ctypes.c_double * 8)()
        n = (ctypes.c_int64 * 8)()
        _check(load_library().dgr_profile_read(self._h, ms, n))
        return {k: ms[i] for i, k in enumerate(self.STAGES)}, {k: int(n[i]) for i, k in enumerate(self.STAGES)}

    @property
    def iteration(self) -> int:
        return self.info()["k"]

    def host_input_bytes(self) -> int:
        return self._d.host_bytes()

    def close(self):
        if getattr(self, "_h", None) and self._h.value:
            load_library().dgr_free(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class BuiltForest:
    """Row f1: a routing DAG forest built on the GPU from the nets' pins (dgr_build_forest).
    The device arrays are owned by libdgr; download() copies them into host numpy arrays."""

    def __init__(self, X: int, Y: int, net_pin_off, pin_xy, n_tree_cand: int = 2, z_cap: int = 15, seed: int = 1,
                 stream=None, c_cap: int = 0):
        import torch
        if not torch.cuda.is_available():
            raise DgrError("libdgr needs a CUDA device (no CPU fallback)")
        L = load_library()
        self.X, self.Y = int(X), int(Y)
        npo = np.ascontiguousarray(net_pin_off, np.int64)
        pxy = np.ascontiguousarray(np.asarray(pin_xy, np.int32).reshape(-1))
        st = stream if stream is not None else torch.cuda.current_stream()
        d = _PinsDesc(self.X, self.Y, len(npo) - 1, npo.ctypes.data, pxy.ctypes.data, int(n_tree_cand), int(z_cap),
                      int(seed), int(c_cap))
        self._h = ctypes.c_void_p()
        _check(L.dgr_build_forest(ctypes.byref(d), ctypes.c_void_p(st.cuda_stream), ctypes.byref(self._h)))
        sz = np.zeros(6, np.int64)
        _check(L.dgr_built_forest_sizes(self._h, sz.ctypes.data_as(ctypes.POINTER(ctypes.c_int64))))
        self.n_nets, self.n_trees, self.n_subnets, self.n_paths, self.n_segs, self.n_tps = (int(v) for v in sz)

    def download(self) -> dict:
        out = dict(net_tree_off=np.zeros(self.n_nets + 1, np.int64), tree_sub_off=np.zeros(self.n_trees + 1, np.int64),
                   sub_path_off=np.zeros(self.n_subnets + 1, np.int64),
                   path_seg_off=np.zeros(self.n_paths + 1, np.int64), path_tp_off=np.zeros(self.n_paths + 1, np.int64),
                   sub_xy=np.zeros((self.n_subnets, 4), np.int32), seg=np.zeros((self.n_segs, 4), np.int32),
                   tp_xy=np.zeros((self.n_tps, 2), np.int32), w_tree0=np.zeros(self.n_trees, np.float32),
                   w_path0=np.zeros(self.n_paths, np.float32))
        order = ("net_tree_off", "tree_sub_off", "sub_path_off", "path_seg_off", "path_tp_off", "sub_xy", "seg",
                 "tp_xy", "w_tree0", "w_path0")
        _check(load_library().dgr_built_forest_download(self._h, *[ctypes.c_void_p(out[k].ctypes.data) for k in order]))
        return out

    def close(self):
        if getattr(self, "_h", None) and self._h.value:
            load_library().dgr_built_forest_free(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def build_forest(X, Y, net_pin_off, pin_xy, n_tree_cand=2, z_cap=15, seed=1, stream=None, c_cap=0) -> BuiltForest:
    """dgr_build_forest (row f1): the routing DAG forest of the nets' pins, built on the GPU."""
    return BuiltForest(X, Y, net_pin_off, pin_xy, n_tree_cand, z_cap, seed, stream, c_cap)

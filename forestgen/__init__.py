"""forestgen — seeded synthetic placement + routing-DAG-forest generator (shared input module).

Both implementations consume what this module emits: the oracle (``oracle/``) and
the CUDA path (``paper_conf_dac_0159layhrr24_b200``).  It holds none of the
solver's arithmetic.  The C++ generator (``forestgen.cpp``, C ABI in
``include/forestgen.h``) stands in for PAPER.md §4.2: tree
candidates, 2-pin decomposition, L/Z path enumeration, Eq. (1) capacities and
random initial logits.  The workload recipes below are the BASELINE.json
``configs`` with the distributions of SURVEY.md §8(d).

``.dgrf`` is a flat little-endian container of the CSR arrays (``write_dgrf`` /
``read_dgrf``) so that a forest can be generated once and replayed.
"""
from __future__ import annotations

import ctypes
import hashlib
import math
import os
import struct
from dataclasses import dataclass, field

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libforestgen.so")
_lib = None

GUMBEL_SEED = 0xD6A5EED  # Gumbel seed unless stated


class _Config(ctypes.Structure):
    _fields_ = [
        ("X", ctypes.c_int32), ("Y", ctypes.c_int32), ("n_nets", ctypes.c_int64),
        ("pins_mode", ctypes.c_int32), ("pins_min", ctypes.c_int32), ("pins_max", ctypes.c_int32),
        ("box_mode", ctypes.c_int32), ("box_min", ctypes.c_int32), ("box_max", ctypes.c_int32),
        ("box_mu", ctypes.c_double), ("cluster_frac", ctypes.c_double), ("n_hotspots", ctypes.c_int32),
        ("track", ctypes.c_double), ("beta_pin", ctypes.c_double), ("n_tree_cand", ctypes.c_int32),
        ("z_cap", ctypes.c_int32), ("seed", ctypes.c_uint64), ("local_weight", ctypes.c_double),
        ("c_cap", ctypes.c_int32), ("m_cap", ctypes.c_int32),
    ]


_P64 = ctypes.POINTER(ctypes.c_int64)
_P32 = ctypes.POINTER(ctypes.c_int32)
_PF = ctypes.POINTER(ctypes.c_float)


class _View(ctypes.Structure):
    _fields_ = [
        ("X", ctypes.c_int32), ("Y", ctypes.c_int32),
        ("n_nets", ctypes.c_int64), ("n_trees", ctypes.c_int64), ("n_subnets", ctypes.c_int64),
        ("n_paths", ctypes.c_int64), ("n_segs", ctypes.c_int64), ("n_tps", ctypes.c_int64),
        ("n_local_nets", ctypes.c_int64), ("n_pins", ctypes.c_int64),
        ("net_tree_off", _P64), ("tree_sub_off", _P64), ("sub_path_off", _P64),
        ("path_seg_off", _P64), ("path_tp_off", _P64),
        ("seg", _P32), ("tp_xy", _P32), ("sub_xy", _P32),
        ("cap_h", _PF), ("cap_v", _PF), ("w_tree0", _PF), ("w_path0", _PF),
        ("net_pin_off", _P64), ("pin_xy", _P32),
    ]


def build(verbose: bool = False) -> str:
    """Compile libforestgen.so in-tree (g++, OpenMP)."""
    import subprocess
    src = os.path.join(_HERE, "forestgen.cpp")
    inc = os.path.join(os.path.dirname(_HERE), "include")
    cmd = ["g++", "-O2", "-std=c++17", "-fopenmp", "-shared", "-fPIC", "-I" + inc, "-o", _LIB_PATH, src]
    if verbose:
        print(" ".join(cmd))
    subprocess.check_call(cmd)
    return _LIB_PATH


def _load():
    global _lib
    if _lib is None:
        src = os.path.join(_HERE, "forestgen.cpp")
        if not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(src):
            build()
        lib = ctypes.CDLL(_LIB_PATH)
        lib.forestgen_generate.argtypes = [ctypes.POINTER(_Config), ctypes.POINTER(ctypes.c_void_p)]
        lib.forestgen_generate.restype = ctypes.c_int
        lib.forestgen_get_view.argtypes = [ctypes.c_void_p, ctypes.POINTER(_View)]
        lib.forestgen_free.argtypes = [ctypes.c_void_p]
        lib.forestgen_last_error.restype = ctypes.c_char_p
        _lib = lib
    return _lib


# --------------------------------------------------------------------------------------
# workload recipes (BASELINE.json configs; SURVEY.md §8(d) "Concrete synthetic inputs")
# --------------------------------------------------------------------------------------
def _sweep(n: int) -> dict:
    side = int(round(1000 * math.sqrt(n / 1e6)))
    return dict(X=side, Y=side, n_nets=n, pins_mode=1, box_mode=1, box_mu=5.0, cluster_frac=0.3,
                n_hotspots=max(1, int(round(32 * side * side / 1e6))), track=4.0, beta_pin=0.25,
                n_tree_cand=2, z_cap=15, seed=1)


# PAPER.md Table 1: (grid side, cap_e, #nets, box) of the ILP comparison rows.  Three
# G-cells drawn in a box per net as pins, L-shape candidates only, uniform
# capacity.  "Every 2-pin pair" is read as the MST's two sub-nets (ambiguous; the
# printed overflows are not reproducible and stay unpinned).
TABLE1_ROWS = [(20, 1, 20, 4), (50, 1, 50, 10), (50, 1, 100, 10), (50, 2, 100, 10), (50, 1, 1000, 10),
               (50, 10, 1000, 10), (50, 10, 10000, 10), (100, 2, 1000, 20), (100, 2, 10000, 20),
               (1000, 1, 100000, 200)]
TABLE1_DGR = [30, 173, 1028, 0, 35445, 7407, 364536, 48846, 785664, 80237614]   # DGR* overflow column


def _table1(side, cap, nets, box):
    return dict(X=side, Y=side, n_nets=nets, pins_mode=0, pins_min=3, pins_max=3, box_mode=0, box_min=box,
                box_max=box, cluster_frac=0.0, n_hotspots=0, track=float(cap), beta_pin=0.0, local_weight=0.0,
                n_tree_cand=1, z_cap=-1, seed=1)


CONFIGS: dict[str, dict] = {
    # 16x16, 40 nets of 2-4 pins in boxes U{2..8}, 2 trees, L+Z uncapped, T=1 uniform
    "tiny": dict(X=16, Y=16, n_nets=40, pins_mode=0, pins_min=2, pins_max=4, box_mode=0, box_min=2,
                 box_max=8, cluster_frac=0.0, n_hotspots=0, track=1.0, beta_pin=0.0, n_tree_cand=2,
                 z_cap=0, seed=1),
    # 256x256, ~1e4 nets, uniform capacity T=1
    "c1e4": dict(X=256, Y=256, n_nets=10_000, pins_mode=1, box_mode=1, box_mu=8.0, cluster_frac=0.0,
                 n_hotspots=0, track=1.0, beta_pin=0.25, n_tree_cand=2, z_cap=15, seed=1),
    # ISPD'18-shaped: 600x600, ~1e5 nets, T=2, 8 hotspots, 30% clustered
    "ispd18": dict(X=600, Y=600, n_nets=100_000, pins_mode=1, box_mode=1, box_mu=6.0, cluster_frac=0.3,
                   n_hotspots=8, track=2.0, beta_pin=0.25, n_tree_cand=2, z_cap=15, seed=1),
    # ISPD'19-shaped (north star): 1000x1000, ~1e6 nets, T=4, 32 hotspots, 30% clustered
    "ispd19": dict(X=1000, Y=1000, n_nets=1_000_000, pins_mode=1, box_mode=1, box_mu=5.0,
                   cluster_frac=0.3, n_hotspots=32, track=4.0, beta_pin=0.25, n_tree_cand=2, z_cap=15,
                   seed=1),
    # row f4 (C-shape detours, Q14b): groups stay <= 32 (2 L + 2x11 Z + up to 2x2x2 C)
    "tiny_c": dict(X=16, Y=16, n_nets=40, pins_mode=0, pins_min=2, pins_max=4, box_mode=0, box_min=2,
                   box_max=8, cluster_frac=0.0, n_hotspots=0, track=1.0, beta_pin=0.0, n_tree_cand=2,
                   z_cap=0, c_cap=2, seed=3),
    "c1e4_c": dict(X=256, Y=256, n_nets=10_000, pins_mode=1, box_mode=1, box_mu=8.0, cluster_frac=0.0,
                   n_hotspots=0, track=1.0, beta_pin=0.25, n_tree_cand=2, z_cap=11, c_cap=2, seed=1),
    # row f4' (reading Q14c): monotone staircases (4 turning points) and groups > 32 (uncapped Z)
    "tiny_m": dict(X=32, Y=32, n_nets=40, pins_mode=0, pins_min=2, pins_max=4, box_mode=0, box_min=14,
                   box_max=24, cluster_frac=0.0, n_hotspots=0, track=1.0, beta_pin=0.0, n_tree_cand=2,
                   z_cap=0, c_cap=1, m_cap=2, seed=7),
    "c1e4_m": dict(X=256, Y=256, n_nets=10_000, pins_mode=1, box_mode=1, box_mu=8.0, cluster_frac=0.0,
                   n_hotspots=0, track=1.0, beta_pin=0.25, n_tree_cand=2, z_cap=24, c_cap=1, m_cap=2, seed=1),
    "ispd18_m": dict(X=600, Y=600, n_nets=100_000, pins_mode=1, box_mode=1, box_mu=6.0, cluster_frac=0.3,
                     n_hotspots=8, track=2.0, beta_pin=0.25, n_tree_cand=2, z_cap=24, c_cap=1, m_cap=2, seed=1),
    "ispd19_c": dict(X=1000, Y=1000, n_nets=1_000_000, pins_mode=1, box_mode=1, box_mu=5.0,
                     cluster_frac=0.3, n_hotspots=32, track=4.0, beta_pin=0.25, n_tree_cand=2, z_cap=11,
                     c_cap=2, seed=1),
    **{f"table1_r{i + 1}": _table1(*row) for i, row in enumerate(TABLE1_ROWS)},
    "sweep1e4": _sweep(10_000),
    "sweep1e5": _sweep(100_000),
    "sweep1e6": _sweep(1_000_000),
    "sweep4e6": _sweep(4_000_000),
}


@dataclass
class Forest:
    """Flat CSR forest, the shape of include/dgr.h's dgr_forest_desc."""
    X: int
    Y: int
    net_tree_off: np.ndarray
    tree_sub_off: np.ndarray
    sub_path_off: np.ndarray
    path_seg_off: np.ndarray
    path_tp_off: np.ndarray
    seg: np.ndarray        # [n_segs, 4] int32 {dir, line, lo, hi}
    tp_xy: np.ndarray      # [n_tps, 2] int32
    sub_xy: np.ndarray     # [n_subnets, 4] int32
    cap_h: np.ndarray      # [Y, X] float32
    cap_v: np.ndarray      # [Y, X] float32
    w_tree0: np.ndarray    # [n_trees] float32
    w_path0: np.ndarray    # [n_paths] float32
    seed: int = GUMBEL_SEED
    net_pin_off: np.ndarray | None = None
    pin_xy: np.ndarray | None = None
    n_local_nets: int = 0
    meta: dict = field(default_factory=dict)

    @property
    def n_nets(self): return len(self.net_tree_off) - 1
    @property
    def n_trees(self): return len(self.tree_sub_off) - 1
    @property
    def n_subnets(self): return len(self.sub_path_off) - 1
    @property
    def n_paths(self): return len(self.path_seg_off) - 1
    @property
    def n_segs(self): return int(self.seg.shape[0])
    @property
    def n_tps(self): return int(self.tp_xy.shape[0])

    def stats(self) -> dict:
        return dict(X=self.X, Y=self.Y, nets=self.n_nets, trees=self.n_trees, subnets=self.n_subnets,
                    paths=self.n_paths, segs=self.n_segs, tps=self.n_tps, local_nets=self.n_local_nets,
                    max_group=int(np.diff(self.sub_path_off).max()) if self.n_subnets else 0)

    def sha256(self) -> str:
        h = hashlib.sha256()
        for a in (self.net_tree_off, self.tree_sub_off, self.sub_path_off, self.path_seg_off,
                  self.path_tp_off, self.seg, self.tp_xy, self.sub_xy, self.cap_h, self.cap_v,
                  self.w_tree0, self.w_path0):
            h.update(np.ascontiguousarray(a).tobytes())
        h.update(struct.pack("<iiQ", self.X, self.Y, self.seed))
        return h.hexdigest()


def generate(config: str | dict, seed: int | None = None, gumbel_seed: int = GUMBEL_SEED, **overrides) -> Forest:
    """Generate a forest from a named recipe (``CONFIGS``) or an explicit dict."""
    if isinstance(config, str):
        if config.startswith("sweep") and config not in CONFIGS:
            cfg = _sweep(int(float(config[5:])))
        else:
            cfg = dict(CONFIGS[config])
    else:
        cfg = dict(config)
    cfg.update(overrides)
    if seed is not None:
        cfg["seed"] = seed
    c = _Config()
    defaults = dict(pins_min=2, pins_max=4, box_min=2, box_max=8, box_mu=5.0, cluster_frac=0.0,
                    n_hotspots=0, track=1.0, beta_pin=0.0, n_tree_cand=2, z_cap=15, seed=1,
                    pins_mode=0, box_mode=0, local_weight=1.0, c_cap=0, m_cap=0)
    for k, v in {**defaults, **cfg}.items():
        setattr(c, k, v)
    lib = _load()
    h = ctypes.c_void_p()
    rc = lib.forestgen_generate(ctypes.byref(c), ctypes.byref(h))
    if rc != 0:
        raise ValueError("forestgen: " + lib.forestgen_last_error().decode())
    try:
        v = _View()
        lib.forestgen_get_view(h, ctypes.byref(v))

        def arr(ptr, n, dt, shape=None):
            if n == 0:
                a = np.zeros(0, dtype=dt)
            else:
                a = np.ctypeslib.as_array(ptr, shape=(n,)).copy()
            return a.reshape(shape) if shape is not None else a

        nn, nt, ns, npth = v.n_nets, v.n_trees, v.n_subnets, v.n_paths
        f = Forest(
            X=v.X, Y=v.Y,
            net_tree_off=arr(v.net_tree_off, nn + 1, np.int64),
            tree_sub_off=arr(v.tree_sub_off, nt + 1, np.int64),
            sub_path_off=arr(v.sub_path_off, ns + 1, np.int64),
            path_seg_off=arr(v.path_seg_off, npth + 1, np.int64),
            path_tp_off=arr(v.path_tp_off, npth + 1, np.int64),
            seg=arr(v.seg, v.n_segs * 4, np.int32, (v.n_segs, 4)),
            tp_xy=arr(v.tp_xy, v.n_tps * 2, np.int32, (v.n_tps, 2)),
            sub_xy=arr(v.sub_xy, ns * 4, np.int32, (ns, 4)),
            cap_h=arr(v.cap_h, v.X * v.Y, np.float32, (v.Y, v.X)),
            cap_v=arr(v.cap_v, v.X * v.Y, np.float32, (v.Y, v.X)),
            w_tree0=arr(v.w_tree0, nt, np.float32),
            w_path0=arr(v.w_path0, npth, np.float32),
            seed=gumbel_seed,
            net_pin_off=arr(v.net_pin_off, nn + 1, np.int64),
            pin_xy=arr(v.pin_xy, v.n_pins * 2, np.int32, (v.n_pins, 2)),
            n_local_nets=v.n_local_nets,
            meta=dict(config=cfg),
        )
    finally:
        lib.forestgen_free(h)
    return f


# --------------------------------------------------------------------------------------
# .dgrf container
# --------------------------------------------------------------------------------------
_MAGIC = b"DGRF"
_VERSION = 1
_ARRAYS = [("net_tree_off", np.int64), ("tree_sub_off", np.int64), ("sub_path_off", np.int64),
           ("path_seg_off", np.int64), ("path_tp_off", np.int64), ("seg", np.int32), ("tp_xy", np.int32),
           ("sub_xy", np.int32), ("cap_h", np.float32), ("cap_v", np.float32), ("w_tree0", np.float32),
           ("w_path0", np.float32)]


def write_dgrf(f: Forest, path: str) -> None:
    with open(path, "wb") as fh:
        fh.write(_MAGIC + struct.pack("<IiiQq", _VERSION, f.X, f.Y, f.seed, f.n_local_nets))
        for name, dt in _ARRAYS:
            a = np.ascontiguousarray(getattr(f, name), dtype=dt)
            fh.write(struct.pack("<q", a.size))
            fh.write(a.tobytes())


def read_dgrf(path: str) -> Forest:
    with open(path, "rb") as fh:
        head = fh.read(4 + struct.calcsize("<IiiQq"))
        if head[:4] != _MAGIC:
            raise ValueError("not a .dgrf file")
        ver, X, Y, seed, nloc = struct.unpack("<IiiQq", head[4:])
        if ver != _VERSION:
            raise ValueError(f"unsupported .dgrf version {ver}")
        vals = {}
        for name, dt in _ARRAYS:
            (n,) = struct.unpack("<q", fh.read(8))
            vals[name] = np.frombuffer(fh.read(n * np.dtype(dt).itemsize), dtype=dt).copy()
    vals["seg"] = vals["seg"].reshape(-1, 4)
    vals["tp_xy"] = vals["tp_xy"].reshape(-1, 2)
    vals["sub_xy"] = vals["sub_xy"].reshape(-1, 4)
    vals["cap_h"] = vals["cap_h"].reshape(Y, X)
    vals["cap_v"] = vals["cap_v"].reshape(Y, X)
    return Forest(X=X, Y=Y, seed=seed, n_local_nets=nloc, **vals)


def subset(f: Forest, net_lo: int, net_hi: int) -> Forest:
    """The sub-forest of nets [net_lo, net_hi) (offsets rebased; caps and seed kept)."""
    t0, t1 = int(f.net_tree_off[net_lo]), int(f.net_tree_off[net_hi])
    s0, s1 = int(f.tree_sub_off[t0]), int(f.tree_sub_off[t1])
    p0, p1 = int(f.sub_path_off[s0]), int(f.sub_path_off[s1])
    g0, g1 = int(f.path_seg_off[p0]), int(f.path_seg_off[p1])
    q0, q1 = int(f.path_tp_off[p0]), int(f.path_tp_off[p1])
    return Forest(
        X=f.X, Y=f.Y,
        net_tree_off=f.net_tree_off[net_lo:net_hi + 1] - t0,
        tree_sub_off=f.tree_sub_off[t0:t1 + 1] - s0,
        sub_path_off=f.sub_path_off[s0:s1 + 1] - p0,
        path_seg_off=f.path_seg_off[p0:p1 + 1] - g0,
        path_tp_off=f.path_tp_off[p0:p1 + 1] - q0,
        seg=f.seg[g0:g1].copy(), tp_xy=f.tp_xy[q0:q1].copy(), sub_xy=f.sub_xy[s0:s1].copy(),
        cap_h=f.cap_h, cap_v=f.cap_v,
        w_tree0=f.w_tree0[t0:t1].copy(), w_path0=f.w_path0[p0:p1].copy(), seed=f.seed,
    )


def _ranges(off: np.ndarray, sel: np.ndarray) -> np.ndarray:
    """Concatenation of the index ranges [off[i], off[i+1]) for i in sel (vectorised)."""
    off = np.asarray(off, np.int64)
    lo, hi = off[sel], off[np.asarray(sel) + 1]
    n = hi - lo
    if n.sum() == 0:
        return np.zeros(0, np.int64)
    start = np.repeat(lo - np.concatenate([[0], np.cumsum(n)[:-1]]), n)
    return start + np.arange(int(n.sum()), dtype=np.int64)


def _gather_paths(f: Forest, order: np.ndarray) -> dict:
    """CSR path arrays (segments, turning points, initial logits) with the paths in `order`."""
    order = np.asarray(order, np.int64)
    nseg = np.diff(f.path_seg_off)[order]
    ntp = np.diff(f.path_tp_off)[order]
    return dict(path_seg_off=np.concatenate([[0], np.cumsum(nseg)]).astype(np.int64),
                path_tp_off=np.concatenate([[0], np.cumsum(ntp)]).astype(np.int64),
                seg=f.seg[_ranges(f.path_seg_off, order)].copy(), tp_xy=f.tp_xy[_ranges(f.path_tp_off, order)].copy(),
                w_path0=f.w_path0[order].copy())


def shuffle_candidates(f: Forest, seed: int = 0) -> Forest:
    """The same forest with every sub-net's path candidates in a random order (a valid forest the
    tile kernel's canonical order does not cover: it runs on the general path, row f4')."""
    rng = np.random.default_rng(seed)
    order = np.concatenate([f.sub_path_off[s] + rng.permutation(int(f.sub_path_off[s + 1] - f.sub_path_off[s]))
                            for s in range(f.n_subnets)]).astype(np.int64) if f.n_subnets else np.zeros(0, np.int64)
    g = Forest(X=f.X, Y=f.Y, net_tree_off=f.net_tree_off.copy(), tree_sub_off=f.tree_sub_off.copy(),
               sub_path_off=f.sub_path_off.copy(), sub_xy=f.sub_xy.copy(), cap_h=f.cap_h, cap_v=f.cap_v,
               w_tree0=f.w_tree0.copy(), seed=f.seed, **_gather_paths(f, order))
    g.meta = dict(f.meta, shuffled_candidates=seed)
    return g


def shuffle_nets(f: Forest, seed: int = 0) -> Forest:
    """The same forest with its nets in a random order (trees, sub-nets and paths follow their net)."""
    rng = np.random.default_rng(seed)
    nets = rng.permutation(f.n_nets)
    trees = _ranges(f.net_tree_off, nets)
    subs = _ranges(f.tree_sub_off, trees)
    paths = _ranges(f.sub_path_off, subs)
    g = Forest(X=f.X, Y=f.Y,
               net_tree_off=np.concatenate([[0], np.cumsum(np.diff(f.net_tree_off)[nets])]).astype(np.int64),
               tree_sub_off=np.concatenate([[0], np.cumsum(np.diff(f.tree_sub_off)[trees])]).astype(np.int64),
               sub_path_off=np.concatenate([[0], np.cumsum(np.diff(f.sub_path_off)[subs])]).astype(np.int64),
               sub_xy=f.sub_xy[subs].copy(), cap_h=f.cap_h, cap_v=f.cap_v, w_tree0=f.w_tree0[trees].copy(),
               seed=f.seed, **_gather_paths(f, paths))
    g.meta = dict(f.meta, shuffled_nets=seed)
    return g

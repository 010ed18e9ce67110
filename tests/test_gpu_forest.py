"""Row f1 on the GPU: dgr_build_forest (net-parallel forest construction) against the f1 oracle
(oracle/forest_oracle.c), bit for bit; malformed pins rejected on the host (no GPU needed)."""
import ctypes

import numpy as np
import pytest

import forestgen
import oracle
import paper_conf_dac_0159layhrr24_b200 as dgr
from paper_conf_dac_0159layhrr24_b200 import dgr as binding


def _oracle(X, Y, net_pin_off, pin_xy, n_tree_cand, z_cap, seed, c_cap=0):
    return oracle.build_forest(X, Y, net_pin_off, pin_xy, n_tree_cand, z_cap, seed, c_cap)


def _assert_same(gpu: dict, ref: dict):
    for k, v in ref.items():
        np.testing.assert_array_equal(gpu[k].reshape(v.shape), v, err_msg=k)


@pytest.mark.gpu
@pytest.mark.parametrize("name,kw", [("tiny", {}), ("c1e4", {}), ("ispd18", {}), ("c1e4", {"n_tree_cand": 1}),
                                     ("c1e4", {"z_cap": -1}), ("c1e4", {"z_cap": 0}), ("tiny_c", {}),
                                     ("c1e4_c", {})])
def test_gpu_forest_equals_oracle(name, kw):
    f = forestgen.generate(name, **kw)
    c = f.meta["config"]
    b = dgr.build_forest(f.X, f.Y, f.net_pin_off, f.pin_xy, c["n_tree_cand"], c["z_cap"], c["seed"],
                         c_cap=c.get("c_cap", 0))
    _assert_same(b.download(), _oracle(f.X, f.Y, f.net_pin_off, f.pin_xy, c["n_tree_cand"], c["z_cap"], c["seed"],
                                       c.get("c_cap", 0)))


@pytest.mark.gpu
def test_gpu_forest_full_size_ispd19():
    """The bench workload's 956,622 nets: every array equal to the oracle's."""
    f = forestgen.generate("ispd19")
    c = f.meta["config"]
    b = dgr.build_forest(f.X, f.Y, f.net_pin_off, f.pin_xy, c["n_tree_cand"], c["z_cap"], c["seed"])
    _assert_same(b.download(), _oracle(f.X, f.Y, f.net_pin_off, f.pin_xy, c["n_tree_cand"], c["z_cap"], c["seed"]))


def _synthetic_pins(rng, n_nets, kmin, kmax, X, Y, box):
    off, pts = [0], []
    for _ in range(n_nets):
        k = int(rng.integers(kmin, kmax + 1))
        x0, y0 = int(rng.integers(0, X - box)), int(rng.integers(0, Y - box))
        seen = set()
        while len(seen) < k:
            p = (x0 + int(rng.integers(0, box)), y0 + int(rng.integers(0, box)))
            if p not in seen:
                seen.add(p)
                pts.append(p)
        off.append(len(pts))
    return np.asarray(off, np.int64), np.asarray(pts, np.int32)


@pytest.mark.gpu
@pytest.mark.parametrize("kmin,kmax,box", [(2, 2, 5), (8, 9, 6), (32, 32, 12), (3, 5, 3), (2, 32, 40)])
def test_gpu_forest_edge_cases(kmin, kmax, box):
    """2-pin nets, the 8/9-pin switch between 1-Steiner and the re-rooted MST, 32-pin nets,
    crowded boxes (many aligned / colinear pins), mixed sizes."""
    rng = np.random.default_rng(kmin * 100 + kmax)
    off, pts = _synthetic_pins(rng, 700, kmin, kmax, 64, 64, box)
    for ntc, zc, cc in ((2, 15, 0), (2, 0, 0), (1, -1, 0), (2, 11, 2), (2, 3, 5)):
        b = dgr.build_forest(64, 64, off, pts, ntc, zc, 7, c_cap=cc)
        _assert_same(b.download(), _oracle(64, 64, off, pts, ntc, zc, 7, cc))


@pytest.mark.gpu
def test_gpu_forest_empty():
    b = dgr.build_forest(8, 8, np.zeros(1, np.int64), np.zeros((0, 2), np.int32))
    d = b.download()
    assert b.n_nets == 0 and b.n_paths == 0 and d["net_tree_off"].tolist() == [0]


@pytest.mark.gpu
def test_gpu_built_forest_solves_like_the_generator():
    """Pins -> GPU forest -> solver gives the same iterations as the generator's forest."""
    f = forestgen.generate("c1e4")
    c = f.meta["config"]
    b = dgr.build_forest(f.X, f.Y, f.net_pin_off, f.pin_xy, c["n_tree_cand"], c["z_cap"], c["seed"]).download()
    g = forestgen.Forest(X=f.X, Y=f.Y, cap_h=f.cap_h, cap_v=f.cap_v, seed=f.seed, **b)
    s1, s2 = dgr.Solver(f), dgr.Solver(g)
    l1 = s1.step(20, 0.8, 0.3)
    l2 = s2.step(20, 0.8, 0.3)
    np.testing.assert_array_equal(l1, l2)
    np.testing.assert_array_equal(s1.logits()[1], s2.logits()[1])


@pytest.mark.parametrize("mutate,msg", [
    (lambda off, pts: (off, np.concatenate([pts[:1], pts[:1], pts[2:]])), "distinct"),   # duplicate pin
    (lambda off, pts: (off, np.where(np.arange(len(pts))[:, None] == 0, 99, pts)), "inside the grid"),
    (lambda off, pts: (np.asarray([0, 1] + [o for o in off[1:]], np.int64)[:len(off)], pts), "2.."),  # 1-pin net
])
def test_malformed_pins_rejected_on_host(mutate, msg):
    """Validation happens before any device work (runs without a GPU)."""
    off = np.asarray([0, 3, 6], np.int64)
    pts = np.asarray([[0, 0], [3, 1], [5, 5], [1, 1], [2, 2], [6, 0]], np.int32)
    off2, pts2 = mutate(off, pts)
    off2 = np.ascontiguousarray(off2, np.int64)
    pts2 = np.ascontiguousarray(pts2, np.int32)
    L = dgr.load_library()
    d = binding._PinsDesc(8, 8, len(off2) - 1, off2.ctypes.data, pts2.ctypes.data, 2, 15, 1)
    h = ctypes.c_void_p()
    rc = L.dgr_build_forest(ctypes.byref(d), None, ctypes.byref(h))
    assert rc == -1 and msg in L.dgr_last_error().decode()

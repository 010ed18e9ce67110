"""The C-ABI boundary without a GPU: the library loads, exports every symbol include/dgr.h
declares, shards nets, and rejects malformed forests with DGR_EINVAL (host-only calls)."""
import ctypes
import os
import re

import numpy as np
import pytest

import forestgen
import paper_conf_dac_0159layhrr24_b200 as dgr
from paper_conf_dac_0159layhrr24_b200 import dgr as binding

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared(header):
    txt = open(os.path.join(ROOT, "include", header)).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(dgr_[a-z_0-9]+)\s*\(", txt)))


def test_library_exports_every_declared_symbol():
    lib = dgr.load_library()
    names = _declared("dgr.h")
    assert {"dgr_forest_load", "dgr_step", "dgr_get_demand", "dgr_induce"} <= set(names)
    for n in names:
        assert hasattr(lib, n), n


def test_library_is_sm100a_cubin():
    import subprocess
    out = subprocess.run(["cuobjdump", "--list-elf", dgr.lib_path()], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_product_package_does_not_touch_the_oracle():
    pkg = os.path.join(ROOT, "paper_conf_dac_0159layhrr24_b200")
    for dirpath, _, files in os.walk(pkg):
        for fn in files:
            if fn.endswith((".py", ".cu", ".h", ".cpp")):
                txt = open(os.path.join(dirpath, fn)).read()
                assert "import oracle" not in txt and "from oracle" not in txt and "odgr_" not in txt, fn


def test_partition_contiguous_and_balanced(c1e4):
    for world in (1, 2, 3, 4, 8):
        part = dgr.partition(c1e4, world)
        assert part[0] == 0 and part[-1] == c1e4.n_nets and np.all(np.diff(part) >= 0)
        work = []
        for r in range(world):
            t0, t1 = c1e4.net_tree_off[part[r]], c1e4.net_tree_off[part[r + 1]]
            s0, s1 = c1e4.tree_sub_off[t0], c1e4.tree_sub_off[t1]
            p0, p1 = c1e4.sub_path_off[s0], c1e4.sub_path_off[s1]
            work.append((p1 - p0) + c1e4.path_seg_off[p1] - c1e4.path_seg_off[p0])
        assert max(work) - min(work) <= 2 * 200      # within ~one net's work of each other


def _ws(f):
    lib = dgr.load_library()
    d = binding._DescHolder(f)
    return lib.dgr_workspace_size(ctypes.byref(d.desc), None), lib.dgr_last_error().decode()


def test_workspace_size_of_valid_forest(tiny):
    n, err = _ws(tiny)
    assert n > 0 and err == ""


def test_dist_needs_nccl_id_or_allreduce_callback(tiny):
    """dgr_dist: world > 1 needs an NCCL id or a caller-supplied allreduce (host-only check)."""
    lib = dgr.load_library()
    d = binding._DescHolder(tiny)
    none = binding._Dist(0, 2, None)
    assert lib.dgr_workspace_size(ctypes.byref(d.desc), ctypes.byref(none)) == 0   # 0 on error
    assert "allreduce callback" in lib.dgr_last_error().decode()
    cb = binding.ALLREDUCE_FN(lambda *a: 0)
    for r in range(2):
        ok = binding._Dist(r, 2, None, cb, None)
        assert lib.dgr_workspace_size(ctypes.byref(d.desc), ctypes.byref(ok)) > 0, lib.dgr_last_error()
    bad = binding._Dist(2, 2, None, cb, None)
    assert lib.dgr_workspace_size(ctypes.byref(d.desc), ctypes.byref(bad)) == 0


@pytest.mark.parametrize("mutate,msg", [
    (lambda f: f.sub_path_off.__setitem__(3, f.sub_path_off[2]), "empty group"),
    (lambda f: f.net_tree_off.__setitem__(1, 0), "empty group"),
    (lambda f: f.seg.__setitem__((0, 3), f.seg[0, 2]), "malformed"),                 # empty segment
    (lambda f: f.tp_xy.__setitem__((0, 0), (f.tp_xy[0, 0] + 1) % f.X), "malformed"),  # turning point off the path
    (lambda f: f.seg.__setitem__((0, 1), f.Y + 3), "malformed"),                      # segment line outside the grid
    (lambda f: f.sub_xy.__setitem__((0, 2), 99), "outside the grid"),
    (lambda f: f.path_seg_off.__setitem__(2, f.path_seg_off[3] + 1), "monotone"),
])
def test_invalid_forest_rejected(tiny, mutate, msg):
    import copy
    f = copy.deepcopy(tiny)
    mutate(f)
    n, err = _ws(f)
    assert n == 0 and msg in err, err


def _info(f):
    lib = dgr.load_library()
    d = binding._DescHolder(f)
    out = (ctypes.c_int64 * 8)()
    rc = lib.dgr_plan_info(ctypes.byref(d.desc), None, out)
    return rc, lib.dgr_last_error().decode()


def test_general_nets_accepted():
    """Row f4' (reading Q14c): groups above 32 (uncapped Z), monotone staircases (4 turning points)
    and candidates in any order are planned onto the general path, not rejected."""
    f = forestgen.generate("c1e4", z_cap=0)          # uncapped Z: groups above 32 exist
    assert np.diff(f.sub_path_off).max() > 32
    n, err = _ws(f)
    assert n > 0 and err == "", err
    g = forestgen.generate("tiny_m")
    assert (np.diff(g.path_seg_off) == 5).any()
    assert _info(g)[0] == 0
    # a shuffled candidate order (reverse the candidates of every sub-net: CSR arrays rebuilt)
    h = forestgen.shuffle_candidates(forestgen.generate("tiny"), seed=3)
    assert _info(h)[0] == 0, _info(h)[1]


def test_group_above_limit_rejected():
    """More than kGenMaxGroup = 1024 candidates in one sub-net is DGR_EINVAL."""
    for seed in range(1, 200):
        f = forestgen.generate(dict(X=1200, Y=1200, n_nets=1, pins_mode=0, pins_min=2, pins_max=2, box_mode=0,
                                    box_min=1190, box_max=1190, track=1.0, n_tree_cand=1, z_cap=0, seed=seed))
        if f.n_subnets and np.diff(f.sub_path_off).max() > 1024:
            break
    assert np.diff(f.sub_path_off).max() > 1024
    n, err = _ws(f)
    assert n == 0 and "> 1024 candidates" in err, err


def test_gpu_required_without_cuda(tiny):
    import torch
    if torch.cuda.is_available():
        pytest.skip("has a GPU")
    with pytest.raises(dgr.DgrError):
        dgr.Solver(tiny)


@pytest.mark.parametrize("name", ["tiny", "c1e4", "ispd18"])
def test_plan_tiles_cover_the_forest(name):
    f = forestgen.generate(name)
    pi = dgr.plan_info(f)
    assert pi["n_paths"] == f.n_paths
    assert pi["n_slots"] >= f.n_paths and pi["n_slots"] % 32 == 0
    assert pi["n_slots"] <= 1.25 * f.n_paths + 32 * pi["n_tiles"]      # padding stays bounded
    assert pi["max_window"] <= 2048
    assert pi["global_paths"] <= 0.01 * f.n_paths                       # almost all tiles use SMEM windows
    for world in (2, 3):
        tot = sum(dgr.plan_info(f, rank=r, world=world)["n_paths"] for r in range(world))
        assert tot == f.n_paths


def _permute_candidates(f, s, order):
    """Copy of forest f with sub-net s's candidates listed in `order` (CSR arrays rebuilt)."""
    import copy
    g = copy.deepcopy(f)
    p0 = int(f.sub_path_off[s])
    perm = np.arange(f.n_paths)
    perm[p0:p0 + len(order)] = p0 + np.asarray(order)
    segs, tps, so, to = [], [], [0], [0]
    for i in perm:
        a, b = f.path_seg_off[i], f.path_seg_off[i + 1]
        segs.append(f.seg[a:b]); so.append(so[-1] + b - a)
        a, b = f.path_tp_off[i], f.path_tp_off[i + 1]
        tps.append(f.tp_xy[a:b]); to.append(to[-1] + b - a)
    g.seg = np.ascontiguousarray(np.concatenate(segs)).astype(f.seg.dtype)
    g.tp_xy = np.ascontiguousarray(np.concatenate(tps)).astype(f.tp_xy.dtype)
    g.path_seg_off = np.asarray(so, dtype=f.path_seg_off.dtype)
    g.path_tp_off = np.asarray(to, dtype=f.path_tp_off.dtype)
    g.w_path0 = np.ascontiguousarray(f.w_path0[perm])
    return g


def test_candidate_order_contract(tiny):
    """dgr.h: any order of a sub-net's candidates is accepted.  The canonical order (HV, VH, Z-HVH...,
    Z-VHV..., C...) runs in the tile kernels, any other on the general path (row f4'); the plan
    reports the general candidates (dgr_get_info info[11] on a bound handle)."""
    n = np.diff(tiny.sub_path_off)
    s = int(np.nonzero(n >= 4)[0][0])
    ok, err = _ws(_permute_candidates(tiny, s, list(range(n[s]))))
    assert ok > 0 and err == ""
    for order in ([1, 0] + list(range(2, n[s])), [2, 0, 1] + list(range(3, n[s]))):
        ws, err = _ws(_permute_candidates(tiny, s, order))
        assert ws > 0 and err == "", err
    s2 = int(np.nonzero(n == 2)[0][0]) if (n == 2).any() else None
    if s2 is not None:
        assert _ws(_permute_candidates(tiny, s2, [1, 0]))[0] > 0


@pytest.mark.parametrize("xm", [-3, -1, "X", "X+2"])
def test_c_shape_detour_outside_grid_rejected(xm):
    """A C-shape detour (reading Q14b) whose x_m lies outside the grid is DGR_EINVAL: its demand
    events and S reads would otherwise index outside the grid."""
    import copy
    f = copy.deepcopy(forestgen.generate("tiny_c"))
    xm = {"X": f.X, "X+2": f.X + 2}.get(xm, xm)
    for i in range(f.n_paths):
        t0, t1 = f.path_tp_off[i], f.path_tp_off[i + 1]
        if t1 - t0 != 2 or f.tp_xy[t0, 0] != f.tp_xy[t0 + 1, 0]:
            continue
        s = int(np.searchsorted(f.sub_path_off, i, side="right") - 1)
        x0, y0, x1, y1 = f.sub_xy[s]
        if min(x0, x1) <= f.tp_xy[t0, 0] <= max(x0, x1):
            continue                                          # a Z, not a C-HVH
        f.tp_xy[t0:t1, 0] = xm
        for g in range(f.path_seg_off[i], f.path_seg_off[i + 1]):
            d, line, lo, hi = f.seg[g]
            if d == 1:
                f.seg[g, 1] = xm
            else:
                xe = x0 if line == y0 else x1
                f.seg[g, 2], f.seg[g, 3] = min(xe, xm), max(xe, xm)
        break
    else:
        pytest.fail("tiny_c has no C-HVH candidate")
    n, err = _ws(f)
    assert n == 0 and "malformed" in err, err


def test_plan_restores_a_spatial_net_order():
    """the plan takes nets in a spatial (Morton) order when the caller's order is
    not spatially coherent, so a net-shuffled forest tiles like the sorted one (dgr_plan_info)."""
    f = forestgen.generate("c1e4")
    g = forestgen.shuffle_nets(f, seed=5)
    a, b = dgr.plan_info(f), dgr.plan_info(g)
    assert b["n_paths"] == a["n_paths"]
    assert b["n_tiles"] <= 1.1 * a["n_tiles"] and b["n_global_tiles"] <= a["n_global_tiles"] + 2, (a, b)

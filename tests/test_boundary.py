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


@pytest.mark.parametrize("mutate,msg", [
    (lambda f: f.sub_path_off.__setitem__(3, f.sub_path_off[2]), "empty group"),
    (lambda f: f.net_tree_off.__setitem__(1, 0), "empty group"),
    (lambda f: f.seg.__setitem__((0, 3), f.seg[0, 2]), "pattern"),
    (lambda f: f.tp_xy.__setitem__((0, 0), (f.tp_xy[0, 0] + 1) % f.X), "pattern"),
    (lambda f: f.sub_xy.__setitem__((0, 2), 99), "outside the grid"),
    (lambda f: f.path_seg_off.__setitem__(2, f.path_seg_off[3] + 1), "monotone"),
])
def test_invalid_forest_rejected(tiny, mutate, msg):
    import copy
    f = copy.deepcopy(tiny)
    mutate(f)
    n, err = _ws(f)
    assert n == 0 and msg in err, err


def test_group_of_33_rejected(tiny):
    f = forestgen.generate("c1e4", z_cap=0)          # uncapped Z: groups above 32 exist
    assert np.diff(f.sub_path_off).max() > 32
    n, err = _ws(f)
    assert n == 0 and "> 32 candidates" in err


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

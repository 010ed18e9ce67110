"""The shared input generator: determinism, CSR validity, pattern shapes, .dgrf round trip."""
import os
import subprocess
import sys
import tempfile

import numpy as np
import pytest

import forestgen
from tests import _ref


def _check_forest(f):
    for off in (f.net_tree_off, f.tree_sub_off, f.sub_path_off, f.path_seg_off, f.path_tp_off):
        assert off[0] == 0 and np.all(np.diff(off) >= 0)
    assert np.all(np.diff(f.net_tree_off) >= 1) and np.all(np.diff(f.tree_sub_off) >= 1)
    assert np.all(np.diff(f.sub_path_off) >= 1) and np.all(np.diff(f.sub_path_off) <= 32)
    X, Y = f.X, f.Y
    s = f.seg
    assert np.all((s[:, 0] == 0) | (s[:, 0] == 1))
    assert np.all(s[:, 2] < s[:, 3]) and np.all(s[:, 2] >= 0)
    h, v = s[:, 0] == 0, s[:, 0] == 1
    assert np.all(s[h, 3] <= X - 1) and np.all(s[h, 1] < Y) and np.all(s[v, 3] <= Y - 1) and np.all(s[v, 1] < X)
    x0, y0, x1, y1 = f.sub_xy.T
    assert np.all((x0 < x1) | ((x0 == x1) & (y0 < y1)))          # canonical orientation
    # every candidate is a monotone path from (x0,y0) to (x1,y1): WL = |dx| + |dy|, TP = #seg - 1
    path_sub = np.repeat(np.arange(f.n_subnets), np.diff(f.sub_path_off))
    wl = np.add.reduceat(s[:, 3] - s[:, 2], f.path_seg_off[:-1])
    man = np.abs(x1 - x0) + np.abs(y1 - y0)
    assert np.array_equal(wl, man[path_sub])
    assert np.array_equal(np.diff(f.path_tp_off), np.diff(f.path_seg_off) - 1)


def test_tiny_and_c1e4_valid(tiny, c1e4):
    _check_forest(tiny)
    _check_forest(c1e4)
    assert tiny.n_nets == 40 and tiny.X == 16


def test_turning_points_lie_on_their_paths(tiny):
    for i in range(tiny.n_paths):
        cells = set()
        for d, y, x in _ref.path_edges(tiny, i):
            cells.add((x, y)); cells.add((x + 1, y) if d == 0 else (x, y + 1))
        for tp in _ref.path_tps(tiny, i):
            assert tp in cells


def test_z_cap_and_order(c1e4):
    f = c1e4
    for s in range(0, f.n_subnets, 7):
        a, b = f.sub_path_off[s], f.sub_path_off[s + 1]
        x0, y0, x1, y1 = f.sub_xy[s]
        if x0 == x1 or y0 == y1:
            assert b - a == 1
            continue
        nh = min(x1 - x0 - 1, 15)
        nv = min(abs(y1 - y0) - 1, 15)
        assert b - a == 2 + nh + nv
        xm = [f.seg[f.path_seg_off[i] + 1, 1] for i in range(a + 2, a + 2 + nh)]    # V segment line = x_m
        assert xm == sorted(set(xm)) and all(x0 < x < x1 for x in xm)


def test_deterministic_across_thread_counts():
    code = ("import forestgen,sys; f=forestgen.generate('c1e4'); sys.stdout.write(f.sha256())")
    env = dict(os.environ)
    shas = []
    for th in ("1", "4"):
        env["OMP_NUM_THREADS"] = th
        shas.append(subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True,
                                   cwd=os.path.dirname(os.path.dirname(__file__)), check=True).stdout)
    assert shas[0] == shas[1] and len(shas[0]) == 64


def test_dgrf_round_trip(tiny):
    with tempfile.TemporaryDirectory() as td:
        p = os.path.join(td, "t.dgrf")
        forestgen.write_dgrf(tiny, p)
        g = forestgen.read_dgrf(p)
    assert g.sha256() == tiny.sha256()


def test_morton_order(c1e4):
    f = c1e4
    def part(x):
        x &= 0xFFFF
        x = (x | (x << 8)) & 0x00FF00FF; x = (x | (x << 4)) & 0x0F0F0F0F
        x = (x | (x << 2)) & 0x33333333; x = (x | (x << 1)) & 0x55555555
        return x
    keys = []
    for n in range(f.n_nets):
        p = f.pin_xy[f.net_pin_off[n]:f.net_pin_off[n + 1]]
        keys.append(part(int(p[:, 0].min() + p[:, 0].max())) | (part(int(p[:, 1].min() + p[:, 1].max())) << 1))
    assert np.all(np.diff(keys) >= 0)


def test_capacity_quarters_and_padding(c1e4):
    assert np.all(c1e4.cap_h[:, -1] == 0) and np.all(c1e4.cap_v[-1, :] == 0)
    assert np.all(np.asarray(c1e4.cap_h * 4) == np.round(c1e4.cap_h * 4))


@pytest.mark.parametrize("name", ["c1e4", "ispd18"])
def test_stats_near_survey_estimates(name):
    f = forestgen.generate(name)
    ratio = f.n_paths / f.n_nets
    assert 5 < ratio < 12

"""Row f1 oracle (oracle/forest_oracle.c): routing-DAG-forest construction (§4.2, P:524-539;
readings Q8, Q14, Q17 in DESIGN.md §3), pinned against library routines and closed forms."""
import numpy as np
import pytest
from scipy.sparse.csgraph import minimum_spanning_tree

import forestgen
import oracle


def _built(f):
    c = f.meta["config"]
    return oracle.build_forest(f.X, f.Y, f.net_pin_off, f.pin_xy, c["n_tree_cand"], c["z_cap"], c["seed"],
                               c.get("c_cap", 0))


def _tree_subs(o, n):
    """sub-nets (x0, y0, x1, y1) of each tree of net n"""
    out = []
    for j in range(o["net_tree_off"][n], o["net_tree_off"][n + 1]):
        out.append(o["sub_xy"][o["tree_sub_off"][j]:o["tree_sub_off"][j + 1]])
    return out


def _manhattan_mst(pts):
    d = np.abs(pts[:, None, :] - pts[None, :, :]).sum(-1).astype(float)
    d[d == 0] = 1e-9          # distinct points only; keep zero-length edges representable
    np.fill_diagonal(d, 0)
    return minimum_spanning_tree(d).sum()


@pytest.fixture(scope="module")
def c1e4_built(c1e4):
    return _built(c1e4)


def test_oracle_equals_the_input_generator(tiny, c1e4, c1e4_built):
    """Two independent statements of readings Q8/Q14/Q17 (forestgen's generator and the oracle)
    agree bit for bit on every array."""
    for f, o in ((tiny, _built(tiny)), (c1e4, c1e4_built)):
        for k, v in o.items():
            np.testing.assert_array_equal(np.asarray(getattr(f, k)).reshape(v.shape), v, err_msg=k)


def test_candidate0_is_a_minimum_spanning_tree(c1e4, c1e4_built):
    """Candidate 0 = Prim MST (Q17): its length equals scipy's minimum spanning tree (Manhattan)."""
    o = c1e4_built
    for n in range(0, c1e4.n_nets, 7):
        pins = c1e4.pin_xy[c1e4.net_pin_off[n]:c1e4.net_pin_off[n + 1]]
        t0 = _tree_subs(o, n)[0]
        assert len(t0) == len(pins) - 1
        length = np.abs(t0[:, 2] - t0[:, 0]).sum() + np.abs(t0[:, 3] - t0[:, 1]).sum()
        assert abs(length - _manhattan_mst(pins.astype(np.int64))) < 1e-6


def _components(points, subs):
    idx = {tuple(p): i for i, p in enumerate(points)}
    parent = list(range(len(points)))

    def find(a):
        while parent[a] != a:
            parent[a] = parent[parent[a]]
            a = parent[a]
        return a
    for s in subs:
        a, b = find(idx[(s[0], s[1])]), find(idx[(s[2], s[3])])
        parent[a] = b
    return len({find(i) for i in range(len(points))})


def test_candidate1_is_a_steiner_tree_no_longer_than_the_mst(c1e4, c1e4_built):
    """Candidate 1 (iterated 1-Steiner, k <= 8): a tree over the pins plus Steiner points of degree
    >= 3, no longer than the MST, and exactly the half-perimeter (the RSMT closed form) for 3 pins."""
    o = c1e4_built
    checked3 = 0
    for n in range(c1e4.n_nets):
        pins = c1e4.pin_xy[c1e4.net_pin_off[n]:c1e4.net_pin_off[n + 1]]
        trees = _tree_subs(o, n)
        if len(trees) < 2:
            continue
        t0, t1 = trees
        l0 = np.abs(t0[:, 2] - t0[:, 0]).sum() + np.abs(t0[:, 3] - t0[:, 1]).sum()
        l1 = np.abs(t1[:, 2] - t1[:, 0]).sum() + np.abs(t1[:, 3] - t1[:, 1]).sum()
        pts = {tuple(p) for p in pins}
        ends = {(s[0], s[1]) for s in t1} | {(s[2], s[3]) for s in t1}
        assert pts <= ends
        steiner = ends - pts
        allp = [tuple(p) for p in pins] + sorted(steiner)
        assert len(t1) == len(allp) - 1 and _components(allp, t1) == 1
        deg = {p: 0 for p in steiner}
        for s in t1:
            for e in ((s[0], s[1]), (s[2], s[3])):
                if e in deg:
                    deg[e] += 1
        assert all(v >= 3 for v in deg.values())
        if len(pins) <= 8:
            assert l1 <= l0
        if len(pins) == 3:
            hp = pins[:, 0].max() - pins[:, 0].min() + pins[:, 1].max() - pins[:, 1].min()
            assert l1 == hp
            checked3 += 1
    assert checked3 > 50


def test_candidate1_is_a_local_optimum_of_the_1_steiner_step(c1e4, c1e4_built):
    """Candidate 1 against the definition of iterated 1-Steiner (reading Q17, Kahng-Robins), checked
    with scipy's MST rather than the oracle's Prim: (a) its edges form a minimum spanning tree of
    pins + Steiner points; (b) it is a fixed point of the 1-Steiner step: adding any further Hanan
    grid point of the pins does not shorten that point set's MST (the loop stops only then).  Nets
    of 3..6 pins (Hanan grids of <= 36 points)."""
    o = c1e4_built
    checked = 0
    for n in range(c1e4.n_nets):
        pins = c1e4.pin_xy[c1e4.net_pin_off[n]:c1e4.net_pin_off[n + 1]].astype(np.int64)
        if not 3 <= len(pins) <= 6:
            continue
        trees = _tree_subs(o, n)
        if len(trees) < 2:
            continue
        t1 = trees[1]
        pset = {tuple(p) for p in pins}
        ends = {(s[0], s[1]) for s in t1} | {(s[2], s[3]) for s in t1}
        pts = np.array([tuple(p) for p in pins] + sorted(ends - pset), np.int64)
        l1 = np.abs(t1[:, 2] - t1[:, 0]).sum() + np.abs(t1[:, 3] - t1[:, 1]).sum()
        mst = _manhattan_mst(pts)
        assert abs(l1 - mst) < 1e-6, (n, l1, mst)                                     # (a)
        have = {tuple(p) for p in pts}
        for hx in np.unique(pins[:, 0]):
            for hy in np.unique(pins[:, 1]):
                if (hx, hy) in have:
                    continue
                grown = _manhattan_mst(np.vstack([pts, [[hx, hy]]]))
                assert grown >= mst - 1e-6, (n, (hx, hy), grown, mst)                   # (b)
        checked += 1
    assert checked > 100


def test_path_candidates_are_the_patterns(tiny):
    """Every candidate is a monotone route between its sub-net's endpoints (length |dx| + |dy|,
    turning points = segments - 1), groups are straight / HV, VH, Z... (Q14, all Z on tiny)."""
    o = _built(tiny)
    for s in range(len(o["sub_path_off"]) - 1):
        x0, y0, x1, y1 = o["sub_xy"][s]
        a, b = o["sub_path_off"][s], o["sub_path_off"][s + 1]
        aligned = x0 == x1 or y0 == y1
        assert (b - a) == (1 if aligned else 2 + max(x1 - x0 - 1, 0) + max(abs(y1 - y0) - 1, 0))
        for i in range(a, b):
            segs = o["seg"][o["path_seg_off"][i]:o["path_seg_off"][i + 1]]
            tps = o["path_tp_off"][i + 1] - o["path_tp_off"][i]
            assert (segs[:, 3] - segs[:, 2]).sum() == (x1 - x0) + abs(y1 - y0)
            assert tps == len(segs) - 1


def test_initial_logits_uniform(c1e4_built):
    w = np.concatenate([c1e4_built["w_tree0"], c1e4_built["w_path0"]])
    assert w.min() >= 0.0 and w.max() < 1.0 and abs(w.mean() - 0.5) < 0.01


def test_single_tree_candidate_and_l_only():
    f = forestgen.generate("c1e4", n_tree_cand=1, z_cap=-1)
    o = _built(f)
    assert np.all(np.diff(o["net_tree_off"]) == 1)
    assert np.diff(o["sub_path_off"]).max() <= 2
    for k, v in o.items():
        np.testing.assert_array_equal(np.asarray(getattr(f, k)).reshape(v.shape), v, err_msg=k)


def test_c_shape_detours():
    """Reading Q14b (row f4): C-HVH / C-VHV candidates after the Z's, x_m (y_m) outside the sub-net's
    span by 1..c_cap on each side inside the grid; length = |dx| + |dy| + 2 x detour, 2 turning points."""
    f = forestgen.generate("tiny_c")
    o = _built(f)
    c = f.meta["config"]["c_cap"]
    nc = 0
    for s in range(len(o["sub_path_off"]) - 1):
        x0, y0, x1, y1 = o["sub_xy"][s]
        a, b = o["sub_path_off"][s], o["sub_path_off"][s + 1]
        if x0 == x1 or y0 == y1:
            assert b - a == 1
            continue
        ylo, yhi = min(y0, y1), max(y0, y1)
        ncx = min(c, x0) + min(c, f.X - 1 - x1)
        ncy = min(c, ylo) + min(c, f.Y - 1 - yhi)
        nz = (x1 - x0 - 1) + (yhi - ylo - 1)          # tiny_c: every Z
        assert b - a == 2 + nz + ncx + ncy
        for r, i in enumerate(range(b - ncx - ncy, b)):
            segs = o["seg"][o["path_seg_off"][i]:o["path_seg_off"][i + 1]]
            tp = o["tp_xy"][o["path_tp_off"][i]:o["path_tp_off"][i + 1]]
            assert len(segs) == 3 and len(tp) == 2
            if r < ncx:    # C-HVH: turning points on column x_m outside [x0, x1]
                m = tp[0, 0]
                assert tp[1, 0] == m and (m < x0 or m > x1)
                det = x0 - m if m < x0 else m - x1
            else:          # C-VHV: turning points on row y_m outside [ylo, yhi]
                m = tp[0, 1]
                assert tp[1, 1] == m and (m < ylo or m > yhi)
                det = ylo - m if m < ylo else m - yhi
            assert 1 <= det <= c
            assert (segs[:, 3] - segs[:, 2]).sum() == (x1 - x0) + (yhi - ylo) + 2 * det
            nc += 1
    assert nc > 100

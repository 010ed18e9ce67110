"""Pins for the oracle's expected demand and cost (Eqs. (2), (9)-(12)).

* one-hot probabilities reduce Eq. (10) to the integer rasterisation of Eq. (2), bit-exactly;
* conservation: sum_e d_e = E[WL] + beta * sum_i pi_i * sum_{v in TP(i)} deg(v);
* brute-force expectation over every discrete selection on small sub-forests (reading Q20);
* the cost equals a torch restatement (library sigmoid/relu) given the same noise.
"""
import numpy as np
import pytest
import torch

import forestgen
import oracle
from tests import _ref


def _one_hot_logits(f, rng):
    """Logits with a winner gap of 1000: fp64 softmax gives exact 0/1 at any t >= 0.5."""
    wt = np.zeros(f.n_trees); wp = np.zeros(f.n_paths)
    tree_pick, path_pick = [], []
    for n in range(f.n_nets):
        a, b = f.net_tree_off[n], f.net_tree_off[n + 1]
        j = int(rng.integers(a, b)); wt[j] = 1000.0; tree_pick.append(j)
    for s in range(f.n_subnets):
        a, b = f.sub_path_off[s], f.sub_path_off[s + 1]
        i = int(rng.integers(a, b)); wp[i] = 1000.0; path_pick.append(i)
    return wt, wp, tree_pick, path_pick


@pytest.mark.parametrize("beta", [0.0, 0.25])
def test_one_hot_demand_equals_integer_rasterisation(tinyx, beta):
    rng = np.random.default_rng(5)
    o = oracle.Oracle(tinyx)
    wt, wp, tree_pick, path_pick = _one_hot_logits(tinyx, rng)
    o.set_logits(wt, wp)
    o.forward(1.0, oracle.weights(beta=beta))
    q, p = o.probs()
    assert set(np.unique(q)) <= {0.0, 1.0} and set(np.unique(p)) <= {0.0, 1.0}
    sel = []
    for j in tree_pick:
        for s in range(tinyx.tree_sub_off[j], tinyx.tree_sub_off[j + 1]):
            sel.append(path_pick[s])
    dh_ref, dv_ref = _ref.rasterise(tinyx, sel, beta=beta)
    dh, dv = o.demand()
    assert np.array_equal(dh, dh_ref) and np.array_equal(dv, dv_ref)


def test_conservation(tinyx):
    beta = 0.25
    o = oracle.Oracle(tinyx)
    out = o.forward(0.8, oracle.weights(beta=beta))
    q, p = o.probs()
    path_tree = np.repeat(np.repeat(np.arange(tinyx.n_trees), np.diff(tinyx.tree_sub_off)), np.diff(tinyx.sub_path_off))
    pi = q[path_tree] * p
    dh, dv = o.demand()
    ewl = out[1]
    via_total = 0.0
    for i in range(tinyx.n_paths):
        for (x, y) in _ref.path_tps(tinyx, i):
            via_total += pi[i] * len(_ref.incident_edges(tinyx.X, tinyx.Y, x, y))
    assert abs(dh.sum() + dv.sum() - (ewl + beta * via_total)) < 1e-9
    o0 = oracle.Oracle(tinyx)
    out0 = o0.forward(0.8, oracle.weights(beta=0.0))
    dh0, dv0 = o0.demand()
    assert abs(dh0.sum() + dv0.sum() - out0[1]) < 1e-9          # beta = 0: sum_e W_e = E[WL]


def _small_subforest(f, max_space=20000):
    """Pick consecutive nets of the tiny forest whose joint selection space is small."""
    def n_opts(n):
        tot = 0
        for j in range(f.net_tree_off[n], f.net_tree_off[n + 1]):
            c = 1
            for s in range(f.tree_sub_off[j], f.tree_sub_off[j + 1]):
                c *= int(f.sub_path_off[s + 1] - f.sub_path_off[s])
            tot += c
        return tot
    picks = []
    for lo in range(f.n_nets - 2):
        space = n_opts(lo) * n_opts(lo + 1) * n_opts(lo + 2)
        has_two_trees = any(f.net_tree_off[n + 1] - f.net_tree_off[n] > 1 for n in range(lo, lo + 3))
        if space <= max_space and has_two_trees:
            picks.append(lo)
    return picks


@pytest.mark.parametrize("which", [0, 1, 2])
def test_brute_force_expectation(tinyx, which):
    """E[D_e], E[WL], E[TP] of Eq. (10)-(12) equal the enumeration of every discrete selection.
    For the staircase recipe (row f4') the enumerable sub-forests come from the same recipe with
    small boxes and one staircase per orientation (its large groups are not enumerable)."""
    if tinyx.meta["config"].get("m_cap", 0):
        tinyx = forestgen.generate(dict(tinyx.meta["config"], box_min=4, box_max=7, z_cap=1, c_cap=0, m_cap=1))
        assert any(np.diff(tinyx.path_seg_off) == 5)
    los = _small_subforest(tinyx)
    assert len(los) > which
    lo = los[which * (len(los) // 3)]
    f = forestgen.subset(tinyx, lo, lo + 3)
    beta = 0.25
    o = oracle.Oracle(f)
    o.iteration = 4
    out = o.forward(0.6, oracle.weights(beta=beta))
    q, p = o.probs()
    dh, dv = o.demand()
    Eh = np.zeros_like(dh); Ev = np.zeros_like(dv); Ewl = 0.0; Etp = 0.0; Ptot = 0.0
    path_sub = np.repeat(np.arange(f.n_subnets), np.diff(f.sub_path_off))
    for trees, paths in _ref.enumerate_selections(f):
        pr = np.prod([q[j] for j in trees]) * np.prod([p[i] for i in paths])
        Ptot += pr
        h, v = _ref.rasterise(f, paths, beta=beta)
        Eh += pr * h; Ev += pr * v
        for i in paths:
            Ewl += pr * sum(int(s[3] - s[2]) for s in f.seg[f.path_seg_off[i]:f.path_seg_off[i + 1]])
            Etp += pr * (f.path_tp_off[i + 1] - f.path_tp_off[i])
    assert abs(Ptot - 1) < 1e-12
    np.testing.assert_allclose(dh, Eh, rtol=0, atol=1e-12)
    np.testing.assert_allclose(dv, Ev, rtol=0, atol=1e-12)
    assert abs(out[1] - Ewl) < 1e-10
    assert abs(out[2] - np.sqrt(5.0) * Etp) < 1e-10
    assert len(path_sub) == f.n_paths


@pytest.mark.parametrize("f_kind,slope", [(0, 1.0), (1, 1.0), (2, 0.01), (3, 0.5), (4, 1.0)])
def test_cost_matches_torch_restatement(tinyx, f_kind, slope):
    """sigmoid, ReLU and the LeakyReLU / exp / CELU alternatives of Fig. 6."""
    W = oracle.weights(f_kind=f_kind, f_slope=slope)
    o = oracle.Oracle(tinyx)
    o.iteration = 2
    t = 0.9
    out = o.forward(t, W)
    g = torch.tensor(_ref.path_noise(tinyx, 2), dtype=torch.float64)
    gt = torch.tensor([oracle.gumbel(tinyx.seed, j, 2, 1) for j in range(tinyx.n_trees)], dtype=torch.float64)
    cost, d, ewl, etp, of, _, _ = _ref.torch_cost(tinyx, torch.tensor(tinyx.w_tree0, dtype=torch.float64),
                                                  torch.tensor(tinyx.w_path0, dtype=torch.float64), gt, g, t, W)
    assert abs(out[0] - cost.item()) <= 1e-11 * abs(cost.item())
    assert abs(out[1] - ewl.item()) < 1e-10
    assert abs(out[3] - of.item()) < 1e-9
    dh, dv = o.demand()
    np.testing.assert_allclose(np.concatenate([dh.reshape(-1), dv.reshape(-1)]), d.numpy(), atol=1e-12)


def test_weights_are_the_papers(tiny):
    """The default weights are the ICCAD'19 metric weights printed at P:582-583 (golden file)."""
    import os
    gold = {}
    for line in open(os.path.join(os.path.dirname(__file__), "golden", "hyperparams.txt")):
        if line.startswith("#") or not line.strip():
            continue
        k, v = line.split()[:2]
        gold[k] = float(v)
    W = oracle.weights()
    assert (W.a_wl, W.a_via, W.a_of) == (gold["a_wl"], gold["a_via"], gold["a_of"])


def test_fig4_candidate_pattern():
    """Fig. 4: aligned sub-nets -> one straight candidate with 0 vias; others -> two L
    candidates of equal WL with 1 via each (L-only forest, as in the paper's §4.2 construction)."""
    import os
    gold = [tuple(int(v) for v in line.split()) for line in
            open(os.path.join(os.path.dirname(__file__), "golden", "fig4_wl_via.txt"))
            if line.strip() and not line.startswith("#")]
    assert {(v, m) for _, v, m in gold} == {(0, 1), (1, 2)}
    f = forestgen.generate("tiny", z_cap=-1)
    for s in range(f.n_subnets):
        a, b = f.sub_path_off[s], f.sub_path_off[s + 1]
        wls = [sum(int(g[3] - g[2]) for g in f.seg[f.path_seg_off[i]:f.path_seg_off[i + 1]]) for i in range(a, b)]
        vias = [int(f.path_tp_off[i + 1] - f.path_tp_off[i]) for i in range(a, b)]
        assert (b - a, tuple(sorted(set(vias)))) in {(1, (0,)), (2, (1,))}
        assert len(set(wls)) == 1

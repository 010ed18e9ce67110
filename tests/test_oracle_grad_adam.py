"""Pins for the oracle's reverse pass and Adam (P:841-847 autograd, P:913-914 Adam).

* central finite differences of the oracle's own cost (fp64);
* torch autograd of a torch restatement of Eqs. (9)-(12) (library gradient);
* softmax shift invariance => per-group sum of dw is zero;
* the oracle's Adam vs torch.optim.Adam fed the same gradient stream.
"""
import numpy as np
import pytest
import torch

import oracle
from tests import _ref


def _grad(f, k, t, W):
    o = oracle.Oracle(f)
    o.iteration = k
    o.forward(t, W)
    return o, o.backward(t, W)


@pytest.mark.parametrize("beta", [0.0, 0.25])
def test_gradient_central_differences(tiny, beta):
    W = oracle.weights(beta=beta)
    t, k = 0.8, 3
    o, (dw, du) = _grad(tiny, k, t, W)
    wt0, wp0 = o.logits()
    rng = np.random.default_rng(1)
    # cost ~ 1e5: fp64 cancellation ~ eps*|L|/h ~ 1e-7 and truncation ~ h^2 at h = 1e-4
    h = 1e-4
    for i in rng.choice(tiny.n_paths, 12, replace=False):
        vals = []
        for sgn in (1, -1):
            oo = oracle.Oracle(tiny); oo.iteration = k
            wp = wp0.copy(); wp[i] += sgn * h
            oo.set_logits(wt0, wp)
            vals.append(oo.forward(t, W)[0])
        fd = (vals[0] - vals[1]) / (2 * h)
        assert abs(fd - dw[i]) <= 1e-5 * max(1.0, abs(dw[i])), (i, fd, dw[i])
    multi = [j for n in range(tiny.n_nets) if tiny.net_tree_off[n + 1] - tiny.net_tree_off[n] > 1
             for j in range(tiny.net_tree_off[n], tiny.net_tree_off[n + 1])]
    for j in rng.choice(multi, 8, replace=False):
        vals = []
        for sgn in (1, -1):
            oo = oracle.Oracle(tiny); oo.iteration = k
            wt = wt0.copy(); wt[j] += sgn * h
            oo.set_logits(wt, wp0)
            vals.append(oo.forward(t, W)[0])
        fd = (vals[0] - vals[1]) / (2 * h)
        assert abs(fd - du[j]) <= 1e-5 * max(1.0, abs(du[j])), (j, fd, du[j])


def test_gradient_central_differences_relu_away_from_kinks(tiny):
    """ReLU f (Table 1 objective): FD agrees wherever no edge sits within h of d == cap."""
    W = oracle.weights(f_kind=1)
    t, k = 0.6, 1
    o, (dw, du) = _grad(tiny, k, t, W)
    wt0, wp0 = o.logits()
    h = 1e-7
    rng = np.random.default_rng(2)
    checked = 0
    for i in rng.choice(tiny.n_paths, 20, replace=False):
        vals = []
        for sgn in (1, -1):
            oo = oracle.Oracle(tiny); oo.iteration = k
            wp = wp0.copy(); wp[i] += sgn * h
            oo.set_logits(wt0, wp)
            vals.append(oo.forward(t, W)[0])
        fd = (vals[0] - vals[1]) / (2 * h)
        if abs(fd - dw[i]) <= 1e-5 * max(1.0, abs(dw[i])):
            checked += 1
    assert checked >= 15


@pytest.mark.parametrize("f_kind,slope", [(0, 1.0), (1, 1.0), (2, 0.01), (3, 0.5), (4, 1.0)])
def test_gradient_matches_torch_autograd(tinyx, f_kind, slope):
    W = oracle.weights(f_kind=f_kind, f_slope=slope)
    t, k = 0.7, 5
    o, (dw, du) = _grad(tinyx, k, t, W)
    g = torch.tensor(_ref.path_noise(tinyx, k), dtype=torch.float64)
    gt = torch.tensor([oracle.gumbel(tinyx.seed, j, k, 1) for j in range(tinyx.n_trees)], dtype=torch.float64)
    wp = torch.tensor(tinyx.w_path0, dtype=torch.float64, requires_grad=True)
    wt = torch.tensor(tinyx.w_tree0, dtype=torch.float64, requires_grad=True)
    cost, *_ = _ref.torch_cost(tinyx, wt, wp, gt, g, t, W)
    cost.backward()
    np.testing.assert_allclose(dw, wp.grad.numpy(), rtol=1e-9, atol=1e-9)
    np.testing.assert_allclose(du, wt.grad.numpy(), rtol=1e-9, atol=1e-9)


def test_group_gradient_sums_to_zero(tinyx):
    o, (dw, du) = _grad(tinyx, 0, 1.0, oracle.weights())
    for s in range(tinyx.n_subnets):
        a, b = tinyx.sub_path_off[s], tinyx.sub_path_off[s + 1]
        assert abs(dw[a:b].sum()) <= 1e-9 * max(1.0, np.abs(dw[a:b]).max())
    for n in range(tinyx.n_nets):
        a, b = tinyx.net_tree_off[n], tinyx.net_tree_off[n + 1]
        assert abs(du[a:b].sum()) <= 1e-9 * max(1.0, np.abs(du[a:b]).max())


def test_adam_matches_torch_optim(tiny):
    """Iterate the oracle; feed each iteration's gradient to torch.optim.Adam (fp64, lr 0.3)."""
    W = oracle.weights()
    lr = 0.3
    o = oracle.Oracle(tiny)
    wt0, wp0 = o.logits()
    pt = torch.nn.Parameter(torch.tensor(wt0)); pp = torch.nn.Parameter(torch.tensor(wp0))
    opt = torch.optim.Adam([pt, pp], lr=lr)
    for it in range(25):
        t = 0.9 ** (it // 10)
        o.forward(t, W)
        dw, du = o.backward(t, W)
        o.adam(lr, dw, du)
        o.next_iteration()
        opt.zero_grad()
        pt.grad = torch.tensor(du); pp.grad = torch.tensor(dw)
        opt.step()
        wt, wp = o.logits()
        np.testing.assert_allclose(wp, pp.detach().numpy(), rtol=1e-12, atol=1e-12)
        np.testing.assert_allclose(wt, pt.detach().numpy(), rtol=1e-12, atol=1e-12)
    mt, vt, mp, vp = o.adam_state()
    st = opt.state[pp]
    np.testing.assert_allclose(mp, st["exp_avg"].numpy(), rtol=1e-12, atol=1e-15)
    np.testing.assert_allclose(vp, st["exp_avg_sq"].numpy(), rtol=1e-12, atol=1e-20)


def test_step_equals_manual_loop_and_split_calls(tiny):
    """dgr_step contract: 10x10 iterations == 1x100 at equal t; iters=0 is forward only."""
    W = oracle.weights()
    a, b = oracle.Oracle(tiny), oracle.Oracle(tiny)
    la = a.step(20, 0.9, 0.3, W)
    for _ in range(4):
        lb = b.step(5, 0.9, 0.3, W)
    np.testing.assert_array_equal(a.logits()[1], b.logits()[1])
    np.testing.assert_array_equal(la, lb)
    assert a.iteration == 20
    c = oracle.Oracle(tiny)
    c.step(0, 1.0, 0.3, W)
    assert c.iteration == 0
    np.testing.assert_array_equal(c.logits()[1], tiny.w_path0.astype(np.float64))


def test_annealed_solve_decreases_cost_and_sharpens(tiny):
    """Quality sanity (not parity): 1000 annealed iterations lower the cost and make q near one-hot."""
    W = oracle.weights()
    o = oracle.Oracle(tiny)
    first = o.forward(1.0, W, noise=False)[0]
    for k in range(10):
        o.step(100, 0.9 ** k, 0.3, W)
    last = o.forward(0.9 ** 9, W, noise=False)[0]
    assert last < first
    q, p = o.probs()
    multi = [n for n in range(tiny.n_nets) if tiny.net_tree_off[n + 1] - tiny.net_tree_off[n] > 1]
    qmax = [q[tiny.net_tree_off[n]:tiny.net_tree_off[n + 1]].max() for n in multi]
    assert np.mean(np.array(qmax) > 0.99) > 0.8

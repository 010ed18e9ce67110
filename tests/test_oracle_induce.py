"""Pins for the oracle's discrete induction (§4.5; readings Q12, Q13, Q23)."""
import numpy as np

import oracle
from tests import _ref


def test_ranks_ties_and_nucleus_rules(tiny):
    o = oracle.Oracle(tiny)
    wt = np.zeros(tiny.n_trees); wp = np.zeros(tiny.n_paths)      # all ties
    o.set_logits(wt, wp)
    r = o.induce(top_p=0.0, t_final=1.0)
    for n in range(tiny.n_nets):
        assert r.tree_choice[n] == tiny.net_tree_off[n]                # argmax ties -> lowest index
    for s in range(tiny.n_subnets):
        if r.route[s] >= 0:
            assert r.route[s] == tiny.sub_path_off[s]                  # ties -> lowest index
            assert r.nucleus_off[s + 1] - r.nucleus_off[s] == 1          # top_p = 0 keeps one path
    # uniform p_hat over m paths: the nucleus for top_p is the smallest prefix with cumsum >= top_p
    r = o.induce(top_p=0.5, t_final=1.0)
    for s in range(tiny.n_subnets):
        if r.route[s] < 0:
            continue
        m = int(tiny.sub_path_off[s + 1] - tiny.sub_path_off[s])
        size = r.nucleus_off[s + 1] - r.nucleus_off[s]
        assert size == int(np.ceil(0.5 * m - 1e-9))
        np.testing.assert_array_equal(r.nucleus[r.nucleus_off[s]:r.nucleus_off[s + 1]],
                                      np.arange(tiny.sub_path_off[s], tiny.sub_path_off[s] + size))


def test_route_is_argmax_and_nucleus_is_sorted(tiny):
    o = oracle.Oracle(tiny)
    rng = np.random.default_rng(11)
    wt = rng.normal(size=tiny.n_trees); wp = rng.normal(size=tiny.n_paths) * 2
    o.set_logits(wt, wp)
    r = o.induce(top_p=0.9, t_final=0.7)
    for n in range(tiny.n_nets):
        a, b = tiny.net_tree_off[n], tiny.net_tree_off[n + 1]
        assert r.tree_choice[n] == a + int(np.argmax(wt[a:b]))
    for s in range(tiny.n_subnets):
        if r.route[s] < 0:
            continue
        a, b = tiny.sub_path_off[s], tiny.sub_path_off[s + 1]
        assert r.route[s] == a + int(np.argmax(wp[a:b]))
        nuc = r.nucleus[r.nucleus_off[s]:r.nucleus_off[s + 1]]
        ph = np.exp((wp[a:b] - wp[a:b].max()) / 0.7); ph /= ph.sum()
        assert np.all(np.diff(wp[nuc]) <= 0)
        c = np.cumsum(ph[nuc - a])
        assert c[-1] >= 0.9 - 1e-12 and (len(c) == 1 or c[-2] < 0.9)
        if ph.max() >= 0.9:
            assert len(nuc) == 1


def test_unchosen_trees_have_no_routes(tiny):
    o = oracle.Oracle(tiny)
    r = o.induce(top_p=0.9)
    for n in range(tiny.n_nets):
        for j in range(tiny.net_tree_off[n], tiny.net_tree_off[n + 1]):
            for s in range(tiny.tree_sub_off[j], tiny.tree_sub_off[j + 1]):
                assert (r.route[s] >= 0) == (j == r.tree_choice[n])


def test_induced_demand_and_metrics(tiny):
    o = oracle.Oracle(tiny)
    o.step(50, 1.0, 0.3, oracle.weights())
    beta = 0.25
    r = o.induce(top_p=0.9, beta=beta)
    routes = [int(i) for i in r.route if i >= 0]
    dh, dv = _ref.rasterise(tiny, routes, beta=0.0)
    assert np.array_equal(r.D_h, dh.astype(np.int32)) and np.array_equal(r.D_v, dv.astype(np.int32))
    V = np.zeros((tiny.Y, tiny.X))
    for i in routes:
        for (x, y) in _ref.path_tps(tiny, i):
            V[y, x] += 1
    oh = dh[:, :-1] + beta * (V[:, :-1] + V[:, 1:]) - tiny.cap_h[:, :-1]
    ov = dv[:-1, :] + beta * (V[:-1, :] + V[1:, :]) - tiny.cap_v[:-1, :]
    allo = np.concatenate([oh.reshape(-1), ov.reshape(-1)])
    pos = allo[allo > 0]
    assert abs(r.metrics[0] - pos.sum()) < 1e-9
    assert r.metrics[1] == len(pos)
    assert r.metrics[2] == (pos.max() if len(pos) else 0.0)
    assert r.metrics[3] == dh.sum() + dv.sum()
    assert r.metrics[4] == sum(len(_ref.path_tps(tiny, i)) for i in routes)


def test_no_overflow_term_prefers_fewest_turns(tiny):
    """a3 = 0: every candidate of a sub-net has the same WL, so the cost prefers the fewest
    turning points — straight or L, never Z (Eqs. (11)/(12))."""
    W = oracle.weights(a_of=0.0)
    o = oracle.Oracle(tiny)
    for k in range(3):
        o.step(100, 0.9 ** k, 0.3, W)
    r = o.induce(top_p=0.9)
    tp = np.diff(tiny.path_tp_off)
    bad = 0
    for s in range(tiny.n_subnets):
        if r.route[s] < 0:
            continue
        a, b = tiny.sub_path_off[s], tiny.sub_path_off[s + 1]
        bad += tp[r.route[s]] != tp[a:b].min()
    assert bad == 0

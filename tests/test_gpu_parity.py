"""Parity of the sm_100a path (through the C ABI) against the fp64 oracle, element by element.

Tolerance (BASELINE.json north_star; reading Q21): floats |gpu - oracle| <= 1e-4 * max(|oracle|, 1)
elementwise for demand and logits, relative 1e-4 for the scalar loss terms; integer outputs
(one-hot demand, induced routes where the top-1/top-2 margin exceeds 1e-3) bit-exact.
"""
import copy

import numpy as np
import pytest

import forestgen
import oracle
import paper_conf_dac_0159layhrr24_b200 as dgr
from tests import _ref

pytestmark = pytest.mark.gpu

TOL = 1e-4


def assert_close(a, b, tol=TOL, what=""):
    a = np.asarray(a, np.float64); b = np.asarray(b, np.float64)
    err = np.abs(a - b) / np.maximum(np.abs(b), 1.0)
    i = int(np.argmax(err)) if err.size else 0
    assert err.size == 0 or err.max() <= tol, f"{what}: max scaled err {err.max():.3e} at {i}: gpu {a.flat[i]} oracle {b.flat[i]}"


def assert_rel(a, b, tol=TOL, what=""):
    assert abs(a - b) <= tol * max(abs(b), 1e-12), f"{what}: gpu {a} oracle {b}"


def ow(w: dgr.Weights):
    return oracle.weights(a_wl=w.a_wl, a_via=w.a_via, a_of=w.a_of, beta=w.beta_via, n_layers=w.n_layers,
                          f_kind=w.f_kind, f_slope=w.f_slope)


@pytest.fixture(scope="module")
def forests():
    fs = {n: forestgen.generate(n) for n in ("tiny", "c1e4", "ispd18", "tiny_c", "c1e4_c", "tiny_m", "c1e4_m")}
    # row f4': candidates in a random order per sub-net (the general path, like the staircases)
    fs["c1e4_shuf"] = forestgen.shuffle_candidates(fs["c1e4"], seed=7)
    # nets in a random order: the plan restores a spatial order (Morton)
    fs["c1e4_nshuf"] = forestgen.shuffle_nets(fs["c1e4"], seed=5)
    return fs


def run_both(f, schedule, W=None, lr=0.3):
    """schedule: list of (iters, t).  Returns (solver, oracle, gpu losses, oracle losses)."""
    W = W or dgr.Weights()
    s = dgr.Solver(f)
    o = oracle.Oracle(f)
    gl, ol = [], []
    for iters, t in schedule:
        gl.append(s.step(iters, t, lr, W))
        ol.append(o.step(iters, t, lr, ow(W)))
    return s, o, gl, ol


def probes(f, schedule, W=None):
    """Conditioning probe: the oracle source built with real = float (the paper's presumed fp32,
    rounding everywhere), replaying the same schedule."""
    W = ow(W or dgr.Weights())
    o = oracle.Oracle(f, fp32=True)
    for iters, t in schedule:
        o.step(iters, t, 0.3, W)
    return o


def scaled_err(a, b):
    a = np.asarray(a, np.float64); b = np.asarray(b, np.float64)
    return np.abs(a - b) / np.maximum(np.abs(b), 1.0)


# The float parity contract (readings Q21, Q21b, Q21c).  An element passes
#   strict:   |gpu - fp64| <= TOL max(|fp64|, 1);
#   exempt:   (logits after ONE Adam step) the fp64 gradient is below the resolution of an fp32
#             evaluation of the paper's formulation (first_step_exempt): Adam's first step is
#             lr g / (|g| + eps), so such a coordinate may land anywhere in [w0 - lr, w0 + lr];
#   probe:    (multi-iteration runs) the fp32 probe -- the oracle's own source built with real = float
#             -- is itself beyond TOL there, and |gpu - fp64| <= K_PROBE |probe - fp64| and <= 2 lr;
#   chaotic:  (multi-iteration runs) beyond TOL where the probe is not: a trajectory that took a
#             different rounding path earlier.  Allowed only up to as many elements as the fp32 probe
#             deviates at in total (the GPU is no less accurate than fp32 evaluation of the same
#             formulas), each within CHAOS_DEMAND (demand) / 2 lr (logits).
# Anything else fails.  Every clause's count is recorded (tests/conftest.py prints them and writes
# $DGR_PARITY_COUNTS).
K_PROBE = float(__import__("os").environ.get("DGR_K_PROBE", "2.0"))   # env: data-gathering runs only
KAPPA = 2.0 ** -16          # fp32 resolution of a gradient relative to the terms it is formed from
CHAOS_DEMAND = 20 * TOL
LR = 0.3
ADAM_EPS = 1e-8             # torch.optim.Adam default (reading Q9)
PARITY_COUNTS = {}   # test -> field -> clause counts (printed in the session summary, tests/conftest.py)


def _record(what, nm, **kv):
    PARITY_COUNTS.setdefault(what, {})[nm] = kv


def first_step_exempt(f, W=None, t=1.0):
    """Coordinates whose fp64 first-step gradient is below the resolution of an fp32 evaluation of the
    paper's formulation (reading Q21b): dw_i = (p_i q_j / t)(c_i - sum_k p_k c_k) is formed from absolute
    costs c (PyTorch autograd of Eq. (9) through the softmaxes), so fp32 resolves it only to
    ~eps_p (p_i q_j / t)(|c_i| + sum_k p_k |c_k|), eps_p the relative error of the fp32 probabilities;
    likewise du_j = (q_j / t)(dq_j - sum_l q_l dq_l) with dq_j = sum_{i in j} p_i c_i.  eps_p: z = (w + g)/t
    in fp32 carries 2^-24 |z| of rounding (|z| <~ 20 at the first step), and exp's argument reduction
    as much again, so eps_p <~ 2^-24 * 2 * 20 = 2.4e-6 and the gradient's error <~ 2 eps_p (terms);
    KAPPA = 2^-16 = 1.5e-5 leaves a factor 3.  A coordinate is exempt when its gradient's sign is
    not resolved (|g| < KAPPA terms), or when Adam's first step lr g / (|g| + eps) (bias-corrected
    from zero moments) amplifies that resolution beyond TOL: its derivative in g is
    lr eps / (|g| + eps)^2, so lr eps KAPPA terms / (|g| + eps)^2 > TOL max(|w|, 1) (|g| near eps).
    Returns (tree mask, path mask)."""
    W = ow(W or dgr.Weights())
    o = oracle.Oracle(f)
    o.forward(t, W)
    dw, du, c = o.backward(t, W, costs=True)
    q, p = o.probs()
    path_sub = np.repeat(np.arange(f.n_subnets), np.diff(f.sub_path_off))
    sub_tree = np.repeat(np.arange(f.n_trees), np.diff(f.tree_sub_off))
    tree_net = np.repeat(np.arange(f.n_nets), np.diff(f.net_tree_off))
    path_tree = sub_tree[path_sub]
    grp = np.zeros(f.n_subnets)
    np.add.at(grp, path_sub, p * np.abs(c))
    r_path = KAPPA * p * q[path_tree] / t * (np.abs(c) + grp[path_sub])
    dq = np.zeros(f.n_trees)
    np.add.at(dq, path_tree, p * c)
    ngrp = np.zeros(f.n_nets)
    np.add.at(ngrp, tree_net, q * np.abs(dq))
    r_tree = KAPPA * q / t * (np.abs(dq) + ngrp[tree_net])
    wt0 = np.asarray(f.w_tree0, np.float64); wp0 = np.asarray(f.w_path0, np.float64)

    def ill(g, r, w0):
        step_sens = LR * ADAM_EPS * r / (np.abs(g) + ADAM_EPS) ** 2   # d(first step)/dg x resolution
        return (np.abs(g) < r) | (step_sens > TOL * np.maximum(np.abs(w0), 1.0))
    return ill(du, r_tree, wt0), ill(dw, r_path, wp0)


def compare_state(s, o, what, probe=None, max_ill=0.01, exempt=None, chaos=False, k_probe=K_PROBE):
    """Element-wise parity of demand and logits under the contract above.  `exempt` = (tree mask,
    path mask) of first_step_exempt (one-iteration runs); `probe` = the fp32 oracle replaying the same
    schedule; `chaos` allows the chaotic clause (multi-iteration runs)."""
    gdh, gdv = s.demand()
    odh, odv = o.demand()
    gwt, gwp = s.logits()
    owt, owp = o.logits()
    pr = None
    if probe is not None:
        pdh, pdv = probe.demand()
        pwt, pwp = probe.logits()
        pr = (pdh, pdv, pwp, pwt)
    ex_t, ex_p = exempt if exempt is not None else (None, None)
    fields = ((gdh, odh, "d_h", None), (gdv, odv, "d_v", None), (gwp, owp, "w_path", ex_p), (gwt, owt, "w_tree", ex_t))
    for fi, (g, r, nm, ex) in enumerate(fields):
        g = np.asarray(g, np.float64); r = np.asarray(r, np.float64)
        eg = scaled_err(g, r)
        dif = np.abs(g - r)
        strict = eg <= TOL
        e32 = scaled_err(pr[fi], r) if pr is not None else np.zeros_like(eg)
        n32 = int((e32 > TOL).sum())
        relaxed = ~strict & (e32 > TOL) & (eg <= k_probe * e32) & (dif <= 2 * LR + 1e-6)
        rest = ~strict & ~relaxed
        exempted = np.zeros_like(rest)
        if ex is not None:
            exempted = rest & ex.reshape(rest.shape) & (dif <= 2 * LR + 1e-6)
            rest &= ~exempted
        chaotic = np.zeros_like(rest)
        if chaos:
            bound = (eg <= CHAOS_DEMAND) if nm.startswith("d_") else (dif <= 2 * LR + 1e-6)
            chaotic = rest & bound
            rest &= ~chaotic
        bad = rest
        ratio = (eg / np.maximum(e32, 1e-300))[relaxed]
        _record(what, nm, n=int(eg.size), strict=int(strict.sum()), probe=int(relaxed.sum()),
                exempt=int(exempted.sum()), chaotic=int(chaotic.sum()), bad=int(bad.sum()),
                fp32_beyond_tol=n32, fp32_max_err=float(e32.max(initial=0.0)),
                max_err=float(eg.max(initial=0.0)), max_probe_ratio=float(ratio.max(initial=0.0)),
                max_err_chaotic=float(eg[chaotic].max(initial=0.0)))
        i = int(np.argmax(np.where(bad, eg, -1))) if bad.any() else 0
        assert not bad.any(), (f"{what} {nm}: {bad.sum()} elements outside every clause; "
                               f"worst {i}: gpu {g.flat[i]} fp64 {r.flat[i]}"
                               + (f" fp32 {pr[fi].flat[i]}" if pr is not None else ""))
        assert relaxed.mean() <= max_ill, f"{what} {nm}: {relaxed.sum()} of {relaxed.size} need the fp32 clause"
        assert exempted.mean() <= max_ill, f"{what} {nm}: {exempted.sum()} of {exempted.size} exempt"
        assert chaotic.sum() <= max(n32, 1), f"{what} {nm}: {chaotic.sum()} chaotic elements > the fp32 probe's {n32}"


@pytest.mark.parametrize("beta", [0.0, 0.25])
@pytest.mark.parametrize("name", ["c1e4", "c1e4_c", "c1e4_m", "c1e4_shuf"])
def test_one_hot_demand_is_bit_exact(forests, beta, name):
    f = copy.deepcopy(forests[name])
    rng = np.random.default_rng(0)
    wt = np.zeros(f.n_trees, np.float32); wp = np.zeros(f.n_paths, np.float32)
    pick = [int(rng.integers(f.sub_path_off[sn], f.sub_path_off[sn + 1])) for sn in range(f.n_subnets)]
    wp[pick] = 1000.0                       # winner gap 1000: exact 0/1 probabilities in fp32 and fp64
    sel = []
    for n in range(f.n_nets):
        j = int(rng.integers(f.net_tree_off[n], f.net_tree_off[n + 1])); wt[j] = 1000.0
        sel += [pick[sn] for sn in range(f.tree_sub_off[j], f.tree_sub_off[j + 1])]
    f.w_tree0, f.w_path0 = wt, wp
    W = dgr.Weights(beta_via=beta)
    s = dgr.Solver(f)
    s.step(0, 1.0, 0.3, W)
    gdh, gdv = s.demand()
    rdh, rdv = _ref.rasterise(f, sel, beta=beta)
    assert np.array_equal(gdh.astype(np.float64), rdh) and np.array_equal(gdv.astype(np.float64), rdv)
    o = oracle.Oracle(f)
    o.forward(1.0, ow(W))
    odh, odv = o.demand()
    assert np.array_equal(gdh.astype(np.float64), odh) and np.array_equal(gdv.astype(np.float64), odv)


@pytest.mark.parametrize("name", ["tiny", "c1e4", "ispd18", "tiny_c", "c1e4_c", "tiny_m", "c1e4_m"])
@pytest.mark.parametrize("f_kind", [0, 1, 2, 3, 4])
def test_forward_parity(forests, name, f_kind):
    """sigmoid, ReLU and the LeakyReLU / exp / CELU of Fig. 6."""
    W = dgr.Weights(f_kind=f_kind, f_slope=0.5 if f_kind == 3 else None)
    f = forests[name]
    s, o, gl, ol = run_both(f, [(0, 0.7)], W)
    gdh, gdv = s.demand()
    odh, odv = o.demand()
    assert_close(gdh, odh, what="d_h"); assert_close(gdv, odv, what="d_v")
    for i, nm in enumerate(("total", "wl", "via", "overflow")):
        assert_rel(gl[0][i], ol[0][i], what=nm)
    assert s.iteration == 0


@pytest.mark.parametrize("name", ["tiny", "c1e4", "ispd18", "tiny_c", "c1e4_c", "tiny_m", "c1e4_m", "c1e4_shuf",
                                  "c1e4_nshuf"])
def test_one_iteration_parity(forests, name):
    """After one Adam step the update of a coordinate whose gradient is ~eps depends on that
    gradient's last bits (Q21b), so the fp32 probe applies from the first step on."""
    s, o, gl, ol = run_both(forests[name], [(1, 1.0)])
    compare_state(s, o, name, exempt=first_step_exempt(forests[name]), max_ill=1e-3)
    assert s.iteration == 1


@pytest.mark.parametrize("name,schedule", [
    ("tiny", [(100, 1.0), (100, 0.9)]),                  # BASELINE.json: tiny, 200 iterations
    ("c1e4", [(100, 1.0)]),
    ("tiny_c", [(100, 1.0), (100, 0.9)]),                # row f4: C-shape detours
    ("c1e4_c", [(100, 1.0)]),
    ("tiny_m", [(100, 1.0), (100, 0.9)]),                # row f4': staircases, groups > 32
    ("c1e4_m", [(100, 1.0)]),
    ("c1e4_shuf", [(100, 1.0)]),                         # any candidate order
    ("c1e4_nshuf", [(100, 1.0)]),                        # any net order
])
def test_trajectory_parity(forests, name, schedule):
    f = forests[name]
    s, o, gl, ol = run_both(f, schedule)
    compare_state(s, o, name, probe=probes(f, schedule), chaos=True)
    for i, nm in enumerate(("total", "wl", "via", "overflow")):
        assert_rel(gl[-1][i], ol[-1][i], what=nm)


@pytest.mark.parametrize("name", ["ispd18", "ispd19"])
def test_trajectory_parity_100_iterations_full_size(name):
    """BASELINE.json north_star: "the logits after 100 iterations in fp32 within 1e-4", at configs[2]
    (ispd18, ~1e5 nets) and configs[3] (ispd19, ~1e6 nets, the bench workload), in the bench's launch
    configuration: 100 iterations at t = 1 with Adam at lr 0.3, then every demand element
    and every logit against the fp64 oracle, and the loss of the 100th forward (reading Q11)."""
    f = forestgen.generate(name)
    sched = [(100, 1.0)]
    s, o, gl, ol = run_both(f, sched)
    compare_state(s, o, name + " 100 it", probe=probes(f, sched), max_ill=1e-3, chaos=True)
    for i, nm in enumerate(("total", "wl", "via", "overflow")):
        assert_rel(gl[-1][i], ol[-1][i], what=nm)
    assert s.iteration == 100


@pytest.mark.parametrize("f_kind", [2, 3, 4])
def test_alternative_activations_one_iteration(forests, f_kind):
    """Piecewise-linear f (LeakyReLU, CELU's linear branch) make exact cost ties common: the two L
    candidates of a sub-net whose edges all overflow get identical c, so the exact gradient is 0 and
    Adam's first step is 0.  The kernel forms c from prefix-sum differences, whose ~1e-12 rounding
    Adam turns into lr * g / eps <= ~1e-3.  Such exact-tie coordinates (fp64 |dw| < 1e-10) are held
    to 1e-3 and must be rare; every other coordinate follows compare_state."""
    W = dgr.Weights(f_kind=f_kind, f_slope=0.5 if f_kind == 3 else None)
    f = forests["c1e4"]
    s, o, gl, ol = run_both(f, [(1, 1.0)], W)
    o0 = oracle.Oracle(f)
    o0.forward(1.0, ow(W))
    dw0, du0 = o0.backward(1.0, ow(W))
    tie_p, tie_t = np.abs(dw0) < 1e-10, np.abs(du0) < 1e-10
    gwt, gwp = s.logits()
    owt, owp = o.logits()
    _record(f"alt_f{f_kind} ties", "w_path", n=int(tie_p.size), tie=int(tie_p.sum()),
            max_abs_tie=float(np.abs(gwp - owp)[tie_p].max(initial=0)))
    _record(f"alt_f{f_kind} ties", "w_tree", n=int(tie_t.size), tie=int(tie_t.sum()),
            max_abs_tie=float(np.abs(gwt - owt)[tie_t].max(initial=0)))
    assert np.abs(gwp - owp)[tie_p].max(initial=0) <= 1e-3 and np.abs(gwt - owt)[tie_t].max(initial=0) <= 1e-3
    ex_t, ex_p = first_step_exempt(f, W)
    for g, r, ex, tie, nm in ((gwp, owp, ex_p, tie_p, "w_path"), (gwt, owt, ex_t, tie_t, "w_tree")):
        eg = scaled_err(g, r)
        exempted = ~tie & (eg > TOL) & ex & (np.abs(g - r) <= 2 * LR + 1e-6)
        bad = ~tie & (eg > TOL) & ~exempted
        PARITY_COUNTS[f"alt_f{f_kind} ties"][nm].update(exempt_res=int(exempted.sum()), bad=int(bad.sum()),
                                                         strict=int((~tie & (eg <= TOL)).sum()))
        assert not bad.any(), f"f{f_kind} {nm}: {bad.sum()} bad"
        assert exempted.mean() <= 1e-3, f"f{f_kind} {nm}: {exempted.sum()} exempt"
    assert tie_p.mean() < 0.2
    gdh, gdv = s.demand(); odh, odv = o.demand()
    assert_close(gdh, odh, what="d_h"); assert_close(gdv, odv, what="d_v")


def test_relu_trajectory_parity(forests):
    """ReLU's gradient is a step in d: trajectories are piecewise and chaotic, so parity
    is checked over 5 iterations (the Table 1 objective's quality is checked by the oracle tests)."""
    W = dgr.Weights(f_kind=1)
    for name in ("tiny", "c1e4"):
        sched = [(5, 1.0)]
        s, o, gl, ol = run_both(forests[name], sched, W)
        compare_state(s, o, "relu " + name, probe=probes(forests[name], sched, W), chaos=True)


def test_split_calls_and_determinism(forests):
    f = forests["c1e4"]
    a = dgr.Solver(f); b = dgr.Solver(f)
    a.step(10, 0.9, 0.3)
    for _ in range(5):
        b.step(2, 0.9, 0.3)
    assert np.array_equal(a.logits()[1], b.logits()[1]) and np.array_equal(a.logits()[0], b.logits()[0])
    assert all(np.array_equal(x, y) for x, y in zip(a.demand(), b.demand()))


@pytest.mark.parametrize("pinned", [False, True])
def test_step_async_equals_step(forests, pinned):
    """dgr_step_async (no host sync) is dgr_step: same losses, same state.  A pageable loss buffer gets
    a stream-ordered copy; a pinned one is written by the loss kernel itself (no copy in the chain)."""
    import torch
    f = forests["c1e4"]
    a = dgr.Solver(f); b = dgr.Solver(f)
    la = np.array([a.step(1, 0.9, 0.3) for _ in range(5)])
    lb = torch.zeros((5, 4), dtype=torch.float64).pin_memory().numpy() if pinned else np.zeros((5, 4))
    for i in range(5):
        b.step_async(1, 0.9, 0.3, None, lb[i])
    b.sync()
    assert np.array_equal(la, lb)
    assert np.array_equal(a.logits()[1], b.logits()[1]) and np.array_equal(a.logits()[0], b.logits()[0])


@pytest.mark.parametrize("name", ["tiny", "c1e4", "c1e4_c", "tiny_m", "c1e4_m", "c1e4_shuf", "c1e4_nshuf"])
def test_induce_parity(forests, name):
    f = forests[name]
    s, o, _, _ = run_both(f, [(60, 1.0), (40, 0.9)])
    g = s.induce(0.9)
    r = o.induce(0.9, beta=0.25, t_final=0.9)
    sure_tree = r.margin_tree > 1e-3
    assert np.array_equal(g.tree_choice[sure_tree], r.tree_choice[sure_tree])
    # routes: bit-exact where the sub-net's tree choice and top-1 / top-2 margin are clear
    path_tree = np.repeat(np.arange(f.n_trees), np.diff(f.tree_sub_off))
    sub_net = np.repeat(np.arange(f.n_nets), np.diff(f.net_tree_off))[path_tree]
    sure = sure_tree[sub_net] & (r.margin_route > 1e-3)
    assert np.array_equal(g.route[sure], r.route[sure])
    assert sure.mean() > 0.5
    # nuclei where the cumulative sums are clear of top_p
    for sn in np.nonzero(sure & (r.margin_nucleus > 1e-3))[0][:2000]:
        assert np.array_equal(g.nucleus[g.nucleus_off[sn]:g.nucleus_off[sn + 1]],
                              r.nucleus[r.nucleus_off[sn]:r.nucleus_off[sn + 1]])
    # the integer grids and metrics of the GPU's own routes, recomputed independently
    routes = [int(i) for i in g.route if i >= 0]
    dh, dv = _ref.rasterise(f, routes, beta=0.0)
    assert np.array_equal(g.D_h, dh.astype(np.int32)) and np.array_equal(g.D_v, dv.astype(np.int32))
    assert g.metrics[3] == dh.sum() + dv.sum()
    if sure.all():
        assert np.array_equal(g.D_h, r.D_h) and np.array_equal(g.D_v, r.D_v)
        np.testing.assert_allclose(g.metrics, r.metrics, rtol=1e-9)


def test_induce_metrics_exact_on_oracle_routes(forests):
    """Metrics of identical routes: start from w0 (both sides read the same fp32 logits)."""
    f = forests["c1e4"]
    s = dgr.Solver(f); o = oracle.Oracle(f)
    s.step(0, 1.0, 0.3)
    g = s.induce(0.9)
    r = o.induce(0.9, beta=0.25, t_final=1.0)
    assert np.array_equal(g.tree_choice, r.tree_choice)
    assert np.array_equal(g.route, r.route)
    assert np.array_equal(g.D_h, r.D_h) and np.array_equal(g.D_v, r.D_v)
    np.testing.assert_allclose(g.metrics, r.metrics, rtol=1e-12)


def test_empty_and_degenerate_forests():
    # no routed nets at all: demand 0, loss = a3 * sum_e f(cap_e)
    f = forestgen.generate("tiny", n_nets=0)
    s = dgr.Solver(f)
    gl = s.step(3, 1.0, 0.3)
    o = oracle.Oracle(f)
    ol = o.step(3, 1.0, 0.3, ow(dgr.Weights()))
    assert_rel(gl[0], ol[0], what="empty loss")
    assert not s.demand()[0].any()
    # a 2x2 grid
    f = forestgen.generate(dict(X=2, Y=2, n_nets=6, pins_mode=0, pins_min=2, pins_max=4, box_mode=0, box_min=2,
                                box_max=2, track=1.0, n_tree_cand=2, z_cap=0, seed=3))
    s, o, gl, ol = run_both(f, [(20, 1.0)])
    compare_state(s, o, "2x2", probe=probes(f, [(20, 1.0)]), chaos=True)


@pytest.mark.parametrize("name", ["ispd19", "sweep4e6"])
def test_full_size_sampled_parity(name):
    """BASELINE.json configs[3] (ispd19, ~1e6 nets, the bench workload) and the largest sweep point
    of configs[4] (sweep4e6: 3.8e6 nets on 2000x2000) in the bench's launch configuration: full
    demand / loss of the first forward and every logit after one iteration."""
    f = forestgen.generate(name)
    s = dgr.Solver(f)
    o = oracle.Oracle(f)
    gl = s.step(0, 1.0, 0.3)
    ol = o.step(0, 1.0, 0.3, ow(dgr.Weights()))
    for i in range(4):
        assert_rel(gl[i], ol[i], what="loss")
    gdh, gdv = s.demand(); odh, odv = o.demand()
    assert_close(gdh, odh, what="d_h"); assert_close(gdv, odv, what="d_v")
    s.step(1, 1.0, 0.3)
    o.step(1, 1.0, 0.3, ow(dgr.Weights()))
    # reading Q21b at full size: every logit within TOL unless its fp64 gradient is below the fp32
    # resolution of its own terms (first_step_exempt); such coordinates must be rare (<= 1e-5)
    compare_state(s, o, name, max_ill=1e-5, exempt=first_step_exempt(f))


def test_table1_workload_relu_parity_and_optimum():
    """Row f2: overflow-only ReLU, L-only, argmax.  Parity over 3 iterations on a Table-1
    row and the brute-force optimum reached by the GPU on a small instance (best of 5 seeds)."""
    from tests.test_table1 import W_T1, _small, brute_force_overflow
    W = dgr.Weights(a_wl=0.0, a_via=0.0, a_of=1.0, beta_via=0.0, f_kind=1)
    f = forestgen.generate("table1_r5")
    s, o, gl, ol = run_both(f, [(3, 1.0)], W)
    compare_state(s, o, "table1_r5", probe=probes(f, [(3, 1.0)], W), max_ill=0.02, chaos=True)
    g = _small(2)
    opt = brute_force_overflow(g)
    best = None
    rng = np.random.default_rng(0)
    for run in range(5):
        h = copy.deepcopy(g)
        h.seed = 2000 + run
        h.w_path0 = rng.random(g.n_paths).astype(np.float32)
        sv = dgr.Solver(h)
        for k in range(5):
            sv.step(100, 0.9 ** k, 0.3, W, want_loss=False)
        m = sv.induce(0.0).metrics[0]
        best = m if best is None else min(best, m)
    assert best == opt
    assert W_T1["f_kind"] == 1


def test_general_path_is_used(forests):
    """Row f4': the staircase / large-group / shuffled configs do run candidates on the general path
    (dgr_get_info info[11] = general candidates) and the plain configs do not."""
    for name, want in (("c1e4", False), ("c1e4_m", True), ("c1e4_shuf", True), ("tiny_m", True)):
        s = dgr.Solver(forests[name])
        assert (s.info()["n_general_paths"] > 0) == want, name


def test_ispd18_staircases_one_iteration():
    """Row f4' at ISPD'18 scale (configs[2] shape with staircases and groups up to 58)."""
    f = forestgen.generate("ispd18_m")
    s, o, gl, ol = run_both(f, [(1, 1.0)])
    for i in range(4):
        assert_rel(gl[0][i], ol[0][i], what="loss")
    compare_state(s, o, "ispd18_m", exempt=first_step_exempt(f), max_ill=1e-3)


def test_dgr_star_search_reaches_the_optimum():
    """Row f2, DGR* (P:880-885): on an enumerable Table-1-style instance the hyper-parameter search
    (sampled lr in [1e-4, 1], gamma in {0.8, ..., 0.95}) reaches the brute-force optimum."""
    import tools.dgr_star as ds
    from tests.test_table1 import _small, brute_force_overflow
    g = _small(3)
    opt = brute_force_overflow(g)
    default, sampled, best = ds.search(g, runs=12)
    assert min(min(default), best[0]) == opt
    assert all(o >= opt for o, _, _ in sampled)

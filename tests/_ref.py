"""Test-side helpers that restate definitions independently (numpy / torch library routines).

These are NOT the oracle: they implement the *plain definitions* the oracle is pinned to
(Eq. (2) integer rasterisation, brute-force expectation over discrete selections, a torch
autograd statement of Eqs. (9)-(12)) so that a mistake in the oracle's loops shows up as a
mismatch.
"""
import itertools

import numpy as np
import torch

import oracle


def path_noise(f, k):
    """Gumbel noise g_i of every path candidate at iteration k (stream 0), reading Q7:
    a sub-net whose only candidate is a straight path (one segment) draws none (g = 0; its softmax
    is 1 whatever g is); every other candidate takes the next noise index in forest order."""
    g = np.zeros(f.n_paths)
    n = 0
    for s in range(f.n_subnets):
        a, b = int(f.sub_path_off[s]), int(f.sub_path_off[s + 1])
        if b - a == 1 and f.path_seg_off[a + 1] - f.path_seg_off[a] == 1:
            continue
        for i in range(a, b):
            g[i] = oracle.gumbel(f.seed, n, k, 0)
            n += 1
    return g


def path_edges(f, i):
    """Edges of path i as (dir, y, x) triples; dir 0 = H edge (x,y)-(x+1,y), 1 = V edge (x,y)-(x,y+1)."""
    out = []
    for g in range(f.path_seg_off[i], f.path_seg_off[i + 1]):
        d, line, lo, hi = (int(v) for v in f.seg[g])
        for e in range(lo, hi):
            out.append((0, line, e) if d == 0 else (1, e, line))
    return out


def path_tps(f, i):
    return [tuple(int(v) for v in f.tp_xy[u]) for u in range(f.path_tp_off[i], f.path_tp_off[i + 1])]


def incident_edges(X, Y, x, y):
    """Existing G-cell edges incident to G-cell (x,y)."""
    e = []
    if x >= 1: e.append((0, y, x - 1))
    if x <= X - 2: e.append((0, y, x))
    if y >= 1: e.append((1, y - 1, x))
    if y <= Y - 2: e.append((1, y, x))
    return e


def rasterise(f, paths, beta=0.0, weights=None):
    """Eq. (2): d_e = sum over selected paths through e + beta * (turning points at e's end-cells)."""
    dh = np.zeros((f.Y, f.X)); dv = np.zeros((f.Y, f.X))
    for n, i in enumerate(paths):
        wgt = 1.0 if weights is None else weights[n]
        for d, y, x in path_edges(f, i):
            (dh if d == 0 else dv)[y, x] += wgt
        for (x, y) in path_tps(f, i):
            for d, yy, xx in incident_edges(f.X, f.Y, x, y):
                (dh if d == 0 else dv)[yy, xx] += beta * wgt
    return dh, dv


def enumerate_selections(f):
    """All discrete selections (tree per net, path per sub-net of that tree) with their path lists.

    Yields (tree_choice tuple, list of selected paths, tuple of per-net sub-net path choices)."""
    per_net = []
    for n in range(f.n_nets):
        opts = []
        for j in range(f.net_tree_off[n], f.net_tree_off[n + 1]):
            subs = range(f.tree_sub_off[j], f.tree_sub_off[j + 1])
            choices = [range(f.sub_path_off[s], f.sub_path_off[s + 1]) for s in subs]
            for sel in itertools.product(*choices):
                opts.append((j, sel))
        per_net.append(opts)
    for combo in itertools.product(*per_net):
        trees = tuple(c[0] for c in combo)
        paths = [i for c in combo for i in c[1]]
        yield trees, paths


def torch_cost(f, w_tree, w_path, g_tree, g_path, t, W):
    """Eqs. (9)-(12) + P:580-583 in torch (fp64), with segments rasterised through index tensors."""
    X, Y = f.X, f.Y
    path_tree = np.repeat(np.repeat(np.arange(f.n_trees), np.diff(f.tree_sub_off)), np.diff(f.sub_path_off))
    path_sub = np.repeat(np.arange(f.n_subnets), np.diff(f.sub_path_off))
    tree_net = np.repeat(np.arange(f.n_nets), np.diff(f.net_tree_off))
    zp = (w_path + g_path) / t
    zt = (w_tree + g_tree) / t
    ps = torch.zeros_like(zp)
    for s in range(f.n_subnets):
        a, b = int(f.sub_path_off[s]), int(f.sub_path_off[s + 1])
        ps = ps + torch.nn.functional.pad(torch.softmax(zp[a:b], 0), (a, f.n_paths - b))
    qs = torch.zeros_like(zt)
    for n in range(f.n_nets):
        a, b = int(f.net_tree_off[n]), int(f.net_tree_off[n + 1])
        qs = qs + torch.nn.functional.pad(torch.softmax(zt[a:b], 0), (a, f.n_trees - b))
    pi = qs[torch.as_tensor(path_tree)] * ps
    rows, cols, vals = [], [], []
    for i in range(f.n_paths):
        for d, y, x in path_edges(f, i):
            rows.append(d * X * Y + y * X + x); cols.append(i); vals.append(1.0)
        for (x, y) in path_tps(f, i):
            for d, yy, xx in incident_edges(X, Y, x, y):
                rows.append(d * X * Y + yy * X + xx); cols.append(i); vals.append(W.beta)
    A = torch.zeros(2 * X * Y, f.n_paths, dtype=torch.float64)
    A.index_put_((torch.tensor(rows), torch.tensor(cols)), torch.tensor(vals, dtype=torch.float64), accumulate=True)
    d = A @ pi
    cap = torch.tensor(np.concatenate([f.cap_h.reshape(-1), f.cap_v.reshape(-1)]), dtype=torch.float64)
    valid = np.zeros((2, Y, X), bool)
    valid[0, :, : X - 1] = True
    valid[1, : Y - 1, :] = True
    valid = torch.as_tensor(valid.reshape(-1))
    x = d - cap                         # overflow = -(resource)
    F = torch.nn.functional
    if W.f_kind == 0:
        fo = torch.sigmoid(W.f_slope * x)
    elif W.f_kind == 1:
        fo = torch.relu(x)
    elif W.f_kind == 2:
        fo = F.leaky_relu(x, negative_slope=W.f_slope)
    elif W.f_kind == 3:
        fo = torch.exp(W.f_slope * x)
    else:
        fo = F.celu(x, alpha=W.f_slope)
    of = fo[valid].sum()
    wl = torch.tensor([sum(int(s[3] - s[2]) for s in f.seg[f.path_seg_off[i]:f.path_seg_off[i + 1]])
                       for i in range(f.n_paths)], dtype=torch.float64)
    tp = torch.tensor(np.diff(f.path_tp_off), dtype=torch.float64)
    ewl = (pi * wl).sum()
    etp = (pi * tp).sum()
    cost = W.a_wl * ewl + W.a_via * np.sqrt(W.n_layers) * etp + W.a_of * of
    return cost, d, ewl, etp, of, path_sub, tree_net

"""World-size-2 host-side tests of the net-sharded path, on CPU with the gloo backend.

The GPU path shards nets with dgr_partition and exchanges one buffer per iteration — the
demand (difference arrays + turning-point counts) and E[WL], E[TP] — with an allreduce
(include/dgr.h; NCCL on the GPU).  Here the same decomposition is run with the oracle on
each rank (odgr_set_shard) and a gloo allreduce of the partial demand, and must reproduce
the single-rank oracle: nets couple only through d (Eq. (10)).
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, name, iters, out_q):
    import sys
    sys.path.insert(0, ROOT)
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import forestgen
    import oracle
    import paper_conf_dac_0159layhrr24_b200 as dgr
    f = forestgen.generate(name)
    part = dgr.partition(f, world)                       # libdgr's host-only sharding
    plan = dgr.plan_info(f, rank=rank, world=world)
    o = oracle.Oracle(f)
    o.set_shard(int(part[rank]), int(part[rank + 1]))
    W = oracle.weights()
    losses = []
    for it in range(iters):
        t = 0.9 ** (it // 3)
        dh, dv, ewl, etp = o.forward_partial(t, W)
        buf = torch.tensor(np.concatenate([dh.ravel(), dv.ravel(), [ewl, etp]]), dtype=torch.float64)
        dist.all_reduce(buf)                             # the one exchange per iteration
        b = buf.numpy()
        G = f.X * f.Y
        loss = o.forward_finish(b[:G].reshape(f.Y, f.X), b[G:2 * G].reshape(f.Y, f.X), b[-2], b[-1], W)
        losses.append(loss[0])
        dw, du = o.backward(t, W)
        o.adam(0.3, dw, du)
        o.next_iteration()
    wt, wp = o.logits()
    p0, p1 = f.sub_path_off[f.tree_sub_off[f.net_tree_off[part[rank]]]], f.sub_path_off[f.tree_sub_off[f.net_tree_off[part[rank + 1]]]]
    t0, t1 = f.net_tree_off[part[rank]], f.net_tree_off[part[rank + 1]]
    out_q.put((rank, list(part), plan["n_paths"], (int(p0), int(p1)), (int(t0), int(t1)), wp[p0:p1].copy(),
               wt[t0:t1].copy(), losses))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("name", ["tiny", "c1e4"])
def test_sharded_oracle_matches_single_rank(name):
    import forestgen
    import oracle
    world, iters = 2, 6
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, name, iters, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    res.sort()
    f = forestgen.generate(name)
    o = oracle.Oracle(f)
    W = oracle.weights()
    ref_losses = []
    for it in range(iters):
        ref_losses.append(o.step(1, 0.9 ** (it // 3), 0.3, W)[0])
    wt, wp = o.logits()
    assert res[0][1] == res[1][1]
    assert sum(r[2] for r in res) == f.n_paths          # the plans cover every candidate once
    for r in res:
        (p0, p1), (t0, t1) = r[3], r[4]
        np.testing.assert_allclose(r[5], wp[p0:p1], rtol=1e-9, atol=1e-9)
        np.testing.assert_allclose(r[6], wt[t0:t1], rtol=1e-9, atol=1e-9)
        np.testing.assert_allclose(r[7], ref_losses, rtol=1e-12)

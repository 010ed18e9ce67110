"""The sharded (world > 1) device path on one GPU: R ranks in one process, one thread per rank, the
demand exchange done by a caller-supplied allreduce (dgr_dist.allreduce) instead of NCCL.

SURVEY §8(e) / DESIGN.md §7: nets are sharded over the ranks (dgr_partition), Gumbel noise is keyed
on global indices and the exchanged demand is exact fixed point, so every rank count must reproduce
the single-rank run BIT-EXACTLY: demand grids, loss, every logit (each from the rank that owns it),
induced tree choices / routes / integer grids / metrics.  This exercises everything of the NCCL path
except NCCL itself (which needs one process per GPU).
"""
import threading

import numpy as np
import pytest

import forestgen
import paper_conf_dac_0159layhrr24_b200 as dgr

pytestmark = pytest.mark.gpu


class _DevArray:
    """A device buffer of the library as a torch tensor (CUDA array interface, no copy)."""

    def __init__(self, ptr: int, n: int, dtype: int):
        self.__cuda_array_interface__ = {"shape": (int(n),), "typestr": ("<i8", "<i4", "<f8", "<f4")[dtype],
                                         "data": (int(ptr), False), "version": 3}


class ThreadAllreduce:
    """In-place sum over R threads' device buffers: every rank synchronises the device, rank 0 sums
    the R buffers in rank order and writes the sum back into all of them."""

    def __init__(self, world: int):
        import torch
        self.torch = torch
        self.world = world
        self.bufs = [None] * world
        self.barrier = threading.Barrier(world)
        self.calls = 0

    def for_rank(self, rank: int):
        def fn(buf, n, dtype, stream):
            torch = self.torch
            try:
                torch.cuda.synchronize()
                self.bufs[rank] = torch.as_tensor(_DevArray(buf, n, dtype), device="cuda")
                self.barrier.wait()
                if rank == 0:
                    tot = self.bufs[0].clone()
                    for t in self.bufs[1:]:
                        tot += t
                    for t in self.bufs:
                        t.copy_(tot)
                    torch.cuda.synchronize()
                    self.calls += 1
                self.barrier.wait()
                return 0
            except Exception:   # a failing exchange must fail the dgr_* call, not pass silently
                self.barrier.abort()
                return 1
        return fn


def _run(solvers, body):
    out, errs = [None] * len(solvers), []

    def work(r):
        try:
            out[r] = body(solvers[r])
        except Exception as e:   # pragma: no cover - surfaced below
            errs.append(e)

    th = [threading.Thread(target=work, args=(r,)) for r in range(len(solvers))]
    for t in th:
        t.start()
    for t in th:
        t.join()
    if errs:
        raise errs[0]
    return out


def _schedule(s):
    losses = [s.step(6, 1.0, 0.3), s.step(4, 0.9, 0.3)]
    return losses, s.demand(), s.logits(), s.induce(0.9)


@pytest.mark.parametrize("name,world", [("c1e4", 2), ("c1e4", 3), ("ispd18", 4), ("ispd19", 8), ("c1e4_m", 3), ("c1e4_nshuf", 2)])
def test_sharded_ranks_reproduce_one_rank_bit_exactly(name, world):
    f = forestgen.shuffle_nets(forestgen.generate("c1e4"), seed=5) if name == "c1e4_nshuf" else forestgen.generate(name)
    ref = dgr.Solver(f)
    ref_losses, (rdh, rdv), (rwt, rwp), rind = _schedule(ref)
    ref.close()

    ex = ThreadAllreduce(world)
    solvers = [dgr.Solver(f, rank=r, world=world, allreduce=ex.for_rank(r)) for r in range(world)]
    res = _run(solvers, _schedule)
    assert ex.calls >= 10 + 2, "the exchange ran once per iteration and twice in induction"

    part = dgr.partition(f, world)
    tree_off, sub_off, path_off = (np.asarray(f.net_tree_off), np.asarray(f.tree_sub_off),
                                   np.asarray(f.sub_path_off))
    for r, (losses, (dh, dv), (wt, wp), ind) in enumerate(res):
        # replicated: the global demand, the loss and the induced grids / metrics of every rank
        for a, b in zip(losses, ref_losses):
            assert np.array_equal(a, b), (r, a, b)
        assert np.array_equal(dh, rdh) and np.array_equal(dv, rdv)
        assert np.array_equal(ind.D_h, rind.D_h) and np.array_equal(ind.D_v, rind.D_v)
        assert np.array_equal(ind.metrics, rind.metrics)
        # rank-local: its nets' tree logits, path logits, tree choices and routes
        n0, n1 = part[r], part[r + 1]
        t0, t1 = tree_off[n0], tree_off[n1]
        s0, s1 = sub_off[t0], sub_off[t1]
        p0, p1 = path_off[s0], path_off[s1]
        assert np.array_equal(wt[t0:t1], rwt[t0:t1])
        assert np.array_equal(wp[p0:p1], rwp[p0:p1])
        assert np.array_equal(ind.tree_choice[n0:n1], rind.tree_choice[n0:n1])
        assert np.array_equal(ind.route[s0:s1], rind.route[s0:s1])
    for s in solvers:
        s.close()


def test_failing_exchange_is_reported():
    f = forestgen.generate("tiny")
    solvers = [dgr.Solver(f, rank=r, world=2, allreduce=lambda *a: 7) for r in range(2)]
    with pytest.raises(dgr.DgrError, match="allreduce callback returned 7"):
        solvers[0].step(1, 1.0, 0.3)
    for s in solvers:
        s.close()


def test_failed_step_leaves_no_stale_events():
    """A dgr_step that fails after its forward (here: the exchange) must not leave that forward's
    demand events behind for the next call to add onto (dgr.h: an error leaves no partial state).
    Rank 0 of 2 with an exchange that adds nothing (the other rank's share is zero): after one
    failed call, the next call equals the same call on a fresh handle."""
    f = forestgen.generate("tiny")
    calls = {"n": 0}

    def flaky(*a):
        calls["n"] += 1
        return 7 if calls["n"] == 1 else 0

    a = dgr.Solver(f, rank=0, world=2, allreduce=flaky)
    b = dgr.Solver(f, rank=0, world=2, allreduce=lambda *a: 0)
    with pytest.raises(dgr.DgrError, match="allreduce callback returned 7"):
        a.step(1, 1.0, 0.3)
    assert np.array_equal(a.step(2, 1.0, 0.3), b.step(2, 1.0, 0.3))
    assert all(np.array_equal(x, y) for x, y in zip(a.demand(), b.demand()))
    assert all(np.array_equal(x, y) for x, y in zip(a.logits(), b.logits()))
    a.close()
    b.close()


def test_slow_tiles_equal_pipelined_tiles(monkeypatch):
    """A net gives bit-identical results whichever tile kind it lands in (the kind can depend on the
    tile's composition, hence on the rank count): every tile on the slow / global-memory path
    (DGR_ALL_SLOW, read at plan time) against the normal plan."""
    f = forestgen.generate("c1e4")
    a = dgr.Solver(f)
    monkeypatch.setenv("DGR_ALL_SLOW", "1")
    b = dgr.Solver(f)
    monkeypatch.delenv("DGR_ALL_SLOW")
    assert b.info()["n_pipe_tiles"] == 0 and a.info()["n_pipe_tiles"] > 0
    for t in (1.0, 1.0, 0.9):
        assert np.array_equal(a.step(2, t, 0.3), b.step(2, t, 0.3))
    assert all(np.array_equal(x, y) for x, y in zip(a.demand(), b.demand()))
    assert all(np.array_equal(x, y) for x, y in zip(a.logits(), b.logits()))
    a.close()
    b.close()


def test_tma_window_equals_cp_async_window(monkeypatch):
    """The S window of a pipelined tile arrives by two 2-D TMA tensor copies, or (windows wider or
    taller than 256 cells, or DGR_NO_TMA_WINDOW at plan time) by cp.async: bit-identical results."""
    f = forestgen.generate("c1e4_c")
    a = dgr.Solver(f)
    monkeypatch.setenv("DGR_NO_TMA_WINDOW", "1")
    b = dgr.Solver(f)
    monkeypatch.delenv("DGR_NO_TMA_WINDOW")
    for t in (1.0, 0.9):
        assert np.array_equal(a.step(3, t, 0.3), b.step(3, t, 0.3))
    assert all(np.array_equal(x, y) for x, y in zip(a.demand(), b.demand()))
    assert all(np.array_equal(x, y) for x, y in zip(a.logits(), b.logits()))
    a.close()
    b.close()


@pytest.mark.parametrize("name", ["c1e4", "c1e4_m", "ispd18"])
def test_one_rank_nccl_exchange_reproduces_single_gpu(name):
    """The band exchange through a real NCCL communicator (one rank: dgr_dist with world 1 and an NCCL
    id, include/dgr.h): ncclReduceScatter / ncclAllGather / ncclAllReduce in groups on the handle's
    stream, the band clears and the polling wait, bit-identical to the plain single-GPU path."""
    f = forestgen.generate(name)
    ref = dgr.Solver(f)
    r_losses, (rdh, rdv), (rwt, rwp), rind = _schedule(ref)
    ref.close()
    s = dgr.Solver(f, nccl_id=dgr.nccl_unique_id())
    losses, (dh, dv), (wt, wp), ind = _schedule(s)
    s.close()
    for a, b in zip(losses, r_losses):
        assert np.array_equal(a, b)
    assert np.array_equal(dh, rdh) and np.array_equal(dv, rdv)
    assert np.array_equal(wt, rwt) and np.array_equal(wp, rwp)
    assert np.array_equal(ind.tree_choice, rind.tree_choice) and np.array_equal(ind.route, rind.route)
    assert np.array_equal(ind.D_h, rind.D_h) and np.array_equal(ind.metrics, rind.metrics)


_ABORT_SCRIPT = r"""
import os, sys
import numpy as np
import forestgen
import paper_conf_dac_0159layhrr24_b200 as dgr
s = dgr.Solver(forestgen.generate("ispd19"), nccl_id=dgr.nccl_unique_id())
s.step(2, 1.0, 0.3)
os.environ["DGR_NCCL_TIMEOUT_MS"] = "0"
try:
    s.step(100, 1.0, 0.3)
    sys.exit("no timeout")
except dgr.DgrError as e:
    assert "communicator aborted" in str(e), e
del os.environ["DGR_NCCL_TIMEOUT_MS"]
try:
    s.step(1, 1.0, 0.3)
    sys.exit("step after abort succeeded")
except dgr.DgrError as e:
    assert "aborted" in str(e), e
s.close()
t = dgr.Solver(forestgen.generate("tiny"))
assert np.isfinite(t.step(2, 1.0, 0.3)).all()
t.close()
print("ABORT-OK")
"""


def test_nccl_timeout_aborts_the_communicator():
    """A synchronising call that finds the NCCL exchange unfinished after DGR_NCCL_TIMEOUT_MS aborts
    the communicator (ncclCommAbort) and fails with DGR_ENCCL instead of hanging; later calls fail
    with DGR_ESTATE; the device stays usable.  A timeout of 0 ms trips on the first poll of a long
    call (100 ispd19 iterations, ~20 ms).  In a subprocess: an abort with work in flight must not
    take this test process's CUDA context with it if it goes wrong."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, "-c", _ABORT_SCRIPT], cwd=root, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0 and "ABORT-OK" in r.stdout, (r.returncode, r.stdout[-2000:], r.stderr[-2000:])


def test_tile_bundle_target_does_not_change_results(monkeypatch):
    """Small forests get tiles of fewer bundles (a full wave of resident tiles, make_plan); the tile
    composition never changes a result: auto against 32 and 4 group bundles per tile, bit-identical."""
    f = forestgen.generate("c1e4")
    outs = []
    for tb in (None, "32", "4"):
        if tb is None:
            monkeypatch.delenv("DGR_TILE_BUNDLES", raising=False)
        else:
            monkeypatch.setenv("DGR_TILE_BUNDLES", tb)
        s = dgr.Solver(f)
        monkeypatch.delenv("DGR_TILE_BUNDLES", raising=False)
        outs.append((s.info()["n_tiles"], _schedule(s)))
        s.close()
    assert outs[0][0] != outs[1][0] and outs[2][0] > outs[1][0]
    for _, (losses, (dh, dv), (wt, wp), ind) in outs[1:]:
        r_losses, (rdh, rdv), (rwt, rwp), rind = outs[0][1]
        assert all(np.array_equal(a, b) for a, b in zip(losses, r_losses))
        assert np.array_equal(dh, rdh) and np.array_equal(dv, rdv)
        assert np.array_equal(wt, rwt) and np.array_equal(wp, rwp)
        assert np.array_equal(ind.tree_choice, rind.tree_choice) and np.array_equal(ind.metrics, rind.metrics)

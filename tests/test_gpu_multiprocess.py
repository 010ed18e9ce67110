"""The N > 1 plumbing across PROCESSES on one GPU: one process per
rank under torchrun (127.0.0.1), the demand exchange through torch.distributed (gloo) via the
dgr_dist.allreduce callback instead of NCCL (NCCL cannot put two ranks on one GPU).  Everything else
is the production multi-rank path: per-rank plans, reduce-scatter of the demand bands, band-local KG,
all-gather of S, the induction exchange; the result must equal one rank bit-exactly."""
import json
import os
import socket
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _torchrun(nproc, *args, timeout=900):
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={nproc}",
           "--master-addr", "127.0.0.1", f"--master-port={_port()}", *args]
    r = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True, timeout=timeout)
    ranks = "\n".join(ln for ln in (r.stdout + r.stderr).splitlines() if "[rank" in ln)
    assert r.returncode == 0, ranks[-4000:] + r.stderr[-2000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout[-3000:] + r.stderr[-3000:]
    return json.loads(lines[0])


@pytest.mark.parametrize("name,nproc", [("c1e4", 2), ("c1e4_m", 3)])
def test_processes_reproduce_one_rank_bit_exactly(name, nproc):
    out = _torchrun(nproc, os.path.join("tools", "mp_parity.py"), name)
    assert out["ok"], out


def test_bench_two_ranks_through_torch_distributed():
    """bench.py's N > 1 path (launch, rendezvous, sharded solve, max-over-ranks timing, one JSON line
    from rank 0) with --exchange torch."""
    out = _torchrun(2, "bench.py", "--gpus", "2", "--exchange", "torch", "--config", "c1e4", "--steps", "3",
                    "--warmup", "3", "--no-quality", "--no-cpu-baseline", "--e2e-iters", "10")
    assert out["n_gpus"] == 2 and out["value"] > 0 and "gloo" in out["config"]["parallelism"]

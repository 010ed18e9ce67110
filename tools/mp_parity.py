"""Two (or more) processes, one rank each, exchanging through torch.distributed (gloo) via
dgr_dist.allreduce -- run under torchrun (127.0.0.1); every rank may share one GPU.  Rank 0 compares
the gathered demand, losses, logits and induction with a single-rank run of the same forest and
prints one JSON line ({"ok": true, ...}).  Used by tests/test_gpu_multiprocess.py.

    python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \\
        --master-port 29517 tools/mp_parity.py c1e4
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402
import torch.distributed as tdist  # noqa: E402

import forestgen  # noqa: E402
import paper_conf_dac_0159layhrr24_b200 as dgr  # noqa: E402


def schedule(s):
    losses = [s.step(6, 1.0, 0.3), s.step(4, 0.9, 0.3)]
    dh, dv = s.demand()
    wt, wp = s.logits()
    ind = s.induce(0.9)
    return dict(losses=np.array(losses), dh=dh, dv=dv, wt=wt, wp=wp, tree_choice=ind.tree_choice, route=ind.route,
                D_h=ind.D_h, D_v=ind.D_v, metrics=ind.metrics)


def main():
    name = sys.argv[1] if len(sys.argv) > 1 else "c1e4"
    rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
    torch.cuda.set_device(int(os.environ.get("LOCAL_RANK", 0)) % torch.cuda.device_count())
    tdist.init_process_group("gloo")
    f = forestgen.generate(name)
    s = dgr.Solver(f, rank=rank, world=world, allreduce=dgr.torch_allreduce())
    mine = schedule(s)
    part = dgr.partition(f, world)
    outs = [None] * world
    tdist.all_gather_object(outs, (part[rank], part[rank + 1], mine))
    if rank == 0:
        ref = schedule(dgr.Solver(f))
        ok = {}
        for key in ("losses", "dh", "dv", "D_h", "D_v", "metrics"):      # global on every rank
            ok[key] = all(np.array_equal(o[2][key], ref[key]) for o in outs)
        wt = np.full(f.n_trees, np.nan, np.float32); wp = np.full(f.n_paths, np.nan, np.float32)
        tc = np.full(f.n_nets, -2, np.int32); rt = np.full(f.n_subnets, -2, np.int32)
        for lo, hi, o in outs:   # each logit / choice from the rank that owns the net
            t0, t1 = f.net_tree_off[lo], f.net_tree_off[hi]
            s0, s1 = f.tree_sub_off[t0], f.tree_sub_off[t1]
            p0, p1 = f.sub_path_off[s0], f.sub_path_off[s1]
            wt[t0:t1] = o["wt"][t0:t1]; wp[p0:p1] = o["wp"][p0:p1]
            tc[lo:hi] = o["tree_choice"][lo:hi]; rt[s0:s1] = o["route"][s0:s1]
        ok["w_tree"] = bool(np.array_equal(wt, ref["wt"]))
        ok["w_path"] = bool(np.array_equal(wp, ref["wp"]))
        ok["tree_choice"] = bool(np.array_equal(tc, ref["tree_choice"]))
        ok["route"] = bool(np.array_equal(rt, ref["route"]))
        print(json.dumps({"ok": all(ok.values()), "checks": ok, "world": world, "forest": name}), flush=True)
    tdist.barrier()   # rank 0 has reported; process exit closes the gloo group


if __name__ == "__main__":
    main()

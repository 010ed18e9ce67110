"""Where does the world-8 emulation first diverge from world 1 (ispd19)?"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, forestgen
import paper_conf_dac_0159layhrr24_b200 as dgr
from tests.test_gpu_multirank import ThreadAllreduce, _run
name = sys.argv[1] if len(sys.argv) > 1 else "ispd19"; W = int(sys.argv[2]) if len(sys.argv) > 2 else 8
f = forestgen.generate(name)
ref = dgr.Solver(f)
ex = ThreadAllreduce(W)
sol = [dgr.Solver(f, rank=r, world=W, allreduce=ex.for_rank(r)) for r in range(W)]
part = dgr.partition(f, W)
to, so, po = np.asarray(f.net_tree_off), np.asarray(f.tree_sub_off), np.asarray(f.sub_path_off)
def gather(res):
    wt = np.zeros(f.n_trees, np.float32); wp = np.zeros(f.n_paths, np.float32)
    for r, (a, b) in enumerate(res):
        n0, n1 = part[r], part[r + 1]; t0, t1 = to[n0], to[n1]; p0, p1 = po[so[t0]], po[so[t1]]
        wt[t0:t1] = a[t0:t1]; wp[p0:p1] = b[p0:p1]
    return wt, wp
sched = [(1, 1.0)] * 6 + [(1, 0.9)] * 4 if os.environ.get("SPLIT") else [(6, 1.0), (4, 0.9)]
for it, (n_it, t) in enumerate(sched):
    lr_ = ref.step(n_it, t, 0.3)
    res = _run(sol, lambda s: (s.step(n_it, t, 0.3), s.demand(), s.logits()))
    dh, dv = res[0][1]; rdh, rdv = ref.demand()
    rwt, rwp = ref.logits(); wt, wp = gather([x[2] for x in res])
    print(f"it {it}: loss eq {np.array_equal(res[0][0], lr_)} {res[0][0] - lr_}  demand eq {np.array_equal(dh, rdh) and np.array_equal(dv, rdv)}"
          f"  (#diff H {int((dh != rdh).sum())} V {int((dv != rdv).sum())})  wt diff {int((wt != rwt).sum())}  wp diff {int((wp != rwp).sum())}")
    if (wp != rwp).any():
        idx = np.nonzero(wp != rwp)[0][:10]
        sub = np.searchsorted(po, idx, side="right") - 1; tree = np.searchsorted(so, sub, side="right") - 1
        net = np.searchsorted(to, tree, side="right") - 1
        print("  first differing paths", idx, "nets", net, "rank", np.searchsorted(part, net, side="right") - 1,
              "max |dw|", np.abs(wp - rwp).max())
    if (wt != rwt).any():
        idx = np.nonzero(wt != rwt)[0][:10]
        net = np.searchsorted(to, idx, side="right") - 1
        print("  first differing trees", idx, "nets", net)

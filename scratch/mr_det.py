"""Are two world-8 emulations (same schedule) bit-identical to each other?  (race vs partition effect)"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, forestgen
import paper_conf_dac_0159layhrr24_b200 as dgr
from tests.test_gpu_multirank import ThreadAllreduce, _run
name = sys.argv[1]; W = int(sys.argv[2])
f = forestgen.generate(name)
sets = []
for k in range(2):
    ex = ThreadAllreduce(W)
    sets.append([dgr.Solver(f, rank=r, world=W, allreduce=ex.for_rank(r)) for r in range(W)])
ref = dgr.Solver(f)
for it in range(6):
    outs = [_run(S, lambda s: (s.step(1, 1.0, 0.3), s.demand())) for S in sets]
    lr_ = ref.step(1, 1.0, 0.3); rd = ref.demand()
    a, b = outs
    print(f"it {it}: A==B loss {np.array_equal(a[0][0], b[0][0])} demand H {int((a[0][1][0] != b[0][1][0]).sum())} V {int((a[0][1][1] != b[0][1][1]).sum())} | A==ref demand H {int((a[0][1][0] != rd[0]).sum())} V {int((a[0][1][1] != rd[1]).sum())}", flush=True)

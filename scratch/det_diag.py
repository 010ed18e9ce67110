"""Run-to-run determinism of one rank at full size: two solvers, same schedule, bit-compare."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, forestgen
import paper_conf_dac_0159layhrr24_b200 as dgr
f = forestgen.generate(sys.argv[1] if len(sys.argv) > 1 else "ispd19")
A = dgr.Solver(f); B = dgr.Solver(f)
for it in range(6):
    la = A.step(1, 1.0, 0.3); lb = B.step(1, 1.0, 0.3)
    (ah, av), (bh, bv) = A.demand(), B.demand()
    (awt, awp), (bwt, bwp) = A.logits(), B.logits()
    d = np.nonzero(awp != bwp)[0]
    print(f"it {it}: loss eq {np.array_equal(la, lb)} demand diff H {int((ah != bh).sum())} V {int((av != bv).sum())} wt diff {int((awt != bwt).sum())} wp diff {len(d)} {d[:6]}", flush=True)

"""Do slow (global-path) tiles compute bit-identically to pipelined tiles?  world 1, DGR_ALL_SLOW
toggled between two solvers (the env is read at plan time)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, forestgen
import paper_conf_dac_0159layhrr24_b200 as dgr
f = forestgen.generate(sys.argv[1] if len(sys.argv) > 1 else "c1e4")
A = dgr.Solver(f)
os.environ["DGR_ALL_SLOW"] = "1"; B = dgr.Solver(f); del os.environ["DGR_ALL_SLOW"]
print("B tiles", B.info())
for it in range(6):
    la = A.step(1, 1.0, 0.3); lb = B.step(1, 1.0, 0.3)
    (ah, av), (bh, bv) = A.demand(), B.demand()
    (awt, awp), (bwt, bwp) = A.logits(), B.logits()
    d = np.nonzero(awp != bwp)[0]
    print(f"it {it}: loss eq {np.array_equal(la, lb)} {la - lb} demand diff H {int((ah != bh).sum())} V {int((av != bv).sum())} wt diff {int((awt != bwt).sum())} wp diff {len(d)} max {np.abs(awp-bwp).max():.3g}", flush=True)

"""Driver for compute-sanitizer: forward, a few fused iterations and induction on one config.

    compute-sanitizer --tool racecheck python tools/san_run.py tiny
DGR_ALL_SLOW=1 (read at plan time) puts every tile on the global-memory path."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import forestgen  # noqa: E402
import paper_conf_dac_0159layhrr24_b200 as dgr  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "tiny"
iters = int(sys.argv[2]) if len(sys.argv) > 2 else 2
f = forestgen.generate(name)
s = dgr.Solver(f)
s.step(0, 1.0, 0.3)                 # KF + KG + KL
s.step(iters, 1.0, 0.3)             # KG + KBF per iteration
s.step(1, 0.9, 0.3)                 # new temperature: stale events cleared, KF again
r = s.induce(0.9)                   # KI kernels
torch.cuda.synchronize()
print("san_run ok", name, s.info()["k"], float(r.metrics[0]))

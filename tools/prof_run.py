"""Minimal driver for ncu: load a forest, warm up, then run a few iterations (no timing)."""
import sys
import os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import forestgen
import paper_conf_dac_0159layhrr24_b200 as dgr

name = sys.argv[1] if len(sys.argv) > 1 else "ispd19"
iters = int(sys.argv[2]) if len(sys.argv) > 2 else 3
f = forestgen.generate(name.replace("+nshuf", ""))
if name.endswith("+nshuf"):   # the nets in a random order (the plan restores a spatial one)
    f = forestgen.shuffle_nets(f, seed=5)
s = dgr.Solver(f)
s.step(2, 1.0, 0.3, want_loss=False)
torch.cuda.synchronize()
s.step(iters, 1.0, 0.3, want_loss=True)
torch.cuda.synchronize()
print("done", s.info())

"""Host-side cost of the e2e step loop: 220 x step(1) in three forms (wall clock)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, forestgen
import paper_conf_dac_0159layhrr24_b200 as dgr
f = forestgen.generate("ispd19")
W = dgr.Weights()
s = dgr.Solver(f)
s.step(5, 1.0, 0.3, W)
n = 220
buf = torch.empty((n, 4), dtype=torch.float64).pin_memory().numpy()
for rep in range(2):
    torch.cuda.synchronize(); t = time.perf_counter()
    for i in range(n): s.step(1, 1.0, 0.3, W, want_loss=True)
    torch.cuda.synchronize(); a = time.perf_counter() - t
    t = time.perf_counter()
    for i in range(n): s.step_async(1, 1.0, 0.3, W, buf[i])
    s.sync(); b = time.perf_counter() - t
    t = time.perf_counter()
    for i in range(n): s.step(1, 1.0, 0.3, W, want_loss=False)
    torch.cuda.synchronize(); c = time.perf_counter() - t
    t = time.perf_counter()
    s.step(n, 1.0, 0.3, W, want_loss=False)
    torch.cuda.synchronize(); d = time.perf_counter() - t
    print(f"ms/step: sync-loss {a/n*1e3:.4f}  async-loss {b/n*1e3:.4f}  no-loss {c/n*1e3:.4f}  one-call {d/n*1e3:.4f}")

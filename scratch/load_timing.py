import sys, os, time
sys.path.insert(0, os.getcwd())
import torch
import forestgen
import paper_conf_dac_0159layhrr24_b200 as dgr
f = forestgen.generate("ispd19")
torch.cuda.init(); torch.zeros(1, device="cuda")
for r in range(3):
    t0 = time.perf_counter(); pi = dgr.plan_info(f); t1 = time.perf_counter()
    s = dgr.Solver(f); torch.cuda.synchronize(); t2 = time.perf_counter()
    s.step(1, 1.0, 0.3, want_loss=True); t3 = time.perf_counter()
    for _ in range(20): s.step(1, 1.0, 0.3, want_loss=True)
    t4 = time.perf_counter()
    print(f"plan_info {1e3*(t1-t0):.1f} ms  Solver() {1e3*(t2-t1):.1f} ms  first step {1e3*(t3-t2):.1f} ms  step(1)+loss {1e3*(t4-t3)/20:.3f} ms", flush=True)
    s.close()

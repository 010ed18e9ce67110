import sys, os, time
sys.path.insert(0, os.getcwd())
import forestgen
import paper_conf_dac_0159layhrr24_b200 as dgr
t=time.perf_counter(); f = forestgen.generate("ispd19"); print("gen", time.perf_counter()-t)
for r in range(3):
    t0 = time.perf_counter(); pi = dgr.plan_info(f); t1 = time.perf_counter()
    print(f"plan_info {1e3*(t1-t0):.1f} ms", flush=True)

"""Split of the e2e load: descriptor marshalling, dgr_forest_plan (host), workspace, dgr_bind_workspace."""
import ctypes, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, forestgen
import paper_conf_dac_0159layhrr24_b200 as dgr
from paper_conf_dac_0159layhrr24_b200 import dgr as B
f = forestgen.generate("ispd19")
torch.zeros(1, device="cuda")
L = B.load_library()
st = torch.cuda.current_stream()
print("omp threads", os.cpu_count(), flush=True)
for r in range(5):
    t0 = time.perf_counter(); d = B._DescHolder(f); t1 = time.perf_counter()
    h = ctypes.c_void_p()
    B._check(L.dgr_forest_plan(ctypes.byref(d.desc), None, ctypes.c_void_p(st.cuda_stream), ctypes.byref(h)))
    t2 = time.perf_counter()
    n = L.dgr_handle_workspace_size(h); ws = torch.empty(int(n), dtype=torch.uint8, device="cuda"); t3 = time.perf_counter()
    B._check(L.dgr_bind_workspace(h, ctypes.byref(d.desc), None, ctypes.c_void_p(ws.data_ptr()), int(n)))
    torch.cuda.synchronize(); t4 = time.perf_counter()
    L.dgr_free(h); del ws
    print(f"desc {1e3*(t1-t0):.1f}  plan {1e3*(t2-t1):.1f}  alloc {1e3*(t3-t2):.1f}  bind {1e3*(t4-t3):.1f} ms", flush=True)

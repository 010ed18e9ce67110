"""Same-box A/B timing of libdgr builds: python tools/ab_time.py CONFIG [iters] [reps]
(DGR_LIB selects the build).  Prints one JSON line: iterations/s (CUDA events around dgr_step(iters),
best of reps) and the per-stage milliseconds of one profiled repeat."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import forestgen  # noqa: E402
import paper_conf_dac_0159layhrr24_b200 as dgr  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "ispd19"
iters = int(sys.argv[2]) if len(sys.argv) > 2 else 200
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
f = forestgen.generate(name.replace("+nshuf", ""))
if name.endswith("+nshuf"):   # the same forest with its nets in a random order (the plan restores a spatial one)
    f = forestgen.shuffle_nets(f, seed=5)
s = dgr.Solver(f)
s.step(20, 1.0, 0.3, want_loss=False)
st = torch.cuda.current_stream()
best = 0.0
for _ in range(reps):
    e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record(st)
    s.step(iters, 1.0, 0.3, want_loss=False)
    e1.record(st)
    torch.cuda.synchronize()
    best = max(best, iters / (e0.elapsed_time(e1) * 1e-3))
# host enqueue time of the same call (dgr_step without a loss read does not synchronise): if it is
# below the device time per iteration, launches are not what bounds the loop
import time  # noqa: E402
torch.cuda.synchronize()
h0 = time.perf_counter()
s.step(iters, 1.0, 0.3, want_loss=False)
host_us = (time.perf_counter() - h0) / iters * 1e6
torch.cuda.synchronize()
s.profile(True)
s.step(iters, 1.0, 0.3, want_loss=False)
ms, n = s.profile_read()
s.profile(False)
print(json.dumps({"lib": os.path.basename(os.environ.get("DGR_LIB", "libdgr.so")), "kg_cta": bool(os.environ.get("DGR_KG_CTA")),
                  "config": name, "tile_bundles": os.environ.get("DGR_TILE_BUNDLES", "auto"),
                  "tiles": s.info()["n_tiles"], "iters_per_s": best, "host_enqueue_us_per_iter": host_us,
                  "stage_ms": {k: ms[k] / n[k] for k in ms if n[k]}}))

#!/bin/bash
# e2e / load A/B of the in-tree build against gpurun_scratch_head.so (bench lines without CPU baselines), then -m gpu
O=gpurun_out/$1; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/build_smoke.log 2>&1 || { tail -30 $O/build_smoke.log; exit 1; }
for round in 1 2; do
  for lib in gpurun_scratch_head.so paper_conf_dac_0159layhrr24_b200/libdgr.so; do
    DGR_LIB=$PWD/$lib timeout 900 python bench.py --no-cpu-baseline --no-quality > $O/b.log 2>&1
    python - $O/b.log $lib <<'PY'
import json, sys
l = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
print(sys.argv[2].split('/')[-1], round(l["value"]), "e2e", round(l["e2e"]["value"]), l["e2e"].get("split"))
PY
  done
done 2>&1 | tee $O/e2e.txt
DGR_PLAN_TIMING=1 timeout 300 python -c "
import time, forestgen, paper_conf_dac_0159layhrr24_b200 as dgr
f = forestgen.generate('ispd19')
for _ in range(2):
    t = time.perf_counter(); s = dgr.Solver(f); print('load_ms', (time.perf_counter() - t) * 1e3); s.close()
" > $O/plan_timing.txt 2>&1
DGR_PARITY_COUNTS=$O/parity_counts.json timeout 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -3 | tee $O/pytest_gpu.log

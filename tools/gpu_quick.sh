#!/bin/bash
# build + gpu tests (optional) + bench line; usage: tools/gpu_quick.sh TAG [tests|notests] [bench args...]
TAG=${1:-run}; MODE=${2:-tests}; shift; shift
O=gpurun_out/$TAG; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/build_smoke.log 2>&1 || { tail -30 $O/build_smoke.log; exit 1; }
tail -1 $O/build_smoke.log
if [ "$MODE" = tests ]; then
  timeout 1200 python -m pytest tests -q -m gpu -x > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
  tail -15 $O/pytest_gpu.log
fi
timeout 900 python bench.py --no-quality --no-cpu-baseline "$@" > $O/bench.log 2>&1; tail -1 $O/bench.log | cut -c1-300
python - <<'PY' $O/bench.log
import json,sys
l=open(sys.argv[1]).read().strip().split('\n')[-1]
try:
    d=json.loads(l); print('VALUE', d['value'], d.get('stage_ms_per_launch'), d['roofline']['frac'])
except Exception as e: print('bench parse failed', e)
PY

#!/bin/bash
# A/B bench of libdgr variants: scratch/ab.sh lib1 lib2 ...
for lib in "$@"; do
  for r in 1 2; do
    DGR_LIB=$lib python bench.py --no-quality --no-cpu-baseline --steps 300 --warmup 20 2>/dev/null | python -c "
import json,sys
d=json.loads(sys.stdin.read().strip().splitlines()[-1]); s=d['stage_ms_per_launch']
print('$lib', round(d['value'],1), 'KBF', round(s['KBF'],4), 'KG', round(s['KG'],4), 'e2e', round(d['e2e']['value'],1))"
  done
done

#!/bin/bash
# A/B of libdgr variants with optional env: scratch/ab2.sh lib1 "VAR=1@lib2" ...
for spec in "$@"; do
  envs=""; lib=$spec
  if [[ "$spec" == *@* ]]; then envs=${spec%@*}; lib=${spec#*@}; fi
  for r in 1 2; do
    env $envs DGR_LIB=$lib python bench.py --no-quality --no-cpu-baseline --steps 300 --warmup 20 2>/dev/null | python -c "
import json,sys
d=json.loads(sys.stdin.read().strip().splitlines()[-1]); s=d['stage_ms_per_launch']
print('$spec', round(d['value'],1), 'KBF', round(s['KBF'],4), 'KG', round(s['KG'],4), 'e2e', round(d['e2e']['value'],1), d['e2e'].get('split'))"
  done
done

#!/bin/bash
# A/B of libdgr variants (optionally with env): scratch/ab3.sh "lib[:ENV=V]" ...  (2 reps each)
for spec in "$@"; do
  lib=${spec%%:*}; envs=""; [[ "$spec" == *:* ]] && envs=${spec#*:}
  for r in 1 2; do
    env $envs DGR_LIB=$lib python bench.py --no-quality --no-cpu-baseline --steps 300 --warmup 20 2>/dev/null | python -c "
import json,sys
d=json.loads(sys.stdin.read().strip().splitlines()[-1]); s=d['stage_ms_per_launch']
print('$spec', round(d['value'],1), 'KBF', round(s['KBF'],4), 'KG', round(s['KG'],4))"
  done
done

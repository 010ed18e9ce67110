#!/bin/bash
# one bench per environment setting: scratch/ko.sh "VAR=1" ...
for env in "" "$@"; do
  env $env python bench.py --no-quality --no-cpu-baseline --steps 300 --warmup 20 2>/dev/null | python -c "
import json,sys
d=json.loads(sys.stdin.read().strip().splitlines()[-1]); s=d['stage_ms_per_launch']
print('[$env]', round(d['value'],1), 'KBF', round(s['KBF'],4), 'KG', round(s['KG'],4))"
done

#!/bin/bash
# same-box A/B of run-time switches of the in-tree build: tools/gpu_ab_env.sh TAG "cfg1 cfg2" "ENV=1" "ENV2=1" ...
# ("-" = no switch); two rounds, interleaved
TAG=$1; CFGS=$2; shift 2
O=gpurun_out/$TAG; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
for round in 1 2; do
  for cfg in $CFGS; do
    for e in "$@"; do
      if [ "$e" = - ]; then python tools/ab_time.py $cfg 200 3 | sed 's/^/{"env": "-", "d": /; s/$/}/'
      else env $e python tools/ab_time.py $cfg 200 3 | sed "s|^|{\"env\": \"$e\", \"d\": |; s|\$|}|"; fi
    done
  done
done 2>&1 | grep -v Warning | tee $O/ab.jsonl | python -c "
import sys, json
for l in sys.stdin:
    try: d = json.loads(l)
    except Exception: print(l.strip()[:200]); continue
    print(d['env'], d['d']['config'], round(d['d']['iters_per_s']), {k: round(v*1e3, 1) for k, v in d['d']['stage_ms'].items()})
"

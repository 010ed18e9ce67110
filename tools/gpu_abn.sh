#!/bin/bash
# same-box A/B of several libdgr builds: tools/gpu_abn.sh TAG "cfg1 cfg2" lib1.so lib2.so ... ("default" = the in-tree build)
TAG=$1; CFGS=$2; shift 2
O=gpurun_out/$TAG; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
for round in 1 2; do
  for cfg in $CFGS; do
    for lib in "$@"; do
      if [ "$lib" = default ]; then python tools/ab_time.py $cfg 200 3; else DGR_LIB=$PWD/$lib python tools/ab_time.py $cfg 200 3; fi
    done
  done
done 2>&1 | grep -v Warning | tee $O/ab.jsonl | python -c "
import sys, json
for l in sys.stdin:
    try: d = json.loads(l)
    except Exception: print(l.strip()[:200]); continue
    print(d['lib'], d['config'], round(d['iters_per_s']), {k: round(v*1e3, 1) for k, v in d['stage_ms'].items()})
"

#!/bin/bash
# KBF knock-out table (timing only, results invalid): a -DDGR_DIAG=1 build timed with each phase of the
# tile kernel switched off (DGR_DEBUG_SKIP bits: 1 flush, 2 path noise, 4 forward events, 8 path cost, 512 global tiles,
# 16 whole tile body, 32 S window, 64 reverse, 128 net level); the marginal cost of each phase.
# usage: tools/gpu_ko.sh TAG [CONFIG] [skip values...]
TAG=${1:-ko}; CFG=${2:-ispd19}; shift; shift
O=gpurun_out/$TAG; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
DGR_NVCC_EXTRA="-DDGR_DIAG=1 $KO_EXTRA" python -c "
import paper_conf_dac_0159layhrr24_b200.build as b, shutil
b.build(force=True); shutil.copy(b.LIB, 'gpurun_diag.so')" > $O/diag_build.log 2>&1 || { tail -30 $O/diag_build.log; exit 1; }
SKIPS=${@:-0 1 2 4 8 64 128 32 40 16}
for round in 1 2; do
  python tools/ab_time.py $CFG 200 3 | sed 's/^/{"skip": "default", "d": /; s/$/}/'
  for sk in $SKIPS; do
    DGR_LIB=$PWD/gpurun_diag.so DGR_DEBUG_SKIP=$sk python tools/ab_time.py $CFG 200 3 | sed "s/^/{\"skip\": $sk, \"d\": /; s/\$/}/"
  done
done 2>&1 | grep -v Warning | tee $O/ko.jsonl | python -c "
import sys, json
for l in sys.stdin:
    try: d = json.loads(l)
    except Exception: print(l.strip()[:200]); continue
    print(d['skip'], round(d['d']['iters_per_s']), {k: round(v*1e3, 1) for k, v in d['d']['stage_ms'].items()})
"

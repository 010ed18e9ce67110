#!/bin/bash
# same-box A/B of the default build against gpurun_scratch_head.so on CONFIGS, then the -m gpu suite
# usage: tools/gpu_ab2.sh TAG "cfg1 cfg2 ..." [pytest -k expr]
TAG=$1; CFGS=$2; K=$3
O=gpurun_out/$TAG; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/build_smoke.log 2>&1 || { tail -30 $O/build_smoke.log; exit 1; }
for round in 1 2; do
  for cfg in $CFGS; do
    for lib in gpurun_scratch_head.so paper_conf_dac_0159layhrr24_b200/libdgr.so; do
      DGR_LIB=$PWD/$lib python tools/ab_time.py $cfg 200 3
    done
  done
done 2>&1 | grep -v Warning | tee $O/ab.jsonl | cut -c1-200
if [ -n "$K" ]; then
  DGR_PARITY_COUNTS=$O/parity_counts.json timeout 1500 python -m pytest tests -m gpu -q -x -k "$K" 2>&1 | tail -4 | tee $O/pytest_gpu.log
else
  DGR_PARITY_COUNTS=$O/parity_counts.json timeout 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -4 | tee $O/pytest_gpu.log
fi

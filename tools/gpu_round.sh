#!/bin/bash
# One GPU-box pass: build, gpu tests, bench line, ncu launch list + one full capture of the top kernel.
# usage: tools/gpu_round.sh TAG [tests|notests]
TAG=${1:-run}; MODE=${2:-tests}
O=gpurun_out/$TAG; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/build_smoke.log 2>&1 || { tail -30 $O/build_smoke.log; exit 1; }
if [ "$MODE" = tests ]; then
  timeout 1500 python -m pytest tests -q -m gpu -x > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
  tail -3 $O/pytest_gpu.log
fi
timeout 900 python bench.py > $O/bench.log 2>&1; tail -1 $O/bench.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -s 10 -c 60 --csv --log-file $O/launches.csv python tools/prof_run.py ispd19 8 > $O/ncu_launch.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:tile_bulk -s 3 -c 1 -o $O/kbf python tools/prof_run.py ispd19 3 > $O/ncu_full.log 2>&1
timeout 600 ncu --set full --clock-control none -k regex:kg_kernel -s 3 -c 1 -o $O/kg python tools/prof_run.py ispd19 3 > $O/ncu_kg.log 2>&1
ls -la $O

#!/bin/bash
# Full GPU pass: build + smoke, all -m gpu tests (parity counts), bench lines for ispd19 (default),
# c1e4 (configs[1]) and ispd18 (configs[2]), the ncu launch list of the bench workload.
# usage: tools/gpu_full.sh TAG
TAG=${1:-full}; O=gpurun_out/$TAG; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/build_smoke.log 2>&1 || { tail -30 $O/build_smoke.log; exit 1; }
DGR_PARITY_COUNTS=$O/parity_counts.json timeout 2400 python -m pytest tests -q -m gpu -rf > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
grep -E "passed|failed|Error" $O/pytest_gpu.log | tail -8
timeout 900 python bench.py > $O/bench.log 2>&1; tail -1 $O/bench.log | cut -c1-400
for c in c1e4 ispd18; do
  timeout 900 python bench.py --config $c --no-cpu-baseline > $O/bench_$c.log 2>&1; tail -1 $O/bench_$c.log | cut -c1-300
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -s 10 -c 60 --csv --log-file $O/launches.csv python tools/prof_run.py ispd19 8 > $O/ncu_launch.log 2>&1
cp paper_conf_dac_0159layhrr24_b200/csrc/dgr_kernels.cu $O/
timeout 900 ncu --set full --clock-control none --import-source on -k regex:tile_bulk -s 3 -c 1 -o $O/kbf python tools/prof_run.py ispd19 3 > $O/ncu_full.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:kg_kernel -s 3 -c 1 -o $O/kg python tools/prof_run.py ispd19 3 > $O/ncu_kg.log 2>&1
ls $O

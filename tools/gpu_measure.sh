#!/bin/bash
# The round's measurement pass on one B200: build + smoke, the -m gpu suite (parity counts), bench lines
# (ispd19 default with cpu_baseline + quality; c1e4 = configs[1]; ispd18 = configs[2]; ispd19_c; sweep4e6),
# the sweep, host plan phase times, the ncu launch list of the bench workload and one ncu --set full
# capture each of KBF and KG (with source), per-tile phase clocks (diagnostic build).
# usage: tools/gpu_measure.sh TAG [notests]
TAG=${1:-measure}; MODE=${2:-tests}
O=gpurun_out/$TAG; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.limit --format=csv > $O/smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/build_smoke.log 2>&1 || { tail -30 $O/build_smoke.log; exit 1; }
if [ "$MODE" = tests ]; then
  DGR_PARITY_COUNTS=$O/parity_counts.json timeout 2400 python -m pytest tests -q -m gpu -rf > $O/pytest_gpu.log 2>&1
  echo "pytest rc=$?" >> $O/pytest_gpu.log; grep -E "passed|failed|rc=" $O/pytest_gpu.log | tail -3
fi
timeout 900 python bench.py > $O/bench.log 2>&1; tail -1 $O/bench.log | cut -c1-300
for c in c1e4 ispd18 ispd19_c sweep4e6; do
  timeout 900 python bench.py --config $c --no-cpu-baseline --no-quality > $O/bench_$c.log 2>&1; tail -1 $O/bench_$c.log | cut -c1-200
done
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > $O/bench_reference.log 2>&1; tail -1 $O/bench_reference.log | cut -c1-200
timeout 900 python tools/sweep.py > $O/sweep.jsonl 2>$O/sweep.err; tail -4 $O/sweep.jsonl | cut -c1-160
DGR_PLAN_TIMING=1 timeout 300 python -c "
import time, forestgen, paper_conf_dac_0159layhrr24_b200 as dgr
f = forestgen.generate('ispd19')
for _ in range(2):
    t = time.perf_counter(); s = dgr.Solver(f); print('load_ms', (time.perf_counter() - t) * 1e3); s.close()
" > $O/plan_timing.txt 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -s 10 -c 60 --csv --log-file $O/launches.csv python tools/prof_run.py ispd19 8 > $O/ncu_launch.log 2>&1
cp paper_conf_dac_0159layhrr24_b200/csrc/dgr_kernels.cu $O/
timeout 900 ncu --set full --clock-control none --import-source on -k regex:tile_bulk -s 3 -c 1 -o $O/kbf python tools/prof_run.py ispd19 3 > $O/ncu_full.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:kg_kernel -s 3 -c 1 -o $O/kg python tools/prof_run.py ispd19 3 > $O/ncu_kg.log 2>&1
# per-tile phase clocks: a diagnostic build (-DDGR_DIAG=1) loaded through DGR_LIB, then the normal build back
DGR_NVCC_EXTRA="-DDGR_DIAG=1" python -c "
import paper_conf_dac_0159layhrr24_b200.build as b, shutil
b.build(force=True); shutil.copy(b.LIB, 'gpurun_diag.so')" > $O/diag_build.log 2>&1
python -c "import paper_conf_dac_0159layhrr24_b200.build as b; b.build(force=True)" >> $O/diag_build.log 2>&1
DGR_LIB=$PWD/gpurun_diag.so timeout 300 python tools/tprof.py ispd19 > $O/tile_phases.txt 2>&1; head -12 $O/tile_phases.txt
ls $O
